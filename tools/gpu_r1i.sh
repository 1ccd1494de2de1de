cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python bench.py --steps 5 --warmup 3 > gpurun_out/bench_B.log 2>&1; echo "rc=$?" >> gpurun_out/bench_B.log
tail -2 gpurun_out/bench_B.log
timeout 900 python tools/state_reduction.py > gpurun_out/state_reduction.log 2>&1; echo "rc=$?" >> gpurun_out/state_reduction.log
tail -3 gpurun_out/state_reduction.log
