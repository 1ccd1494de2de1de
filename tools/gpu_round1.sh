cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -q --maxfail=20 --timeout 300 > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 300 python bench.py --config A --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/bench_A.log 2>&1; echo "rc=$?" >> gpurun_out/bench_A.log
timeout 900 python bench.py --steps 5 --warmup 3 > gpurun_out/bench_B.log 2>&1; echo "rc=$?" >> gpurun_out/bench_B.log
tail -30 gpurun_out/pytest_gpu.log; tail -3 gpurun_out/bench_A.log; tail -3 gpurun_out/bench_B.log
