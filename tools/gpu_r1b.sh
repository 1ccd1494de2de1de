cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 300 ./tools/probe_ce > gpurun_out/probe_ce.log 2>&1
timeout 1500 python -m pytest tests -m gpu -q --maxfail=10 --timeout 300 > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 900 python bench.py --steps 5 --warmup 3 > gpurun_out/bench_B.log 2>&1; echo "rc=$?" >> gpurun_out/bench_B.log
timeout 300 python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/bench_ref.log 2>&1; echo "rc=$?" >> gpurun_out/bench_ref.log
cat gpurun_out/probe_ce.log; tail -15 gpurun_out/pytest_gpu.log; tail -2 gpurun_out/bench_B.log; tail -2 gpurun_out/bench_ref.log
