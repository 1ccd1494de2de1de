cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_multirank.py -m gpu -q --timeout 600 > gpurun_out/pytest_multirank.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_multirank.log
timeout 900 python bench.py --steps 5 --warmup 3 > gpurun_out/bench_B.log 2>&1; echo "rc=$?" >> gpurun_out/bench_B.log
tail -30 gpurun_out/pytest_multirank.log; tail -2 gpurun_out/bench_B.log
