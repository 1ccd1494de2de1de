cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q --maxfail=10 --timeout 300 > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 900 python bench.py --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/bench_B.log 2>&1; echo "rc=$?" >> gpurun_out/bench_B.log
timeout 900 python bench.py --steps 3 --warmup 3 --no-cpu-baseline --no-compare --checksum xxh64 > gpurun_out/bench_B_xxh.log 2>&1; echo "rc=$?" >> gpurun_out/bench_B_xxh.log
tail -15 gpurun_out/pytest_gpu.log; tail -2 gpurun_out/bench_B.log; tail -2 gpurun_out/bench_B_xxh.log
