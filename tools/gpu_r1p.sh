cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 1800 python -m pytest tests -m gpu -q --maxfail=5 --timeout 600 > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
tail -3 gpurun_out/pytest_gpu.log
timeout 900 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-compare > gpurun_out/bench_B.log 2>&1
grep -o '"roofline_verify[^}]*}' gpurun_out/bench_B.log; grep -o '"swap_in_latency_s": [0-9.]*' gpurun_out/bench_B.log
