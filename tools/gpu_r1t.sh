cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 1800 python -m pytest tests -m gpu -q --timeout 600 > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
tail -4 gpurun_out/pytest_gpu.log
timeout 600 python bench.py --config A --steps 20 --warmup 5 --no-cpu-baseline > gpurun_out/bench_A.log 2>&1
tail -2 gpurun_out/bench_A.log | head -1 | cut -c1-200; grep -o '"swap_in_latency_s": [0-9.]*\|"roofline_verify[^}]*}\|"mechanisms": {[^}]*}[^}]*}[^}]*}[^}]*}[^}]*}' gpurun_out/bench_A.log
timeout 900 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-compare > gpurun_out/bench_B.log 2>&1
grep -o '"swap_in_latency_s": [0-9.]*\|"achieved": [0-9.]*' gpurun_out/bench_B.log
