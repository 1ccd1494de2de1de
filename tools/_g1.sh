cd "${GRAFT_REPO_ROOT:-.}"; mkdir -p gpurun_out
timeout 1500 python -m pytest tests/test_gpu_multirank.py tests/test_gpu_parity.py tests/test_gpu_large_region.py -q -x --timeout 900 2>&1 | tail -5
timeout 900 python bench.py > gpurun_out/bench_B_r02b.log 2>&1; echo "bench rc=$?"; tail -1 gpurun_out/bench_B_r02b.log | cut -c1-300
