cd "${GRAFT_REPO_ROOT:-.}"; mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_dp_replicas.py -q -x --timeout 300 2>&1 | tail -15
timeout 2400 python -m pytest tests -m gpu -q --timeout 900 > gpurun_out/pytest_gpu_r02.log 2>&1; echo "tests rc=$?"; tail -5 gpurun_out/pytest_gpu_r02.log
timeout 300 python __graft_entry__.py smoke 2>&1 | tail -2
timeout 900 python bench.py --checksum xxh64 --no-compare > gpurun_out/bench_B_xxh64_r02.log 2>&1; echo "bench rc=$?"; tail -1 gpurun_out/bench_B_xxh64_r02.log | cut -c1-300
