cd "${GRAFT_REPO_ROOT:-.}"; mkdir -p gpurun_out
timeout 2700 python -m pytest tests -m gpu -q --timeout 900 > gpurun_out/pytest_gpu_r02b.log 2>&1; echo "tests rc=$?"; tail -3 gpurun_out/pytest_gpu_r02b.log
timeout 300 python __graft_entry__.py smoke 2>&1 | tail -2
timeout 900 python bench.py > gpurun_out/bench_B_r02c.log 2>&1; echo "bench rc=$?"; tail -1 gpurun_out/bench_B_r02c.log | cut -c1-200
