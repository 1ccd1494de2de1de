cd "${GRAFT_REPO_ROOT:-.}"; mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_dp_replicas.py tests/test_gpu_multirank.py -q -x --timeout 600 2>&1 | tail -25
