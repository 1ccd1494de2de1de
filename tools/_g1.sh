cd "${GRAFT_REPO_ROOT:-.}"; mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_dp_replicas.py -q -x --timeout 600 2>&1 | tail -20
timeout 1800 python -m pytest tests/test_gpu_fullsize.py -q -x --timeout 900 -k "xxh64" 2>&1 | tail -5
