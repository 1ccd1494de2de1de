cd "${GRAFT_REPO_ROOT:-.}"; mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_dp_replicas.py -q -x --timeout 600 2>&1 | tail -8
timeout 300 python tools/sanitize_case.py 2>&1 | tail -2
bash tools/sanitize.sh
