cd "${GRAFT_REPO_ROOT:-.}"; mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_helpers.py tests/test_gpu_multirank.py -q -x --timeout 600 2>&1 | tail -4
timeout 300 python tools/seg_ab.py 2>&1 | tail -6
timeout 600 python bench.py --config A --steps 20 --warmup 5 > gpurun_out/bench_A_r02c.log 2>&1; echo "benchA rc=$?"; tail -1 gpurun_out/bench_A_r02c.log | cut -c1-200
