cd "${GRAFT_REPO_ROOT:-.}"; mkdir -p gpurun_out
( time timeout 900 python bench.py --impl reference > gpurun_out/bench_ref_r02.log 2>&1 ) 2>&1 | tail -3; tail -1 gpurun_out/bench_ref_r02.log | cut -c1-400
timeout 900 python -m pytest tests/test_gpu_multirank.py -q -x --timeout 600 2>&1 | tail -3
