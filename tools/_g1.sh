cd "${GRAFT_REPO_ROOT:-.}"; mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_xxh_variants.py -q -x --timeout 600 2>&1 | tail -3
for C in 16777216 4194304 1048576 262144; do
  timeout 600 python tools/hash_bench.py --checksum xxh64 --chunk $C --reps 8 --variants dyn,dyn_x,quad,quad_x,quad1k,lane8 2>&1 | grep -v Warn
done
