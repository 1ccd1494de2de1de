cd "${GRAFT_REPO_ROOT:-.}"; mkdir -p gpurun_out
for C in 262144 524288 2097152 8388608 16777216; do
  timeout 600 python tools/hash_bench.py --checksum xxh64 --chunk $C --reps 8 --variants quad,quad2,quad3k,quad1k,lane8,dyn 2>&1 | grep -v Warn
done
timeout 600 python tools/hash_bench.py --checksum crc32c --chunk 1048576 --reps 8 2>&1 | grep -v Warn
