cd "${GRAFT_REPO_ROOT:-.}"; mkdir -p gpurun_out
timeout 600 python tools/hash_bench.py --checksum crc32c --chunk 1048576 --reps 10 --variants base,b0f,zb,zbb0f 2>&1 | grep -v Warn
timeout 600 python tools/hash_bench.py --checksum crc32c --chunk 16777216 --reps 6 --variants base,b0f,zb,zbb0f 2>&1 | grep -v Warn
timeout 600 python tools/hash_bench.py --checksum crc32c --chunk 4096 --gib 8 --reps 6 --variants base,b0f,zb,zbb0f 2>&1 | grep -v Warn
