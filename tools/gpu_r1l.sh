cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
df -h /tmp . | tail -3; mount | grep -E " / | /tmp " | head
timeout 900 python -m pytest tests/test_gpu_storage.py tests/test_gpu_parity.py -k "storage or save or xxh64_hash or bit_exact" -m gpu -q --timeout 600 > gpurun_out/pytest_storage.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_storage.log
tail -5 gpurun_out/pytest_storage.log
timeout 900 python bench.py --steps 3 --warmup 3 --no-cpu-baseline --no-compare --checksum xxh64 > gpurun_out/bench_B_xxh.log 2>&1
grep -o '"roofline_verify[^}]*}' gpurun_out/bench_B_xxh.log
timeout 1200 python tools/storage_bench.py /tmp/swap_bench.img > gpurun_out/storage.log 2>&1; echo "rc=$?" >> gpurun_out/storage.log
tail -3 gpurun_out/storage.log
