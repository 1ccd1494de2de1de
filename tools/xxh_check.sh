cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests/test_gpu_xxh_variants.py tests/test_gpu_parity.py -k "xxh" -m gpu -q --timeout 600 > gpurun_out/pytest_xxh.log 2>&1; echo "rc=$?"; tail -2 gpurun_out/pytest_xxh.log
timeout 900 python bench.py --steps 3 --warmup 2 --no-cpu-baseline --no-compare --checksum xxh64 > gpurun_out/bench_xxh.log 2>&1
grep -o '"roofline_verify[^}]*}' gpurun_out/bench_xxh.log
