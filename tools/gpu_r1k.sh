cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 1800 python -m pytest tests -m gpu -q --maxfail=5 --timeout 600 > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
tail -6 gpurun_out/pytest_gpu.log
timeout 900 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-compare > gpurun_out/bench_B.log 2>&1; echo "rc=$?" >> gpurun_out/bench_B.log
grep -o '"roofline_verify[^}]*}' gpurun_out/bench_B.log; grep -o '"swap_in_latency_s": [0-9.]*' gpurun_out/bench_B.log
timeout 1200 python tools/sweep.py --gib 8 --checksums crc32c --mechs ce_region --out gpurun_out/sweep_crc > gpurun_out/sweep_crc.log 2>&1
cat gpurun_out/sweep_crc.md | tail -5
