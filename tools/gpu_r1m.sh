cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 1800 python -m pytest tests -m gpu -q --maxfail=5 --timeout 600 > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
tail -4 gpurun_out/pytest_gpu.log
timeout 900 python bench.py --steps 3 --warmup 3 --no-cpu-baseline --no-compare --checksum xxh64 > gpurun_out/bench_B_xxh.log 2>&1
grep -o '"roofline_verify[^}]*}' gpurun_out/bench_B_xxh.log
timeout 900 python bench.py --config C --steps 3 --warmup 3 --no-cpu-baseline --no-compare > gpurun_out/bench_C.log 2>&1; echo "rc=$?" >> gpurun_out/bench_C.log
tail -2 gpurun_out/bench_C.log | cut -c1-700
timeout 900 python bench.py --config D --steps 3 --warmup 3 --no-cpu-baseline --no-compare > gpurun_out/bench_D.log 2>&1; echo "rc=$?" >> gpurun_out/bench_D.log
tail -2 gpurun_out/bench_D.log | cut -c1-700
