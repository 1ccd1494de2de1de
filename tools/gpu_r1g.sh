cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_arena.py tests/test_gpu_parity.py -k "arena or xxh64_hash" -m gpu -q --timeout 300 > gpurun_out/pytest_arena.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_arena.log
tail -15 gpurun_out/pytest_arena.log
timeout 1500 python tools/trace_e.py --duration 180 --seed 0 --out gpurun_out/trace_e_180.json > gpurun_out/trace_e.log 2>&1; echo "rc=$?" >> gpurun_out/trace_e.log
tail -20 gpurun_out/trace_e.log
