cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_arena.py -m gpu -q --timeout 600 > gpurun_out/pytest_arena.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_arena.log
tail -5 gpurun_out/pytest_arena.log
timeout 900 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-compare > gpurun_out/bench_B.log 2>&1; echo "rc=$?" >> gpurun_out/bench_B.log
tail -2 gpurun_out/bench_B.log | cut -c1-300; grep -o '"swap_in_with[^,]*,\|"hbm_reacquire_s[^,]*,\|"swap_in_with_overlapped[^,]*,' gpurun_out/bench_B.log
timeout 900 python tools/state_reduction.py > gpurun_out/state_reduction.log 2>&1; echo "rc=$?" >> gpurun_out/state_reduction.log
tail -2 gpurun_out/state_reduction.log
timeout 1800 python tools/trace_e.py --duration 300 --seed 1 --out gpurun_out/trace_e_300.json > gpurun_out/trace_e.log 2>&1; echo "rc=$?" >> gpurun_out/trace_e.log
tail -2 gpurun_out/trace_e.log
