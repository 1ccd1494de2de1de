cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_arena.py -m gpu -q --timeout 600 -x > gpurun_out/pytest_arena.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_arena.log
tail -15 gpurun_out/pytest_arena.log
timeout 1500 python tools/trace_e.py --duration 300 --seed 1 --out gpurun_out/trace_e_300_seq.json > gpurun_out/trace_seq.log 2>&1; echo "rc=$?" >> gpurun_out/trace_seq.log
timeout 1500 python tools/trace_e.py --duration 300 --seed 1 --duplex --out gpurun_out/trace_e_300_duplex.json > gpurun_out/trace_dup.log 2>&1; echo "rc=$?" >> gpurun_out/trace_dup.log
tail -2 gpurun_out/trace_seq.log | cut -c1-1200; tail -3 gpurun_out/trace_dup.log | cut -c1-1200
