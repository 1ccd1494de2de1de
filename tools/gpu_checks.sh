# One GPU-box job (run with: gpurun --timeout 3600 -- 'bash tools/gpu_checks.sh [what ...]').
#   tests   : pytest -m gpu                       smoke  : __graft_entry__.smoke()
#   bench   : bench.py config B (default line)    benchA : bench.py --config A
#   launches: ncu launch list of the bench        sweep  : tools/sweep.py 8 GiB
#   trace   : tools/trace_e.py 300 s, sequential and full duplex
#   sanitize: tools/sanitize.sh
# Logs land in gpurun_out/.
cd "${GRAFT_REPO_ROOT:-.}"
mkdir -p gpurun_out
what="${*:-tests smoke bench}"
for w in $what; do
  case $w in
    tests) timeout 1800 python -m pytest tests -m gpu -q --timeout 600 > gpurun_out/pytest_gpu.log 2>&1
           echo "tests rc=$?"; tail -3 gpurun_out/pytest_gpu.log ;;
    smoke) timeout 300 python __graft_entry__.py smoke 2>&1 | tail -2 ;;
    bench) timeout 900 python bench.py > gpurun_out/bench_B.log 2>&1; echo "bench rc=$?"; tail -1 gpurun_out/bench_B.log | cut -c1-400 ;;
    benchA) timeout 600 python bench.py --config A --steps 20 --warmup 5 > gpurun_out/bench_A.log 2>&1; tail -1 gpurun_out/bench_A.log | cut -c1-400 ;;
    launches) timeout 1200 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_B.csv \
                python bench.py --steps 2 --warmup 1 --no-compare --no-cpu-baseline > gpurun_out/ncu_launches.log 2>&1; echo "launches rc=$?" ;;
    sweep) timeout 2400 python tools/sweep.py --gib 8 --out gpurun_out/sweep > gpurun_out/sweep.log 2>&1; cat gpurun_out/sweep.md ;;
    trace) timeout 1800 python tools/trace_e.py --duration 300 --seed 1 --out gpurun_out/trace_seq.json > /dev/null 2>&1
           timeout 1800 python tools/trace_e.py --duration 300 --seed 1 --duplex --out gpurun_out/trace_duplex.json > /dev/null 2>&1
           cat gpurun_out/trace_seq.json gpurun_out/trace_duplex.json | cut -c1-400 ;;
    sanitize) bash tools/sanitize.sh ;;
    *) echo "unknown: $w" ;;
  esac
done
