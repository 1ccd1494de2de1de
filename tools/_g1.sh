cd "${GRAFT_REPO_ROOT:-.}"; mkdir -p gpurun_out
timeout 600 ncu --replay-mode app-range --metrics pcie__read_bytes.sum,pcie__write_bytes.sum,dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum \
  --csv --log-file gpurun_out/counters_tma.csv tools/probe_tma ranges > gpurun_out/counters_tma.log 2>&1; echo "tma rc=$?"; cat gpurun_out/counters_tma.log | tail -8
timeout 1200 ncu --replay-mode app-range --metrics pcie__read_bytes.sum,pcie__write_bytes.sum,dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum \
  --csv --log-file gpurun_out/counters8.csv python tools/counters.py --gib 8 --chunks 1048576,16777216 --cases-out gpurun_out/counter_cases8.json > gpurun_out/counters8.log 2>&1
echo "counters8 rc=$?"
