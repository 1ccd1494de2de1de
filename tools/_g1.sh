cd "${GRAFT_REPO_ROOT:-.}"; mkdir -p gpurun_out
timeout 1200 ncu --replay-mode app-range --metrics pcie__read_bytes.sum,pcie__write_bytes.sum,dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum \
  --csv --log-file gpurun_out/counters.csv python tools/counters.py --cases-out gpurun_out/counter_cases.json > gpurun_out/counters.log 2>&1
echo "counters rc=$?"; tail -5 gpurun_out/counters.log; head -5 gpurun_out/counters.csv
for C in 1048576 4194304; do
  timeout 600 python tools/hash_bench.py --checksum xxh64 --chunk $C --reps 8 --variants quad,quad3k,quad2 2>&1 | grep -v Warn
done
