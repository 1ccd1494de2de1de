cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
for m in sm ce_pipe auto; do
timeout 600 python bench.py --config A --steps 20 --warmup 5 --no-cpu-baseline --no-compare --mechanism $m > gpurun_out/bench_A_$m.log 2>&1
echo "$m: $(grep -o '"swap_in_latency_s": [0-9.]*' gpurun_out/bench_A_$m.log) $(grep -o '"restore_GBps_per_gpu": [0-9.]*' gpurun_out/bench_A_$m.log)"
done
for g in 0.0625 0.25 1 4; do
timeout 600 python tools/sweep.py --gib $g --chunks 1048576 --checksums crc32c --mechs sm,ce_pipe,ce_batch --reps 5 --out gpurun_out/sw_$g > /dev/null 2>&1; tail -3 gpurun_out/sw_$g.md
done
