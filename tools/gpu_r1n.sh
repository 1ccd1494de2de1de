cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
# launch list of the default bench command (single metric, no replay)
timeout 1200 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_B2.csv python bench.py --steps 2 --warmup 1 --no-compare --no-cpu-baseline > gpurun_out/ncu_launch_bench2.log 2>&1; echo "rc=$?" >> gpurun_out/ncu_launch_bench2.log
tail -2 gpurun_out/ncu_launch_bench2.log | cut -c1-200
# full captures at 8 GiB: CRC verify kernel, XXH64 verify kernel, SM scatter
timeout 900 ncu --set full --clock-control none --import-source on -k regex:hash_kernel -s 3 -c 1 -o gpurun_out/prof_hash_crc python tools/prof_case.py --gib 8 --mechanism sm > gpurun_out/ncu_hash.log 2>&1; echo "rc=$?" >> gpurun_out/ncu_hash.log
timeout 900 ncu --set full --clock-control none --import-source on -k regex:xxh_lane_kernel -s 1 -c 1 -o gpurun_out/prof_hash_xxh python tools/prof_case.py --gib 16 --mechanism sm --checksum xxh64 --reps 1 > gpurun_out/ncu_xxh.log 2>&1; echo "rc=$?" >> gpurun_out/ncu_xxh.log
timeout 900 ncu --set full --clock-control none --import-source on -k regex:mover_kernel -s 2 -c 2 -o gpurun_out/prof_sm_movers python tools/prof_case.py --gib 4 --mechanism sm --reps 2 > gpurun_out/ncu_sm.log 2>&1; echo "rc=$?" >> gpurun_out/ncu_sm.log
tail -1 gpurun_out/ncu_hash.log gpurun_out/ncu_xxh.log gpurun_out/ncu_sm.log
timeout 2400 python tools/trace_e.py --duration 600 --seed 0 --out gpurun_out/trace_e_600.json > gpurun_out/trace_e600.log 2>&1; echo "rc=$?" >> gpurun_out/trace_e600.log
tail -2 gpurun_out/trace_e600.log | cut -c1-600
