cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 600 ./tools/probe_tma > gpurun_out/probe_tma.log 2>&1; echo "rc=$?" >> gpurun_out/probe_tma.log
# launch list of the default bench command (single-metric pass, no replay)
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_B.csv python bench.py --steps 2 --warmup 1 --no-compare --no-cpu-baseline > gpurun_out/ncu_launch_bench.log 2>&1; echo "rc=$?" >> gpurun_out/ncu_launch_bench.log
# full capture of the three movers (gather, scatter, hash_check) on config A, warm step
timeout 900 ncu --set full --clock-control none --import-source on -k regex:mover_kernel -s 6 -c 3 -o gpurun_out/prof_A python bench.py --config A --steps 2 --warmup 2 --no-compare --no-cpu-baseline > gpurun_out/ncu_full_A.log 2>&1; echo "rc=$?" >> gpurun_out/ncu_full_A.log
cat gpurun_out/probe_tma.log; tail -3 gpurun_out/ncu_launch_bench.log; tail -3 gpurun_out/ncu_full_A.log
