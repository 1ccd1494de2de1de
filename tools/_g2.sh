cd "${GRAFT_REPO_ROOT:-.}"; mkdir -p gpurun_out
timeout 1500 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_B_r02.csv \
  python bench.py --steps 2 --warmup 1 --no-compare --no-cpu-baseline > gpurun_out/ncu_launches_r02.log 2>&1; echo "launches rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:hash_kernel -c 2 -o gpurun_out/ncu_verify_A -f \
    python tools/prof_case.py --config A --mechanism sm --checksum crc32c --reps 1 > gpurun_out/ncu_verify_A.log 2>&1; echo "A rc=$?"
ncu -i gpurun_out/ncu_verify_A.ncu-rep --page details > gpurun_out/ncu_verify_A_details.txt 2>/dev/null
ncu -i gpurun_out/ncu_verify_A.ncu-rep --page source --csv --print-source sass > gpurun_out/ncu_verify_A_sass.csv 2>/dev/null
rm -f gpurun_out/*.ncu-rep
