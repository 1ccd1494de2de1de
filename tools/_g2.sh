cd "${GRAFT_REPO_ROOT:-.}"; mkdir -p gpurun_out
timeout 1500 python -m pytest tests/test_gpu_parity.py -q -x --timeout 900 2>&1 | tail -2
timeout 900 ncu --set full --clock-control none --import-source on -k regex:mover_kernel -c 3 -o gpurun_out/ncu_mover_xxh_A -f \
    python tools/prof_case.py --config A --mechanism sm --checksum xxh64 --reps 1 > gpurun_out/ncu_mover_xxh_A.log 2>&1; echo "rc=$?"
ncu -i gpurun_out/ncu_mover_xxh_A.ncu-rep --page details > gpurun_out/ncu_mover_xxh_A_details.txt 2>/dev/null
ncu -i gpurun_out/ncu_mover_xxh_A.ncu-rep --page source --csv --print-source sass > gpurun_out/ncu_mover_xxh_A_sass.csv 2>/dev/null
rm -f gpurun_out/*.ncu-rep
