cd "${GRAFT_REPO_ROOT:-.}"; mkdir -p gpurun_out
timeout 900 ncu --set full --clock-control none --import-source on -k regex:xxh_quad -c 1 -o gpurun_out/ncu_verify_B_xxh64_r02 -f \
    python tools/prof_case.py --config B --mechanism sm --checksum xxh64 --reps 1 > gpurun_out/ncu_verify_B_xxh64_r02.log 2>&1; echo "xxh rc=$?"
ncu -i gpurun_out/ncu_verify_B_xxh64_r02.ncu-rep --page details > gpurun_out/ncu_verify_B_xxh64_r02_details.txt 2>/dev/null
ncu -i gpurun_out/ncu_verify_B_xxh64_r02.ncu-rep --page raw --csv > gpurun_out/ncu_verify_B_xxh64_r02_raw.csv 2>/dev/null
timeout 900 ncu --set full --clock-control none --import-source on -k regex:hash_kernel -c 1 -o gpurun_out/ncu_verify_B_crc_r02 -f \
    python tools/prof_case.py --config B --mechanism sm --checksum crc32c --reps 1 > gpurun_out/ncu_verify_B_crc_r02.log 2>&1; echo "crc rc=$?"
ncu -i gpurun_out/ncu_verify_B_crc_r02.ncu-rep --page details > gpurun_out/ncu_verify_B_crc_r02_details.txt 2>/dev/null
ncu -i gpurun_out/ncu_verify_B_crc_r02.ncu-rep --page raw --csv > gpurun_out/ncu_verify_B_crc_r02_raw.csv 2>/dev/null
ncu -i gpurun_out/ncu_verify_B_crc_r02.ncu-rep --page source --csv --print-source sass > gpurun_out/ncu_verify_B_crc_r02_sass.csv 2>/dev/null
rm -f gpurun_out/*.ncu-rep
