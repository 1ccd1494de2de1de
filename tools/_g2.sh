cd "${GRAFT_REPO_ROOT:-.}"; mkdir -p gpurun_out
for C in 16777216; do
  SWAP_XXH_KERNEL=quad timeout 900 ncu --set full --clock-control none --import-source on -k regex:xxh_quad -c 1 -o gpurun_out/ncu_quadt_$C -f \
    python tools/prof_case.py --config B --mechanism sm --checksum xxh64 --chunk $C --reps 1 > gpurun_out/ncu_quadt_$C.log 2>&1
  echo "ncu $C rc=$?"
  ncu -i gpurun_out/ncu_quadt_$C.ncu-rep --page details > gpurun_out/ncu_quadt_${C}_details.txt 2>/dev/null
  ncu -i gpurun_out/ncu_quadt_$C.ncu-rep --page raw --csv > gpurun_out/ncu_quadt_${C}_raw.csv 2>/dev/null
  ncu -i gpurun_out/ncu_quadt_$C.ncu-rep --page source --csv --print-source sass > gpurun_out/ncu_quadt_${C}_sass.csv 2>/dev/null
done
