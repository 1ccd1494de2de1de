# ncu --set full captures of the HBM verify pass (a8) on the full bench workload (config B, 52.57 GB):
# checkpoint/restore use the SM movers, so the only hash kernel launched is the verify pass.
# Run with: gpurun --timeout 2400 -- "bash tools/ncu_verify.sh [crc32c] [xxh64]". Reports land in gpurun_out/.
cd "${GRAFT_REPO_ROOT:-.}"
mkdir -p gpurun_out
for ck in ${@:-crc32c xxh64}; do
  k=$([ $ck = crc32c ] && echo "regex:hash_kernel|crc_ts_kernel|crc_mx_kernel" || echo regex:xxh_)
  timeout 1200 ncu --set full --clock-control none --import-source on -k $k -c 1 -o gpurun_out/ncu_verify_B_$ck -f \
    python tools/prof_case.py --config B --mechanism sm --checksum $ck --reps 1 > gpurun_out/ncu_verify_B_$ck.log 2>&1
  echo "$ck rc=$?"
  ncu -i gpurun_out/ncu_verify_B_$ck.ncu-rep --page raw --csv > gpurun_out/ncu_verify_B_${ck}_raw.csv 2>/dev/null
  ncu -i gpurun_out/ncu_verify_B_$ck.ncu-rep --page details > gpurun_out/ncu_verify_B_${ck}_details.txt 2>/dev/null
done
