cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 ncu --set full --clock-control none --import-source on -k regex:hash_kernel -s 1 -c 1 -o gpurun_out/prof_hash_crc python tools/prof_case.py --gib 8 --mechanism sm > gpurun_out/ncu_hash.log 2>&1; echo "rc=$?" >> gpurun_out/ncu_hash.log
timeout 900 ncu --set full --clock-control none --import-source on -k regex:xxh_lane_kernel -s 1 -c 1 -o gpurun_out/prof_hash_xxh python tools/prof_case.py --gib 8 --mechanism sm --checksum xxh64 --chunk 262144 > gpurun_out/ncu_xxh.log 2>&1; echo "rc=$?" >> gpurun_out/ncu_xxh.log
tail -2 gpurun_out/ncu_hash.log gpurun_out/ncu_xxh.log
