cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 ncu --set full --clock-control none --import-source on -k regex:hash_kernel -s 1 -c 1 -o gpurun_out/prof_hash_crc2 python tools/prof_case.py --gib 8 --mechanism sm > gpurun_out/ncu_hash2.log 2>&1; echo "rc=$?"
