cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
bash tools/sanitize.sh
timeout 2400 python tools/sweep.py --gib 8 --out gpurun_out/sweep > gpurun_out/sweep.log 2>&1; echo "rc=$?" >> gpurun_out/sweep.log
tail -3 gpurun_out/sweep.log; cat gpurun_out/sweep.md
