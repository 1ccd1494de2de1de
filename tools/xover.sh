cd $GRAFT_REPO_ROOT
for g in 0.015625 0.0625 0.25 1 4 16; do
timeout 900 python tools/sweep.py --gib $g --chunks 1048576 --checksums crc32c --mechs sm,ce_batch,ce_pipe,ce_region --reps 5 --out gpurun_out/xo_$g > /dev/null 2>&1
python - <<PY
import json
for l in open("gpurun_out/xo_$g.jsonl"):
    r=json.loads(l); P=r["payload"]
    ti=P/r["restore_GBps"]/1e9+P/r["verify_GBps"]/1e9
    print("$g", r["mechanism"], "restore", r["restore_GBps"], "ckpt", r["checkpoint_GBps"], "swapin_GBps", round(P/ti/1e9,2))
PY
done
