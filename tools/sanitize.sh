# compute-sanitizer over the smoke path (config-B mix, 8 MiB + edge sizes, CRC32C and XXH64, SM mover)
# and one CE_PIPE round trip. Run on the GPU box.
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
cat > /tmp/san_case.py <<'PY'
import sys, os
sys.path.insert(0, os.environ.get("GRAFT_REPO_ROOT", "."))
import __graft_entry__ as g
g.smoke()
import torch, numpy as np, workloads as W
from paper_conf_sc_stoyanovsracb25_b200 import swap
specs = W.config_a(3)
host, offs = W.host_arena(specs, 3)
arena = torch.from_numpy(host).cuda()
regions = [(arena.data_ptr() + o, r.nbytes, r.kind, i) for i, (r, o) in enumerate(zip(specs, offs))]
s = torch.cuda.Stream()
for mech in ("ce_pipe", "sm"):
    with swap.Swapper(regions, chunk_bytes=1 << 16, mechanism=mech, pipe_mib=8) as sw, torch.cuda.stream(s):
        sw.checkpoint(s); sw.restore(s); assert sw.verify(s)["status"] == 0
print("case ok")
PY
for tool in memcheck racecheck synccheck initcheck; do
  timeout 1200 compute-sanitizer --tool $tool --print-limit 20 python /tmp/san_case.py > gpurun_out/sanitize_$tool.log 2>&1
  echo "$tool rc=$?" >> gpurun_out/sanitize_$tool.log
  tail -4 gpurun_out/sanitize_$tool.log
done
