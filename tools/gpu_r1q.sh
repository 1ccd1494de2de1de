cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_xxh_variants.py -m gpu -q --timeout 600 > gpurun_out/pytest_xxh.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_xxh.log
tail -12 gpurun_out/pytest_xxh.log
for v in lane quad ring; do
  SWAP_XXH_KERNEL=$v timeout 900 python bench.py --steps 3 --warmup 2 --no-cpu-baseline --no-compare --checksum xxh64 > gpurun_out/bench_xxh_$v.log 2>&1
  echo "$v: $(grep -o '"achieved": [0-9.]*, "peak": 6549.4' gpurun_out/bench_xxh_$v.log)"
done
SWAP_XXH_KERNEL=quad timeout 900 python tools/sweep.py --gib 8 --checksums xxh64 --mechs ce_region --out gpurun_out/sweep_xxh_quad > /dev/null 2>&1; tail -4 gpurun_out/sweep_xxh_quad.md
SWAP_XXH_KERNEL=ring timeout 900 python tools/sweep.py --gib 8 --checksums xxh64 --mechs ce_region --out gpurun_out/sweep_xxh_ring > /dev/null 2>&1; tail -4 gpurun_out/sweep_xxh_ring.md
