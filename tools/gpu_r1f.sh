cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q --maxfail=10 --timeout 300 > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
tail -5 gpurun_out/pytest_gpu.log
timeout 1200 python tools/sweep.py --gib 8 --checksums xxh64 --mechs sm,ce_region,ce_pipe --out gpurun_out/sweep_xxh > gpurun_out/sweep_xxh.log 2>&1; echo "rc=$?" >> gpurun_out/sweep_xxh.log
cat gpurun_out/sweep_xxh.md
