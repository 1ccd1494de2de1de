cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_helpers.py -m gpu -q --timeout 600 > gpurun_out/pytest_helpers.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_helpers.log
tail -25 gpurun_out/pytest_helpers.log
