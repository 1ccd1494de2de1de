# compute-sanitizer over every kernel family and mover (tools/sanitize_case.py). Run on the GPU box.
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
for tool in memcheck racecheck synccheck initcheck; do
  timeout 1500 compute-sanitizer --tool $tool --print-limit 20 python tools/sanitize_case.py > gpurun_out/sanitize_$tool.log 2>&1
  echo "$tool rc=$?" >> gpurun_out/sanitize_$tool.log
  grep -E "SUMMARY|rc=|case ok" gpurun_out/sanitize_$tool.log
done
