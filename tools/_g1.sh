cd "${GRAFT_REPO_ROOT:-.}"; mkdir -p gpurun_out
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fuzz.py tests/test_gpu_xxh_variants.py -q -x --timeout 900 2>&1 | tail -3
for C in 65536 1048576 4194304 16777216; do
timeout 600 python bench.py --config A --checksum xxh64 --chunk $C --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/bench_A_xxh_$C.log 2>&1; echo "rc=$?"
tail -1 gpurun_out/bench_A_xxh_$C.log | python -c "
import json,sys; d=json.loads(sys.stdin.read()); print($C, d['value'], d['config']['mechanism'], json.dumps(d['mechanisms']))"
done
