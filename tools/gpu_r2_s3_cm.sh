cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_records.py -m gpu -q --timeout 900 -p no:cacheprovider -x -k "checkpointed or dense or memoized or vr_others or records or configs_small or full_size_other or literal" > gpurun_out/cm_pytest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/cm_pytest.log
: > gpurun_out/cm.log
for c in c3 c3s; do timeout 600 python bench.py --config $c --steps 10 --warmup 3 --e2e-steps 0 --no-cpu-baseline --no-per-dfa > gpurun_out/cm_$c.log 2>&1; echo "$c $(grep -o '"value": [0-9.]*, "unit"\|"ms_per_step": [0-9.]*\|"gpu_launches": [0-9]*' gpurun_out/cm_$c.log | head -3 | tr '\n' ' ')" >> gpurun_out/cm.log; done
