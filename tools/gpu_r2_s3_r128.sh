cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
: > gpurun_out/r128.log
echo "mixed" >> gpurun_out/r128.log; timeout 300 python tools/ck_probe.py c3 sre 4 >> gpurun_out/r128.log 2>&1
echo "row64" >> gpurun_out/r128.log; GSPEC_CK_ROW=64 timeout 300 python tools/ck_probe.py c3 sre 4 >> gpurun_out/r128.log 2>&1
for c in c3 c3s; do timeout 600 python bench.py --config $c --steps 10 --warmup 3 --e2e-steps 0 --no-cpu-baseline --no-per-dfa > gpurun_out/r128_$c.log 2>&1; echo "$c $(grep -o '"value": [0-9.]*, "unit"\|"ms_per_step": [0-9.]*' gpurun_out/r128_$c.log | head -2 | tr '\n' ' ')" >> gpurun_out/r128.log; done
CK_PROFILE_LAST=1 timeout 600 ncu --profile-from-start off --metrics gpu__time_duration.sum,smsp__inst_executed.sum --clock-control none --csv --log-file gpurun_out/r128_launches_c3.csv python tools/ck_probe.py c3 sre 3 > gpurun_out/r128_ncu.log 2>&1
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_records.py -m gpu -q --timeout 900 -p no:cacheprovider -x -k "checkpointed or dense or memoized or vr_others or records or configs_small or full_size_other" > gpurun_out/r128_pytest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/r128_pytest.log
