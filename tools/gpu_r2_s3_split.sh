cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
: > gpurun_out/sp_probe.log
for c in c3 c3s; do echo "$c" >> gpurun_out/sp_probe.log; timeout 300 python tools/ck_probe.py $c sre 4 >> gpurun_out/sp_probe.log 2>&1; done
for c in c2 c3 c4 c1; do timeout 600 python bench.py --config $c --steps 10 --warmup 3 --e2e-steps 0 --no-cpu-baseline --no-per-dfa > gpurun_out/sp_bench_$c.log 2>&1; done
CK_PROFILE_LAST=1 timeout 600 ncu --profile-from-start off --metrics gpu__time_duration.sum,smsp__inst_executed.sum --clock-control none --csv --log-file gpurun_out/sp_launches_c3.csv python tools/ck_probe.py c3 sre 3 > gpurun_out/sp_ncu.log 2>&1
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_records.py -m gpu -q --timeout 900 -p no:cacheprovider -x > gpurun_out/sp_pytest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/sp_pytest.log
