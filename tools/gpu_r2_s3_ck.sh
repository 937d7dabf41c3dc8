# R30 checkpointed dense rounds: parity tests touching dense rounds, then C3 / C3s bench lines (SRE, RR, NF)
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_records.py -m gpu -q --timeout 900 -p no:cacheprovider -x \
  -k "checkpointed or dense or memoized or vr_others or records or configs_small or full_size_other" > gpurun_out/ck_pytest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/ck_pytest.log
for c in c3 c3s; do
  timeout 600 python bench.py --config $c --steps 10 --warmup 3 --e2e-steps 0 --no-cpu-baseline --no-per-dfa > gpurun_out/ck_bench_$c.log 2>&1
  GSPEC_CK=0 timeout 600 python bench.py --config $c --steps 10 --warmup 3 --e2e-steps 0 --no-cpu-baseline --no-per-dfa > gpurun_out/ck0_bench_$c.log 2>&1
done
for s in rr nf; do
  timeout 600 python bench.py --config c3 --scheme $s --steps 10 --warmup 3 --e2e-steps 0 --no-cpu-baseline --no-per-dfa > gpurun_out/ck_bench_c3_$s.log 2>&1
done
for ck in 256 1024; do
  GSPEC_CK=$ck timeout 600 python bench.py --config c3 --steps 10 --warmup 3 --e2e-steps 0 --no-cpu-baseline --no-per-dfa > gpurun_out/ck${ck}_bench_c3.log 2>&1
done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/ck_launches_c3.csv python tools/profile_spec.py c3 sre 2 > gpurun_out/ck_ncu_launch_c3.log 2>&1
