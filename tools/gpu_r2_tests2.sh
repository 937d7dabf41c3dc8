cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
nproc > gpurun_out/r2_nproc.txt
timeout 900 python -m pytest tests/test_gpu_shard.py tests/test_gpu_parity.py -q --timeout 600 -p no:cacheprovider -k "invalid_symbol_in or failed or nonmerging or dense_recovery or vr_others or enum_bound or input_sensitive or configs_small" > gpurun_out/r2_t2.log 2>&1; echo "rc=$?" >> gpurun_out/r2_t2.log
for s in sre rr nf; do
  timeout 600 python bench.py --config c3 --scheme $s --steps 5 --warmup 3 --e2e-steps 0 --no-cpu-baseline --no-per-dfa > gpurun_out/r2_c3_$s.log 2>&1
  timeout 600 python bench.py --config c3s --scheme $s --steps 5 --warmup 3 --e2e-steps 0 --no-cpu-baseline --no-per-dfa > gpurun_out/r2_c3s_$s.log 2>&1
done
