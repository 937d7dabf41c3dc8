cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_shard.py -q --timeout 600 -p no:cacheprovider -k "dense_recovery or vr_others or configs_small or random_dfas or chained or nonmerging or failed or invalid_symbol_in" > gpurun_out/r2_t3.log 2>&1; echo "rc=$?" >> gpurun_out/r2_t3.log
for s in rr nf; do
  timeout 600 python bench.py --config c3 --scheme $s --steps 5 --warmup 3 --e2e-steps 0 --no-cpu-baseline --no-per-dfa > gpurun_out/r2_c3_$s.log 2>&1
  timeout 600 python bench.py --config c3s --scheme $s --steps 5 --warmup 3 --e2e-steps 0 --no-cpu-baseline --no-per-dfa > gpurun_out/r2_c3s_$s.log 2>&1
done
