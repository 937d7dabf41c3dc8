cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_records.py tests/test_gpu_shard.py -q --timeout 900 -p no:cacheprovider -k "memoized or dense_recovery or vr_others or configs_small or random_dfas or true_walk or chained or nccl_single" > gpurun_out/r2_t10.log 2>&1; echo "rc=$?" >> gpurun_out/r2_t10.log
for s in rr nf sre; do
  timeout 600 python bench.py --config c3 --scheme $s --steps 10 --warmup 3 --e2e-steps 0 --no-cpu-baseline --no-per-dfa > gpurun_out/r2_lazy_c3_$s.log 2>&1
  timeout 600 python bench.py --config c3s --scheme $s --steps 10 --warmup 3 --e2e-steps 0 --no-cpu-baseline --no-per-dfa > gpurun_out/r2_lazy_c3s_$s.log 2>&1
done
GSPEC_LAZY_HELPERS=0 timeout 600 python bench.py --config c3 --scheme rr --steps 10 --warmup 3 --e2e-steps 0 --no-cpu-baseline --no-per-dfa > gpurun_out/r2_eager_c3_rr.log 2>&1
