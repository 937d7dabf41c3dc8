cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_records.py tests/test_gpu_shard.py -q --timeout 900 -p no:cacheprovider -k "memoized or dense_recovery or true_walk or nccl_single or configs_small" > gpurun_out/r2_t11.log 2>&1; echo "rc=$?" >> gpurun_out/r2_t11.log
for s in rr nf sre; do timeout 600 python bench.py --config c3 --scheme $s --steps 10 --warmup 3 --e2e-steps 0 --no-cpu-baseline --no-per-dfa > gpurun_out/r2_final_c3_$s.log 2>&1; done
timeout 600 python bench.py --steps 20 --warmup 3 --e2e-steps 0 --no-cpu-baseline --no-per-dfa > gpurun_out/r2_final_c2.log 2>&1
