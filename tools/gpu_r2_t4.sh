cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_shard.py tests/test_gpu_dist.py -q --timeout 900 -p no:cacheprovider -k "lookback or cse_spec16 or fake_collective or spread or pm_tree or run_sharded" > gpurun_out/r2_t4.log 2>&1; echo "rc=$?" >> gpurun_out/r2_t4.log
for c in c2 c3 c4; do timeout 600 python bench.py --config $c --scheme cse --steps 5 --warmup 3 --e2e-steps 0 --no-cpu-baseline --no-per-dfa > gpurun_out/r2_cse_$c.log 2>&1; done
