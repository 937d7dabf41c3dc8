cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_shard.py -q --timeout 900 -p no:cacheprovider -k "lookback or cse_spec16 or fake_collective or spread or pm_tree or inline_round0 or configs_small or random_dfas or edge_lengths or full_size or async or bank_aware" > gpurun_out/r2_t5.log 2>&1; echo "rc=$?" >> gpurun_out/r2_t5.log
for v in 1 0; do
  GSPEC_V0=$v timeout 600 python bench.py --config c2 --steps 20 --warmup 3 --e2e-steps 0 --no-cpu-baseline --no-per-dfa > gpurun_out/r2_v0_$v_c2.log 2>&1
  GSPEC_V0=$v timeout 600 python bench.py --config c2 --steps 20 --warmup 3 --e2e-steps 0 --no-cpu-baseline --no-per-dfa > gpurun_out/r2_v0${v}_c2.log 2>&1
  GSPEC_V0=$v timeout 600 python bench.py --config c4 --steps 10 --warmup 3 --e2e-steps 0 --no-cpu-baseline --no-per-dfa > gpurun_out/r2_v0${v}_c4.log 2>&1
done
timeout 600 python bench.py --config c3 --steps 10 --warmup 3 --e2e-steps 0 --no-cpu-baseline --no-per-dfa > gpurun_out/r2_c3_after.log 2>&1
