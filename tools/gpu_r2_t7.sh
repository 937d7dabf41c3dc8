# ENUM with 64-entry maps + selector bound + shard ENUM path; experiment analogues if not done
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_shard.py -q --timeout 900 -p no:cacheprovider -k "enum_bound or random_dfas or div7_c1 or nonmerging or fake_collective" > gpurun_out/r2_t7.log 2>&1; echo "rc=$?" >> gpurun_out/r2_t7.log
for e in 0 1; do for p in 0 1; do
  GSPEC_TMA_EVICT=$e GSPEC_TMA_PROMO=$p timeout 600 python bench.py --config c4 --steps 10 --warmup 3 --e2e-steps 0 --no-cpu-baseline --no-per-dfa > gpurun_out/r2_tma_c4_e${e}p${p}.log 2>&1
  GSPEC_TMA_EVICT=$e GSPEC_TMA_PROMO=$p timeout 600 python bench.py --config c2 --steps 20 --warmup 3 --e2e-steps 0 --no-cpu-baseline --no-per-dfa > gpurun_out/r2_tma_c2_e${e}p${p}.log 2>&1
done; done
GSPEC_TMA_EVICT=1 timeout 900 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none -k regex:k_spec_tma -s 2 -c 1 --csv python tools/profile_spec.py c4 sre 3 > gpurun_out/r2_tma_c4_evictnormal_dram.csv 2>&1
timeout 900 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none -k regex:k_spec_tma -s 2 -c 1 --csv python tools/profile_spec.py c4 sre 3 > gpurun_out/r2_tma_c4_default_dram.csv 2>&1
