cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_shard.py tests/test_gpu_dist.py -q --timeout 900 -p no:cacheprovider -k "enum or c1 or div7 or random_dfas or multi_rank" > gpurun_out/r2_t22.log 2>&1; echo "rc=$?" >> gpurun_out/r2_t22.log
timeout 900 python bench.py --config c5 --c5-dfa c1 --steps 5 --warmup 3 2>&1 | tail -1 > gpurun_out/r2_t22_c5c1.log
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 60 --csv --log-file gpurun_out/r2_t22_launch_c1.csv python bench.py --config c5 --c5-dfa c1 --steps 1 --warmup 3 > /dev/null 2>&1
timeout 600 python bench.py --config c1 --steps 20 --warmup 3 --e2e-steps 0 --no-cpu-baseline --no-per-dfa 2>&1 | tail -1 > gpurun_out/r2_t22_c1.log
