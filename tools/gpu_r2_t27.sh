cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_shard.py tests/test_gpu_dist.py tests/test_gpu_batch.py -q --timeout 900 -p no:cacheprovider -k "enum or c1 or div7 or random_dfas or multi_rank or batch" > gpurun_out/r2_t27.log 2>&1; echo "rc=$?" >> gpurun_out/r2_t27.log
for f in 1 0; do GSPEC_TK=$f timeout 600 python bench.py --config c1 --steps 50 --warmup 5 --e2e-steps 0 --no-cpu-baseline --no-per-dfa 2>&1 | tail -1 > gpurun_out/r2_t27_c1_tk$f.log; done
