cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_shard.py -q --timeout 900 -p no:cacheprovider -k "enum or c1 or div7 or random_dfas" > gpurun_out/r2_t20.log 2>&1; echo "rc=$?" >> gpurun_out/r2_t20.log
for f in 1 0; do GSPEC_TK=$f timeout 900 python bench.py --config c5 --c5-dfa c1 --steps 5 --warmup 3 2>&1 | tail -1 > gpurun_out/r2_t20_c5c1_t4$f.log; done
timeout 600 python bench.py --config c1 --steps 20 --warmup 3 --e2e-steps 0 --no-cpu-baseline --no-per-dfa 2>&1 | tail -1 > gpurun_out/r2_t20_c1.log
