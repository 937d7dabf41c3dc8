cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 1200 python -m pytest tests/test_gpu_bench.py -q --timeout 900 -p no:cacheprovider -k "more_steps" > gpurun_out/r2_t28.log 2>&1; echo "rc=$?" >> gpurun_out/r2_t28.log
for f in 1 0; do GSPEC_TK=$f timeout 600 python bench.py --config c1 --steps 50 --warmup 5 --e2e-steps 0 --no-cpu-baseline --no-per-dfa 2>&1 | tail -1 > gpurun_out/r2_t28_c1_tk$f.log; done
timeout 600 python bench.py --steps 100 --warmup 5 --e2e-steps 0 --no-cpu-baseline --no-per-dfa 2>&1 | tail -1 > gpurun_out/r2_t28_c2_100.log
