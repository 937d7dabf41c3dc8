cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
for k in 10 20 50; do timeout 600 python bench.py --steps $k --warmup 3 --e2e-steps 0 --no-cpu-baseline --no-per-dfa 2>&1 | tail -1 >> gpurun_out/r2_t39.jsonl; done
timeout 600 python bench.py --config c3 --steps 10 --warmup 3 --e2e-steps 0 --no-cpu-baseline --no-per-dfa 2>&1 | tail -1 >> gpurun_out/r2_t39.jsonl
timeout 900 python -m pytest tests/test_gpu_bench.py -q --timeout 900 -p no:cacheprovider > gpurun_out/r2_t39.log 2>&1; echo rc=$? >> gpurun_out/r2_t39.log
