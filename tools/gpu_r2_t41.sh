cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
for k in 10 50; do timeout 600 python bench.py --steps $k --warmup 3 --e2e-steps 0 --no-cpu-baseline --no-per-dfa 2>&1 | tail -1 >> gpurun_out/r2_t41.jsonl; done
timeout 600 python bench.py --config c4 --steps 10 --warmup 3 --e2e-steps 0 --no-cpu-baseline --no-per-dfa 2>&1 | tail -1 >> gpurun_out/r2_t41.jsonl
