cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
for c in "" max; do
  GSPEC_CARVEOUT=$c GSPEC_STAMPS=1 python tools/timeline.py c2 > gpurun_out/r2_t36_tl_$c.log 2>&1
  for i in 1 2; do GSPEC_CARVEOUT=$c timeout 600 python bench.py --steps 50 --warmup 5 --e2e-steps 0 --no-cpu-baseline --no-per-dfa 2>&1 | tail -1 >> gpurun_out/r2_t36_c2_$c.jsonl; done
  GSPEC_CARVEOUT=$c timeout 600 python bench.py --config c4 --steps 10 --warmup 3 --e2e-steps 0 --no-cpu-baseline --no-per-dfa 2>&1 | tail -1 >> gpurun_out/r2_t36_c2_$c.jsonl
  GSPEC_CARVEOUT=$c timeout 600 python bench.py --config c3 --steps 10 --warmup 3 --e2e-steps 0 --no-cpu-baseline --no-per-dfa 2>&1 | tail -1 >> gpurun_out/r2_t36_c2_$c.jsonl
done
