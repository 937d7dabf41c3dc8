# Bench line of every BASELINE config (c1..c4, + the input-sensitive c3s) on one GPU.
# Usage (from gpurun): bash tools/gpu_configs.sh
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
for c in c1 c2 c3 c3s c4; do
  timeout 900 python bench.py --config $c --steps 10 --warmup 3 --e2e-steps 1 > gpurun_out/bench_$c.log 2>&1
done
for s in sre rr nf pm; do
  timeout 900 python bench.py --config c3 --scheme $s --steps 5 --warmup 3 --e2e-steps 0 --no-cpu-baseline > gpurun_out/bench_c3_$s.log 2>&1
done
