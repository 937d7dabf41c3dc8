# Iteration check: full GPU test suite, then c2/c3/c4 bench lines (no CPU baseline).
# Usage (from gpurun): bash tools/gpu_iter2.sh
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q -x --timeout 900 -p no:cacheprovider > gpurun_out/pytest_iter.log 2>&1
echo "pytest rc=$?" >> gpurun_out/pytest_iter.log
for c in c2 c3 c4; do
  timeout 600 python bench.py --config $c --steps 10 --warmup 3 --e2e-steps 0 --no-cpu-baseline > gpurun_out/bench_iter_$c.log 2>&1
done
