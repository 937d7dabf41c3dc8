# CSE scheme check: parity tests touching schemes, then CSE / PM bench lines.
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q -x --timeout 900 -p no:cacheprovider -k "div7 or configs_small or random_dfas or dense or edge" > gpurun_out/pytest_cse.log 2>&1
echo "pytest rc=$?" >> gpurun_out/pytest_cse.log
for c in c1 c2 c3 c4; do
  for s in cse pm; do
    timeout 600 python bench.py --config $c --scheme $s --steps 5 --warmup 3 --e2e-steps 0 --no-cpu-baseline > gpurun_out/bench_${s}_$c.log 2>&1
  done
done
