# Round 2 start: GPU tests, smoke, default bench line and every config's bench line.
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 2400 python -m pytest tests -m gpu -q --timeout 1200 -p no:cacheprovider > gpurun_out/r2_pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/r2_pytest_gpu.log
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r2_smoke.log 2>&1
timeout 900 python bench.py > gpurun_out/r2_bench_default.log 2>&1
for c in c1 c3 c3s c4; do
  timeout 900 python bench.py --config $c --steps 10 --warmup 3 --e2e-steps 1 --no-cpu-baseline > gpurun_out/r2_bench_$c.log 2>&1
done
for s in rr nf; do
  timeout 900 python bench.py --config c3 --scheme $s --steps 5 --warmup 3 --e2e-steps 0 --no-cpu-baseline > gpurun_out/r2_bench_c3_$s.log 2>&1
done
