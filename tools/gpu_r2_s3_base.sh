# Session-3 baseline after the container restore: GPU tests, smoke, default bench line.
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 2400 python -m pytest tests -m gpu -q --timeout 1500 -p no:cacheprovider --durations=15 > gpurun_out/s3_pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/s3_pytest_gpu.log
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/s3_smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/s3_smoke.log
timeout 1200 python bench.py > gpurun_out/s3_bench_default.log 2>&1
timeout 900 python bench.py --config c4 --steps 10 --warmup 3 --e2e-steps 0 --no-cpu-baseline --no-per-dfa > gpurun_out/s3_bench_c4.log 2>&1
