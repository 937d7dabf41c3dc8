# Last check of the session's final tree: full GPU tests, smoke, default bench line
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 2400 python -m pytest tests -m gpu -q --timeout 1500 -p no:cacheprovider > gpurun_out/last_pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/last_pytest_gpu.log
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/last_smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/last_smoke.log
timeout 1200 python bench.py > gpurun_out/last_bench_default.log 2>&1
