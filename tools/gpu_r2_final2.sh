# Round-2 final check 2 (after the K-symbol ENUM tables and the bench in-flight window).
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 2400 python -m pytest tests -m gpu -q --timeout 1500 -p no:cacheprovider --durations=10 > gpurun_out/g_pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/g_pytest_gpu.log
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/g_smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/g_smoke.log
timeout 1200 python bench.py > gpurun_out/g_bench_default.log 2>&1
timeout 1200 python bench.py --impl reference --steps 2 --warmup 1 > gpurun_out/g_bench_reference.log 2>&1
