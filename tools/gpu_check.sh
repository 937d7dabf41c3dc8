cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q -x --timeout 600 -p no:cacheprovider > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 600 python bench.py --steps 20 --warmup 3 > gpurun_out/bench.log 2>&1
timeout 600 python bench.py --config c3 --scheme sre --steps 3 --warmup 3 --e2e-steps 0 --no-cpu-baseline > gpurun_out/bench_c3_sre.log 2>&1
