cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q --timeout 900 -p no:cacheprovider > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 600 python bench.py --steps 20 --warmup 3 > gpurun_out/bench.log 2>&1
timeout 600 python bench.py --config c3 --scheme sre --steps 3 --warmup 3 --e2e-steps 0 --no-cpu-baseline > gpurun_out/bench_c3_sre.log 2>&1
timeout 300 python tools/profile_spec.py c2 sre 5 > gpurun_out/phases_c2.log 2>&1
timeout 300 python tools/profile_spec.py c3 sre 3 > gpurun_out/phases_c3.log 2>&1
