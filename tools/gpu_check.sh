cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "dense or configs_small" --timeout 600 -p no:cacheprovider > gpurun_out/pytest_dense.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_dense.log
timeout 1500 python -m pytest tests -m gpu -q --timeout 600 -p no:cacheprovider > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
for s in sre; do timeout 600 python bench.py --config c3 --scheme $s --steps 3 --warmup 3 --e2e-steps 0 --no-cpu-baseline > gpurun_out/bench_c3_$s.log 2>&1; done
timeout 600 python bench.py --steps 20 --warmup 3 > gpurun_out/bench.log 2>&1
GSPEC_DIST_BACKEND=gloo timeout 600 torchrun --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29611 bench.py --gpus 2 --steps 3 --warmup 3 --e2e-steps 2 > gpurun_out/bench_2rank.log 2>&1; echo "rc=$?" >> gpurun_out/bench_2rank.log
