# Device-driven dense rounds: full GPU suite, C2/C3/C3s/C4 bench lines, memcheck of the dense tests.
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q -x --timeout 900 -p no:cacheprovider > gpurun_out/pytest_dense.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_dense.log
for c in c2 c3 c3s c4; do timeout 300 python bench.py --config $c --steps 10 --warmup 3 --e2e-steps 0 --no-cpu-baseline > gpurun_out/bench_dense_$c.log 2>&1; done
timeout 900 /usr/local/cuda/bin/compute-sanitizer --tool memcheck python -m pytest tests/test_gpu_parity.py -q -x -p no:cacheprovider -k "dense or chained" > gpurun_out/memcheck_dense.log 2>&1; echo "memcheck rc=$?" >> gpurun_out/memcheck_dense.log
