cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
GSPEC_DEBUG_ERR=1 timeout 1500 python -m pytest tests -m gpu -q --timeout 900 -p no:cacheprovider > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
for v in 1 0; do
GSPEC_PDL=$v timeout 600 python bench.py --steps 20 --warmup 3 --e2e-steps 0 --no-cpu-baseline > gpurun_out/bench_pdl$v.log 2>&1
done
