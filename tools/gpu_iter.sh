# Iteration check: GPU tests, then c2 bench (with and without the run timeline) and c3 auto.
# Usage (from gpurun): bash tools/gpu_iter.sh [pytest -k expr]
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
K=${1:-}
if [ -n "$K" ]; then
  timeout 1500 python -m pytest tests -m gpu -q -x --timeout 900 -p no:cacheprovider -k "$K" > gpurun_out/pytest_iter.log 2>&1
else
  timeout 1500 python -m pytest tests -m gpu -q -x --timeout 900 -p no:cacheprovider > gpurun_out/pytest_iter.log 2>&1
fi
echo "pytest rc=$?" >> gpurun_out/pytest_iter.log
timeout 600 python bench.py --steps 20 --warmup 3 --e2e-steps 0 --no-cpu-baseline > gpurun_out/bench_iter_c2.log 2>&1
GSPEC_STAMPS=1 timeout 600 python tools/timeline.py c2 > gpurun_out/timeline_c2.log 2>&1
timeout 600 python bench.py --config c3 --steps 5 --warmup 3 --e2e-steps 0 --no-cpu-baseline > gpurun_out/bench_iter_c3.log 2>&1
