# Chained relaxation passes: full GPU suite, C1 PM/CSE bench lines, C2/C3 default lines, experiments.
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q -x --timeout 900 -p no:cacheprovider > gpurun_out/pytest_chain.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_chain.log
for s in cse pm rr nf; do timeout 300 python bench.py --config c1 --scheme $s --steps 5 --warmup 3 --e2e-steps 0 --no-cpu-baseline > gpurun_out/bench_chain_c1_$s.log 2>&1; done
for c in c2 c3 c4; do timeout 300 python bench.py --config $c --steps 10 --warmup 3 --e2e-steps 0 --no-cpu-baseline > gpurun_out/bench_chain_$c.log 2>&1; done
timeout 1200 python tools/experiments.py --mib 64 --out gpurun_out/r01_experiments.md > gpurun_out/experiments.log 2>&1
