cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -q --timeout 600 -p no:cacheprovider -k "pm_tree or literal" > gpurun_out/r2_pm.log 2>&1; echo "rc=$?" >> gpurun_out/r2_pm.log
timeout 600 python tools/literal_vs_pipeline.py > gpurun_out/r2_lit_vs_pipe.log 2>&1
for c in c2 c4; do timeout 600 python bench.py --config $c --scheme pm_tree --steps 5 --warmup 3 --e2e-steps 0 --no-cpu-baseline --no-per-dfa > gpurun_out/r2_pmtree_$c.log 2>&1; done
