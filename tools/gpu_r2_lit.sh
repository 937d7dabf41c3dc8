cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -q --timeout 600 -p no:cacheprovider -k "literal" > gpurun_out/r2_lit.log 2>&1; echo "rc=$?" >> gpurun_out/r2_lit.log
timeout 600 python tools/literal_vs_pipeline.py > gpurun_out/r2_lit_vs_pipe.log 2>&1
