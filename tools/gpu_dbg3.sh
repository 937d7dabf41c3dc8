cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
GSPEC_DEBUG_ERR=1 CUDA_LAUNCH_BLOCKING=1 timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -p no:cacheprovider -k "test_lookback_long" > gpurun_out/r2_dbg3.log 2>&1
