cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
CUDA_LAUNCH_BLOCKING=1 timeout 300 python tools/dbg_lookback2.py > gpurun_out/r2_dbg4.log 2>&1
