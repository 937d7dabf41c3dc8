cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
CUDA_LAUNCH_BLOCKING=1 timeout 300 python tools/dbg_lookback.py > gpurun_out/r2_dbg.log 2>&1
timeout 600 compute-sanitizer --tool memcheck python tools/dbg_lookback.py > gpurun_out/r2_dbg_memcheck.log 2>&1
