cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 600 compute-sanitizer --tool memcheck --show-backtrace host python tools/dbg_lookback2.py > gpurun_out/r2_dbg5.log 2>&1
