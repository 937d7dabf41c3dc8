cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 300 python tools/clock_probe.py 3000 > gpurun_out/clock_probe.log 2>&1
