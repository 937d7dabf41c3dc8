# C3 recovery profile: ncu launch list of two C3 runs (per-kernel durations of the
# dense task rounds), plus the run timeline.  Usage (from gpurun): bash tools/gpu_c3prof.sh
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches_c3.csv python tools/profile_spec.py c3 sre 2 > gpurun_out/ncu_launch_c3.log 2>&1
GSPEC_STAMPS=1 timeout 600 python tools/timeline.py c3 > gpurun_out/timeline_c3.log 2>&1
