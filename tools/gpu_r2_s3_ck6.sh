cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
CK_PROFILE_LAST=1 timeout 600 ncu --profile-from-start off --metrics gpu__time_duration.sum,smsp__inst_executed.sum,smsp__warps_launched.sum --clock-control none --csv --log-file gpurun_out/ck6_launches.csv python tools/ck_probe.py c3 sre 3 > gpurun_out/ck6_ncu.log 2>&1
echo pdl > gpurun_out/ck6_probe.log; GSPEC_PDL=1 timeout 300 python tools/ck_probe.py c3 sre 4 >> gpurun_out/ck6_probe.log 2>&1
