cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 300 python tools/ck_probe.py c3 sre 4 > gpurun_out/ck2_probe.log 2>&1
GSPEC_CK=0 timeout 300 python tools/ck_probe.py c3 sre 4 >> gpurun_out/ck2_probe.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_task_ck -s 1 -c 1 -o /tmp/ck_task -f python tools/ck_probe.py c3 sre 3 > gpurun_out/ck2_ncu.log 2>&1
ncu -i /tmp/ck_task.ncu-rep --page raw --csv > gpurun_out/ck2_task_raw.csv 2>&1
ncu -i /tmp/ck_task.ncu-rep --page details --csv > gpurun_out/ck2_task_details.csv 2>&1
ncu -i /tmp/ck_task.ncu-rep --page source --csv > gpurun_out/ck2_task_source.csv 2>&1
