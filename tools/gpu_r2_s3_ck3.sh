cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
CK_PROFILE_LAST=1 timeout 600 ncu --profile-from-start off --set full --clock-control none --import-source on -k regex:k_task_ck -c 1 -o /tmp/ck_task -f python tools/ck_probe.py c3 sre 3 > gpurun_out/ck3_ncu.log 2>&1
ncu -i /tmp/ck_task.ncu-rep --page raw --csv > gpurun_out/ck3_task_raw.csv 2>&1
ncu -i /tmp/ck_task.ncu-rep --page details --csv > gpurun_out/ck3_task_details.csv 2>&1
ncu -i /tmp/ck_task.ncu-rep --page source --csv > gpurun_out/ck3_task_source.csv 2>&1
