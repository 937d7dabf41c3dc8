cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
for wp in 28 20 16 12 8; do echo "warps $wp" >> gpurun_out/ck4_probe.log; GSPEC_CK_WARPS=$wp timeout 300 python tools/ck_probe.py c3 sre 4 >> gpurun_out/ck4_probe.log 2>&1; done
echo "ck 256" >> gpurun_out/ck4_probe.log; GSPEC_CK=256 timeout 300 python tools/ck_probe.py c3 sre 4 >> gpurun_out/ck4_probe.log 2>&1
echo "c3s" >> gpurun_out/ck4_probe.log; timeout 300 python tools/ck_probe.py c3s sre 4 >> gpurun_out/ck4_probe.log 2>&1
CK_PROFILE_LAST=1 timeout 600 ncu --profile-from-start off --set full --clock-control none --import-source on -k regex:k_task_ck -c 1 -o /tmp/ck_task -f python tools/ck_probe.py c3 sre 3 > gpurun_out/ck4_ncu.log 2>&1
ncu -i /tmp/ck_task.ncu-rep --page raw --csv > gpurun_out/ck4_task_raw.csv 2>&1
ncu -i /tmp/ck_task.ncu-rep --page details --csv > gpurun_out/ck4_task_details.csv 2>&1
ncu -i /tmp/ck_task.ncu-rep --page source --csv > gpurun_out/ck4_task_source.csv 2>&1
