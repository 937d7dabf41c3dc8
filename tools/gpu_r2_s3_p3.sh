cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
CK_PROFILE_LAST=1 timeout 600 ncu --profile-from-start off --set full --clock-control none --import-source on -k regex:k_task_seg -s 3 -c 1 -o /tmp/p3_seg -f python tools/ck_probe.py c3 sre 3 > gpurun_out/p3_ncu.log 2>&1
ncu -i /tmp/p3_seg.ncu-rep --page raw --csv > gpurun_out/p3_seg_raw.csv 2>&1
ncu -i /tmp/p3_seg.ncu-rep --page source --csv > gpurun_out/p3_seg_source.csv 2>&1
ncu -i /tmp/p3_seg.ncu-rep --page details --csv > gpurun_out/p3_seg_details.csv 2>&1
