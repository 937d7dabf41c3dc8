cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
: > gpurun_out/nc_probe.log
echo "nc2 default" >> gpurun_out/nc_probe.log; timeout 300 python tools/ck_probe.py c3 sre 4 >> gpurun_out/nc_probe.log 2>&1
echo "nc1" >> gpurun_out/nc_probe.log; GSPEC_CK_NC=1 timeout 300 python tools/ck_probe.py c3 sre 4 >> gpurun_out/nc_probe.log 2>&1
for sg in 1024 4096; do echo "nc2 seg $sg" >> gpurun_out/nc_probe.log; GSPEC_CK_SEG=$sg timeout 300 python tools/ck_probe.py c3 sre 4 >> gpurun_out/nc_probe.log 2>&1; done
echo "c3s" >> gpurun_out/nc_probe.log; timeout 300 python tools/ck_probe.py c3s sre 4 >> gpurun_out/nc_probe.log 2>&1
for s in rr nf; do echo "c3 $s" >> gpurun_out/nc_probe.log; timeout 300 python tools/ck_probe.py c3 $s 4 >> gpurun_out/nc_probe.log 2>&1; done
CK_PROFILE_LAST=1 timeout 600 ncu --profile-from-start off --metrics gpu__time_duration.sum,smsp__inst_executed.sum --clock-control none --csv --log-file gpurun_out/nc_launches_c3.csv python tools/ck_probe.py c3 sre 3 > gpurun_out/nc_ncu.log 2>&1
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_records.py -m gpu -q --timeout 900 -p no:cacheprovider -x -k "checkpointed or dense or memoized or vr_others or records or configs_small or full_size_other" > gpurun_out/nc_pytest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/nc_pytest.log
