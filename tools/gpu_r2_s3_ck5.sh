cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
: > gpurun_out/ck5_probe.log
for sg in def 1024 4096 512; do echo "seg $sg" >> gpurun_out/ck5_probe.log; if [ $sg = def ]; then timeout 300 python tools/ck_probe.py c3 sre 4 >> gpurun_out/ck5_probe.log 2>&1; else GSPEC_CK_SEG=$sg timeout 300 python tools/ck_probe.py c3 sre 4 >> gpurun_out/ck5_probe.log 2>&1; fi; done
echo "ck 256 seg 1024" >> gpurun_out/ck5_probe.log; GSPEC_CK=256 GSPEC_CK_SEG=1024 timeout 300 python tools/ck_probe.py c3 sre 4 >> gpurun_out/ck5_probe.log 2>&1
for s in rr nf; do echo "c3 $s" >> gpurun_out/ck5_probe.log; timeout 300 python tools/ck_probe.py c3 $s 4 >> gpurun_out/ck5_probe.log 2>&1; done
echo "c3s" >> gpurun_out/ck5_probe.log; timeout 300 python tools/ck_probe.py c3s sre 4 >> gpurun_out/ck5_probe.log 2>&1
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_records.py -m gpu -q --timeout 900 -p no:cacheprovider \
  -k "checkpointed or dense or memoized or vr_others or records or configs_small or full_size_other" > gpurun_out/ck5_pytest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/ck5_pytest.log
