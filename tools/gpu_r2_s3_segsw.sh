cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
: > gpurun_out/segsw.log
for sg in 1024 1536 3072 4096; do echo "seg $sg" >> gpurun_out/segsw.log; GSPEC_CK_SEG=$sg timeout 300 python tools/ck_probe.py c3 sre 4 >> gpurun_out/segsw.log 2>&1; done
echo "ck256" >> gpurun_out/segsw.log; GSPEC_CK=256 timeout 300 python tools/ck_probe.py c3 sre 4 >> gpurun_out/segsw.log 2>&1
echo "ck1024" >> gpurun_out/segsw.log; GSPEC_CK=1024 timeout 300 python tools/ck_probe.py c3 sre 4 >> gpurun_out/segsw.log 2>&1
