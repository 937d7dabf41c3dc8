cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
for e in 0 2; do GSPEC_TMA_EVICT=$e timeout 900 python bench.py --config c5 --c5-dfa c1 --steps 5 --warmup 3 2>&1 | tail -1 > gpurun_out/r2_t25_c5c1_e$e.log; done
GSPEC_ENUM_TMA=0 timeout 900 python bench.py --config c5 --c5-dfa c1 --steps 5 --warmup 3 2>&1 | tail -1 > gpurun_out/r2_t25_c5c1_k1.log
