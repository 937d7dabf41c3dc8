cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_shard.py tests/test_gpu_dist.py -q --timeout 900 -p no:cacheprovider -k "enum or c1 or div7 or random_dfas or multi_rank" > gpurun_out/r2_t24.log 2>&1; echo "rc=$?" >> gpurun_out/r2_t24.log
for t in 1 0; do GSPEC_ENUM_TMA=$t timeout 900 python bench.py --config c5 --c5-dfa c1 --steps 5 --warmup 3 2>&1 | tail -1 > gpurun_out/r2_t24_c5c1_tma$t.log; done
cat > /tmp/enum_prof.py <<'PY'
import sys; sys.path.insert(0, ".")
import torch, gen
import paper_conf_ipps_wangwqw22_b200 as gs
L = 2 << 30
w = gen.workload("c1", length=L)
x = torch.empty(L, dtype=torch.uint8, device="cuda"); w.device(x)
fsm = gs.FSM.load(w.table, w.start, w.accept)
for i in range(3):
    r = fsm.run(x, scheme="enum", chunk_bytes=4096)
torch.cuda.synchronize(); print(r.final_state, r.accept_count)
PY
timeout 900 ncu --set full --clock-control none --kernel-name-base mangled -k regex:k_spec_tmaILi1ELi8ELi3ELb0ELb0ELi2E -s 1 -c 1 -o /tmp/enum_tma -f python /tmp/enum_prof.py > gpurun_out/r2_t24_ncu.log 2>&1
if [ -f /tmp/enum_tma.ncu-rep ]; then ncu -i /tmp/enum_tma.ncu-rep --page raw --csv > gpurun_out/r2_t24_enum_tma_raw.csv 2>&1; fi
