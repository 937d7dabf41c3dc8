cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
cat > /tmp/enum_prof.py <<'PY'
import sys; sys.path.insert(0, '.')
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
timeout 900 ncu --set full --clock-control none --import-source on --kernel-name-base mangled -k regex:k_spec_tmaILi1ELi8ELi3ELb0ELb0ELi2E -s 1 -c 1 -o /tmp/enum_tma -f python /tmp/enum_prof.py > gpurun_out/r2_t23_ncu.log 2>&1
GSPEC_ENUM_TMA=0 timeout 900 ncu --set full --clock-control none --import-source on --kernel-name-base mangled -k regex:k_enum_walkILi1ELi8ELi32ELb1E -s 1 -c 1 -o /tmp/enum_k1 -f python /tmp/enum_prof.py > gpurun_out/r2_t23_ncu_k1.log 2>&1
for r in enum_tma enum_k1; do
  if [ -f /tmp/$r.ncu-rep ]; then ncu -i /tmp/$r.ncu-rep --page raw --csv > gpurun_out/r2_t23_${r}_raw.csv 2>&1; ncu -i /tmp/$r.ncu-rep --page details --csv > gpurun_out/r2_t23_${r}_details.csv 2>&1; fi
done
