# compute-sanitizer over the GPU paths changed this session: the TMA-gather dense task
# rounds (C3 SRE/CSE), u16d pre-multiplied codes (C4), CSE path fusion (C2).
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
CS=/usr/local/cuda/bin/compute-sanitizer
timeout 1200 $CS --tool memcheck python -m pytest tests/test_gpu_parity.py -q -x -p no:cacheprovider -k "dense or (configs_small and (c4 or c2) and (sre or cse))" > gpurun_out/memcheck.log 2>&1; echo "memcheck rc=$?" >> gpurun_out/memcheck.log
cat > /tmp/rc.py <<'PY'
import sys; sys.path.insert(0, '.')
import torch, gen, numpy as np, oracle
import paper_conf_ipps_wangwqw22_b200 as gs
for name, n, scheme in (("c3", 32 << 20, "sre"), ("c3", 32 << 20, "cse"), ("c4", 8 << 20, "sre"), ("c2", 8 << 20, "cse")):
    w = gen.workload(name, length=n); h = w.host()
    fsm = gs.FSM.load(w.table, w.start, w.accept)
    r = fsm.run(torch.from_numpy(h).cuda(), scheme=scheme)
    ref = oracle.run(w.table, w.start, w.accept, h, 4096)
    print(name, scheme, r.final_state == ref["final"], r.accept_count == ref["count"], r.stats["rounds"], r.stats["tasks_total"])
PY
timeout 1800 $CS --tool racecheck python /tmp/rc.py > gpurun_out/racecheck.log 2>&1; echo "racecheck rc=$?" >> gpurun_out/racecheck.log
timeout 1800 $CS --tool synccheck python /tmp/rc.py > gpurun_out/synccheck.log 2>&1; echo "synccheck rc=$?" >> gpurun_out/synccheck.log
