"""Run the bench workload's fsm_run a few times (for ncu captures).
usage: python tools/profile_spec.py [config] [scheme] [reps] [chunk_bytes]"""
import sys
sys.path.insert(0, '.')
import torch
import gen
import paper_conf_ipps_wangwqw22_b200 as gs
cfg = sys.argv[1] if len(sys.argv) > 1 else 'c2'
scheme = sys.argv[2] if len(sys.argv) > 2 else 'sre'
reps = int(sys.argv[3]) if len(sys.argv) > 3 else 3
w = gen.workload(cfg)
x = torch.empty(w.length, dtype=torch.uint8, device='cuda')
w.device(x)
prof = torch.empty(1 << 20, dtype=torch.uint8, device='cuda')
w.device(prof, offset=w.length)  # disjoint training trace, as bench.py
fsm = gs.FSM.load(w.table, w.start, w.accept, profile=prof.cpu().numpy())
_, feats = fsm.select_scheme(x)  # as bench.py (spread profile, R20): dense-round slots, fused round 0
B = int(sys.argv[4]) if len(sys.argv) > 4 else feats["chunk_bytes"]  # as bench.py: the R29 recommendation
for i in range(reps):
    r = fsm.run(x, scheme=scheme, chunk_bytes=B)
torch.cuda.synchronize()
print(r.final_state, r.accept_count, r.stats['ms_spec'], r.stats['ms_verify'])
print("verify phase times (us):", [round(v, 1) for v in fsm.phase_times()])
