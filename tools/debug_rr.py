import sys, numpy as np, torch
sys.path.insert(0, '.')
import gen, oracle
import paper_conf_ipps_wangwqw22_b200 as gs
w = gen.workload('rand:218:242:4', length=176279, seed=4)
d = w.host()
x = torch.from_numpy(d).cuda()
refs = {B: oracle.run(w.table, w.start, w.accept, d, B) for B in (16, 48, 4096)}
def chk(tag, fsm, scheme, B):
    r = fsm.run(x, scheme=scheme, chunk_bytes=B)
    ref = refs[B]
    ce = r.chunk_ends.cpu().numpy().view(np.uint32)
    ok = r.final_state == ref['final'] and r.accept_count == ref['count'] and (ce == ref['chunk_end']).all()
    print(tag, scheme, B, 'OK' if ok else f'BAD count {r.accept_count} vs {ref["count"]}', r.stats['rounds'], r.stats['tasks_helper'], flush=True)
    return ok
f1 = gs.FSM.load(w.table, w.start, w.accept)
for i in range(3): chk('fresh', f1, 'rr', 16)
f2 = gs.FSM.load(w.table, w.start, w.accept)
for s in ['seq', 'pm', 'sre']:
    for B in (16, 48, 4096): chk('warm', f2, s, B)
for i in range(3): chk('reused', f2, 'rr', 16)
f3 = gs.FSM.load(w.table, w.start, w.accept)
chk('f3', f3, 'sre', 4096)
chk('f3', f3, 'rr', 16)
f4 = gs.FSM.load(w.table, w.start, w.accept)
chk('f4', f4, 'pm', 16)
chk('f4', f4, 'rr', 16)
f5 = gs.FSM.load(w.table, w.start, w.accept)
chk('f5', f5, 'rr', 48)
chk('f5', f5, 'rr', 16)
