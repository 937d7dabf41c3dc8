"""Offline shared-memory bank model of the classed (u16) lookup (no GPU).
Warps of 32 lanes walk 32 consecutive chunks in lockstep over a config's input;
per warp-step it counts wavefronts (max over banks of distinct 4-byte words) of
the row lookup for several hot-table layouts:
  row     T[t][cl] at (t*C + cl)*2                      (current)
  rowpad  rows padded to an odd number of words
  col     T[cl][t] at (cl*Hp + t)*2, Hp = H rounded so Hp/2 is odd (class-major)
and of the u16d branchy variant (hot lanes: row lookup; cold lanes: descriptor +
base row).  usage: python tools/bank_sim_u16.py c4 [H]"""
import sys

import numpy as np

sys.path.insert(0, '.')
import gen  # noqa: E402
import oracle  # noqa: E402

name = sys.argv[1] if len(sys.argv) > 1 else 'c4'
H = int(sys.argv[2]) if len(sys.argv) > 2 else 512
w = gen.workload(name, length=1 << 23)
data = w.host()
perm, inv, freq, tt, acc = oracle.transform(w.table, w.accept)
n = w.nstates
nt = n + 1
# byte classes (identical columns) of the transformed table
cols = {}
cls = np.zeros(256, np.int64)
for b in range(256):
    k = tt[:, b].tobytes()
    cls[b] = cols.setdefault(k, len(cols))
C = len(cols)
B = 4096
nw = 48
r = oracle.run(w.table, w.start, w.accept, data, B)
ends = np.concatenate([[w.start], r['chunk_end']])
st = np.array([[perm[ends[wi * 32 + L]] for L in range(32)] for wi in range(nw)], np.int64)
steps = 1024
byts = np.stack([[data[(wi * 32 + L) * B:(wi * 32 + L) * B + steps] for L in range(32)] for wi in range(nw)])
Hp = H + (2 - (H // 2) % 2) * 2 if (H // 2) % 2 == 0 else H
rw = (C * 2 + 3) // 4
padw = rw if rw % 2 == 1 else rw + 1


def wf(words):
    banks = words % 32
    m = 0
    for b in np.unique(banks):
        m = max(m, len(np.unique(words[banks == b])))
    return m


# greedy bank-aware row placement (the u8 placement of fsm_load, on class words):
# states by profile visits; each takes the free row slot whose bank rotation
# (slot * padw mod 32) puts its word histogram on the least-loaded banks
prof = data[: 1 << 20]
visits = np.zeros(nt)
hist = np.zeros((nt, padw))
t0 = perm[w.start]
pcl = cls[prof]
tcur = t0
for i in range(len(prof)):
    visits[tcur] += 1
    hist[tcur, pcl[i] // 2] += 1
    tcur = tt[tcur, prof[i]]
slot_of = np.zeros(nt, np.int64)
nslots = ((nt + 31) // 32 + 1) * 32
free = np.ones(nslots, bool)
load = np.zeros(32)
for q in np.argsort(-visits, kind='stable'):
    if visits[q] == 0:
        r = int(np.nonzero(free)[0][0])
    else:
        best, bc = -1, 0
        for rot in range(32):
            cand = np.nonzero(free[rot::32])[0]
            if len(cand) == 0:
                continue
            r0 = rot + 32 * int(cand[0])
            cost = sum(hist[q, wd] * load[(wd + r0 * padw) % 32] for wd in range(padw))
            if best < 0 or cost < bc:
                best, bc = r0, cost
        r = best
    free[r] = False
    slot_of[q] = r
    for wd in range(padw):
        load[(wd + r * padw) % 32] += hist[q, wd]

res = {k: 0 for k in ("row", "rowpad", "col", "greedy", "cold_lanes", "any_cold")}
for s in range(steps):
    cl = cls[byts[:, :, s]]
    for wi in range(nw):
        t = st[wi]
        c = cl[wi]
        hot = t < H
        th = np.where(hot, t, 0)
        res["row"] += wf(((th * C + c) * 2) // 4)
        res["rowpad"] += wf(th * padw + (c * 2) // 4)
        res["col"] += wf(((c * Hp + th) * 2) // 4)
        res["greedy"] += wf(slot_of[t] * padw + (c * 2) // 4)
        res["cold_lanes"] += (~hot).sum()
        res["any_cold"] += (~hot).any()
    st = tt[st, byts[:, :, s]]
N = steps * nw
print(f"{name}: n={n} C={C} H={H} Hp={Hp} row words={rw} padded={padw}")
for k, v in res.items():
    print(f"  {k:10s} {v / N:.3f} per warp-step")
