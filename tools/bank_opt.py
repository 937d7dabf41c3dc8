"""Local-search row placement for the u8 table (model only, no GPU).
Warps of 32 lanes walk 32 consecutive chunks of a profile trace in lockstep;
lane L reads byte b of row code(state): word = code*65 + b//4 (260-B rows),
bank = (code + b//4) mod 32.  Wavefronts per warp-step = max over banks of the
distinct words.  Compares the rank-order codes, the greedy bank-aware placement
of fsm_load, and a local search over the residues (code mod 32) of the hottest
states.  usage: python tools/bank_opt.py [c2] [MiB]"""
import sys
import time

import numpy as np

sys.path.insert(0, '.')
import gen  # noqa: E402
import oracle  # noqa: E402

name = sys.argv[1] if len(sys.argv) > 1 else 'c2'
mib = int(sys.argv[2]) if len(sys.argv) > 2 else 2
w = gen.workload(name, length=(mib << 20) * 2)
data = w.host()
perm, inv, freq, tt, acc = oracle.transform(w.table, w.accept)
nt = w.nstates + 1
B = 4096
prof = data[: mib << 20]            # training trace (profile)
test = data[mib << 20:]             # held-out trace (evaluation)


def warpsteps(d, steps=4096):
    N = len(d) // B
    nw = N // 32
    r = oracle.run(w.table, w.start, w.accept, d, B)
    ends = np.concatenate([[w.start], r['chunk_end']])
    S = np.zeros((nw * steps, 32), np.int64)
    W = np.zeros((nw * steps, 32), np.int64)
    for wi in range(nw):
        st = np.array([perm[ends[wi * 32 + L]] for L in range(32)])
        for i in range(steps):
            b = d[(wi * 32 + np.arange(32)) * B + i].astype(np.int64)
            S[wi * steps + i] = st
            W[wi * steps + i] = b >> 2
            st = tt[st, b]
    return S, W


def wavefronts(S, W, res):
    pid = S * 64 + W
    srt = np.sort(pid, axis=1)
    first = np.ones_like(srt, bool)
    first[:, 1:] = srt[:, 1:] != srt[:, :-1]
    s_u = srt // 64
    w_u = srt % 64
    bank = (res[s_u] + w_u) % 32
    cnt = np.zeros((S.shape[0], 32), np.int32)
    rows = np.repeat(np.arange(S.shape[0]), 32).reshape(S.shape)
    np.add.at(cnt, (rows[first], bank[first]), 1)
    return cnt.max(axis=1).mean()


t0 = time.time()
Sp, Wp = warpsteps(prof)
St, Wt = warpsteps(test)
print(f"{name}: {Sp.shape[0]} profile warp-steps, {St.shape[0]} test warp-steps ({time.time() - t0:.1f}s)")
# rank-order codes: non-accepting 0.., accepting 128..
code = np.zeros(nt, np.int64)
na = ac = 0
for t in range(nt):
    if acc[t]:
        code[t] = 128 + ac; ac += 1
    else:
        code[t] = na; na += 1
print("rank order  ", round(wavefronts(St, Wt, code % 32), 3))
# local search over residues with capacity: each residue hosts <= 4 non-accepting and <= 4 accepting rows
res = code % 32
visits = np.bincount(Sp.ravel(), minlength=nt)
hot = np.argsort(-visits)[:40]
cap = {0: np.zeros(32, int), 1: np.zeros(32, int)}
for t in range(nt):
    cap[int(acc[t])][res[t]] += 1
best = wavefronts(Sp, Wp, res)
for sweep in range(3):
    improved = False
    for t in hot:
        if visits[t] == 0:
            continue
        a = int(acc[t])
        cur = res[t]
        for r in range(32):
            if r == cur or cap[a][r] >= 4:
                continue
            res[t] = r
            v = wavefronts(Sp, Wp, res)
            if v < best - 1e-6:
                cap[a][cur] -= 1; cap[a][r] += 1
                best, cur, improved = v, r, True
            else:
                res[t] = cur
    print(f"sweep {sweep}: profile {best:.3f}  held-out {wavefronts(St, Wt, res):.3f}  ({time.time() - t0:.0f}s)")
    if not improved:
        break
