"""Offline shared-memory bank-conflict model of the spec-exec lookup (no GPU).
Simulates warps of 32 lanes walking 32 consecutive chunks in lockstep over the
real C2 workload and counts wavefronts per warp-step for several table layouts."""
import sys
import numpy as np
sys.path.insert(0, '.')
import gen, oracle

w = gen.workload(sys.argv[1] if len(sys.argv) > 1 else 'c2', length=1 << 22)
data = w.host()
perm, inv, freq, tt, acc = oracle.transform(w.table, w.accept)
n = w.nstates
nt = n + 1
# u8 codes as in api.cpp: non-accepting tids -> 0.., accepting -> 128..
code = np.zeros(nt, np.int64)
na = ac = 0
for t in range(nt):
    if acc[t]:
        code[t] = 128 + ac; ac += 1
    else:
        code[t] = na; na += 1
B = 4096
nwarps = 32
T = np.zeros((nwarps, 32), np.int64)  # current tid per lane
# start each lane at the true state (speculation ~always right for c2)
r = oracle.run(w.table, w.start, w.accept, data, B)
ends = np.concatenate([[w.start], r['chunk_end']])
for wi in range(nwarps):
    for L in range(32):
        c = wi * 32 + L
        T[wi, L] = perm[ends[c]]
def wavefronts(addr_bytes):
    # addr_bytes: [32] byte addresses -> number of wavefronts (max distinct words per bank)
    words = addr_bytes // 4
    banks = words % 32
    wf = 0
    for b in np.unique(banks):
        wf = max(wf, len(np.unique(words[banks == b])))
    return wf
layouts = {
    'stride256': lambda cd, b, L: cd * 256 + b,
    'stride260': lambda cd, b, L: cd * 260 + b,
    'stride260+2rep': lambda cd, b, L: (L & 1) * 40000 + cd * 260 + b + (L & 1) * 64,
    'stride272': lambda cd, b, L: cd * 272 + b,
    'stride264': lambda cd, b, L: cd * 264 + b,
}
tot = {k: 0 for k in layouts}
tot['stride260_rootskip'] = 0
steps = 0
root = perm[w.start]
starts_lit = set(int(L[0]) for L in w.literals)
for i in range(0, 1024):
    for wi in range(nwarps):
        pos = np.array([(wi * 32 + L) * B + i for L in range(32)])
        b = data[pos].astype(np.int64)
        cd = code[T[wi]]
        for k, f in layouts.items():
            tot[k] += wavefronts(f(cd, b, np.arange(32)))
        act = ~((T[wi] == root) & np.array([x not in starts_lit for x in b]))
        if act.any():
            tot['stride260_rootskip'] += wavefronts((cd * 260 + b)[act])
        T[wi] = tt[T[wi], b]
        steps += 1
for k, v in tot.items():
    print(f'{k:24s} {v / steps:.3f} wavefronts/warp-step')
print('root fraction', np.mean(T == root))

# ---- bank-aware code assignment (greedy) ----
visits = np.zeros(nt)
hist = np.zeros((nt, 64))  # word-index histogram of the next byte per state
s = perm[w.start]
prof = data[:1 << 20]
for x in prof:
    visits[s] += 1
    hist[s, x >> 2] += 1
    s = tt[s, x]
order = np.argsort(-visits, kind='stable')
load = np.zeros(32)  # expected accesses per bank (weighted)
free_na = list(range(128)); free_a = list(range(128, 256))
code2 = np.zeros(nt, np.int64)
for t in order:
    pool = free_a if acc[t] else free_na
    best, bestv = None, None
    hw = hist[t] / max(1, hist[t].sum()) * visits[t]
    for cd in pool:
        sh = cd % 32  # rotation of row cd with stride 260 is cd*65 mod 32 = cd mod 32
        banks = (np.arange(64) + sh) % 32
        cost = np.sum(hw * load[banks])
        if bestv is None or cost < bestv - 1e-12:
            best, bestv = cd, cost
    pool.remove(best)
    code2[t] = best
    banks = (np.arange(64) + best % 32) % 32
    np.add.at(load, banks, hw)
T2 = np.zeros((nwarps, 32), np.int64)
for wi in range(nwarps):
    for L in range(32):
        T2[wi, L] = perm[ends[wi * 32 + L]]
tot2 = 0; steps2 = 0
for i in range(0, 1024):
    for wi in range(nwarps):
        pos = np.array([(wi * 32 + L) * B + i for L in range(32)])
        b = data[pos].astype(np.int64)
        tot2 += wavefronts(code2[T2[wi]] * 260 + b)
        T2[wi] = tt[T2[wi], b]
        steps2 += 1
print(f'{"stride260+bankaware":24s} {tot2 / steps2:.3f} wavefronts/warp-step')
