"""Offline bank-conflict model of the u16d (C4) row lookup (no GPU): warps of 32 lanes walk
32 consecutive chunks in lockstep over the real C4 workload; counts wavefronts per warp-step of
the hot-row LDS.U16 for the library's row order (slot = tid) and for a bank-aware order (each
hot tid, in visit order, takes the free slot whose bank offset (21 * slot mod 32 for 42
classes) minimises the expected collisions with the rows placed before it)."""
import sys
import numpy as np
sys.path.insert(0, '.')
import gen, oracle

name = sys.argv[1] if len(sys.argv) > 1 else 'c4'
NW = int(sys.argv[2]) if len(sys.argv) > 2 else 48
STEPS = int(sys.argv[3]) if len(sys.argv) > 3 else 1024
H = int(sys.argv[4]) if len(sys.argv) > 4 else 457
B = 4096
w = gen.workload(name, length=NW * 32 * B)
data = w.host()
table = np.asarray(w.table, np.uint32)
n, ns = table.shape
perm, inv, freq, tt, acc = oracle.transform(w.table, w.accept)
# byte classes as api.cpp: identical columns, first-occurrence order (+ poison class if nsyms < 256)
cols = {}
cls = np.zeros(256, np.int64)
for b in range(ns):
    key = table[:, b].tobytes()
    cls[b] = cols.setdefault(key, len(cols))
C = len(cols) + (1 if ns < 256 else 0)
cls[ns:] = len(cols)
print("n", n, "C", C, "H", H)
r = oracle.run(w.table, w.start, w.accept, data, B)
ends = np.concatenate([[w.start], r['chunk_end']])
T0 = perm[ends[:NW * 32]].reshape(NW, 32).astype(np.int64)
ttc = np.zeros((n + 1, C), np.int64)  # transformed tid x class (tt is [tid][byte])
for b in range(ns):
    ttc[:, cls[b]] = np.append(tt[:, b], n)[: n + 1] if tt.shape[0] == n else tt[:, b]
ttc[n, :] = n

# first pass: visit counts and per-tid word histograms (word index within the row = cl // 2)
T = T0.copy()
visits = np.zeros(n + 1)
hist = np.zeros((n + 1, 32))
trace = []
for i in range(STEPS):
    pos = (np.arange(NW * 32).reshape(NW, 32)) * B + i
    cl = cls[data[pos]]
    trace.append((T.copy(), cl.copy()))
    np.add.at(visits, T.ravel(), 1)
    np.add.at(hist, (T.ravel(), (cl.ravel() // 2) % 32), 1)
    T = ttc[T, cl]

def wavefronts(words):
    """per warp: max over banks of distinct words"""
    tot = 0
    for row in words:
        banks = row % 32
        m = 0
        for b in np.unique(banks):
            m = max(m, len(np.unique(row[banks == b])))
        tot += m
    return tot

def measure(slot):
    tot, hot_steps, lanes_cold = 0, 0, 0
    for T, cl in trace:
        hot = T < H
        lanes_cold += (~hot).sum()
        words = np.where(hot, slot[np.minimum(T, H)] * (C // 2) + cl // 2, -1 - np.arange(32)[None, :] * 1000)
        # cold lanes: excluded (their base-row read is a separate, predicated path in this model)
        tot += sum(wavefronts(wr[None, hot_r]) if hot_r.any() else 0 for wr, hot_r in zip(words, hot))
        hot_steps += len(T)
    return tot / hot_steps, lanes_cold / (hot_steps * 32)

ident = np.arange(H + 1)
wf0, cold = measure(ident)
print(f"identity order: {wf0:.3f} hot-row wavefronts / warp-step (cold lane-steps {cold:.3%})")
# bank-aware: tids in visit order; offset of slot s = (s * C/2) mod 32 (C even)
assert C % 2 == 0
order = np.argsort(-visits[:H], kind="stable")
free = list(range(H))
load = np.zeros(32)
slot = np.zeros(H + 1, np.int64)
slot[H] = H
off = lambda s: (s * (C // 2)) % 32
for t in order:
    h = hist[t] / max(1, hist[t].sum()) * visits[t]
    best, bs = None, None
    seen = set()
    for s in free:
        o = off(s)
        if o in seen:
            continue
        seen.add(o)
        cost = float((h * load[(o + np.arange(32)) % 32]).sum())
        if best is None or cost < best:
            best, bs = cost, s
    free.remove(bs)
    slot[t] = bs
    load[(off(bs) + np.arange(32)) % 32] += h
wf1, _ = measure(slot)
print(f"bank-aware order: {wf1:.3f} hot-row wavefronts / warp-step")
