"""Spec-kernel time vs SM clock under sustained load (c2, 1 GiB): long queued
run with nvidia-smi sampled every 50 ms, plus isolated runs.
usage: python tools/clock_probe.py [steps]"""
import subprocess
import sys
import time

sys.path.insert(0, '.')
import numpy as np
import torch

import gen
import paper_conf_ipps_wangwqw22_b200 as gs

steps = int(sys.argv[1]) if len(sys.argv) > 1 else 3000
w = gen.workload('c2')
x = torch.empty(w.length, dtype=torch.uint8, device='cuda')
w.device(x)
prof = torch.empty(1 << 20, dtype=torch.uint8, device='cuda')
w.device(prof, offset=w.length)
fsm = gs.FSM.load(w.table, w.start, w.accept, profile=prof.cpu().numpy())
ce = torch.empty(gs.fsm_num_chunks(w.length, 4096), dtype=torch.int32, device='cuda')
iso, fl = [], []
junk = torch.empty(512 << 20, dtype=torch.uint8, device='cuda')
for _ in range(30):
    r = fsm.run(x, scheme='sre', chunk_ends=True)
    iso.append(r.stats['ms_spec'])
    junk.fill_(1)  # L2 flush (512 MiB write) before the next run
    torch.cuda.synchronize()
    r = fsm.run(x, scheme='sre', chunk_ends=True)
    fl.append(r.stats['ms_spec'])
    time.sleep(0.01)
print('isolated runs: ms_spec median %.4f min %.4f' % (np.median(iso), min(iso)))
print('after an L2 flush: ms_spec median %.4f min %.4f' % (np.median(fl), min(fl)))
del junk
smi = subprocess.Popen(['nvidia-smi', '--query-gpu=timestamp,clocks.sm,power.draw,clocks_event_reasons.active',
                        '--format=csv,noheader', '-lms', '50'], stdout=subprocess.PIPE, text=True)
time.sleep(0.3)
torch.cuda.synchronize()
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
e0.record()
pend, res = [], []
for _ in range(steps):
    pend.append(fsm.run_async(x, scheme='sre', chunk_ends=ce))
    if len(pend) >= 16:
        res.append(fsm.wait(pend.pop(0)))
e1.record()
torch.cuda.synchronize()
res += [fsm.wait(t) for t in pend]
time.sleep(0.2)
smi.terminate()
out = smi.communicate()[0]
sp = np.array([r.stats['ms_spec'] for r in res])
ve = np.array([r.stats['ms_verify'] for r in res])
print('queued %d steps: %.4f ms/step' % (steps, e0.elapsed_time(e1) / steps))
for lo, hi in ((0, 100), (100, 1000), (steps - 500, steps)):
    print('  steps %5d-%5d: spec median %.4f  verify median %.4f' % (lo, hi, np.median(sp[lo:hi]), np.median(ve[lo:hi])))
print('nvidia-smi samples:')
print(out)
