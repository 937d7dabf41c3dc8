"""R30 probe: C3 1 GiB SRE with the recommended chunk, prints the dense-round counters
(task_walked_bytes vs reread_bytes) and the per-run times.  usage: python tools/ck_probe.py [cfg] [scheme] [reps]"""
import sys
sys.path.insert(0, '.')
import torch
import gen
import paper_conf_ipps_wangwqw22_b200 as gs
cfg = sys.argv[1] if len(sys.argv) > 1 else 'c3'
scheme = sys.argv[2] if len(sys.argv) > 2 else 'sre'
reps = int(sys.argv[3]) if len(sys.argv) > 3 else 3
w = gen.workload(cfg)
x = torch.empty(w.length, dtype=torch.uint8, device='cuda')
w.device(x)
fsm = gs.FSM.load(w.table, w.start, w.accept)
_, feats = fsm.select_scheme(x)
B = feats["chunk_bytes"]
import os
prof_last = os.environ.get("CK_PROFILE_LAST") == "1"  # ncu --profile-from-start off: capture only the last run
for i in range(reps):
    if prof_last and i == reps - 1:
        torch.cuda.synchronize()
        torch.cuda.cudart().cudaProfilerStart()
    s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    s.record()
    r = fsm.run(x, scheme=scheme, chunk_bytes=B)
    e.record()
    torch.cuda.synchronize()
    if prof_last and i == reps - 1:
        torch.cuda.cudart().cudaProfilerStop()
    st = r.stats
    print(f"B={B} ms={s.elapsed_time(e):.3f} spec={st['ms_spec']:.3f} verify={st['ms_verify']:.3f} tasks={st['tasks_total']} "
          f"reread={st['reread_bytes']} walked={st['task_walked_bytes']} ratio={st['task_walked_bytes'] / max(1, st['reread_bytes']):.3f} "
          f"launches={st['kernel_launches']}", flush=True)
