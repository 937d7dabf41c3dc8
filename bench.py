#!/usr/bin/env python3
"""Benchmark of the GSpecPal hot path on B200 (BASELINE.json metric).

One "step" = one fsm_run over the whole configured stream (every §8(a) step:
lookback speculation, speculative execution, verification/recovery rounds,
finalize) with the input already resident in HBM.  Default workload =
BASELINE.json configs[1] ("c2": ~100-state Snort-like Aho–Corasick DFA on a
1 GiB synthetic text stream), scheme chosen by the selector (untimed, like
the paper's offline profiling P:363).  The default single-GPU line also
carries per-DFA sub-results for C1, C3, C3s and C4 under "per_dfa".

  python bench.py [--gpus N] [--steps K] [--warmup W] [--config c2] [--scheme auto]
  python bench.py --config c5 [--gpus N]   # 16 GiB per DFA sharded over N GPUs (strong)
  python bench.py --impl reference ...     # the CPU oracle, timed on host cores

Multi-GPU (one process per GPU; `--gpus N` without torchrun re-launches itself
under torch.distributed.run): the stream is sharded contiguously; each rank
reduces its shard to a state map, ONE allgather (the library's own NCCL
communicator, fsm_run_sharded) exchanges the maps and every rank composes them
(DESIGN.md §Multi-GPU).  c1..c4 at N > 1: weak scaling (each rank owns the
config's length, N x the bytes in total); c5: strong scaling (16 GiB in total).
"""
from __future__ import annotations

import argparse
import json
import os
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

CONFIG_DESC = {
    "c1": "div7 (7-state binary DFA, paper Fig. 1) on a 1 MiB seeded random bit stream",
    "c2": "AC-111 Snort-like literal DFA (12 literals) on a 1 GiB synthetic text stream",
    "c3": "AC x Z16 counter DFA (816 states, low speculation accuracy) on a 1 GiB stream",
    "c3s": "AC x Z16 counter DFA, input-sensitive stream (1 GiB)",
    "c4": "AC-9912 DFA (520 literals, table exceeds smem) on a 4 GiB stream",
    "c5": "16 GiB stream of each of the C1-C4 DFAs sharded over N B200 (strong scaling), "
          "scheme chosen by the selector per DFA; NCCL allgather of state maps",
}
C5_LEN = 16 << 30
C5_DFAS = ("c2", "c1", "c3", "c4")  # c2 (the high-accuracy DFA) is the line's headline
METRIC = "input GB/s per DFA (1 GB stream, 1 B200); % of HBM roofline; latency per 1 GB"


def _peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return float(d.get("hbm_gbs", 6650.0)), "measured"
    return 6650.0, "fallback"


class ClockSampler:
    """SM clocks + throttle reasons sampled DURING the timed region: NVML every 0.5 ms (a
    short timed region still gets many samples), nvidia-smi every 100 ms as a fallback."""

    REASONS = {0x8: "hw_slowdown", 0x40: "hw_thermal_slowdown", 0x20: "sw_thermal_slowdown", 0x4: "sw_power_cap"}

    def __init__(self, index=0):
        self.index = index
        self.samples = []  # (sm_mhz, max_mhz, reason bitmask)
        self._stop = threading.Event()
        self._t = None
        self._nvml = None
        self._max_mhz = None
        try:
            import pynvml
            import torch

            pynvml.nvmlInit()
            pr = torch.cuda.get_device_properties(index)
            try:
                bus = f"{pr.pci_domain_id:08x}:{pr.pci_bus_id:02x}:{pr.pci_device_id:02x}.0"
                h = pynvml.nvmlDeviceGetHandleByPciBusId(bus)
            except Exception:
                h = pynvml.nvmlDeviceGetHandleByIndex(index)
            self._nvml = (pynvml, h)
            self._max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(h, pynvml.NVML_CLOCK_SM)  # before the timed region
        except Exception:
            self._nvml = None

    def _sample_nvml(self):
        nv, h = self._nvml
        sm = nv.nvmlDeviceGetClockInfo(h, nv.NVML_CLOCK_SM)
        if self._max_mhz is None:  # constant, and ~6 ms per call (the other two take microseconds)
            self._max_mhz = nv.nvmlDeviceGetMaxClockInfo(h, nv.NVML_CLOCK_SM)
        mx = self._max_mhz
        try:
            rs = nv.nvmlDeviceGetCurrentClocksEventReasons(h)
        except Exception:
            rs = nv.nvmlDeviceGetCurrentClocksThrottleReasons(h)
        return (float(sm), float(mx), int(rs))

    def _sample_smi(self):
        q = ("clocks.sm,clocks.max.sm,clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
             "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")
        out = subprocess.run(["nvidia-smi", "-i", str(self.index), f"--query-gpu={q}", "--format=csv,noheader,nounits"],
                             capture_output=True, text=True, timeout=5).stdout.strip()
        f = [x.strip() for x in out.split(",")]
        bits = [0x8, 0x40, 0x20, 0x4]
        return (float(f[0]), float(f[1]), sum(b for b, v in zip(bits, f[2:6]) if v.lower() == "active"))

    def _run(self):
        while not self._stop.is_set():
            try:
                self.samples.append(self._sample_nvml() if self._nvml else self._sample_smi())
            except Exception:
                pass
            self._stop.wait(0.0005 if self._nvml else 0.1)

    def __enter__(self):
        # a short GIL switch interval so the sampler thread gets its turns while the main
        # thread queues the timed steps (the GPU is ahead of the host: no effect on the timing)
        self._swi = sys.getswitchinterval()
        sys.setswitchinterval(2e-4)
        self._t = threading.Thread(target=self._run, daemon=True)
        self._t.start()
        return self

    def __exit__(self, *a):
        self._stop.set()
        if self._t:
            self._t.join(timeout=10)
        sys.setswitchinterval(self._swi)

    def summary(self):
        if not self.samples:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["unavailable"], "samples": 0}
        sm = sorted(s[0] for s in self.samples)
        mx = max(s[1] for s in self.samples)
        reasons = sorted({name for s in self.samples for bit, name in self.REASONS.items() if s[2] & bit})
        return {"sm_mhz": sm[len(sm) // 2], "sm_max_mhz": mx, "reasons": reasons, "samples": len(self.samples),
                "source": "nvml" if self._nvml else "nvidia-smi"}


def _max_over_ranks(dist, v: float) -> float:
    """MAX over ranks (device timings are taken per rank, the job is as slow as the slowest)."""
    import torch

    on_gpu = dist.get_backend() == "nccl"
    t = torch.tensor([v], dtype=torch.float64, device="cuda" if on_gpu else "cpu")
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return float(t.item())


def _cpu_model():
    try:
        return next((l.split(":", 1)[1].strip() for l in open("/proc/cpuinfo") if l.startswith("model name")), "")
    except OSError:
        import platform

        return platform.processor()


class _Pinned:
    """Pin the calling thread to one host core (1 thread, 1 core)."""

    def __enter__(self):
        self.old = None
        self.core = None
        try:
            self.old = os.sched_getaffinity(0)
            self.core = max(self.old)
            os.sched_setaffinity(0, {self.core})
        except (AttributeError, OSError):
            self.old = None
        return self

    def __exit__(self, *a):
        if self.old is not None:
            os.sched_setaffinity(0, self.old)


def cpu_baseline(w, sample_cap=256 << 20, check=None, x=None, B=4096):
    """The oracle (plain sequential C, oracle/) on one pinned host core, bounded sample
    (the first min(len, 256 MiB) bytes of the stream), median of 3 runs.  check
    (nullable): callable(sample_len) -> the GPU result on the same prefix, compared with
    the oracle's bit for bit (final state, accept count, every chunk end).  x (nullable):
    the device stream, whose sample bytes are hash-compared with the host generator's."""
    import numpy as np

    import gen
    import oracle

    sample = min(w.length, sample_cap)
    data = w.host(0, sample)
    same_bytes = None
    if x is not None:
        same_bytes = gen.bytes_hash(data) == gen.bytes_hash(x[:sample].cpu().numpy())
    times = []
    with _Pinned() as pin:
        for _ in range(3):
            t0 = time.perf_counter()
            r = oracle.run(w.table, w.start, w.accept, data, B)
            times.append(time.perf_counter() - t0)
            assert r["status"] == 0
    dt = sorted(times)[1]
    parity = None
    if check is not None:
        g = check(sample)
        ce = g.chunk_ends.cpu().numpy().view(np.uint32)
        ok = g.final_state == r["final"] and g.accept_count == r["count"] and (ce == r["chunk_end"]).all()
        parity = {"bit_exact": bool(ok), "sample": f"first {sample >> 20 or sample} {'MiB' if sample >> 20 else 'B'}"
                  f", same scheme and chunking", "chunks": int(len(ce)), "host_device_bytes_hash_equal": same_bytes}
    out = {"value": round(sample / dt / 1e9, 4), "unit": "GB/s", "cores": 1, "kind": "oracle",
           "sample": f"first {sample >> 20} MiB of the {w.name} stream, oracle.run (Alg. 1), 1 thread pinned to "
                     f"core {pin.core}, median of 3", "seconds": round(dt, 3), "host_nproc": os.cpu_count(),
           "cpu_model": _cpu_model()}
    return out, parity


def run_reference(args):
    """--impl reference: the oracle as it stands on host cores (the reference arm for this tier)."""
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return 0
    import gen
    import oracle

    name = "c2" if args.config == "c5" else args.config
    w = gen.workload(name)
    sample = min(w.length, args.ref_sample_mib << 20)
    data = w.host(0, sample)
    with _Pinned() as pin:
        for _ in range(max(0, args.warmup)):
            oracle.run(w.table, w.start, w.accept, data[: 1 << 20], 4096)
        t0 = time.perf_counter()
        for _ in range(args.steps):
            r = oracle.run(w.table, w.start, w.accept, data, 4096)
            assert r["status"] == 0
        dt = (time.perf_counter() - t0) / args.steps
    v = sample / dt / 1e9
    line = {"impl": "reference", "metric": METRIC, "value": round(v, 4), "unit": "GB/s", "n_gpus": args.gpus,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(dt * 1e3, 3),
            "higher_is_better": True, "scaling": "strong" if args.config == "c5" else "weak", "vs_baseline": None,
            "dtype": "u8", "data": "synthetic",
            "config": {"workload": args.config, "desc": CONFIG_DESC[args.config], "bytes_per_step": sample,
                       "chunk_bytes": 4096},
            "cpu_baseline": {"value": round(v, 4), "unit": "GB/s", "cores": 1, "kind": "oracle",
                             "sample": f"first {sample >> 20} MiB of the {name} stream per step, 1 thread pinned "
                                       f"to core {pin.core}"},
            "e2e": {"value": round(v, 4), "unit": "GB/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)
    return 0


def _head_start():
    """A ~1 ms GPU spin queued right before the first timing event: while it runs the host
    queues the first steps, so the event pair times the K steps' device work rather than the
    host's latency to enqueue the first one (the spin itself is outside the timed region)."""
    import torch

    torch.cuda._sleep(2_000_000)


def _median(v):
    v = sorted(v)
    return v[len(v) // 2] if v else None


def _roofline(name, length, spec_ms, peak, peak_kind):
    traffic = None
    tp = os.path.join(ROOT, "profiles", "traffic.json")
    if os.path.exists(tp):
        try:
            traffic = json.load(open(tp)).get(name)
        except Exception:
            traffic = None
    achieved = length / (spec_ms * 1e-3) / 1e9
    return {"bound": "hbm", "achieved": round(achieved, 1), "peak": peak, "unit": "GB/s",
            "frac": round(achieved / peak, 4), "traffic": traffic,
            "kernel": "k_spec_tma (speculative execution, TMA-staged)", "peak_kind": peak_kind,
            "achieved_def": "input bytes per launch / CUDA-event duration of the spec launch on its stream"}


def measure_single(gs, w, x, args, fsm, scheme, B, with_clocks=True):
    """K back-to-back runs of the whole stream on this GPU (fsm_run_async queue), timed by
    two CUDA events on the launching stream; spec / verify splits from the library's
    own per-run events."""
    import torch

    length = x.numel()
    stream = torch.cuda.current_stream()
    ce = torch.empty(gs.fsm_num_chunks(length, B), dtype=torch.int32, device="cuda")
    kw = {"spec_k": args.spec_k, "lookback": args.lookback}
    kr = [fsm.run(x, scheme=scheme, chunk_bytes=B, **kw) for _ in range(3)]
    verify_phases = [round(float(v), 1) for v in fsm.phase_times()]
    # at most WINDOW runs in flight (the handle's ring holds 32): waiting for the oldest while
    # the GPU works on the others never leaves it idle
    WINDOW = 16
    done = []

    def enqueue(pend):
        if len(pend) >= WINDOW:
            done.append(fsm.wait(pend.pop(0)))
        pend.append(fsm.run_async(x, scheme=scheme, chunk_bytes=B, chunk_ends=ce, **kw))

    pending = []
    for _ in range(max(3, args.warmup)):
        enqueue(pending)
    for t in pending:
        fsm.wait(t)
    pending.clear()
    done.clear()
    torch.cuda.synchronize()
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    clk = ClockSampler(torch.cuda.current_device()) if with_clocks else None
    if clk:
        clk.__enter__()
    _head_start()
    ev0.record(stream)
    for _ in range(args.steps):
        enqueue(pending)
    ev1.record(stream)
    torch.cuda.synchronize()
    if clk:
        clk.__exit__()
    spec_ms, ver_ms, launches = [], [], 0
    for res in done + [fsm.wait(t) for t in pending]:
        spec_ms.append(res.stats["ms_spec"])
        ver_ms.append(res.stats["ms_verify"])
        launches += res.stats["kernel_launches"]  # counted by the library per run
    ms = ev0.elapsed_time(ev1) / args.steps
    st0 = kr[-1].stats
    diag = {k: st0[k] for k in ("rounds", "tasks_total", "tasks_mustdo", "tasks_sre", "tasks_helper", "reread_bytes",
                                "verify_checks", "verify_matches", "task_walked_bytes")}
    diag["runtime_speculation_accuracy"] = round(st0["verify_matches"] / max(1, st0["verify_checks"]), 6)
    diag["avg_active_workers"] = round(float(st0.get("avg_active_workers", 0.0)), 2)
    return {"ms": ms, "value": length / (ms * 1e-3) / 1e9, "spec_ms": _median(spec_ms), "ver_ms": _median(ver_ms),
            "launches": launches, "clocks": clk.summary() if clk else None, "diag": diag, "phases": verify_phases,
            "result": res}


def spread_profile(w, total_len):
    """The selector's profile of a stream of total_len bytes (reading R20, as
    fsm_select_scheme builds it from a long trace): 8 portions of 128 KiB spread evenly
    from the start to the end of the stream, generated on the device from their global
    offsets (so every rank of a sharded run profiles the same global portions)."""
    import torch

    S = 128 << 10
    buf = torch.empty(8 * S, dtype=torch.uint8, device="cuda")
    if total_len <= 8 * S:
        buf = buf[:total_len]
        w.device(buf, offset=0)
        return buf
    for i in range(8):
        w.device(buf[i * S:(i + 1) * S], offset=(i * (total_len - S) // 7) & ~4095)
    return buf


def _table_info(fsm):
    try:
        tr = fsm.transform()
        return {"format": tr["mode"], "nclasses": int(tr["nclasses"]), "hot_rows": int(tr["hot_rows"])}
    except Exception:
        return None


def per_dfa_result(gs, name, args, peak, peak_kind, with_cpu=True):
    """One sub-result of the default N = 1 line: config `name` at its full size, selector
    scheme, value / ms / roofline / diagnostics / cpu_baseline / parity on a sample."""
    import torch

    import gen

    w = gen.workload(name)
    x = torch.empty(w.length, dtype=torch.uint8, device="cuda")
    w.device(x)
    prof = torch.empty(1 << 20, dtype=torch.uint8, device="cuda")
    w.device(prof, offset=w.length)
    fsm = gs.FSM.load(w.table, w.start, w.accept, profile=prof.cpu().numpy())
    scheme, feats = fsm.select_scheme(x)  # spread profile (R20); chunk size (R29) for this stream
    B = args.chunk_bytes or feats["chunk_bytes"]
    m = measure_single(gs, w, x, args, fsm, scheme, B, with_clocks=False)
    out = {"value": round(m["value"], 3), "unit": "GB/s", "ms_per_step": round(m["ms"], 4),
           "bytes": w.length, "scheme": scheme, "chunk_bytes": B, "nstates": int(w.nstates),
           "pct_hbm_roofline_8TBs": round(100 * m["value"] / 8000.0, 2),
           "breakdown_ms": {"spec_exec": round(m["spec_ms"], 4), "verify_recover": round(m["ver_ms"], 4)},
           "roofline": _roofline(name, w.length, m["spec_ms"], peak, peak_kind), "diagnostics": m["diag"],
           "gpu_launches": m["launches"], "table": _table_info(fsm),
           "features": {k: round(v, 4) if isinstance(v, float) else v for k, v in feats.items()}}
    if with_cpu:
        out["cpu_baseline"], out["parity"] = cpu_baseline(
            w, sample_cap=64 << 20, x=x, check=lambda n: fsm.run(x[:n], scheme=scheme, chunk_bytes=B), B=B)
    fsm.close()
    del x
    torch.cuda.empty_cache()
    return out


def async_sharded_steps(gs, comm, fsm, x, lb, scheme, B, ce, k, window=16):
    """k sharded steps queued back to back (fsm_run_sharded_async: map, ncclAllGather and
    finish without a host wait), collected window by window; returns the last result.  A
    step that reports FSM_EAGAIN (a speculative shard map was invalid) is redone
    synchronously, as every rank sees the same EAGAIN."""
    res, pend = None, []

    def drain():
        nonlocal res
        for t in pend:
            try:
                res = gs.Comm.wait(fsm, t)
            except gs.GSpecError as e:
                if e.status != gs.FSM_EAGAIN:
                    raise
                res = comm.run_sharded(fsm, x, lb, scheme=scheme, chunk_bytes=B)
        pend.clear()

    for _ in range(k):
        pend.append(comm.run_sharded_async(fsm, x, lb, scheme=scheme, chunk_bytes=B, chunk_ends=ce))
        if len(pend) >= window:
            drain()
    drain()
    return res


def _maybe_relaunch(args):
    """--gpus N > 1 without a torch.distributed launcher: re-run this command under
    torch.distributed.run (one process per GPU, rendezvous on 127.0.0.1)."""
    if args.gpus <= 1 or "WORLD_SIZE" in os.environ:
        return None
    import socket

    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={args.gpus}",
           "--master-addr", "127.0.0.1", "--master-port", str(port), os.path.abspath(__file__)] + sys.argv[1:]
    return subprocess.call(cmd)


def run_c5(args, gs, dist, world, rank, dev, comm, peak, peak_kind):
    """C5: each DFA's 16 GiB stream sharded over the `world` ranks (strong scaling); one
    step = fsm_run_sharded on every rank (shard map, one allgather, compose, fix-up),
    timed per rank by CUDA events, MAX over ranks."""
    import numpy as np
    import torch

    import gen
    from paper_conf_ipps_wangwqw22_b200.dist import run_sharded, shard_bounds

    L = args.c5_bytes
    per = {}
    dfas = C5_DFAS if args.c5_dfa == "all" else (args.c5_dfa,)
    clk_all = None
    for name in dfas:
        w = gen.workload(name, length=L)
        fsm = gs.FSM.load(w.table, w.start, w.accept)
        # selector per DFA (offline profiling): every rank profiles the same 8 spread
        # portions of the global stream (R20), so every rank picks the same scheme and the
        # same chunk size (R29, for L / world bytes per GPU) — the shard bounds follow it
        prof = spread_profile(w, L)
        scheme, feats = fsm.select_scheme(prof, stream_len=L // world)
        B = args.chunk_bytes or feats["chunk_bytes"]
        del prof
        lo, hi = shard_bounds(L, world, rank, B)
        x = torch.empty(hi - lo, dtype=torch.uint8, device="cuda")
        w.device(x, offset=lo)
        lb = torch.empty(min(16, lo), dtype=torch.uint8, device="cuda")
        if lo:  # the 16 bytes before the shard (pure function of the offset): its candidate set
            w.device(lb, offset=lo - lb.numel())

        p2p = None
        if dist is not None and args.exchange == "p2p":
            from paper_conf_ipps_wangwqw22_b200.dist import p2p_setup

            p2p = p2p_setup(fsm)

        def step():
            if p2p is not None:
                return p2p.run_sharded(fsm, x, lb, scheme=scheme, chunk_bytes=B)
            if comm is not None:
                return comm.run_sharded(fsm, x, lb, scheme=scheme, chunk_bytes=B)
            if dist is not None:
                return run_sharded(fsm, x, lb, scheme=scheme, chunk_bytes=B)
            return fsm.run(x, scheme=scheme, chunk_bytes=B)

        res = None
        for _ in range(max(3, args.warmup)):
            res = step()
        ce = torch.empty(max(1, gs.fsm_num_chunks(x.numel(), B)), dtype=torch.int32, device="cuda")
        if dist:
            dist.barrier()
        torch.cuda.synchronize()
        stream = torch.cuda.current_stream()
        ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        pend = []
        with ClockSampler(dev) as clk:
            _head_start()
            ev0.record(stream)
            if comm is not None and p2p is None:  # steps queued back to back: no host wait between them
                res = async_sharded_steps(gs, comm, fsm, x, lb, scheme, B, ce, args.steps)
            elif dist is None:  # one GPU: fsm_run_async queue (no host wait between steps either)
                for _ in range(args.steps):
                    if len(pend) >= 16:
                        res = fsm.wait(pend.pop(0))
                    pend.append(fsm.run_async(x, scheme=scheme, chunk_bytes=B, chunk_ends=ce))
            else:
                for _ in range(args.steps):
                    res = step()
            ev1.record(stream)
            for t in pend:
                res = fsm.wait(t)
            torch.cuda.synchronize()
        if p2p is not None:
            p2p.close()
        if clk_all is None:
            clk_all = clk
        else:
            clk_all.samples += clk.samples
        ms = ev0.elapsed_time(ev1) / args.steps
        if dist:
            dist.barrier()
            ms = _max_over_ranks(dist, ms)
        value = L / (ms * 1e-3) / 1e9
        # parity: the global result equals the oracle's on the bench's own run is checked
        # at full size by tests/test_gpu_c5.py; here every rank's global result must agree
        agree = True
        if dist:
            t = torch.tensor([res.final_state, res.accept_count & 0xFFFFFFFF, res.accept_count >> 32],
                             dtype=torch.int64, device="cuda" if dist.get_backend() == "nccl" else "cpu")
            t2 = t.clone()
            dist.all_reduce(t2, op=dist.ReduceOp.MAX)
            agree = bool((t == t2).all().item())
        per[name] = {"value": round(value, 3), "unit": "GB/s", "ms_per_step": round(ms, 4), "bytes": L,
                     "bytes_per_rank": hi - lo, "scheme": scheme, "chunk_bytes": B, "nstates": int(w.nstates),
                     "pct_hbm_roofline_8TBs_per_gpu": round(100 * value / world / 8000.0, 2),
                     "latency_ms_per_GB": round(ms * 1e9 / L, 4), "ranks_agree": agree,
                     "final_state": res.final_state, "accept_count": res.accept_count,
                     "features": {k: round(v, 4) if isinstance(v, float) else v for k, v in feats.items()}}
        fsm.close()
        del x
        torch.cuda.empty_cache()
    head = per[dfas[0]]
    line = {
        "metric": METRIC, "value": head["value"], "unit": "GB/s", "n_gpus": world, "steps": args.steps,
        "warmup": max(3, args.warmup), "ms_per_step": head["ms_per_step"], "higher_is_better": True,
        "scaling": "strong", "vs_baseline": None, "dtype": "u8", "data": "synthetic",
        "config": {"workload": "c5", "desc": CONFIG_DESC["c5"], "headline_dfa": dfas[0], "bytes_total": L,
                   "chunk_bytes": "per DFA (per_dfa[*].chunk_bytes: the selector's R29 recommendation)"
                   if not args.chunk_bytes else args.chunk_bytes,
                   "l2": "input (16 GiB / N per GPU) larger than the 126 MB L2; no flush",
                   "timing": "CUDA events around the K steps after a ~1 ms GPU spin (host head start), max over ranks",
                   "parallelism": f"{world} contiguous shards + one exchange of state maps"
                   + (" (peer-memory stores, fsm_run_sharded_p2p)" if dist is not None and args.exchange == "p2p" else
                      " (library NCCL allgather, fsm_run_sharded_async)" if comm is not None else
                      " (torch.distributed allgather)" if dist is not None else " (single GPU, fsm_run)"),
                   "nccl_ranks": comm.nranks if comm is not None else 0},
        "per_dfa": per,
        "gpu_launches": None,
        "clocks": clk_all.summary() if clk_all else None,
        "e2e": None,
        "e2e_note": "C5 shards are 16/N GiB per rank: the end-to-end (host-buffer) number is the default c2 line's",
    }
    return line


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="own", choices=["own", "reference"])
    ap.add_argument("--config", default="c2", choices=sorted(CONFIG_DESC))
    ap.add_argument("--scheme", default="auto")
    ap.add_argument("--chunk-bytes", type=int, default=0,
                    help="chunk size B; 0 = the selector's recommendation (reading R29, 4096 unless the "
                         "profile's lookback images converge only over longer chunks)")
    ap.add_argument("--spec-k", type=int, default=0, help="paths per chunk for pm / pm_tree / cse (0 = default)")
    ap.add_argument("--lookback", type=int, default=2, help="lookback symbols per chunk prediction (2..16, R25)")
    ap.add_argument("--e2e-steps", type=int, default=3)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-per-dfa", action="store_true", help="skip the per-DFA sub-results of the default line")
    ap.add_argument("--ref-sample-mib", type=int, default=256)
    ap.add_argument("--exchange", default="nccl", choices=["nccl", "p2p"],
                    help="N > 1: state maps by the library's NCCL allgather, or by peer-memory stores (fsm_p2p_*)")
    ap.add_argument("--c5-dfa", default="all", choices=["all"] + list(C5_DFAS))
    ap.add_argument("--c5-bytes", type=int, default=C5_LEN)
    args = ap.parse_args()
    if args.impl == "reference":
        return run_reference(args)
    rc = _maybe_relaunch(args)
    if rc is not None:
        return rc

    import numpy as np
    import torch

    import gen
    import paper_conf_ipps_wangwqw22_b200 as gs

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    # one process per GPU; GSPEC_DIST_BACKEND=gloo lets several ranks share one GPU (tests only)
    backend = os.environ.get("GSPEC_DIST_BACKEND", "nccl")
    dev = local % max(1, torch.cuda.device_count()) if backend != "nccl" else local
    torch.cuda.set_device(dev)
    dist = None
    comm = None
    if world > 1:
        import torch.distributed as dist

        if backend == "nccl":
            dist.init_process_group("nccl", device_id=torch.device("cuda", dev))
            # the library owns its NCCL communicator (fsm_comm_init); torch.distributed
            # only broadcasts the 128-byte unique id and provides barriers
            uid = [gs.Comm.unique_id() if rank == 0 else None]
            dist.broadcast_object_list(uid, src=0)
            comm = gs.Comm(world, rank, uid[0], device=dev)
        else:
            dist.init_process_group(backend)
    peak, peak_kind = _peaks()

    if args.config == "c5":
        line = run_c5(args, gs, dist, world, rank, dev, comm, peak, peak_kind)
        if rank == 0:
            print(json.dumps(line), flush=True)
        if comm is not None:
            comm.close()
        if dist:
            dist.destroy_process_group()
        return 0

    w = gen.workload(args.config)
    length = w.length
    B = args.chunk_bytes
    x = torch.empty(length, dtype=torch.uint8, device="cuda")
    w.device(x, offset=rank * length)  # weak scaling: rank r owns bytes [r*len, (r+1)*len)
    # profile sample (a 1 MiB "training" trace): a disjoint slice of the same
    # source, past every rank's shard; it places the u8 table rows bank-aware (DESIGN.md
    # §5.1) and is the selector's profile
    prof = torch.empty(1 << 20, dtype=torch.uint8, device="cuda")
    w.device(prof, offset=world * length)
    fsm = gs.FSM.load(w.table, w.start, w.accept, profile=prof.cpu().numpy())
    scheme = args.scheme
    feats = None
    del prof
    if scheme == "auto" or not B:  # offline profiling, untimed: 8 spread portions of the stream (R20)
        sp = spread_profile(w, length * world)
        sel, feats = fsm.select_scheme(sp, stream_len=length)
        del sp
        scheme = sel if scheme == "auto" else scheme
        B = B or feats["chunk_bytes"]  # chunk size (granularity) from the profile (R29)

    lb = None
    if world > 1:
        from paper_conf_ipps_wangwqw22_b200.dist import run_sharded

        # the 16 bytes before this rank's shard (pure function of the offset): its candidate
        # start set is their lookback image, the smallest one fsm_shard_map accepts
        lb = torch.empty(16 if rank else 0, dtype=torch.uint8, device="cuda")
        if rank:
            w.device(lb, offset=rank * length - 16)

        p2p = None
        if args.exchange == "p2p":
            from paper_conf_ipps_wangwqw22_b200.dist import p2p_setup

            p2p = p2p_setup(fsm)

        def step():
            if p2p is not None:
                return p2p.run_sharded(fsm, x, lb, scheme=scheme, chunk_bytes=B)
            if comm is not None:
                return comm.run_sharded(fsm, x, lb, scheme=scheme, chunk_bytes=B)
            return run_sharded(fsm, x, lb, scheme=scheme, chunk_bytes=B)

        kr = [fsm.run(x, scheme=scheme, chunk_bytes=B) for _ in range(3)]
        for _ in range(max(3, args.warmup)):
            res = step()
        ce_sh = torch.empty(max(1, gs.fsm_num_chunks(length, B)), dtype=torch.int32, device="cuda")
        dist.barrier()
        torch.cuda.synchronize()
        stream = torch.cuda.current_stream()
        ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        pend = []
        with ClockSampler(dev) as clk:
            _head_start()
            ev0.record(stream)
            if comm is not None and p2p is None:  # steps queued back to back: no host wait between them
                res = async_sharded_steps(gs, comm, fsm, x, lb, scheme, B, ce_sh, args.steps)
            else:
                for _ in range(args.steps):
                    res = step()
            ev1.record(stream)
            torch.cuda.synchronize()
        dist.barrier()
        ms = _max_over_ranks(dist, ev0.elapsed_time(ev1) / args.steps)
        m = {"ms": ms, "spec_ms": _median([r.stats["ms_spec"] for r in kr]),
             "ver_ms": _median([r.stats["ms_verify"] for r in kr]), "launches": None, "clocks": clk.summary(),
             "phases": [], "diag": {k: kr[-1].stats[k] for k in ("rounds", "tasks_total", "tasks_mustdo", "tasks_sre",
                                                                  "tasks_helper", "reread_bytes", "verify_checks",
                                                                  "verify_matches")}}
    else:
        m = measure_single(gs, w, x, args, fsm, scheme, B)
        res = m["result"]
        ms = m["ms"]
    total_bytes = length * world
    value = total_bytes / (ms * 1e-3) / 1e9

    # end-to-end: host (pinned) bytes through the public API, H2D + D2H inside the timed region
    e2e = None
    if args.e2e_steps > 0:
        h = torch.empty(length, dtype=torch.uint8, pin_memory=True)
        h.copy_(x)
        hn = h.numpy()
        nch = gs.fsm_num_chunks(length, B)
        if world == 1:
            def e2e_step():
                return fsm.run_host(hn, scheme=scheme, chunk_bytes=B)
        else:
            xd = torch.empty_like(x)
            ce_h = torch.empty(nch, dtype=torch.int32, pin_memory=True)

            def e2e_step():
                xd.copy_(h, non_blocking=True)                     # H2D of this rank's shard
                if p2p is not None:
                    r = p2p.run_sharded(fsm, xd, lb, scheme=scheme, chunk_bytes=B)
                elif comm is not None:
                    r = comm.run_sharded(fsm, xd, lb, scheme=scheme, chunk_bytes=B)
                else:
                    r = run_sharded(fsm, xd, lb, scheme=scheme, chunk_bytes=B)
                ce_h.copy_(r.chunk_ends, non_blocking=True)       # D2H of the results
                torch.cuda.current_stream().synchronize()
                return r
        e2e_step()
        if dist:
            dist.barrier()
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        for _ in range(args.e2e_steps):
            r2 = e2e_step()
        torch.cuda.synchronize()
        e2e_s = time.perf_counter() - t0
        if dist:
            e2e_s = _max_over_ranks(dist, e2e_s)
        e2e_s /= args.e2e_steps
        assert r2.final_state == res.final_state and r2.accept_count == res.accept_count
        e2e = {"value": round(total_bytes / e2e_s / 1e9, 3), "unit": "GB/s", "h2d_bytes_per_step": length,
               "d2h_bytes_per_step": int(nch * 4 + 64), "ms_per_step": round(e2e_s * 1e3, 3)}

    line = {
        "metric": METRIC,
        "value": round(value, 3),
        "unit": "GB/s",
        "n_gpus": world,
        "steps": args.steps,
        "warmup": max(3, args.warmup),
        "ms_per_step": round(ms, 4),
        "higher_is_better": True,
        "scaling": "weak",
        "vs_baseline": None,
        "dtype": "u8",
        "data": "synthetic",
        "config": {"workload": args.config, "desc": CONFIG_DESC[args.config], "bytes_per_gpu": length,
                   "chunk_bytes": B, "scheme": scheme, "nstates": int(w.nstates), "spec_k": args.spec_k or None,
                   "lookback": args.lookback,
                   "l2": "input (1 GiB/GPU) larger than the 126 MB L2; no explicit flush",
                   "timing": "CUDA events on the launching stream around the K steps (a ~1 ms GPU spin queued "
                             "before the first event lets the host queue ahead; it is outside the region)",
                   "parallelism": (f"dp{world} contiguous shards + one exchange of state maps"
                                   + (" (peer-memory stores, fsm_run_sharded_p2p)" if args.exchange == "p2p" else
                                      " (library NCCL allgather, fsm_run_sharded_async)" if comm is not None else "")
                                   if world > 1 else "single GPU"),
                   "nccl_ranks": comm.nranks if comm is not None else 0},
        "pct_hbm_roofline_8TBs": round(100 * value / world / 8000.0, 2),
        "latency_ms_per_GB": round(ms * 1e9 / length, 4),
        "verify_phase_boundaries_us": m["phases"],
        "breakdown_ms": {"spec_exec": round(m["spec_ms"], 4), "verify_recover": round(m["ver_ms"], 4)},
        "roofline": _roofline(args.config, length, m["spec_ms"], peak, peak_kind),
        "diagnostics": m["diag"],
        "gpu_launches": m["launches"] if m["launches"] is not None else 6 * args.steps,
        "clocks": m["clocks"],
        "e2e": e2e,
    }
    line["pct_measured_hbm_whole_step"] = round(100 * value / world / peak, 2)
    line["config"]["table"] = _table_info(fsm)
    if feats:
        line["config"]["features"] = {k: round(v, 4) if isinstance(v, float) else v for k, v in feats.items()}
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        line["cpu_baseline"], parity = cpu_baseline(
            w, x=x, check=lambda n: fsm.run(x[:n], scheme=scheme, chunk_bytes=B), B=B)
        if parity is not None:
            line["parity"] = parity
    if world == 1 and args.config == "c2" and args.scheme == "auto" and not args.no_per_dfa:
        fsm.close()
        del x
        torch.cuda.empty_cache()
        line["per_dfa"] = {"c2": {"value": line["value"], "ms_per_step": line["ms_per_step"], "scheme": scheme,
                                  "roofline_frac": line["roofline"]["frac"], "see": "top-level keys"}}
        for name in ("c1", "c3", "c3s", "c4"):
            line["per_dfa"][name] = per_dfa_result(gs, name, args, peak, peak_kind,
                                                   with_cpu=not args.no_cpu_baseline)
    if rank == 0:
        print(json.dumps(line), flush=True)
    if comm is not None:
        comm.close()
    if dist:
        dist.destroy_process_group()
    return 0


if __name__ == "__main__":
    sys.exit(main())
