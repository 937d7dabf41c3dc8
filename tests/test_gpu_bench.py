"""bench.py's own launch paths on one GPU: the C5 line (per-DFA sharded runs) at N = 1 and,
with ranks sharing cuda:0 over gloo, at N = 2 through bench.py's self-relaunch under
torch.distributed.run (the driver's 8-GPU run uses the same code with NCCL)."""
import json
import os
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _bench(*args, env=None):
    e = dict(os.environ)
    e.update(env or {})
    out = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py")] + list(args), capture_output=True, text=True,
                         timeout=900, env=e, cwd=ROOT)
    assert out.returncode == 0, out.stderr[-3000:]
    lines = [l for l in out.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1, out.stdout[-2000:]
    return json.loads(lines[0])


@pytest.mark.parametrize("gpus,exchange", [(1, "nccl"), (2, "nccl"), (2, "p2p")])
def test_bench_c5_line(gpus, exchange):
    import gen
    import oracle

    L = 64 << 20
    d = _bench("--config", "c5", "--gpus", str(gpus), "--steps", "2", "--warmup", "3", "--c5-bytes", str(L),
               "--exchange", exchange, env={"GSPEC_DIST_BACKEND": "gloo"} if gpus > 1 else None)
    assert d["n_gpus"] == gpus and d["scaling"] == "strong" and d["config"]["workload"] == "c5"
    assert set(d["per_dfa"]) == {"c1", "c2", "c3", "c4"}
    for name, r in d["per_dfa"].items():
        assert r["value"] > 0 and r["ranks_agree"]
        w = gen.workload(name, length=L)
        ref = oracle.run(w.table, w.start, w.accept, w.host(), 4096)
        assert r["final_state"] == ref["final"] and r["accept_count"] == ref["count"], name
        assert r["scheme"] == {"c1": "enum", "c2": "sre", "c3": "sre", "c4": "sre"}[name]


def test_fused_round0_verification_path():
    """The opt-in fused round-0 verification (GSPEC_V0=1, read once per process: run the
    oracle-parity tests of the SRE round-0 path in a child process with it on)."""
    e = dict(os.environ)
    e["GSPEC_V0"] = "1"
    out = subprocess.run([sys.executable, "-m", "pytest", os.path.join(ROOT, "tests", "test_gpu_parity.py"), "-q",
                          "-p", "no:cacheprovider", "-k", "inline_round0 or full_size_bench or edge_lengths or async"],
                         capture_output=True, text=True, timeout=900, env=e, cwd=ROOT)
    assert out.returncode == 0, out.stdout[-3000:] + out.stderr[-2000:]
    assert " passed" in out.stdout


@pytest.mark.parametrize("config,steps", [("c1", 40), ("c2", 35)])
def test_bench_more_steps_than_the_run_ring(config, steps):
    """The driver picks K: more timed steps than a handle keeps runs in flight (32) must still
    produce one line (bench.py keeps at most 16 runs queued, waiting for the oldest)."""
    line = _bench("--config", config, "--steps", str(steps), "--warmup", "3", "--e2e-steps", "0",
                  "--no-cpu-baseline", "--no-per-dfa")
    assert line["steps"] == steps and line["value"] > 0 and line["gpu_launches"] >= steps


def test_bench_default_line_two_ranks():
    """The default line under bench.py's own relaunch at N = 2 (ranks sharing cuda:0 over gloo;
    the driver's multi-GPU run takes the same path with NCCL): weak scaling, 1 GiB per rank
    shard of one global stream, the end-to-end leg, one JSON line from rank 0."""
    d = _bench("--gpus", "2", "--steps", "3", "--warmup", "3", "--e2e-steps", "1", "--no-cpu-baseline",
               env={"GSPEC_DIST_BACKEND": "gloo"})
    assert d["n_gpus"] == 2 and d["scaling"] == "weak" and d["config"]["workload"] == "c2"
    assert d["value"] > 0 and d["e2e"]["value"] > 0 and d["e2e"]["h2d_bytes_per_step"] == 1 << 30
    assert d["roofline"]["frac"] > 0 and d["gpu_launches"] > 0
