"""Host-side logic of bench.py (no GPU): the N > 1 launch (re-exec under torchrun),
the rank-consistent open-loop submission of serve_poisson over a world-size-2 gloo
group, max-over-ranks timing, and the fixed-latency interpolation of the BASELINE
metric (SURVEY §8(d) operating points)."""
import os
import sys

import numpy as np
import pytest
import torch.distributed as dist
import torch.multiprocessing as mp

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import bench  # noqa: E402


def test_req_s_at_latency_interpolation():
    pts = [dict(req_s=2.0, mean_s=0.2), dict(req_s=4.0, mean_s=0.3), dict(req_s=6.0, mean_s=0.7)]
    assert bench.req_s_at_latency(pts, 0.5) == pytest.approx(5.0)     # between points 2 and 3
    assert bench.req_s_at_latency(pts, 0.3) == pytest.approx(4.0)
    assert bench.req_s_at_latency(pts, 0.8) == pytest.approx(6.0)     # every point within L
    assert bench.req_s_at_latency(pts, 0.1) is None                   # none within L


def test_gpus_n_relaunches_under_torchrun(monkeypatch):
    calls = []
    monkeypatch.setattr(bench.subprocess, "call", lambda cmd: calls.append(cmd) or 0)
    monkeypatch.delenv("WORLD_SIZE", raising=False)
    monkeypatch.setattr(sys, "argv", ["bench.py", "--gpus", "2", "--steps", "3"])
    assert bench.main() == 0
    cmd = calls[0]
    assert cmd[1:3] == ["-m", "torch.distributed.run"]
    assert "--nproc-per-node=2" in cmd and "--master-addr=127.0.0.1" in cmd
    assert cmd[-4:] == ["--gpus", "2", "--steps", "3"]


class FakeEngine:
    """Stands in for LigerEngine: records the submission order; batches finish at once."""

    class Res:
        def __init__(self, arrival):
            self.arrival_s, self.finish_s = arrival, arrival + 0.01

    def __init__(self):
        self.subs = []

    def submit(self, tokens, b, s, n, arrival):
        self.subs.append((b, s, n))
        self.arr = getattr(self, "arr", []) + [arrival]
        return len(self.subs) - 1

    def step(self):
        return 2

    def drain(self):
        pass

    def poll(self, bid):
        return FakeEngine.Res(self.arr[bid]), None


def _rank(r, port, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=r, world_size=2)
    import bench as B
    g = B.DistGroup.__new__(B.DistGroup)
    g.dist, g.world, g.rank, g.gloo = dist, 2, r, dist.group.WORLD
    B.DistGroup.barrier = lambda self: dist.barrier()
    from liger_inputs import make_trace
    tr = make_trace(6, 200.0, seed=1, vocab=100, prompt_range=(4, 8), n_decode=2)
    eng = FakeEngine()
    res = B.serve_poisson(eng, g, tr)
    mx = g.max(float(r + 1))
    # every engine a rank creates gets a fresh communicator id, the same on all ranks
    made = iter(range(100, 200))
    new_uid = B.uid_factory(g, lambda: b"uid-%d" % next(made))
    uids = [new_uid() for _ in range(3)]
    q.put((r, eng.subs, mx, res["req_s"] > 0, uids))
    dist.destroy_process_group()


def test_serve_poisson_submits_identically_on_two_gloo_ranks():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = bench._free_port()
    ps = [ctx.Process(target=_rank, args=(r, port, q)) for r in range(2)]
    for p in ps:
        p.start()
    out = sorted(q.get(timeout=120) for _ in range(2))
    for p in ps:
        p.join(timeout=60)
    (_, s0, m0, ok0, u0), (_, s1, m1, ok1, u1) = out
    assert s0 == s1 and len(s0) == 6     # the same batches in the same order on both ranks
    assert m0 == m1 == 2.0               # max over ranks
    assert ok0 and ok1
    # one fresh communicator id per engine (an ncclUniqueId bootstraps one communicator),
    # identical on both ranks
    assert u0 == u1 == [b"uid-100", b"uid-101", b"uid-102"]


def test_trace_summary_hand_computed():
    """bench.trace_summary on hand-made CTA records (2 SMs, span 100 ns): GEMM CTAs work in
    [10, 40] and [30, 60] (union 50 ns -> no GEMM working 0.5 of the span), a fixup CTA in
    [60, 100] (its entry t0 = 0 starts the span); SM-time shares 60 / 200 and 40 / 200."""
    dt = np.dtype([("kid", "<u4"), ("cta", "<u4"), ("smid", "<u4"), ("pad", "<u4"),
                   ("t0", "<u8"), ("t1", "<u8"), ("t2", "<u8")])
    rec = np.array([(1, 0, 0, 0, 5, 10, 40), (1, 1, 1, 0, 5, 30, 60), (2, 0, 1, 0, 0, 60, 100)], dtype=dt)
    out = bench.trace_summary(rec)
    assert out["sms"] == 2 and out["span_ms"] == round(100 / 1e6, 2)
    assert out["sm_time_share"] == {"gemm": 0.3, "splitk_fixup": 0.2}
    assert out["no_gemm_working_frac"] == 0.5


def test_trace_launches_groups_by_cta_repeat():
    """bench.trace_launches: CTA records of one kernel kind, in entry order, split into launches
    where a CTA index repeats (PDL: the next launch's CTAs enter before this one's exit); each
    launch -> (first PDL-wait release, last exit, CTAs)."""
    dt = np.dtype([("kid", "<u4"), ("cta", "<u4"), ("smid", "<u4"), ("pad", "<u4"),
                   ("t0", "<u8"), ("t1", "<u8"), ("t2", "<u8")])
    rows = [(1, 0, 0, 0, 10, 20, 50), (1, 1, 1, 0, 11, 21, 55), (2, 0, 0, 0, 12, 56, 60),
            (1, 0, 2, 0, 40, 61, 90), (1, 1, 3, 0, 41, 62, 95), (1, 2, 4, 0, 42, 63, 99)]
    rec = np.array(rows, dtype=dt)
    assert bench.trace_launches(rec, 1) == [(20, 55, 2), (61, 99, 3)]
    assert bench.trace_launches(rec, 2) == [(56, 60, 1)]
