"""Pins of the Algorithm 1 oracle (CPU only): the hand-computed worked example
and the invariants the paper states (P:159-166 principles, P:248 contention
factor guarantee, P:149 degeneration to intra-op)."""
import json
import os
import random
from collections import deque

import pytest

from oracle.scheduler import Kernel, Scheduler, plan_round
from oracle import metrics as om

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def _kernels(bid, spec):
    out = []
    for name, typ, d in spec:
        durs = tuple(d) if isinstance(d, list) else (d,)
        out.append(Kernel(bid, name, typ, durs, decomposable=len(durs) > 1))
    return out


def test_worked_example():
    ex = json.load(open(os.path.join(GOLD, "algorithm1_worked_example.json")))
    lists = [deque(_kernels(b["id"], b["kernels"])) for b in ex["batches"]]
    for want in ex["rounds"]:
        r = plan_round(lists, ex["cf"])
        assert r.type == want["type"]
        assert r.time0 == pytest.approx(want["time0"])
        assert [[p.batch, p.name, p.u0, p.u1] for p in r.sub0] == want["sub0"]
        assert [[p.batch, p.name, p.u0, p.u1] for p in r.sub1] == want["sub1"]
    # after round 2 the FC1 remainder (6/8) stays at the head of batch 1
    assert lists[1][0].name == "FC1" and lists[1][0].left == 6


def _random_batch(rng, bid, F=8, n_layers=3):
    ks = []
    for _ in range(n_layers):
        for name, typ, dec in (("LN", "C", False), ("QKV", "C", True), ("attn", "C", False),
                               ("out", "C", True), ("AR1", "M", True), ("LN2", "C", False),
                               ("FC1", "C", True), ("FC2", "C", True), ("AR2", "M", True)):
            d = rng.uniform(1, 100)
            if dec:   # monotone, sub-additive-ish piece durations, full = d
                durs = tuple(d * (0.15 + 0.85 * k / F) if k < F else d for k in range(1, F + 1))
            else:
                durs = (d,)
            ks.append(Kernel(bid, name, typ, durs, decomposable=dec))
    return ks


@pytest.mark.parametrize("seed", range(20))
@pytest.mark.parametrize("cf", [1.0, 1.1, 1.3])
def test_invariants(seed, cf):
    rng = random.Random(seed)
    nb = rng.randint(1, 5)
    batches = {b: _random_batch(rng, b) for b in range(nb)}
    order = {b: [(k.name, k.units) for k in ks] for b, ks in batches.items()}
    sch = Scheduler(list_size=rng.randint(1, 4), cf=cf)
    for b in range(nb):
        sch.submit(b, batches[b])
    rounds = sch.run()
    seen = {b: [] for b in range(nb)}
    for r in rounds:
        # P1 / P:248: the scaled secondary never exceeds the primary
        assert r.time1_scaled <= r.time0 + 1e-9
        assert all(p.type != r.type for p in r.sub1)
        assert all(p.type == r.type for p in r.sub0)
        prim = {p.batch for p in r.sub0}
        assert len(prim) == 1
        assert not any(p.batch in prim for p in r.sub1)
        for p in r.sub0 + r.sub1:
            seen[p.batch].append(p)
    for b, pieces in seen.items():
        # per-batch order preserved; every kernel runs exactly once; the pieces of
        # a decomposed kernel are contiguous and their fractions sum to 1
        i, u = 0, 0
        for p in pieces:
            assert (p.name, p.units) == order[b][i] and p.u0 == u and p.u1 > p.u0
            u = p.u1
            if u == p.units:
                i, u = i + 1, 0
        assert i == len(order[b]) and u == 0


def test_list_size_one_is_serial_intra_op():
    """at low load (one batch in flight) interleaving degenerates to intra-op."""
    rng = random.Random(7)
    batches = [_random_batch(rng, b) for b in range(3)]
    expect = [(b, k.name) for b in range(3) for k in batches[b]]
    sch = Scheduler(list_size=1, cf=1.1)
    for b in range(3):
        sch.submit(b, batches[b])
    got = []
    for r in sch.run():
        assert r.sub1 == []
        got += [(p.batch, p.name) for p in r.sub0]
        assert all(p.u0 == 0 and p.u1 == p.units for p in r.sub0)
    assert got == expect


def test_fifo_admission():
    sch = Scheduler(list_size=2)
    for b in range(4):
        sch.submit(b, [Kernel(b, "k", "C", (1.0,))])
    sch.update_list()
    assert [b for b, _ in sch.processing] == [0, 1]


def test_metrics_toy():
    ex = json.load(open(os.path.join(GOLD, "metrics_toy.json")))
    lat = om.latencies(ex["arrivals"], ex["finishes"])
    assert lat == pytest.approx(ex["latencies"])
    assert om.mean(lat) == pytest.approx(ex["mean"])
    assert om.p_nearest_rank(lat, 99) == pytest.approx(ex["p99"])
    assert om.p_nearest_rank(lat, 50) == pytest.approx(ex["p50"])
    assert om.throughput(ex["arrivals"], ex["finishes"]) == pytest.approx(ex["throughput"])
