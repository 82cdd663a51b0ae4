"""Tensor-parallel serving on ONE GPU with the loopback communicator: t ranks are
threads of this process, each with its own liger context (own shard, streams,
scheduler), collectives via host rendezvous + rank-ordered device reductions.

This runs the complete t > 1 path of the product -- all-reduces on the
communication stream, Algorithm 1 rounds with real secondary subsets,
runtime decomposition, hybrid E1/E2 synchronisation, the vocab-parallel LM
head's all-gather -- and checks BASELINE.json's requirements on the tiny
config (TP=2): greedy tokens identical to the oracle, and interleaved and
non-interleaved runs bit-exact with each other."""
import threading

import numpy as np
import pytest
import torch

from liger_inputs import get_config, make_trace
from oracle import model as om

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def E():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_ppopp_duwjchcl24_b200.engine import LigerEngine
    return LigerEngine


def serve_tp(E, cfg, world, trace, durations=None, **kw):
    """Run `trace` on `world` loopback ranks; returns (tokens per batch, stats) of each rank."""
    uid = E.loopback_id()
    out = [None] * world
    err = []

    def rank_main(r):
        try:
            torch.cuda.set_device(0)
            eng = E(cfg, world=world, rank=r, nccl_uid=uid, **kw)
            for args in durations or ():
                eng.set_duration(*args)
            ids = [eng.submit(t["tokens"], t["batch"], t["seq_len"], t["n_decode"], t["arrival_s"]) for t in trace]
            eng.drain()
            toks = [eng.poll(i, want_tokens=True)[1] for i in ids]
            out[r] = (toks, eng.stats())
            eng.close()
        except Exception as e:   # surfaced in the main thread
            err.append(repr(e))

    ths = [threading.Thread(target=rank_main, args=(r,)) for r in range(world)]
    for t in ths:
        t.start()
    for t in ths:
        t.join(timeout=600)
    assert not err, err
    assert all(o is not None for o in out)
    return out


def test_tiny_tp2_greedy_tokens_match_oracle(E):
    """BASELINE.json configs[0]: tiny, TP=2, batch 2, prompt 32 + 8 decode tokens."""
    cfg = get_config("tiny")
    prompt = np.random.default_rng(0).integers(0, cfg.vocab, size=(2, 32))
    ref, logits = om.greedy_generate(cfg, 0, prompt, 8, return_logits=True)
    assert om.top2_margin(logits).min() > 0.02 * np.sqrt((logits ** 2).mean())
    trace = [dict(tokens=prompt.reshape(-1).astype(np.int32), batch=2, seq_len=32, n_decode=8, arrival_s=0.0)]
    res = serve_tp(E, cfg, 2, trace, mode="interleaved", max_batch=2, max_seq=32, max_new=8, seed=0)
    for toks, st in res:
        assert np.array_equal(toks[0], ref)
        assert st["comm_kernels"] > 0


@pytest.mark.parametrize("world", [2, 4])
def test_interleaved_equals_serial_bit_exact(E, world):
    """Several batches in flight: Algorithm 1 interleaves one batch's all-reduces
    with another's GEMMs (secondary subsets, decomposition pieces); the tokens
    must be bit-identical to serial intra-op TP and to every rank's."""
    import os
    cfg = get_config("tiny")
    trace = make_trace(5, float("inf"), seed=11, batch_sizes=(1, 2, 3), prompt_range=(8, 40), n_decode=6,
                       vocab=cfg.vocab)
    # tiny messages: let every all-reduce be decomposable (and, at t > 2, issued as
    # atomic 1/F chunks) so the pieces path is exercised
    os.environ["LIGER_AR_DECOMP_MIN_KB"] = "0"
    try:
        base = serve_tp(E, cfg, world, trace, mode="serial", max_batch=4, max_seq=64, max_new=8, seed=3)
        inter = serve_tp(E, cfg, world, trace, mode="interleaved", max_batch=4, max_seq=64, max_new=8,
                         max_inflight=3, decomp_factor=8, contention_factor=1.0, seed=3)
    finally:
        os.environ.pop("LIGER_AR_DECOMP_MIN_KB", None)
    ref_toks = base[0][0]
    for toks, st in base + inter:
        for a, b in zip(ref_toks, toks):
            assert np.array_equal(a, b)
    st = inter[0][1]
    assert st["overlapped_rounds"] > 0, st      # secondary subsets were actually scheduled
    assert st["comm_kernels"] > 0
    # and the TP result is the unsharded model's (oracle), where its argmax is unambiguous
    for t, toks in zip(trace[:2], ref_toks[:2]):
        p = t["tokens"].reshape(t["batch"], t["seq_len"])
        ref, logits = om.greedy_generate(cfg, 3, p, t["n_decode"], return_logits=True)
        ok = om.top2_margin(logits) > 0.02 * np.sqrt((logits ** 2).mean())
        for i in range(t["batch"]):
            n = int(np.argmin(ok[i])) if not ok[i].all() else t["n_decode"]
            assert np.array_equal(toks[i, :n], ref[i, :n])


def test_runtime_decomposition_bit_exact(E):
    """§3.6: with a duration table where the GEMMs are much longer than the
    all-reduce windows, Algorithm 1 must split secondary GEMMs into k/F pieces
    (P:254-262); the result stays bit-identical to serial TP."""
    cfg = get_config("tiny")
    F = 8
    dur = []
    for m in (1, 4096):
        for op in ("qkv", "out", "fc1", "fc2"):
            for k in range(1, F + 1):
                dur.append((op, m, k, 20.0 + 200.0 * k / F))
        for op in ("ar1", "ar2"):
            for k in range(1, F + 1):
                dur.append((op, m, k, 10.0 + 60.0 * k / F))
    trace = make_trace(4, float("inf"), seed=12, batch_sizes=(2,), prompt_range=(16, 32), n_decode=4,
                       vocab=cfg.vocab)
    import os
    os.environ["LIGER_AR_DECOMP_MIN_KB"] = "0"   # tiny messages: all-reduces decomposable too
    try:
        base = serve_tp(E, cfg, 2, trace, mode="serial", max_batch=2, max_seq=32, max_new=4, seed=4)
        inter = serve_tp(E, cfg, 2, trace, durations=dur, mode="interleaved", max_batch=2, max_seq=32, max_new=4,
                         max_inflight=2, decomp_factor=F, contention_factor=1.0, seed=4)
    finally:
        os.environ.pop("LIGER_AR_DECOMP_MIN_KB", None)
    for (tb, _), (ti, st) in zip(base, inter):
        for a, b in zip(tb, ti):
            assert np.array_equal(a, b)
    assert inter[0][1]["split_pieces"] > 0, inter[0][1]


@pytest.mark.parametrize("world,mode", [(2, "pipeline"), (3, "pipeline"), (2, "pipeline_th"), (3, "pipeline_th")])
def test_pipeline_baseline_equals_single_gpu(E, world, mode):
    """Inter-operator pipeline baseline: `world` stages of unsharded layers,
    activations and tokens passed stage to stage; several batches in flight.
    The last stage's tokens are bit-identical to the single-GPU run (the same
    unsharded kernels).  Inter-Th issues every projection GEMM as `world`
    partitioned kernels (output-column slices of the full plan): the same bits."""
    from liger_inputs.configs import ModelConfig
    cfg = ModelConfig("tiny6", 6, 256, 4, 1024, 512, 64, "gelu_tanh")
    trace = make_trace(4, float("inf"), seed=13, batch_sizes=(1, 2), prompt_range=(8, 30), n_decode=5,
                       vocab=cfg.vocab)
    eng = E(cfg, mode="serial", max_batch=2, max_seq=32, max_new=8, seed=5)
    ids = [eng.submit(t["tokens"], t["batch"], t["seq_len"], t["n_decode"], 0.0) for t in trace]
    eng.drain()
    ref = [eng.poll(i, want_tokens=True)[1] for i in ids]
    eng.close()
    pipe = serve_tp(E, cfg, world, trace, mode=mode, max_batch=2, max_seq=32, max_new=8, max_inflight=world,
                    seed=5)
    toks, st = pipe[world - 1]
    for a, b in zip(ref, toks):
        assert np.array_equal(a, b)
    assert st["comm_kernels"] > 0


@pytest.mark.parametrize("world", [2, 4])
def test_oneshot_peer_allreduce_equals_rendezvous_reduction(E, world):
    """The one-shot peer-memory all-reduce (csrc/peer_ar.cu: epoch flags, rank-ordered
    fp32 sum) against the loopback backend's rendezvous reduction (same sum order):
    identical tokens, with prefill all-reduces above the one-shot cap (NCCL-style
    path) and decode ones below it, interleaved with decomposition."""
    import os
    cfg = get_config("tiny")
    trace = make_trace(4, float("inf"), seed=5, batch_sizes=(1, 2, 3), prompt_range=(8, 40), n_decode=5,
                       vocab=cfg.vocab)
    res = {}
    for flag in ("0", "1"):
        os.environ["LIGER_ONESHOT_AR"] = flag
        os.environ["LIGER_ONESHOT_MAX_KB"] = "16"   # tiny: decode messages one-shot, most prefill ones not
        try:
            res[flag] = serve_tp(E, cfg, world, trace, mode="interleaved", max_batch=4, max_seq=48, max_new=8,
                                 max_inflight=3, decomp_factor=8, seed=2)
        finally:
            os.environ.pop("LIGER_ONESHOT_AR", None)
            os.environ.pop("LIGER_ONESHOT_MAX_KB", None)
    for r in range(world):
        for a, b in zip(res["0"][r][0], res["1"][r][0]):
            assert np.array_equal(a, b)
        for a, b in zip(res["1"][0][0], res["1"][r][0]):   # every rank holds the same tokens
            assert np.array_equal(a, b)


@pytest.mark.parametrize("sync", ["cpu_gpu", "inter_stream"])
def test_sync_ablation_modes_bit_exact(E, sync):
    """§3.4 Fig. 8 / §4.5 ablation: the CPU-GPU-only and inter-stream-only
    synchronisation variants change when rounds are launched, never what they
    compute -- tokens bit-identical to the hybrid (default) schedule at TP = 2."""
    cfg = get_config("tiny")
    trace = make_trace(4, float("inf"), seed=21, batch_sizes=(1, 2, 3), prompt_range=(8, 40), n_decode=5,
                       vocab=cfg.vocab)
    kw = dict(mode="interleaved", max_batch=4, max_seq=48, max_new=8, max_inflight=3, decomp_factor=8, seed=6)
    hyb = serve_tp(E, cfg, 2, trace, **kw)
    alt = serve_tp(E, cfg, 2, trace, sync=sync, **kw)
    for (th, _), (ta, st) in zip(hyb, alt):
        for a, b in zip(th, ta):
            assert np.array_equal(a, b)
    assert alt[0][1]["overlapped_rounds"] > 0
    if sync == "inter_stream":
        assert alt[0][1]["wait_us"] == 0.0


@pytest.mark.parametrize("world", [2, 4])
def test_fused_gemm_allreduce_bit_exact(E, world):
    """§8(f) next row 4: the row-parallel GEMM's all-reduce fused into its split-K
    fixup (bf16 partial staged in peer-visible memory, epoch published with a
    system-scope release) and the following add + LN (waits for every peer, sums the
    staged rows in rank order) -- no all-reduce kernel.  Serial TP with the fusion
    must give the tokens of serial TP with the one-shot all-reduce kernel, bit for
    bit, on every rank; the config makes the decode projections split K (h = 1024)."""
    import os
    from liger_inputs.configs import ModelConfig
    from paper_conf_ppopp_duwjchcl24_b200 import liger as L
    cfg = ModelConfig("mid2", 2, 1024, 8, 4096, 1024, 96, "relu")
    hl, fl = cfg.hidden // world, cfg.ffn // world
    assert L.gemm_plan(3, cfg.hidden, fl)["splits"] > 1
    trace = make_trace(3, float("inf"), seed=8, batch_sizes=(1, 3), prompt_range=(10, 40), n_decode=5,
                       vocab=cfg.vocab)
    kw = dict(mode="serial", max_batch=4, max_seq=48, max_new=8, seed=9)
    res = {}
    for flag in ("0", "1"):
        os.environ["LIGER_FUSED_AR"] = flag
        try:
            res[flag] = serve_tp(E, cfg, world, trace, **kw)
        finally:
            os.environ.pop("LIGER_FUSED_AR", None)
    for r in range(world):
        for a, b in zip(res["0"][0][0], res["1"][r][0]):
            assert np.array_equal(a, b)
    # the fused run issued fewer all-reduce kernels (only those that could not fuse)
    assert res["1"][0][1]["comm_kernels"] < res["0"][0][1]["comm_kernels"]


def test_gemm_sm_reserve_bit_exact(E):
    """Contention control (§3.5): GEMM grids that leave SMs free for a
    concurrent all-reduce compute the same units, so tokens are bit-identical."""
    import os
    cfg = get_config("tiny")
    trace = make_trace(3, float("inf"), seed=31, batch_sizes=(1, 2), prompt_range=(8, 40), n_decode=5,
                       vocab=cfg.vocab)
    kw = dict(mode="interleaved", max_batch=4, max_seq=48, max_new=8, max_inflight=2, seed=10)
    ref = serve_tp(E, cfg, 2, trace, **kw)
    os.environ["LIGER_GEMM_SM_RESERVE"] = "145"   # 3-CTA grids: units wrap around
    try:
        alt = serve_tp(E, cfg, 2, trace, **kw)
    finally:
        os.environ.pop("LIGER_GEMM_SM_RESERVE", None)
    for (tr, _), (ta, _) in zip(ref, alt):
        for a, b in zip(tr, ta):
            assert np.array_equal(a, b)
