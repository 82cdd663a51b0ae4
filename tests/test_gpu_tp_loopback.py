"""Tensor-parallel serving on ONE GPU with the loopback communicator: t ranks are
threads of this process, each with its own liger context (own shard, streams,
scheduler), collectives via host rendezvous + rank-ordered device reductions (stream
waits on the peers' events; no kernel of one rank waits on another rank's kernel: they
share one GPU, where such kernels are not guaranteed to be co-scheduled).

This runs the complete t > 1 path of the product -- all-reduces on the
communication stream, Algorithm 1 rounds with real secondary subsets, runtime
decomposition, hybrid E1/E2 synchronisation, the vocab-parallel LM head's
all-gather -- and checks BASELINE.json's requirements element by element against
the oracle (tests/engine_check.py: residual, logits shards concatenated, tokens),
plus bit-exactness between the schedules (interleaved vs serial, sync modes, the
pipeline baselines).  The peer-memory all-reduce kernels (one-shot, fused GEMM +
all-reduce) are checked phase by phase in tests/test_gpu_peer_ar.py."""
import os

import numpy as np
import pytest
import torch

from liger_inputs import get_config, make_trace
from liger_inputs.configs import ModelConfig
from engine_check import serve, check_vs_oracle, assert_bit_identical

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def E():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_ppopp_duwjchcl24_b200.engine import LigerEngine
    return LigerEngine


class env:
    def __init__(self, **kv):
        self.kv = kv

    def __enter__(self):
        self.old = {k: os.environ.get(k) for k in self.kv}
        os.environ.update(self.kv)

    def __exit__(self, *a):
        for k, v in self.old.items():
            if v is None:
                os.environ.pop(k, None)
            else:
                os.environ[k] = v


def _mixed_trace(n, seed, cfg, batch_sizes, prompt_range, n_new_choices):
    tr = make_trace(n, float("inf"), seed=seed, batch_sizes=batch_sizes, prompt_range=prompt_range, n_decode=1,
                    vocab=cfg.vocab)
    rng = np.random.default_rng(seed + 1000)
    for t in tr:
        t["n_decode"] = int(rng.choice(n_new_choices))
    return tr


def test_tiny_tp2_matches_oracle(E):
    """BASELINE.json configs[0]: tiny, TP=2, batch 2, prompt 32 + 8 decode tokens --
    residual, logits (both vocabulary shards) and tokens against the oracle; both
    ranks hold the same residual and tokens bit for bit."""
    cfg = get_config("tiny")
    prompt = np.random.default_rng(0).integers(0, cfg.vocab, size=(2, 32)).astype(np.int32)
    trace = [dict(tokens=prompt.reshape(-1), batch=2, seq_len=32, n_decode=8)]
    res = serve(E, cfg, 2, trace, mode="interleaved", max_batch=2, max_seq=32, max_new=8, seed=0)
    check_vs_oracle(cfg, 0, trace, res, world=2)
    assert all(r["stats"]["comm_kernels"] > 0 for r in res)


@pytest.mark.parametrize("world", [2, 4])
def test_interleaved_equals_serial_and_oracle(E, world):
    """Several batches with mixed sizes and mixed numbers of generated tokens in
    flight: Algorithm 1 interleaves one batch's all-reduces with another's GEMMs
    (secondary subsets, decomposition pieces; every all-reduce decomposable, at t > 2
    issued as atomic 1/F chunks).  Serial intra-op TP matches the oracle
    element-wise, and interleaved is bit-identical to it on every rank."""
    cfg = get_config("tiny")
    trace = _mixed_trace(5, 11, cfg, (1, 2, 3), (8, 40), (3, 6, 8))
    with env(LIGER_AR_DECOMP_MIN_KB="0"):
        base = serve(E, cfg, world, trace, mode="serial", max_batch=4, max_seq=64, max_new=8, seed=3)
        inter = serve(E, cfg, world, trace, mode="interleaved", max_batch=4, max_seq=64, max_new=8,
                      max_inflight=3, decomp_factor=8, contention_factor=1.0, seed=3)
    check_vs_oracle(cfg, 3, trace, base, world=world)
    assert_bit_identical(base, inter)
    st = inter[0]["stats"]
    assert st["overlapped_rounds"] > 0, st      # secondary subsets were actually scheduled
    assert st["comm_kernels"] > 0


def test_runtime_decomposition_bit_exact_and_oracle(E):
    """§3.6: with a duration table where the GEMMs are much longer than the
    all-reduce windows, Algorithm 1 splits secondary GEMMs into k/F pieces
    (P:254-262); the result equals the oracle and is bit-identical to serial TP."""
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
    with env(LIGER_AR_DECOMP_MIN_KB="0"):
        base = serve(E, cfg, 2, trace, mode="serial", max_batch=2, max_seq=32, max_new=4, seed=4)
        inter = serve(E, cfg, 2, trace, durations=dur, mode="interleaved", max_batch=2, max_seq=32, max_new=4,
                      max_inflight=2, decomp_factor=F, contention_factor=1.0, seed=4)
    check_vs_oracle(cfg, 4, trace, inter, world=2)
    assert_bit_identical(base, inter)
    assert inter[0]["stats"]["split_pieces"] > 0, inter[0]["stats"]


@pytest.mark.parametrize("world,mode", [(2, "pipeline"), (3, "pipeline"), (2, "pipeline_th"), (3, "pipeline_th")])
def test_pipeline_baselines_match_oracle(E, world, mode):
    """Inter-operator pipeline baseline: `world` stages of unsharded layers,
    activations and tokens passed stage to stage; several batches with mixed numbers
    of generated tokens in flight (stages finish batches out of submit order).  The
    last stage's residual, logits and tokens equal the oracle element-wise and the
    single-GPU run bit for bit.  Inter-Th issues every projection GEMM as
    `world` partitioned kernels (output-column slices of the full plan): the same bits."""
    cfg = ModelConfig("tiny6", 6, 256, 4, 1024, 512, 64, "gelu_tanh")
    trace = _mixed_trace(5, 13, cfg, (1, 2), (8, 30), (2, 5, 8))
    single = serve(E, cfg, 1, trace, mode="serial", max_batch=2, max_seq=32, max_new=8, seed=5)
    pipe = serve(E, cfg, world, trace, mode=mode, max_batch=2, max_seq=32, max_new=8, max_inflight=world, seed=5)
    check_vs_oracle(cfg, 5, trace, pipe, world=world, mode=mode)
    assert_bit_identical(single, [pipe[world - 1]])
    assert pipe[world - 1]["stats"]["comm_kernels"] > 0


def test_full_size_opt13b_tp2_interleaved_equals_serial(E):
    """BASELINE.json configs[1] at full size: OPT-13B (40 layers) at TP = 2 (loopback ranks),
    3 batches of the bench's mixed trace served by Algorithm 1 (interleaved, F = 8, prefill
    all-reduces decomposed, hybrid sync) and by serial intra-op TP: identical tokens, logits
    and last-layer residuals bit for bit on both ranks, with secondary subsets and split
    pieces actually issued."""
    cfg = get_config("opt-13b")
    trace = make_trace(3, float("inf"), seed=4, vocab=cfg.vocab, n_decode=6)
    kw = dict(max_batch=8, max_seq=512, max_new=8, seed=0)
    inter = serve(E, cfg, 2, trace, mode="interleaved", max_inflight=2, decomp_factor=8, **kw)
    ser = serve(E, cfg, 2, trace, mode="serial", **kw)
    assert_bit_identical(inter, ser)
    for a, b in zip(inter[0]["tokens"] + inter[0]["resid"], inter[1]["tokens"] + inter[1]["resid"]):
        assert np.array_equal(a, b)   # both ranks hold the same tokens and residual stream
    st = inter[0]["stats"]
    assert st["overlapped_rounds"] > 0 and st["split_pieces"] > 0 and st["comm_kernels"] > 0


def test_full_size_opt30b_tp4_modes(E):
    """BASELINE.json configs[2] at full size: OPT-30B (48 layers, h = 7168) with 2 request
    batches -- Algorithm 1 interleaving at TP = 4 equals serial TP = 4 bit for bit (tokens,
    logits shards, residuals; all ranks the same residual), and the 4-stage Inter-Op
    pipeline equals the unsharded single-GPU run bit for bit."""
    cfg = get_config("opt-30b")
    trace = make_trace(2, float("inf"), seed=6, vocab=cfg.vocab, n_decode=4, prompt_range=(128, 256))
    kw = dict(max_batch=8, max_seq=256, max_new=4, seed=0)
    inter = serve(E, cfg, 4, trace, mode="interleaved", max_inflight=2, decomp_factor=8, **kw)
    ser = serve(E, cfg, 4, trace, mode="serial", **kw)
    assert_bit_identical(inter, ser)
    for r in range(1, 4):
        for a, b in zip(inter[0]["tokens"] + inter[0]["resid"], inter[r]["tokens"] + inter[r]["resid"]):
            assert np.array_equal(a, b)
    del inter, ser
    pipe = serve(E, cfg, 4, trace, mode="pipeline", max_inflight=4, **kw)
    single = serve(E, cfg, 1, trace, mode="serial", **kw)
    assert_bit_identical(single, [pipe[3]])


def test_full_size_opt66b_tp8_interleaved_equals_serial(E):
    """BASELINE.json configs[3] at full size: OPT-66B (64 layers, h = 9216) at TP = 8 (eight
    loopback ranks, 16.5 GB of weights each, on the one GPU), kernel decomposition on:
    Algorithm 1 interleaving equals serial TP bit for bit, every rank the same residual."""
    cfg = get_config("opt-66b")
    trace = make_trace(2, float("inf"), seed=8, vocab=cfg.vocab, n_decode=3, batch_sizes=(2, 4),
                       prompt_range=(64, 128))
    kw = dict(max_batch=4, max_seq=128, max_new=3, seed=0)
    inter = serve(E, cfg, 8, trace, mode="interleaved", max_inflight=2, decomp_factor=8, **kw)
    ser = serve(E, cfg, 8, trace, mode="serial", **kw)
    assert_bit_identical(inter, ser)
    for r in range(1, 8):
        for a, b in zip(inter[0]["tokens"] + inter[0]["resid"], inter[r]["tokens"] + inter[r]["resid"]):
            assert np.array_equal(a, b)
    assert inter[0]["stats"]["overlapped_rounds"] > 0


def test_glm130b_layer_stack_tp8_cf_sweep(E):
    """BASELINE.json configs[4] shape: a GLM-130B-shaped layer stack (h = 12288, 96 heads,
    FFN 49152, tanh-GELU, vocab 150528; 6 of the 70 layers, which is what fits eight ranks on
    one GPU) at TP = 8 with long prompts of 2048 tokens (100 MB prefill all-reduces,
    decomposed): the contention-factor sweep of the scheduler (cf 1.0 / 1.1 / 1.3)
    changes which kernels overlap, never the results -- every cf's run equals serial TP bit
    for bit."""
    cfg = get_config("glm-130b", 6)
    trace = make_trace(2, float("inf"), seed=12, vocab=cfg.vocab, n_decode=3, batch_sizes=(1, 2),
                       prompt_range=(2048, 2048))
    kw = dict(max_batch=2, max_seq=2048, max_new=3, seed=0)
    ser = serve(E, cfg, 8, trace, mode="serial", **kw)
    rounds = {}
    for cf in (1.0, 1.1, 1.3):
        inter = serve(E, cfg, 8, trace, mode="interleaved", max_inflight=2, decomp_factor=8, contention_factor=cf,
                      **kw)
        assert_bit_identical(inter, ser)
        rounds[cf] = inter[0]["stats"]["overlapped_rounds"]
    assert all(v > 0 for v in rounds.values()), rounds


@pytest.mark.parametrize("lead", ["0", "1000000"])
def test_e1_placement_bit_exact(E, lead):
    """Hybrid sync E1 placement (DESIGN R8): the paper's (before the switch kernel, lead 0)
    and the earliest (before the first SubSet0 kernel, a lead no round reaches) change only
    when the host wakes up -- bit-identical to the default duration-aware placement, which
    matches the oracle element-wise, at TP = 2 with decomposition."""
    cfg = get_config("tiny")
    trace = _mixed_trace(4, 23, cfg, (1, 2, 3), (8, 40), (3, 5))
    kw = dict(mode="interleaved", max_batch=4, max_seq=48, max_new=8, max_inflight=3, decomp_factor=8, seed=7)
    ref = serve(E, cfg, 2, trace, **kw)
    with env(LIGER_E1_LEAD_US=lead):
        alt = serve(E, cfg, 2, trace, **kw)
    check_vs_oracle(cfg, 7, trace, ref, world=2)
    assert_bit_identical(ref, alt)
    assert alt[0]["stats"]["overlapped_rounds"] > 0


@pytest.mark.parametrize("sync", ["cpu_gpu", "inter_stream"])
def test_sync_ablation_modes_bit_exact(E, sync):
    """§3.4 Fig. 8 / §4.5 ablation: the CPU-GPU-only and inter-stream-only
    synchronisation variants change when rounds are launched, never what they
    compute -- bit-identical to the hybrid (default) schedule at TP = 2, which
    matches the oracle element-wise."""
    cfg = get_config("tiny")
    trace = _mixed_trace(4, 21, cfg, (1, 2, 3), (8, 40), (3, 5))
    kw = dict(mode="interleaved", max_batch=4, max_seq=48, max_new=8, max_inflight=3, decomp_factor=8, seed=6)
    hyb = serve(E, cfg, 2, trace, **kw)
    alt = serve(E, cfg, 2, trace, sync=sync, **kw)
    check_vs_oracle(cfg, 6, trace, hyb, world=2)
    assert_bit_identical(hyb, alt)
    assert alt[0]["stats"]["overlapped_rounds"] > 0
    if sync == "inter_stream":
        assert alt[0]["stats"]["wait_us"] == 0.0


def test_gemm_sm_reserve_bit_exact(E):
    """Contention control (§3.5): GEMM grids that leave SMs free for a
    concurrent all-reduce compute the same units, so results are bit-identical."""
    cfg = get_config("tiny")
    trace = make_trace(3, float("inf"), seed=31, batch_sizes=(1, 2), prompt_range=(8, 40), n_decode=5,
                       vocab=cfg.vocab)
    kw = dict(mode="interleaved", max_batch=4, max_seq=48, max_new=8, max_inflight=2, seed=10)
    ref = serve(E, cfg, 2, trace, **kw)
    with env(LIGER_GEMM_SM_RESERVE="145"):   # 3-CTA grids: units wrap around
        alt = serve(E, cfg, 2, trace, **kw)
    assert_bit_identical(ref, alt)


@pytest.mark.parametrize("skip", ["ar2", "fc2"])
def test_broken_tp_layer_fails_the_check(E, skip):
    """The TP checks can fail: skipping a rank's all-reduce #2 (each rank keeps its own
    partial) or its FC2 breaks the element-wise comparison with the oracle."""
    cfg = get_config("tiny")
    prompt = np.random.default_rng(0).integers(0, cfg.vocab, size=(2, 32)).astype(np.int32)
    trace = [dict(tokens=prompt.reshape(-1), batch=2, seq_len=32, n_decode=8)]
    with env(LIGER_DBG_SKIP=skip):
        res = serve(E, cfg, 2, trace, mode="serial", max_batch=2, max_seq=32, max_new=8, seed=0)
    with pytest.raises(AssertionError):
        check_vs_oracle(cfg, 0, trace, res, world=2)


@pytest.mark.parametrize("world", [2, 4])
def test_allreduce_op_vs_oracle_and_decomposition(E, world):
    """a6 / a10 / a13 element-wise: liger_op_allreduce on seeded bf16 partials (one
    per rank), whole and as decomposed pieces, against the oracle's
    allreduce_decomposed (fp64 sum of the bf16 partials).  The sum of t <= 4
    bf16 values of one magnitude range is exact in fp32, so the rank-ordered fp32 sum
    rounded to bf16 must equal bf16_rne(oracle) bit for bit; every split gives the
    bits of the whole all-reduce.  Sizes: a decode-size message and a prefill-size one.
    (The one-shot peer kernel is checked phase by phase in tests/test_gpu_peer_ar.py: the
    loopback backend's ranks share one GPU and never run kernels that wait on each other.)"""
    from liger_inputs import c0_values, bf16_rne
    from oracle import model as om
    cfg = get_config("tiny")
    F = 8
    sizes = (8 * 256, 96 * 256)
    splits = ([8], [2, 3, 3], [1] * 8, [5, 3])
    uid = E.loopback_id()
    # C0 values with magnitudes clipped to [2^-10, 2^-3] (exponent gap <= 7: a sum of
    # four needs <= 17 significant bits, exact in fp32)
    def part(q, n):
        v = c0_values(77, 100 + q, np.arange(n, dtype=np.uint64), -3)
        return np.where(np.abs(v) < 2.0 ** -10, np.where(v < 0, -(2.0 ** -10), 2.0 ** -10), v).astype(np.float32)
    parts = {n: [part(q, n) for q in range(world)] for n in sizes}
    got = {}
    err = []
    import threading
    bar = threading.Barrier(world)

    def rank_main(r):
        # Inputs are staged before any all-reduce, the all-reduces run on the rank's own
        # stream, and results are read after a barrier.
        try:
            torch.cuda.set_device(0)
            eng = E(cfg, world=world, rank=r, nccl_uid=uid, max_batch=2, max_seq=16, max_new=2, seed=0, load=False)
            bufs = {(n, tuple(ks)): torch.from_numpy(parts[n][r]).cuda().bfloat16() for n in sizes for ks in splits}
            torch.cuda.synchronize()
            bar.wait()
            st = torch.cuda.Stream()
            for n in sizes:
                for ks in splits:
                    u = 0
                    for k in ks:
                        eng.allreduce(bufs[(n, tuple(ks))], u, u + k, F, stream=st.cuda_stream)
                        u += k
            st.synchronize()
            bar.wait()
            for key, b in bufs.items():
                got[(r,) + key] = b.float().cpu().numpy()
            bar.wait()
            eng.close()
        except Exception as e:
            err.append(repr(e))
            bar.abort()

    import threading
    ths = [threading.Thread(target=rank_main, args=(r,), daemon=True) for r in range(world)]
    for t in ths:
        t.start()
    for t in ths:
        t.join(timeout=300)
    assert not err, err
    for n in sizes:
        for ks in splits:
            ref = om.allreduce_decomposed([p.astype(np.float64) for p in parts[n]], F, ks)
            want = bf16_rne(ref.astype(np.float32))
            for r in range(world):
                assert np.array_equal(got[(r, n, tuple(ks))].view(np.uint32), want.view(np.uint32)), (r, n, ks)


def _host_shard(cfg, seed, t, r):
    """Rank r's shard of every layer and the embeddings as bf16 torch tensors on the GPU,
    built on the HOST from the numpy C0 generator (liger_inputs; not the library's init)."""
    from liger_inputs import layer_tensor, global_tensor
    h, a, f = cfg.hidden, cfg.n_heads, cfg.ffn
    hl, fl = h // t, f // t
    dev = lambda x: torch.from_numpy(np.ascontiguousarray(x, dtype=np.float32)).cuda().bfloat16()
    layers = []
    for l in range(cfg.n_layers):
        wq = layer_tensor(cfg, seed, l, "w_qkv")                 # [h, 3h] logical
        bq = layer_tensor(cfg, seed, l, "b_qkv")
        cols = np.r_[r * hl:(r + 1) * hl, h + r * hl:h + (r + 1) * hl, 2 * h + r * hl:2 * h + (r + 1) * hl]
        layers.append(dict(
            w_qkv=dev(wq[:, cols].T), b_qkv=dev(bq[cols]),
            w_o=dev(layer_tensor(cfg, seed, l, "w_o")[r * hl:(r + 1) * hl, :].T), b_o=dev(layer_tensor(cfg, seed, l, "b_o")),
            w_1=dev(layer_tensor(cfg, seed, l, "w_1")[:, r * fl:(r + 1) * fl].T),
            b_1=dev(layer_tensor(cfg, seed, l, "b_1")[r * fl:(r + 1) * fl]),
            w_2=dev(layer_tensor(cfg, seed, l, "w_2")[r * fl:(r + 1) * fl, :].T), b_2=dev(layer_tensor(cfg, seed, l, "b_2")),
            ln1_g=dev(layer_tensor(cfg, seed, l, "ln1_g")), ln1_b=dev(layer_tensor(cfg, seed, l, "ln1_b")),
            ln2_g=dev(layer_tensor(cfg, seed, l, "ln2_g")), ln2_b=dev(layer_tensor(cfg, seed, l, "ln2_b"))))
    embed = {k: dev(global_tensor(cfg, seed, k)) for k in ("e_tok", "e_pos", "lnf_g", "lnf_b")}
    return layers, embed


@pytest.mark.parametrize("world", [1, 2])
def test_caller_owned_weights_and_streams(E, world):
    """§8(b) boundary: weights passed in as caller-owned torch tensors
    (liger_load_layer_weights / liger_load_embed_weights, copied by the library) and the
    serving run on caller-owned torch streams (liger_set_streams) give the bits of the
    seeded-init engine and the oracle element-wise, at t = 1 (LN fold) and loopback t = 2."""
    import threading
    cfg = get_config("tiny")
    trace = _mixed_trace(3, 9, cfg, (1, 2), (8, 30), (3, 5))
    kw = dict(mode="interleaved", max_batch=2, max_seq=32, max_new=8, seed=11)
    ref = serve(E, cfg, world, trace, **kw)
    uid = E.loopback_id() if world > 1 else None
    out = [None] * world
    err = []
    bar = threading.Barrier(world)

    def rank_main(r):
        try:
            torch.cuda.set_device(0)
            layers, embed = _host_shard(cfg, 11, world, r)
            eng = E(cfg, world=world, rank=r, nccl_uid=uid, load=False, **kw)
            eng.load_weights(layers, embed)
            s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()
            eng.set_streams(s1.cuda_stream, s2.cuda_stream)
            eng.set_debug_capture()
            ids = [eng.submit(t["tokens"], t["batch"], t["seq_len"], t["n_decode"], 0.0) for t in trace]
            eng.drain()
            out[r] = dict(tokens=[eng.poll(i, want_tokens=True)[1] for i in ids], stats=eng.stats(),
                          logits=[eng.debug_read(i, "logits", t["batch"], t["n_decode"]) for i, t in zip(ids, trace)],
                          resid=[eng.debug_read(i, "resid", t["batch"], t["n_decode"]) for i, t in zip(ids, trace)])
            bar.wait()
            eng.close()
            del layers, embed
        except Exception as e:
            err.append(repr(e))
            bar.abort()

    ths = [threading.Thread(target=rank_main, args=(r,), daemon=True) for r in range(world)]
    for t in ths:
        t.start()
    for t in ths:
        t.join(timeout=300)
    assert not err, err
    assert_bit_identical(ref, out)
    check_vs_oracle(cfg, 11, trace, out, world=world)


def test_profile_and_contention_factor_across_ranks(E):
    """a16: the offline profile and the contention-factor calibration run
    with real cross-rank all-reduces (loopback TP = 2: every all-reduce a collective of the
    two rank threads); the ranks agree on the result (max over ranks), cf >= 1, and the
    agreed tables drive identical plans: interleaved serving on both ranks afterwards stays
    bit-identical to serial TP and equal to the oracle."""
    import threading
    cfg = get_config("tiny")
    uid = E.loopback_id()
    trace = _mixed_trace(3, 9, cfg, (1, 2), (8, 30), (3, 5))
    cfs = [None, None]
    res = [None, None]
    err = []

    def rank_main(r):
        try:
            torch.cuda.set_device(0)
            eng = E(cfg, world=2, rank=r, nccl_uid=uid, mode="interleaved", max_batch=2, max_seq=32, max_new=8,
                    max_inflight=2, seed=11)
            eng.profile([2, 16, 64])
            cf, detail = eng.calibrate_cf([16, 64], set_cf=True)
            cfs[r] = (cf, detail)
            eng.set_debug_capture()
            ids = [eng.submit(t["tokens"], t["batch"], t["seq_len"], t["n_decode"], 0.0) for t in trace]
            eng.drain()
            res[r] = dict(tokens=[eng.poll(i, want_tokens=True)[1] for i in ids], stats=eng.stats(),
                          logits=[eng.debug_read(i, "logits", t["batch"], t["n_decode"]) for i, t in zip(ids, trace)],
                          resid=[eng.debug_read(i, "resid", t["batch"], t["n_decode"]) for i, t in zip(ids, trace)])
            eng.close()
        except Exception as e:
            err.append(repr(e))

    ths = [threading.Thread(target=rank_main, args=(r,), daemon=True) for r in range(2)]
    for t in ths:
        t.start()
    for t in ths:
        t.join(timeout=300)
    assert not err, err
    assert cfs[0][0] == cfs[1][0] and 1.0 <= cfs[0][0] < 100.0, cfs
    assert set(cfs[0][1]) == {16, 64}
    base = serve(E, cfg, 2, trace, mode="serial", max_batch=2, max_seq=32, max_new=8, seed=11)
    assert_bit_identical(base, res)
    check_vs_oracle(cfg, 11, trace, res, world=2)
