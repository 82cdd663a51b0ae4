"""End-to-end serving through liger_init / liger_load_layer / liger_submit /
liger_step / liger_poll on one GPU (t = 1), compared with the fp64 oracle element
by element (tests/engine_check.py): the LM-head input residual and the logits of
every pass through the C-ABI debug readback, and the greedy tokens.  The inputs are
non-degenerate (the oracle's tokens are not the echo of the prompt a model without
layers gives), and a deliberately broken layer makes the checks fail."""
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


def _with_env(env, fn):
    old = {k: os.environ.get(k) for k in env}
    os.environ.update(env)
    try:
        return fn()
    finally:
        for k, v in old.items():
            if v is None:
                os.environ.pop(k, None)
            else:
                os.environ[k] = v


def _mixed_trace(n, seed, cfg, batch_sizes, prompt_range, n_new_choices):
    """make_trace with a per-batch number of generated tokens (mixed n_new)."""
    tr = make_trace(n, float("inf"), seed=seed, batch_sizes=batch_sizes, prompt_range=prompt_range, n_decode=1,
                    vocab=cfg.vocab)
    rng = np.random.default_rng(seed + 1000)
    for t in tr:
        t["n_decode"] = int(rng.choice(n_new_choices))
    return tr


def test_tiny_serving_matches_oracle_elementwise(E):
    """BASELINE.json configs[0] shape (tiny, batch 2, prompt 32 + 8 generated) at t = 1:
    residual, logits and tokens of every pass against the oracle."""
    cfg = get_config("tiny")
    prompt = np.random.default_rng(0).integers(0, cfg.vocab, size=(2, 32)).astype(np.int32)
    trace = [dict(tokens=prompt.reshape(-1), batch=2, seq_len=32, n_decode=8)]
    res = serve(E, cfg, 1, trace, mode="serial", max_batch=4, max_seq=64, max_new=8, seed=0)
    check_vs_oracle(cfg, 0, trace, res)


def test_modes_bit_exact_and_match_oracle(E):
    """Serial intra-op, interleaved with F = 8 and a processing list of 3 (t = 1: the
    two-stream schedule, reading R31) over a trace with mixed batch sizes and mixed
    numbers of generated tokens: every mode equals the oracle element-wise and the
    modes are bit-identical to each other (tokens, logits, residual)."""
    cfg = get_config("tiny")
    trace = _mixed_trace(6, 3, cfg, (1, 2, 3), (5, 40), (2, 6, 8))
    results = {}
    for mode, infl, F in (("serial", 1, 1), ("interleaved", 2, 8), ("interleaved", 3, 1)):
        results[(mode, infl, F)] = serve(E, cfg, 1, trace, mode=mode, max_batch=4, max_seq=64, max_new=8,
                                         max_inflight=infl, decomp_factor=F, seed=1)
        st = results[(mode, infl, F)][0]["stats"]
        assert st["kernels"] > 0 and st["gpu_launches"] > 0
    base = results[("serial", 1, 1)]
    check_vs_oracle(cfg, 1, trace, base)
    for k, v in results.items():
        assert_bit_identical(base, v)


FOLD_CFGS = [ModelConfig("tiny3g", 3, 256, 4, 1024, 512, 96, "gelu_tanh"),
             ModelConfig("mid3", 3, 1024, 8, 4096, 1024, 96, "relu")]


@pytest.mark.parametrize("cfg", FOLD_CFGS, ids=lambda c: c.name)
@pytest.mark.parametrize("fold", ["1", "0"])
def test_ln_fold_decode_matches_oracle(E, cfg, fold):
    """The default t = 1 decode path -- LayerNorm folded into the QKV / FC1 GEMMs
    (W*gamma weights, in-kernel row statistics, u / c epilogue vectors) and the
    residual adds in the out-proj / FC2 epilogues -- and the unfolded path
    (LIGER_LN_FOLD=0), at decode batches b = 1, 2, 8 and 16, element-wise against the
    oracle.  h = 1024 exercises the split-K fixup epilogue, h = 256 the single-chunk one."""
    trace = []
    for i, b in enumerate((1, 2, 8, 16)):
        trace += make_trace(1, float("inf"), seed=40 + i, batch_sizes=(b,), prompt_range=(20, 60), n_decode=6,
                            vocab=cfg.vocab)
    res = _with_env({"LIGER_LN_FOLD": fold}, lambda: serve(E, cfg, 1, trace, mode="interleaved", max_batch=16,
                                                           max_seq=64, max_new=8, seed=7))
    check_vs_oracle(cfg, 7, trace, res)


def test_ln_fold_full_size_opt13b_layer(E):
    """The bench's launch configuration at full width: an OPT-13B-shaped model cut to
    one decoder layer (h = 5120, ffn 20480, vocab 50272, ReLU) served at t = 1 with the
    default folded decode path (split-K QKV / FC1 with the folded LN, out-proj / FC2
    fixups with the residual add), b = 2 and 8, element-wise against the oracle."""
    cfg = ModelConfig("opt13b-L1", 1, 5120, 40, 20480, 50272, 64, "relu")
    trace = (make_trace(1, float("inf"), seed=9, batch_sizes=(2,), prompt_range=(24, 24), n_decode=6,
                        vocab=cfg.vocab) +
             make_trace(1, float("inf"), seed=10, batch_sizes=(8,), prompt_range=(17, 17), n_decode=4,
                        vocab=cfg.vocab))
    res = serve(E, cfg, 1, trace, mode="interleaved", max_batch=8, max_seq=24, max_new=6, seed=1)
    check_vs_oracle(cfg, 1, trace, res)


def test_full_size_opt13b_two_stream_equals_serial(E):
    """bench.py's launch configuration at full size (OPT-13B, 40 layers, t = 1): 4 batches of
    the bench's mixed trace (b in {2, 4, 8}, prompts U[128, 512], 32 generated tokens) served
    by the interleaved mode (the pass-by-pass two-stream schedule, folded LN) and by serial
    intra-op TP give identical tokens, logits and last-layer residuals bit for bit (a
    property that holds at any size; the oracle's element-wise checks run at the sizes it
    finishes in seconds).  The tokens are valid ids, not the echo of the last prompt token."""
    cfg = get_config("opt-13b")
    trace = make_trace(4, float("inf"), seed=3, vocab=cfg.vocab, n_decode=32)
    kw = dict(max_batch=8, max_seq=512, max_new=32, seed=0)
    two = serve(E, cfg, 1, trace, mode="interleaved", **kw)
    ser = serve(E, cfg, 1, trace, mode="serial", **kw)
    assert_bit_identical(two, ser)
    for t, toks, lg in zip(trace, two[0]["tokens"], two[0]["logits"]):
        assert toks.shape == (t["batch"], 32) and toks.min() >= 0 and toks.max() < cfg.vocab
        assert np.isfinite(lg).all()
        assert np.mean(toks != t["tokens"].reshape(t["batch"], -1)[:, -1:]) >= 0.5


@pytest.mark.parametrize("skip", ["fc2", "attn", "out"])
def test_broken_layer_fails_the_check(E, skip):
    """The checks can fail: a decoder-layer kernel skipped (LIGER_DBG_SKIP, a timing
    experiment switch that leaves its output buffer stale) must break the
    element-wise comparison with the oracle."""
    cfg = get_config("tiny")
    prompt = np.random.default_rng(0).integers(0, cfg.vocab, size=(2, 32)).astype(np.int32)
    trace = [dict(tokens=prompt.reshape(-1), batch=2, seq_len=32, n_decode=8)]
    res = _with_env({"LIGER_DBG_SKIP": skip},
                    lambda: serve(E, cfg, 1, trace, mode="serial", max_batch=4, max_seq=64, max_new=8, seed=0))
    with pytest.raises(AssertionError):
        check_vs_oracle(cfg, 0, trace, res)


def test_device_resident_tokens_and_latency_fields(E):
    cfg = get_config("tiny")
    eng = E(cfg, mode="interleaved", max_batch=2, max_seq=16, max_new=4, seed=0)
    toks = torch.randint(0, cfg.vocab, (2 * 16,), dtype=torch.int32, device="cuda")
    bid = eng.submit(None, 2, 16, 4, arrival_s=0.0, device_tokens=toks)
    eng.drain()
    res, _ = eng.poll(bid)
    assert res.done == 1 and res.finish_s >= res.start_s >= res.submit_s > 0
    eng.close()


def test_result_tokens_device_states(E):
    """liger_result_tokens_device: PENDING before the batch finished, the tokens after,
    ESTATE once a later batch reused the slot."""
    import ctypes as C
    from paper_conf_ppopp_duwjchcl24_b200 import liger as L
    cfg = get_config("tiny")
    eng = E(cfg, mode="serial", max_batch=2, max_seq=16, max_new=4, seed=0)
    p = np.random.default_rng(5).integers(0, cfg.vocab, size=2 * 16).astype(np.int32)
    bid = eng.submit(p, 2, 16, 4, 0.0)
    ptr = C.c_void_p()
    assert L.lib().liger_result_tokens_device(eng.ctx, bid, C.byref(ptr)) == L.LIGER_PENDING
    eng.drain()
    assert L.lib().liger_result_tokens_device(eng.ctx, bid, C.byref(ptr)) == L.LIGER_OK
    assert ptr.value
    host = eng.poll(bid, want_tokens=True)[1]
    for _ in range(3):   # serial mode: 2 slots -> the first one is reused
        eng.submit(p, 2, 16, 4, 0.0)
    eng.drain()
    assert L.lib().liger_result_tokens_device(eng.ctx, bid, C.byref(ptr)) == L.LIGER_ESTATE
    assert host.shape == (2, 4)
    eng.close()


def test_submit_rejects_bad_shapes(E):
    from paper_conf_ppopp_duwjchcl24_b200.liger import LigerError
    cfg = get_config("tiny")
    eng = E(cfg, max_batch=2, max_seq=16, max_new=4, seed=0)
    with pytest.raises(LigerError):
        eng.submit(np.zeros(3 * 8, np.int32), 3, 8, 2)     # batch > max_batch
    with pytest.raises(LigerError):
        eng.submit(np.zeros(2 * 17, np.int32), 2, 17, 2)   # prompt > max_seq
    eng.close()


def test_contention_factor_calibration(E):
    """cf = max slowdown of GEMM / all-reduce run concurrently (>= 1)."""
    cfg = get_config("tiny")
    eng = E(cfg, max_batch=2, max_seq=32, max_new=4, seed=0)
    cf, detail = eng.calibrate_cf([16, 64])
    eng.close()
    assert 1.0 <= cf < 10.0
    assert set(detail) == {16, 64} and all(len(v) == 4 for v in detail.values())


def test_nccl_oneshot_setup_and_kernel_single_rank(E):
    """The NCCL backend's one-shot path on real hardware at one rank: liger_calibrate_cf
    at t = 1 runs its all-reduces on a 1-rank NCCL communicator; with LIGER_ONESHOT_AR=1
    its creation sets up the CUDA-IPC staging eagerly (with the NCCL agreement on it)
    and the all-reduces run the one-shot kernel -- with the GEMM SM reserve on."""
    cfg = get_config("tiny")

    def run():
        eng = E(cfg, max_batch=2, max_seq=32, max_new=4, seed=0)
        eng.set_gemm_sm_reserve(16)
        cf, _ = eng.calibrate_cf([16, 64], set_cf=False)
        eng.close()
        return cf
    cf = _with_env({"LIGER_ONESHOT_AR": "1"}, run)
    assert 1.0 <= cf < 10.0
