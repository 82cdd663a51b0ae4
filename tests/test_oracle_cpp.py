"""Pins of the fp32 C++ CPU oracle (oracle/layer_ref.cpp; the BASELINE.md CPU baseline)
against the fp64 numpy oracle (oracle/model.py, itself pinned to HF OPT in
test_oracle_pins.py): prefill and decode steps of one decoder layer, tanh-GELU and
ReLU, within fp32 rounding."""
import ctypes as C

import numpy as np
import pytest

from liger_inputs.configs import ModelConfig
from oracle import model as om


@pytest.fixture(scope="module")
def ref_lib():
    from paper_conf_ppopp_duwjchcl24_b200.build import build_oracle
    _, so = build_oracle()
    lib = C.CDLL(so)
    lib.ref_decoder_layer.restype = C.c_int
    return lib


def _f(a):
    a = np.ascontiguousarray(a, dtype=np.float32)
    return a, a.ctypes.data_as(C.POINTER(C.c_float))


@pytest.mark.parametrize("act", ["gelu_tanh", "relu"])
def test_cpp_layer_matches_numpy_oracle(ref_lib, act):
    cfg = ModelConfig("t", 1, 128, 4, 512, 64, 64, act)
    w = om.layer_weights(cfg, 3, 0)
    h, a, f = cfg.hidden, cfg.n_heads, cfg.ffn
    b, s, cap = 2, 9, 16
    rng = np.random.default_rng(0)
    x = rng.standard_normal((b, s + 2, h)) * 0.3
    keep = []

    def P(arr):
        arr, p = _f(arr)
        keep.append(arr)
        return p
    wt = {k: P(w[k].T) for k in ("w_qkv", "w_o", "w_1", "w_2")}
    vec = {k: P(w[k]) for k in ("b_qkv", "b_o", "b_1", "b_2", "ln1_g", "ln1_b", "ln2_g", "ln2_b")}
    kc = np.zeros((b, a, cap, h // a), np.float32)
    vc = np.zeros_like(kc)

    def run(xin, start):
        xin, xp = _f(xin)
        out = np.zeros_like(xin)
        rc = ref_lib.ref_decoder_layer(b, xin.shape[1], start, h, a, f, 1 if act == "relu" else 2, C.c_float(1e-5),
                                       xp, vec["ln1_g"], vec["ln1_b"], wt["w_qkv"], vec["b_qkv"], wt["w_o"],
                                       vec["b_o"], vec["ln2_g"], vec["ln2_b"], wt["w_1"], vec["b_1"], wt["w_2"],
                                       vec["b_2"], kc.ctypes.data_as(C.POINTER(C.c_float)),
                                       vc.ctypes.data_as(C.POINTER(C.c_float)), cap,
                                       out.ctypes.data_as(C.POINTER(C.c_float)))
        assert rc == 0
        return out
    got_pf = run(x[:, :s], 0)
    got_d1 = run(x[:, s:s + 1], s)
    got_d2 = run(x[:, s + 1:s + 2], s + 1)
    ref_pf, k, v = om.decoder_layer(cfg, w, x[:, :s])
    ref_d1, k, v = om.decoder_layer(cfg, w, x[:, s:s + 1], k, v, start_pos=s)
    ref_d2, k, v = om.decoder_layer(cfg, w, x[:, s + 1:s + 2], k, v, start_pos=s + 1)
    for got, ref in ((got_pf, ref_pf), (got_d1, ref_d1), (got_d2, ref_d2)):
        assert np.abs(got - ref).max() <= 2e-5 * np.abs(ref).max() + 1e-6
    # the cache the C++ layer wrote holds the numpy oracle's K / V
    assert np.abs(kc[:, :, :s + 2] - k).max() <= 1e-5 * np.abs(k).max()
    assert np.abs(vc[:, :, :s + 2] - v).max() <= 1e-5 * np.abs(v).max()


def test_cpp_layer_rejects_bad_shapes(ref_lib):
    z = C.POINTER(C.c_float)()
    assert ref_lib.ref_decoder_layer(1, 4, 14, 128, 3, 512, 1, C.c_float(1e-5), *([z] * 15), 16, z) == -22
