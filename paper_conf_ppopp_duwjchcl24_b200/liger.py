"""Thin ctypes binding of libliger.so (include/liger.h).  Argument marshalling only:
every step of the hot path runs inside the library's CUDA kernels.  There is
no fallback -- if the library is missing or no sm_100 device is present the
calls raise."""
import ctypes as C
import os

HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(HERE, "libliger.so")

LIGER_OK, LIGER_PENDING, LIGER_IDLE = 0, 1, 2
LIGER_EINVAL, LIGER_ENOMEM, LIGER_ECUDA, LIGER_ENCCL, LIGER_ESTATE, LIGER_ETIMEOUT, LIGER_ENODEV = (
    -22, -12, -1000, -1001, -1002, -1003, -1004)
DBG_LOGITS, DBG_RESID = 1, 2
ACT = {"none": 0, "relu": 1, "gelu_tanh": 2}
SYNC = {"hybrid": 0, "cpu_gpu": 1, "inter_stream": 2}
MODE = {"serial": 0, "interleaved": 1, "pipeline": 2, "pipeline_th": 3}
KV_BLOCK = 16
KT_NAMES = ["gemm_decode", "attn", "ln", "allreduce", "gemm_prefill", "lm_head", "splitk_fixup"]   # LIGER_KT_*
OPS = ["embed", "ln1", "qkv", "attn", "out", "ar1", "ln2", "fc1", "fc2", "ar2", "head", "tokg", "pick",
       "recv_x", "send_x", "recv_tok", "send_tok"]


class LigerError(RuntimeError):
    pass


class liger_cfg(C.Structure):
    _fields_ = [("n_layers", C.c_int32), ("hidden", C.c_int32), ("n_heads", C.c_int32), ("ffn", C.c_int32),
                ("vocab", C.c_int32), ("max_pos", C.c_int32), ("act", C.c_int32), ("ln_eps", C.c_float),
                ("max_batch", C.c_int32), ("max_seq", C.c_int32), ("max_new", C.c_int32), ("mode", C.c_int32),
                ("max_inflight", C.c_int32), ("decomp_factor", C.c_int32), ("contention_factor", C.c_float),
                ("seed", C.c_uint64), ("sync_mode", C.c_int32)]


class liger_result(C.Structure):
    _fields_ = [("id", C.c_int64), ("batch", C.c_int32), ("seq_len", C.c_int32), ("n_new", C.c_int32),
                ("done", C.c_int32), ("arrival_s", C.c_double), ("submit_s", C.c_double),
                ("start_s", C.c_double), ("finish_s", C.c_double)]


class liger_layer_weights(C.Structure):
    _fields_ = [(n, C.c_void_p) for n in ("w_qkv", "b_qkv", "w_o", "b_o", "w_1", "b_1", "w_2", "b_2", "ln1_g",
                                          "ln1_b", "ln2_g", "ln2_b")]


class liger_stats_t(C.Structure):
    _fields_ = [("rounds", C.c_int64), ("kernels", C.c_int64), ("comm_kernels", C.c_int64),
                ("split_pieces", C.c_int64), ("overlapped_rounds", C.c_int64), ("host_us", C.c_double),
                ("wait_us", C.c_double), ("gpu_launches", C.c_int64), ("comm_host_us", C.c_double)]


_lib = None

_P, _I, _I64, _F, _SZ, _U64, _D = C.c_void_p, C.c_int, C.c_int64, C.c_float, C.c_size_t, C.c_uint64, C.c_double
_SIGS = {
    "liger_init": (_I, [_I, _I, C.POINTER(liger_cfg), _P, C.POINTER(_P)]),
    "liger_nccl_unique_id": (_I, [_P]),
    "liger_loopback_unique_id": (_I, [_P]),
    "liger_load_layer": (_I, [_P, _I, _U64]),
    "liger_load_embed": (_I, [_P, _U64]),
    "liger_load_layer_weights": (_I, [_P, _I, C.POINTER(liger_layer_weights)]),
    "liger_load_embed_weights": (_I, [_P, _P, _P, _P, _P]),
    "liger_set_streams": (_I, [_P, _P, _P]),
    "liger_submit": (_I64, [_P, _I, _I, _P, _I, _I, _D]),
    "liger_step": (_I, [_P]),
    "liger_drain": (_I, [_P]),
    "liger_poll": (_I, [_P, _I64, C.POINTER(liger_result), _P]),
    "liger_result_tokens_device": (_I, [_P, _I64, C.POINTER(_P)]),
    "liger_set_debug_capture": (_I, [_P, _SZ]),
    "liger_ipc_region_create": (_I, [_SZ, C.POINTER(_P), _P]),
    "liger_ipc_region_open": (_I, [_P, C.POINTER(_P)]),
    "liger_ipc_region_close": (_I, [_P]),
    "liger_ipc_region_free": (_I, [_P]),
    "liger_op_oneshot_allreduce": (_I, [_P, _SZ, _P, _I, _I, _SZ, _U64, _I, _P]),
    "liger_op_oneshot_allreduce_emulated": (_I, [_P, _SZ, _P, _I, _SZ, _U64, _P]),
    "liger_op_gemm_fused_ar_stage": (_I, [_P, _I64, _P, _I, _I, _I, _P, _I, _I, _SZ, _U64, _P, _SZ, _P]),
    "liger_op_add_layernorm_fused_ar": (_I, [_P, _I, _I, _SZ, _U64, _P, _P, _P, _P, _P, _P, _I, _I, _F, _P]),
    "liger_op_allreduce": (_I, [_P, _P, _SZ, _I, _I, _I, _P]),
    "liger_debug_read": (_I, [_P, _I64, _I, _P, _SZ]),
    "liger_stats": (_I, [_P, C.POINTER(liger_stats_t)]),
    "liger_reset_stats": (_I, [_P]),
    "liger_set_gemm_sm_reserve": (_I, [_P, _I]),
    "liger_set_kernel_timing": (_I, [_P, _I]),
    "liger_kernel_timing": (_I, [_P, _P, _P, _P, _P]),
    "liger_set_duration": (_I, [_P, _I, _I, _I, _D]),
    "liger_profile": (_I, [_P, _P, _I]),
    "liger_calibrate_cf": (_I, [_P, _P, _I, _I, _P, _P]),
    "liger_last_error": (C.c_char_p, [_P]),
    "liger_scheduler_name": (C.c_char_p, [_P]),
    "liger_finalize": (_I, [_P]),
    "liger_op_gemm": (_I, [_P, _I64, _P, _I64, _P, _I64, _I, _I, _I, _I, _I, _P, _I, _I, _F, _I, _P, _SZ, _P]),
    "liger_op_gemm_tiled": (_I, [_P, _I64, _P, _P, _I64, _I, _I, _I, _I, _I, _P, _I, _I, _F, _I, _P, _SZ, _P]),
    "liger_op_tile_weight": (_I, [_P, _I64, _P, _I, _I, _P]),
    "liger_gemm_workspace_bytes": (_SZ, [_I, _I, _I]),
    "liger_gemm_plan": (_I, [_I, _I, _I, _P]),
    "liger_op_add_layernorm": (_I, [_P, _P, _P, _P, _P, _P, _P, _I, _I, _I, _I, _F, _P]),
    "liger_op_embed": (_I, [_P, _P, _P, _P, _I, _I, _I, _I, _P]),
    "liger_op_attn_prefill": (_I, [_P, _P, _P, _P, _I, _I, _I, _I, _I, _P]),
    "liger_op_attn_decode": (_I, [_P, _P, _P, _P, _I, _I, _I, _I, _I, _P, _SZ, _P]),
    "liger_attn_decode_workspace_bytes": (_SZ, [_I, _I, _I, _I]),
    "liger_op_argmax": (_I, [_P, _I64, _I, _I, _I, _P, _P, _P]),
    "liger_op_c0_fill": (_I, [_P, _I, _I, _I64, _U64, _U64, _I64, _I64, _I64, _I64, _I, _I, _P]),
    "liger_planner_create": (_I, [_I, _D, C.POINTER(_P)]),
    "liger_planner_submit": (_I, [_P, _I64, _I, _P, _P, _P]),
    "liger_plan_round": (_I, [_P, _P, _I, _P, _P, _P]),
    "liger_planner_destroy": (_I, [_P]),
    "liger_trace_start": (_I, [C.c_uint]),
    "liger_trace_stop": (_I, [_P, C.c_uint, _P]),
}


def lib():
    """Load libliger.so (raises if it has not been built)."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise LigerError(f"{LIB_PATH} not built: run `python -m paper_conf_ppopp_duwjchcl24_b200.build`")
        l = C.CDLL(LIB_PATH, mode=C.RTLD_GLOBAL)
        for name, (res, args) in _SIGS.items():
            f = getattr(l, name, None)
            if f is None:
                continue        # reported by missing_symbols(); calling it raises AttributeError
            f.restype = res
            f.argtypes = args
        _lib = l
    return _lib


def exported_symbols():
    return list(_SIGS)


def missing_symbols():
    l = lib()
    return [n for n in _SIGS if getattr(l, n, None) is None]


def check(rc, ctx=None, what=""):
    if rc < 0:
        msg = lib().liger_last_error(ctx)
        raise LigerError(f"{what}: status {rc}: {msg.decode() if msg else ''}")
    return rc


def _p(t):
    return None if t is None else C.c_void_p(t.data_ptr())


def _s(stream):
    return None if stream is None else C.c_void_p(stream)


# ------------------------------------------------------------------ kernel entry points (torch tensors in)
def gemm(x, w, out, *, n0=0, n1=None, bias=None, act="none", scale_cols=0, scale=1.0, workspace=None,
         stream=None):
    M, K = x.shape
    N = w.shape[0]
    n1 = N if n1 is None else n1
    out_f32 = 1 if out.element_size() == 4 else 0
    ws_b = workspace.numel() * workspace.element_size() if workspace is not None else 0
    check(lib().liger_op_gemm(_p(x), x.stride(0), _p(w), w.stride(0), _p(out), out.stride(0), M, N, K, n0, n1,
                              _p(bias), ACT[act], scale_cols, scale, out_f32, _p(workspace), ws_b, _s(stream)),
          what="liger_op_gemm")


def gemm_tiled(x, w_tiled, out, *, N, n0=0, n1=None, bias=None, act="none", scale_cols=0, scale=1.0,
               workspace=None, stream=None):
    """W given in the tiled layout (see tile_weight)."""
    M, K = x.shape
    n1 = N if n1 is None else n1
    out_f32 = 1 if out.element_size() == 4 else 0
    ws_b = workspace.numel() * workspace.element_size() if workspace is not None else 0
    check(lib().liger_op_gemm_tiled(_p(x), x.stride(0), _p(w_tiled), _p(out), out.stride(0), M, N, K, n0, n1,
                                    _p(bias), ACT[act], scale_cols, scale, out_f32, _p(workspace), ws_b,
                                    _s(stream)), what="liger_op_gemm_tiled")


def ipc_region_create(cap):
    """(region pointer, 64-byte CUDA-IPC handle) of a fresh one-shot staging region."""
    reg = C.c_void_p()
    h = C.create_string_buffer(64)
    check(lib().liger_ipc_region_create(cap, C.byref(reg), h), what="liger_ipc_region_create")
    return reg.value, h.raw


def ipc_region_open(handle):
    p = C.c_void_p()
    check(lib().liger_ipc_region_open(C.create_string_buffer(bytes(handle), 64), C.byref(p)),
          what="liger_ipc_region_open")
    return p.value


AR_PHASE_STAGE, AR_PHASE_REDUCE = 1, 2


def oneshot_allreduce(buf, regions, rank, cap, epoch, phases=AR_PHASE_STAGE | AR_PHASE_REDUCE, stream=None):
    """liger_op_oneshot_allreduce on torch bf16 buffer `buf` (in place)."""
    arr = (C.c_void_p * len(regions))(*regions)
    check(lib().liger_op_oneshot_allreduce(_p(buf), buf.numel(), arr, len(regions), rank, cap, epoch, phases,
                                           _s(stream)),
          what="liger_op_oneshot_allreduce")


def oneshot_allreduce_emulated(bufs, regions, cap, epoch, stream=None):
    """liger_op_oneshot_allreduce_emulated: every rank's one-shot all-reduce of call `epoch` as one
    cooperative launch (test vehicle for the cross-rank protocol on one GPU); bufs summed in place."""
    w = len(bufs)
    pb = (C.c_void_p * w)(*[b.data_ptr() for b in bufs])
    pr = (C.c_void_p * w)(*regions)
    check(lib().liger_op_oneshot_allreduce_emulated(pb, bufs[0].numel(), pr, w, cap, epoch, _s(stream)),
          what="liger_op_oneshot_allreduce_emulated")


def gemm_fused_ar_stage(x, w_tiled, M, N, K, regions, rank, cap, epoch, workspace, stream=None):
    """liger_op_gemm_fused_ar_stage: split-K GEMM whose fixup stages bf16(x W^T) and publishes."""
    arr = (C.c_void_p * len(regions))(*regions)
    check(lib().liger_op_gemm_fused_ar_stage(_p(x), x.stride(0), _p(w_tiled), M, N, K, arr, len(regions), rank, cap,
                                             epoch, _p(workspace), workspace.numel() * workspace.element_size(),
                                             _s(stream)),
          what="liger_op_gemm_fused_ar_stage")


def add_layernorm_fused_ar(regions, rank, cap, epoch, x, add_bias, x_out, y, gamma, beta, eps=1e-5, stream=None):
    """liger_op_add_layernorm_fused_ar: x + sum of the ranks' staged rows + bias, then LN."""
    arr = (C.c_void_p * len(regions))(*regions)
    rows, h = x.shape
    check(lib().liger_op_add_layernorm_fused_ar(arr, len(regions), rank, cap, epoch, _p(x), _p(add_bias), _p(x_out),
                                                _p(y), _p(gamma), _p(beta), rows, h, eps, _s(stream)),
          what="liger_op_add_layernorm_fused_ar")


def tile_weight(w, w_tiled, stream=None):
    N, K = w.shape
    check(lib().liger_op_tile_weight(_p(w), w.stride(0), _p(w_tiled), N, K, _s(stream)), what="liger_op_tile_weight")


def tiled_numel(N, K):
    return (N + 127) // 128 * 128 * K


def gemm_workspace_bytes(M, N, K):
    return lib().liger_gemm_workspace_bytes(M, N, K)


def gemm_plan(M, N, K):
    out = (C.c_int32 * 5)()
    check(lib().liger_gemm_plan(M, N, K, out), what="liger_gemm_plan")
    return dict(zip(("bn", "m_tiles", "kc", "splits", "stages"), list(out)))


def add_layernorm(x, gamma, beta, y, *, add=None, add_bias=None, x_out=None, rows=None, in_row_step=1,
                  in_row_off=0, eps=1e-5, stream=None):
    h = x.shape[-1]
    rows = x.shape[0] if rows is None else rows
    check(lib().liger_op_add_layernorm(_p(x), _p(add), _p(add_bias), _p(x_out), _p(y), _p(gamma), _p(beta), rows,
                                       h, in_row_step, in_row_off, eps, _s(stream)), what="liger_op_add_layernorm")


def embed(ids, e_tok, e_pos, out, *, seq_len, start_pos=0, stream=None):
    check(lib().liger_op_embed(_p(ids), _p(e_tok), _p(e_pos), _p(out), ids.numel(), e_tok.shape[1], seq_len,
                               start_pos, _s(stream)), what="liger_op_embed")


def attn_prefill(qkv, o, kv_pool, page_table, *, b, s, heads, d, stream=None):
    check(lib().liger_op_attn_prefill(_p(qkv), _p(o), _p(kv_pool), _p(page_table), page_table.shape[1], b, s, heads,
                                      d, _s(stream)), what="liger_op_attn_prefill")


def attn_decode(qkv, o, kv_pool, page_table, *, b, pos, heads, d, workspace=None, stream=None):
    ws_b = workspace.numel() * workspace.element_size() if workspace is not None else 0
    check(lib().liger_op_attn_decode(_p(qkv), _p(o), _p(kv_pool), _p(page_table), page_table.shape[1], b, pos,
                                     heads, d, _p(workspace), ws_b, _s(stream)), what="liger_op_attn_decode")


def attn_decode_workspace_bytes(b, heads, d, ctx):
    return lib().liger_attn_decode_workspace_bytes(b, heads, d, ctx)


def argmax(logits, max_out, idx_out, *, idx_offset=0, stream=None):
    rows, n = logits.shape
    check(lib().liger_op_argmax(_p(logits), logits.stride(0), rows, n, idx_offset, _p(max_out), _p(idx_out),
                                _s(stream)), what="liger_op_argmax")


def c0_fill(dst, *, seed, tensor_id, row_off=0, col_off=0, idx_row_stride, idx_col_stride=1, exp=0, kind=0,
            stream=None):
    rows, cols = dst.shape
    check(lib().liger_op_c0_fill(_p(dst), rows, cols, dst.stride(0), seed, tensor_id, row_off, col_off,
                                 idx_row_stride, idx_col_stride, exp, kind, _s(stream)), what="liger_op_c0_fill")


TRACE_KIDS = {1: "gemm", 2: "fixup", 3: "attn_dec", 0x103: "attn_merge", 4: "attn_pre", 5: "add_ln"}


def trace_start(capacity=1 << 20):
    """Diagnostics: start the per-CTA kernel timeline trace (liger_trace_start)."""
    check(lib().liger_trace_start(capacity), None, "liger_trace_start")
    return capacity


def trace_stop(capacity=1 << 20):
    """Stop the trace; returns a numpy structured array (kid, cta, smid, t0, t1, t2 in ns)."""
    import numpy as np
    dt = np.dtype([("kid", "<u4"), ("cta", "<u4"), ("smid", "<u4"), ("pad", "<u4"),
                   ("t0", "<u8"), ("t1", "<u8"), ("t2", "<u8")])
    assert dt.itemsize == 40
    buf = np.zeros(capacity, dtype=dt)
    n = C.c_uint(0)
    check(lib().liger_trace_stop(buf.ctypes.data, capacity, C.byref(n)), None, "liger_trace_stop")
    return buf[:min(n.value, capacity)]
