"""Python convenience layer over the serving calls of libliger.so.

Marshalling only: LigerEngine builds a liger_cfg from a model config, calls
liger_init / liger_load_layer / liger_load_embed, and forwards submit / step /
poll / drain.  All computation happens inside the library.
"""
import ctypes as C

import numpy as np

from . import liger as L


class LigerEngine:
    def __init__(self, model_cfg, *, world=1, rank=0, nccl_uid=None, mode="interleaved", max_batch=8,
                 max_seq=512, max_new=32, max_inflight=2, decomp_factor=8, contention_factor=1.0, seed=0,
                 load=True, sync="hybrid"):
        lib = L.lib()
        cfg = L.liger_cfg()
        cfg.n_layers, cfg.hidden, cfg.n_heads = model_cfg.n_layers, model_cfg.hidden, model_cfg.n_heads
        cfg.ffn, cfg.vocab, cfg.max_pos = model_cfg.ffn, model_cfg.vocab, model_cfg.max_pos
        cfg.act = L.ACT[model_cfg.act]
        cfg.ln_eps = model_cfg.ln_eps
        cfg.max_batch, cfg.max_seq, cfg.max_new = max_batch, max_seq, max_new
        cfg.mode = L.MODE[mode]
        cfg.max_inflight = max_inflight
        cfg.decomp_factor = decomp_factor
        cfg.contention_factor = contention_factor
        cfg.seed = seed
        cfg.sync_mode = L.SYNC[sync]
        self.cfg = cfg
        self.model = model_cfg
        self.world, self.rank = world, rank
        self.seed = seed
        ctx = C.c_void_p()
        uid = None if nccl_uid is None else C.create_string_buffer(bytes(nccl_uid), 128)
        L.check(lib.liger_init(world, rank, C.byref(cfg), uid, C.byref(ctx)), None, "liger_init")
        self.ctx = ctx
        if load:
            self.load(seed)

    @staticmethod
    def unique_id():
        buf = C.create_string_buffer(128)
        L.check(L.lib().liger_nccl_unique_id(buf), None, "liger_nccl_unique_id")
        return buf.raw

    @staticmethod
    def loopback_id():
        """Id for ranks running as threads of this process on one GPU (test vehicle)."""
        buf = C.create_string_buffer(128)
        L.check(L.lib().liger_loopback_unique_id(buf), None, "liger_loopback_unique_id")
        return buf.raw

    def _chk(self, rc, what):
        return L.check(rc, self.ctx, what)

    def load(self, seed):
        lib = L.lib()
        for l in range(self.model.n_layers):
            self._chk(lib.liger_load_layer(self.ctx, l, seed), "liger_load_layer")
        self._chk(lib.liger_load_embed(self.ctx, seed), "liger_load_embed")

    def load_weights(self, layers, embed):
        """Caller-owned weights (liger_load_layer_weights / liger_load_embed_weights): `layers`
        = list of dicts of this rank's bf16 device tensors (nn.Linear layout, see liger.h),
        `embed` = dict(e_tok, e_pos, lnf_g, lnf_b).  The library copies them."""
        lib = L.lib()
        for l, w in enumerate(layers):
            if w is None:
                continue
            st = L.liger_layer_weights(*[w[n].data_ptr() for n, _ in L.liger_layer_weights._fields_])
            self._chk(lib.liger_load_layer_weights(self.ctx, l, C.byref(st)), "liger_load_layer_weights")
        self._chk(lib.liger_load_embed_weights(self.ctx, *[C.c_void_p(embed[k].data_ptr()) for k in
                                                             ("e_tok", "e_pos", "lnf_g", "lnf_b")]),
                  "liger_load_embed_weights")

    def set_streams(self, compute_stream, comm_stream):
        """Run on caller-owned streams (e.g. torch.cuda.Stream().cuda_stream); liger_set_streams."""
        self._chk(L.lib().liger_set_streams(self.ctx, C.c_void_p(compute_stream), C.c_void_p(comm_stream)),
                  "liger_set_streams")

    def profile(self, m_list):
        arr = (C.c_int32 * len(m_list))(*m_list)
        self._chk(L.lib().liger_profile(self.ctx, arr, len(m_list)), "liger_profile")

    def set_duration(self, op, m_tokens, k_of_F, us):
        """Duration-table entry for kernel class `op` (liger.OPS name)."""
        self._chk(L.lib().liger_set_duration(self.ctx, L.OPS.index(op), m_tokens, k_of_F, float(us)),
                  "liger_set_duration")

    def calibrate_cf(self, m_list, set_cf=True):
        arr = (C.c_int32 * len(m_list))(*m_list)
        cf = C.c_double()
        det = (C.c_double * (len(m_list) * 8))()
        self._chk(L.lib().liger_calibrate_cf(self.ctx, arr, len(m_list), int(set_cf), C.byref(cf), det),
                  "liger_calibrate_cf")
        names = ["qkv", "out", "fc1", "fc2"]
        detail = {m: {n: (det[(i * 4 + j) * 2], det[(i * 4 + j) * 2 + 1]) for j, n in enumerate(names)}
                  for i, m in enumerate(m_list)}
        return cf.value, detail

    def submit(self, tokens, batch, seq_len, n_new, arrival_s=-1.0, device_tokens=None):
        """tokens: numpy int32 [batch*seq_len] (host) or None with device_tokens = a device
        int32 tensor (kept alive by the caller until the batch finishes)."""
        lib = L.lib()
        if device_tokens is not None:
            rc = lib.liger_submit(self.ctx, batch, seq_len, C.c_void_p(device_tokens.data_ptr()), 1, n_new,
                                  float(arrival_s))
        else:
            t = np.ascontiguousarray(tokens, dtype=np.int32)
            rc = lib.liger_submit(self.ctx, batch, seq_len, t.ctypes.data_as(C.c_void_p), 0, n_new, float(arrival_s))
        return self._chk(rc, "liger_submit")

    def step(self):
        return self._chk(L.lib().liger_step(self.ctx), "liger_step")

    def drain(self):
        self._chk(L.lib().liger_drain(self.ctx), "liger_drain")

    def poll(self, bid, want_tokens=False):
        res = L.liger_result()
        out = None
        buf = None
        if want_tokens:
            buf = np.zeros(self.cfg.max_batch * self.cfg.max_new, dtype=np.int32)
            out = buf.ctypes.data_as(C.c_void_p)
        rc = self._chk(L.lib().liger_poll(self.ctx, bid, C.byref(res), out), "liger_poll")
        if rc == L.LIGER_PENDING:
            return None
        toks = None
        if want_tokens:
            toks = buf[:res.batch * res.n_new].reshape(res.batch, res.n_new).copy()
        return res, toks

    def allreduce(self, buf, u0=0, u1=1, F=1, stream=None):
        """liger_op_allreduce: in-place bf16 sum over the ranks of units [u0, u1) of F."""
        self._chk(L.lib().liger_op_allreduce(self.ctx, C.c_void_p(buf.data_ptr()), buf.numel(), u0, u1, F,
                                             None if stream is None else C.c_void_p(stream)), "liger_op_allreduce")

    def set_debug_capture(self, arena_bytes=256 << 20):
        """Test readback (liger_set_debug_capture, [collective]): capture per-pass logits and
        LM-head input rows of the batches admitted from now on (0 turns it off)."""
        self._chk(L.lib().liger_set_debug_capture(self.ctx, C.c_size_t(int(arena_bytes))),
                  "liger_set_debug_capture")

    def debug_read(self, bid, what, batch, n_new):
        """liger_debug_read -> numpy: 'logits' fp32 [batch, n_new, V/t] (this rank's shard)
        or 'resid' float32 (bf16 values) [batch, n_new, h]."""
        if what == "logits":
            n = self.model.vocab // (1 if self.cfg.mode >= 2 else self.world)
            buf = np.empty((n_new, batch, n), dtype=np.float32)
            code = L.DBG_LOGITS
        else:
            buf = np.empty((n_new, batch, self.model.hidden), dtype=np.uint16)
            code = L.DBG_RESID
        self._chk(L.lib().liger_debug_read(self.ctx, bid, code, buf.ctypes.data_as(C.c_void_p), buf.nbytes),
                  "liger_debug_read")
        if what != "logits":
            buf = (buf.astype(np.uint32) << 16).view(np.float32)
        return np.ascontiguousarray(buf.transpose(1, 0, 2))

    def scheduler_name(self):
        """The schedule this context runs (liger_scheduler_name)."""
        return L.lib().liger_scheduler_name(self.ctx).decode()

    def stats(self):
        s = L.liger_stats_t()
        self._chk(L.lib().liger_stats(self.ctx, C.byref(s)), "liger_stats")
        return {k: getattr(s, k) for k, _ in s._fields_}

    def reset_stats(self):
        self._chk(L.lib().liger_reset_stats(self.ctx), "liger_reset_stats")

    def set_gemm_sm_reserve(self, reserve):
        self._chk(L.lib().liger_set_gemm_sm_reserve(self.ctx, int(reserve)), "liger_set_gemm_sm_reserve")

    def set_kernel_timing(self, on):
        self._chk(L.lib().liger_set_kernel_timing(self.ctx, int(on)), "liger_set_kernel_timing")

    def kernel_timing(self):
        n = len(L.KT_NAMES)
        cnt = (C.c_int64 * n)()
        ms, by, fl = (C.c_double * n)(), (C.c_double * n)(), (C.c_double * n)()
        self._chk(L.lib().liger_kernel_timing(self.ctx, cnt, ms, by, fl), "liger_kernel_timing")
        names = L.KT_NAMES
        return {n: dict(count=cnt[i], ms=ms[i], bytes=by[i], flops=fl[i]) for i, n in enumerate(names)}

    def close(self):
        if self.ctx:
            L.lib().liger_finalize(self.ctx)
            self.ctx = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass
