"""Benchmark of the Liger hot path (driver contract).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference] [--loopback]

Workload (BASELINE.json configs[1]): OPT-13B random-init bf16, Poisson-shaped
request batches (batch 2/4/8, prompt U[128, 512], 32 generated tokens), served
through the C ABI (liger_submit / liger_step / liger_poll).  One "step" = one
request batch through the whole hot path (prefill pass + 31 decode passes over
all 40 layers).  N GPUs = tensor-parallel degree N (one process per GPU).  Without
torchrun, `--gpus N > 1` re-launches itself under torch.distributed.run with N
processes; `--loopback` instead runs the N ranks as threads sharing ONE GPU (the
loopback communicator: a functional dry run of the t > 1 path, not a speed claim).

value     = requests (sequences) per second of the whole job with the prompts
            already resident in HBM, all K batches offered at once (capacity;
            device time between two synchronised barriers, max over ranks).
e2e       = the same with host prompts copied in and generated tokens copied
            out through the public API inside the timed region.
operating_points = the BASELINE metric itself: Poisson
            traces at rising arrival rates for serial intra-op TP and for the
            interleaved mode on the same traces; L* = 1.5 x serial's mean latency at
            the lowest rate; each mode's req/s at mean latency <= L* (interpolated)
            and mean / p99 latency at 0.5 and 0.8 x serial's saturation rate.
roofline  = the dominant kernel class (by device time) in a timed replay with
            per-launch CUDA events inside the library; at N > 1 also the
            all-reduce class (bus bandwidth) and an NCCL-tests-style sweep.
"""
import argparse
import json
import math
import os
import socket
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)
# stdout carries exactly one JSON line: NCCL prints a version banner at NCCL_DEBUG=WARN/VERSION
os.environ.setdefault("NCCL_DEBUG", "NONE")
_JSON_FD = None


def emit(line):
    """Write the result line to the real stdout (C-level stdout is redirected to stderr)."""
    os.write(_JSON_FD if _JSON_FD is not None else 1, (json.dumps(line) + "\n").encode())


def _redirect_stdout():
    global _JSON_FD
    sys.stdout.flush()
    _JSON_FD = os.dup(1)
    os.dup2(2, 1)


from liger_inputs import get_config, make_trace  # noqa: E402

METRIC = "req/s at fixed mean latency; mean/p99 latency at fixed req/s (OPT, TP=1/2/4/8)"
PEAKS = os.path.join(ROOT, "MEASURED_PEAKS.json")
NVLINK_SPEC_GBS = 900.0   # NVLink 5 per direction per GPU (B200 spec)


def load_peaks():
    try:
        with open(PEAKS) as f:
            p = json.load(f)
        return p["hbm_gbs"], p["bf16_tflops"], p.get("bf16_tflops_sustained", p["bf16_tflops"]), "measured"
    except Exception:
        return 6650.0, 1590.0, 1400.0, "fallback"


class ClockSampler:
    """nvidia-smi clocks / throttle reasons sampled during the timed region."""

    Q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
         "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, gpu_index=0):
        self.idx = gpu_index
        self.p = None

    def start(self):
        try:
            self.p = subprocess.Popen(["nvidia-smi", f"--id={self.idx}", f"--query-gpu={self.Q}",
                                       "--format=csv,noheader,nounits", "-lms", "200"],
                                      stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
        except Exception:
            self.p = None

    def stop(self):
        if self.p is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        self.p.terminate()
        try:
            out, _ = self.p.communicate(timeout=5)
        except Exception:
            self.p.kill()
            out = ""
        sm, mx, reasons = [], None, set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for line in out.strip().splitlines():
            f = [x.strip() for x in line.split(",")]
            if len(f) < 9:
                continue
            try:
                sm.append(float(f[1]))
                mx = float(f[2])
            except ValueError:
                continue
            for n, v in zip(names, f[5:9]):
                if v.lower().startswith("active"):
                    reasons.add(n)
        loaded = [s for s in sm if mx and s > 0.3 * mx] or sm
        return {"sm_mhz": float(np.median(loaded)) if loaded else None, "sm_max_mhz": mx,
                "reasons": sorted(reasons), "samples": len(sm)}


# ----------------------------------------------------------------------------- rank groups
class DistGroup:
    """torch.distributed ranks (one process per GPU): gloo for host values."""

    def __init__(self, world, rank):
        import torch.distributed as dist
        self.dist, self.world, self.rank = dist, world, rank
        self.gloo = dist.new_group(backend="gloo") if world > 1 else None

    def barrier(self):
        import torch
        if self.world > 1:
            self.dist.barrier(group=self.gloo)
        torch.cuda.synchronize()

    def max(self, x):
        if self.world == 1:
            return x
        import torch
        t = torch.tensor([x], dtype=torch.float64)
        self.dist.all_reduce(t, op=self.dist.ReduceOp.MAX, group=self.gloo)
        return float(t.item())

    def bcast(self, obj):
        if self.world == 1:
            return obj
        o = [obj]
        self.dist.broadcast_object_list(o, src=0, group=self.gloo)
        return o[0]


class ThreadShared:
    def __init__(self, world):
        self.world = world
        self.bar = threading.Barrier(world)
        self.slots = [None] * world


class ThreadGroup:
    """Loopback ranks: threads of this process sharing one GPU."""

    def __init__(self, shared, rank):
        self.s, self.world, self.rank = shared, shared.world, rank

    def barrier(self):
        import torch
        torch.cuda.synchronize()
        self.s.bar.wait()

    def _gather(self, x):
        self.s.bar.wait()
        self.s.slots[self.rank] = x
        self.s.bar.wait()
        out = list(self.s.slots)
        self.s.bar.wait()
        return out

    def max(self, x):
        return max(self._gather(x))

    def bcast(self, obj):
        return self._gather(obj)[0]


# ----------------------------------------------------------------------------- CPU oracle baseline
_CPP_ORACLE = []


def _cpp_oracle():
    """The fp32 C++ oracle binary compiled (once per process) for THIS host (-march=native:
    the repo's copy may have been built elsewhere), or None."""
    if not _CPP_ORACLE:
        exe = None
        try:
            import tempfile
            from paper_conf_ppopp_duwjchcl24_b200.build import build_oracle
            exe, _ = build_oracle(os.path.join(tempfile.gettempdir(), f"liger_oracle_{os.getpid()}"))
        except Exception as e:
            print(f"bench.py: C++ oracle unavailable ({e}); timing the numpy oracle", file=sys.stderr)
        _CPP_ORACLE.append(exe)
    return _CPP_ORACLE[0]


def cpu_oracle_sample(cfg, b=2, s=128, n_new=32, threads=None):
    """Time the CPU oracle on a bounded sample of the workload and extrapolate (labelled).

    Preferred: the fp32 C++ OpenMP oracle binary (oracle/layer_ref.cpp; BASELINE.md
    "CPU baseline plan") on one decoder layer -- a prefill over [b, s] and decode
    steps at ctx s + 16 -- with weights generated on the fly, x L layers x n_new passes.
    Fallback (binary not built): the fp64 numpy oracle on the same sample."""
    nproc = os.cpu_count() or 1
    exe = _cpp_oracle()
    if exe and os.path.exists(exe):
        out = {}
        for th in ([threads] if threads else [nproc, 1]):
            cmd = [exe, "--hidden", str(cfg.hidden), "--heads", str(cfg.n_heads), "--ffn", str(cfg.ffn),
                   "--act", cfg.act, "--batch", str(b), "--prompt", str(s), "--decode-steps", "4",
                   "--ctx", str(s + 16), "--budget-s", "12"]
            env = {**os.environ, "OMP_NUM_THREADS": str(th)}
            r = subprocess.run(cmd, capture_output=True, text=True, timeout=600, env=env)
            if r.returncode != 0:
                out = None
                break
            out[th] = json.loads(r.stdout.strip().splitlines()[-1])
        if out:
            main = out[max(out)]
            per_batch = cfg.n_layers * (main["prefill_s"] + (n_new - 1) * main["decode_step_s"])
            res = {"value": b / per_batch, "unit": "req/s", "cores": main["threads"], "kind": "oracle",
                   "sample": (f"fp32 C++ OpenMP oracle (oracle/layer_ref.cpp, -O3 -march=native), one {cfg.name} "
                              f"layer: prefill b={b} s={s} ({main['prefill_s']:.2f} s) + decode steps at ctx "
                              f"{s + 16} ({main['decode_step_s'] * 1e3:.1f} ms each); extrapolated x{cfg.n_layers} "
                              f"layers x {n_new} passes"),
                   "per_batch_s": per_batch}
            if 1 in out and max(out) != 1:
                one = out[1]
                pb1 = cfg.n_layers * (one["prefill_s"] + (n_new - 1) * one["decode_step_s"])
                res["one_thread"] = {"value": b / pb1, "unit": "req/s", "cores": 1}
            return res
    from oracle import model as om
    rng = np.random.default_rng(0)
    h, f = cfg.hidden, cfg.ffn
    w = {"w_qkv": rng.standard_normal((h, 3 * h)) * h ** -0.5, "b_qkv": np.zeros(3 * h),
         "w_o": rng.standard_normal((h, h)) * h ** -0.5, "b_o": np.zeros(h),
         "w_1": rng.standard_normal((h, f)) * h ** -0.5, "b_1": np.zeros(f),
         "w_2": rng.standard_normal((f, h)) * f ** -0.5, "b_2": np.zeros(h),
         "ln1_g": np.ones(h), "ln1_b": np.zeros(h), "ln2_g": np.ones(h), "ln2_b": np.zeros(h)}
    x = rng.standard_normal((b, s, h)) * 0.1
    t0 = time.perf_counter()
    _, k, v = om.decoder_layer(cfg, w, x)
    t_pf = time.perf_counter() - t0
    xd = rng.standard_normal((b, 1, h)) * 0.1
    reps = 0
    t0 = time.perf_counter()
    while reps < 4:
        om.decoder_layer(cfg, w, xd, k, v, start_pos=s)
        reps += 1
    t_dc = (time.perf_counter() - t0) / reps
    per_batch = cfg.n_layers * (t_pf + (n_new - 1) * t_dc)
    return {"value": b / per_batch, "unit": "req/s", "cores": nproc, "kind": "oracle",
            "sample": (f"fp64 numpy oracle, one {cfg.name} layer: prefill b={b} s={s} ({t_pf:.2f}s) + {reps} decode "
                       f"steps at ctx {s + 1} ({t_dc * 1e3:.1f} ms each); extrapolated x{cfg.n_layers} layers x "
                       f"{n_new} passes"),
            "per_batch_s": per_batch}


def run_reference(args):
    """The reference arm of this tier: the CPU oracle as it stands, on the box's host
    cores; each step is one bounded sample (one layer prefill + decode steps) whose
    wall time is ms_per_step; value is the extrapolated whole-workload req/s."""
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return 0
    cfg = get_config(args.config)
    vals, walls = [], []
    for i in range(args.warmup + args.steps):
        t0 = time.perf_counter()
        r = cpu_oracle_sample(cfg, threads=os.cpu_count() or 1)
        if i >= args.warmup:
            vals.append(r["value"])
            walls.append(time.perf_counter() - t0)
    v = float(np.mean(vals))
    line = {"impl": "reference", "metric": METRIC, "value": v, "unit": "req/s", "n_gpus": args.gpus,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * float(np.mean(walls)),
            "higher_is_better": True, "scaling": "strong", "vs_baseline": None,
            "dtype": "f32" if "C++" in r["sample"] else "f64", "data": "synthetic",
            "config": {"workload": f"{args.config} TP={args.gpus}: one-layer prefill + decode sample per step, "
                                   f"req/s extrapolated to {cfg.n_layers} layers x 32 passes (ms_per_step = the "
                                   f"sample's wall time)", "model": args.config},
            "cpu_baseline": {**{k: r[k] for k in ("unit", "cores", "kind", "sample")}, "value": v},
            "e2e": {"value": v, "unit": "req/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    emit(line)
    return 0


# ----------------------------------------------------------------------------- serving helpers
def serve_poisson(eng, group, trace, t_offset=0.0):
    """Open-loop serving of a trace (arrival times on the host clock); all ranks submit
    identically (rank 0 decides which arrivals are due).  Returns per-sequence
    latencies (pending + execution) and the throughput over the run."""
    group.barrier()
    t0 = time.monotonic()
    ids, sizes = [], []
    i = 0
    while True:
        now = time.monotonic() - t0
        due = sum(1 for r in trace[i:] if r["arrival_s"] <= now) if group.rank == 0 else 0
        due = group.bcast(due)
        for r in trace[i:i + due]:
            ids.append(eng.submit(r["tokens"], r["batch"], r["seq_len"], r["n_decode"], t0 + r["arrival_s"]))
            sizes.append(r["batch"])
        i += due
        rc = eng.step()
        if i >= len(trace):
            break
        if rc == 2:   # idle: wait for the next arrival
            time.sleep(max(0.0, min(0.001, trace[i]["arrival_s"] - (time.monotonic() - t0))))
    eng.drain()
    lats, fin = [], []
    for bid, bsz in zip(ids, sizes):
        res, _ = eng.poll(bid)
        lats += [res.finish_s - res.arrival_s] * bsz
        fin.append(res.finish_s)
    lats.sort()
    span = max(fin) - t0
    return {"mean_s": float(np.mean(lats)), "p99_s": float(lats[max(0, math.ceil(0.99 * len(lats)) - 1)]),
            "req_s": sum(sizes) / span}


def req_s_at_latency(points, L):
    """Largest throughput with mean latency <= L, interpolating linearly between the
    swept points in (throughput, mean latency); points sorted by rate."""
    best = None
    for a, b in zip(points, points[1:]):
        if a["mean_s"] <= L:
            best = a["req_s"]
        if a["mean_s"] <= L < b["mean_s"]:
            w = (L - a["mean_s"]) / (b["mean_s"] - a["mean_s"])
            best = a["req_s"] + w * (b["req_s"] - a["req_s"])
            break
    else:
        if points and points[-1]["mean_s"] <= L:
            best = points[-1]["req_s"]
    return best


def allreduce_sweep(eng, group, torch, F=8):
    """NCCL-tests-style bus bandwidth of the library's all-reduce (liger_op_allreduce)
    on the communication stream, 8 B .. 1 GiB, whole vs decomposed into F atomic
    units: busbw = S / t * 2 (t - 1) / t."""
    t = group.world
    st = torch.cuda.Stream()
    out = []
    buf = torch.zeros(1 << 29, dtype=torch.bfloat16, device="cuda")
    for lg in range(3, 31, 3):
        n = max(8, (1 << lg) // 2)
        x = buf[:n]
        row = {"bytes": 2 * n}
        for name, ks in (("whole", [F]), ("chunked", [1] * F)):
            reps = 20 if n < (1 << 24) else 5
            for rep in range(reps + 3):
                if rep == 3:
                    group.barrier()
                    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                    e0.record(st)
                u = 0
                for k in ks:
                    eng.allreduce(x, u, u + k, F, stream=st.cuda_stream)
                    u += k
            e1.record(st)
            e1.synchronize()
            us = group.max(e0.elapsed_time(e1) * 1e3 / reps)
            row[name + "_us"] = round(us, 2)
            row[name + "_busbw_gbs"] = round(2 * n / (us * 1e-6) * 2 * (t - 1) / t / 1e9, 2)
        out.append(row)
    del buf
    return out


# ----------------------------------------------------------------------------- one rank
TRACE_KINDS = {1: "gemm", 2: "splitk_fixup", 3: "attn_decode", 4: "attn_prefill", 5: "add_ln", 6: "embed",
               7: "argmax", 8: "argmax_pick", 9: "fused_ar", 3 | 256: "attn_decode_merge"}


def capacity_trace(eng, trace, torch):
    """Where the schedule that ran spends the GPU: the in-kernel %globaltimer record of every
    CTA (kind, SM, PDL-wait release, exit) while `trace` is served as in the timed region.
    Per kernel kind, its share of the SMs' time (sum over CTAs of release -> exit, divided
    by SMs x span), and the fraction of the span in which no GEMM CTA works."""
    from paper_conf_ppopp_duwjchcl24_b200 import liger as L
    cap = 1 << 23
    torch.cuda.synchronize()
    L.trace_start(cap)
    for r in trace:
        eng.submit(r["tokens"], r["batch"], r["seq_len"], r["n_decode"], 0.0)
    eng.drain()
    torch.cuda.synchronize()
    rec = L.trace_stop(cap)
    if len(rec) == 0 or len(rec) >= cap:
        return None
    return {"batches": len(trace), **trace_summary(rec)}


def trace_launches(rec, kid):
    """Group the CTA records of kernel kind `kid` into launches (launch order = entry order;
    a launch ends when a CTA index repeats): [(first release, last exit, CTAs)]."""
    r = rec[rec["kid"] == kid]
    r = r[np.argsort(r["t0"], kind="stable")]
    out, seen, cur = [], set(), []
    for x in r:
        if int(x["cta"]) in seen:
            out.append(cur)
            seen, cur = set(), []
        seen.add(int(x["cta"]))
        cur.append(x)
    if cur:
        out.append(cur)
    return [(min(int(x["t1"]) for x in c), max(int(x["t2"]) for x in c), len(c)) for c in out]


def decode_gemm_in_situ(eng, cfg, world, torch, b=8, s=256):
    """The decode GEMMs of one whole decode pass with the PDL chain intact (no events between
    kernels): from the in-kernel trace of a batch with 3 generated tokens, the last pass's
    4 L + 1 GEMM launches (projections + LM head); achieved = their weight bytes / the sum of
    their spans (first CTA's PDL-wait release -> last CTA's exit)."""
    from paper_conf_ppopp_duwjchcl24_b200 import liger as L
    ids = torch.from_numpy(np.random.default_rng(4).integers(0, cfg.vocab, size=b * s).astype(np.int32)).cuda()
    per_pass = 4 * cfg.n_layers + 1
    span_us = None
    for _ in range(3):   # best of 3 traced batches
        torch.cuda.synchronize()
        L.trace_start(1 << 20)
        eng.submit(None, b, s, 3, 0.0, device_tokens=ids)
        eng.drain()
        torch.cuda.synchronize()
        g = trace_launches(L.trace_stop(1 << 20), 1)
        if len(g) < 3 * per_pass:
            return None
        us = sum(t2 - t1 for t1, t2, _ in g[-per_pass:]) / 1e3
        span_us = us if span_us is None else min(span_us, us)
    h, f = cfg.hidden, cfg.ffn
    wbytes = (cfg.n_layers * (4 * h * h + 2 * h * f) + cfg.vocab * h) * 2 / world
    return {"launches": per_pass, "sum_span_us": round(span_us, 1), "bytes": round(wbytes),
            "achieved": round(wbytes / (span_us * 1e-6) / 1e9, 1),
            "note": "the last decode pass's projection + LM-head GEMMs (b = %d, prompt %d) with the PDL chain "
                    "intact, spans from the in-kernel trace (first PDL-wait release -> last exit; best of 3), i.e. "
                    "the kernels' own streaming without the per-launch gaps the event-separated replay adds; "
                    "the trace's exit atomics lengthen every span slightly" % (b, s)}


def trace_summary(rec):
    """Per kernel kind: sum over CTAs of (PDL-wait release t1 -> exit t2) / (SMs x span); and
    the fraction of the span [min t0, max t2] in which no GEMM CTA (kid 1) works."""
    t0 = int(rec["t0"].min())
    a = (rec["t1"].astype(np.int64) - t0).astype(np.float64)
    z = (rec["t2"].astype(np.int64) - t0).astype(np.float64)
    span = float(z.max())
    nsm = int(rec["smid"].max()) + 1
    share = {}
    for k in np.unique(rec["kid"]):
        m = rec["kid"] == k
        share[TRACE_KINDS.get(int(k), str(int(k)))] = round(float((z[m] - a[m]).sum()) / (nsm * span), 4)
    g = rec["kid"] == 1
    ev = np.concatenate([a[g], z[g]])
    dv = np.concatenate([np.ones(int(g.sum())), -np.ones(int(g.sum()))])
    o = np.argsort(ev, kind="stable")
    busy = np.cumsum(dv[o])[:-1] > 0
    gemm_cov = float(np.diff(ev[o])[busy].sum()) / span if g.any() else 0.0
    return {"span_ms": round(span / 1e6, 2), "sms": nsm, "cta_records": int(len(rec)),
            "sm_time_share": share, "no_gemm_working_frac": round(1.0 - gemm_cov, 4),
            "note": "in-kernel %globaltimer trace of every CTA while these batches are served as in the timed "
                    "region (release of the PDL wait -> exit); sm_time_share = CTA-time / (SMs x span); "
                    "embedding and argmax kernels are not traced; attn_decode_merge = decode-attention CTAs "
                    "that also merged the splits"}


def uid_factory(group, make):
    """new_uid() for rank_main: at world > 1 every call is a collective in which rank 0
    makes a fresh id (make()) and every rank receives it; None at world 1."""
    if group.world == 1:
        return lambda: None
    return lambda: group.bcast(make() if group.rank == 0 else None)


def rank_main(args, group, local, new_uid, result):
    """One rank.  new_uid(): a fresh communicator id agreed by all ranks (a collective), or
    None at world 1 -- every engine this rank creates gets its own, since an ncclUniqueId
    bootstraps exactly one communicator."""
    import torch
    from paper_conf_ppopp_duwjchcl24_b200.engine import LigerEngine
    torch.cuda.set_device(local)
    world, rank = group.world, group.rank
    cfg = get_config(args.config, args.layers)
    gen = args.workload == "generative"
    trace_kw = (dict(batch_sizes=(32,), prompt_range=(16, 16)) if gen else {})
    ekw = dict(world=world, rank=rank, nccl_uid=new_uid(), max_batch=32 if gen else 8, max_seq=16 if gen else 512,
               max_new=args.n_new, max_inflight=args.inflight, decomp_factor=args.F, contention_factor=args.cf,
               seed=args.seed, sync=args.sync)
    eng = LigerEngine(cfg, mode=args.mode, **ekw)
    eng.profile([8, 64, 256, 512, 1024, 2048, 4096])
    # contention factor: measured GEMM || all-reduce slowdown (1-rank proxy at N=1)
    cf_cal, _ = eng.calibrate_cf([8, 256, 1024], set_cf=args.cf <= 0)
    cf_reserve = {}
    if not args.quick:   # contention control: GEMM grids leaving SMs to the all-reduce
        for rsv in (8, 16, 32):
            eng.set_gemm_sm_reserve(rsv)
            cf_reserve[rsv] = round(eng.calibrate_cf([8, 256, 1024], set_cf=False)[0], 4)
        eng.set_gemm_sm_reserve(int(os.environ.get("LIGER_GEMM_SM_RESERVE", "0")))
    cf_reserve[0] = round(cf_cal, 4)

    trace = make_trace(args.warmup + args.steps, float("inf"), seed=args.seed, vocab=cfg.vocab,
                       n_decode=args.n_new, **trace_kw)
    warm, timed = trace[:args.warmup], trace[args.warmup:]
    seqs = sum(r["batch"] for r in timed)
    dev_tokens = [torch.from_numpy(r["tokens"]).cuda() for r in timed]

    # ---- warm-up (untimed): W batches through the full path
    for r in warm:
        eng.submit(r["tokens"], r["batch"], r["seq_len"], r["n_decode"], 0.0)
    eng.drain()

    def timed_run(host_io):
        eng.reset_stats()
        group.barrier()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        t_host0 = time.perf_counter()
        ids = []
        # NVTX range around the timed region (ncu --nvtx --nvtx-include "timed/" captures just it)
        torch.cuda.nvtx.range_push("timed" if not host_io else "timed_e2e")
        for r, dt in zip(timed, dev_tokens):
            if host_io:
                ids.append(eng.submit(r["tokens"], r["batch"], r["seq_len"], r["n_decode"], 0.0))
            else:
                ids.append(eng.submit(None, r["batch"], r["seq_len"], r["n_decode"], 0.0, device_tokens=dt))
        eng.drain()
        if host_io:
            for bid in ids:
                eng.poll(bid, want_tokens=True)
        torch.cuda.nvtx.range_pop()
        torch.cuda.synchronize()
        e1.record()
        e1.synchronize()
        wall = time.perf_counter() - t_host0
        group.barrier()
        dev_s = group.max(e0.elapsed_time(e1) * 1e-3)
        return dev_s, wall, eng.stats()

    clocks = ClockSampler(local)
    clocks.start()
    dev_s, wall_s, st = timed_run(False)
    clk = clocks.stop()
    value = seqs / dev_s
    e2e_s, _, _ = timed_run(True)
    h2d = sum(r["batch"] * r["seq_len"] * 4 for r in timed) / len(timed)
    d2h = sum(r["batch"] * r["n_decode"] * 4 for r in timed) / len(timed)

    # ---- roofline replay: per-launch CUDA events inside the library
    eng.set_kernel_timing(True)
    for r, dt in zip(timed, dev_tokens):
        eng.submit(None, r["batch"], r["seq_len"], r["n_decode"], 0.0, device_tokens=dt)
    eng.drain()
    kt = eng.kernel_timing()
    eng.set_kernel_timing(False)
    hbm, tc_burst, tc_sus, peak_src = load_peaks()
    total_ms = sum(v["ms"] for v in kt.values()) or 1.0
    shares = {k: v["ms"] / total_ms for k, v in kt.items()}
    classes = {}
    for k, v in kt.items():
        if v["count"] == 0 or v["ms"] <= 0:
            continue
        if k == "gemm_prefill":
            ach = v["flops"] / (v["ms"] * 1e-3) / 1e12
            classes[k] = dict(bound="tensor", achieved=ach, peak=tc_sus, unit="TFLOP/s", frac=ach / tc_sus)
        elif k == "allreduce":
            # bytes = message bytes; bus bandwidth S/t * 2(t-1)/t against NVLink 5 (spec)
            ach = v["bytes"] / (v["ms"] * 1e-3) / 1e9 * 2 * (world - 1) / world
            classes[k] = dict(bound="nvlink", achieved=ach, peak=NVLINK_SPEC_GBS, unit="GB/s (busbw)",
                              frac=ach / NVLINK_SPEC_GBS)
        else:
            ach = v["bytes"] / (v["ms"] * 1e-3) / 1e9
            classes[k] = dict(bound="hbm", achieved=ach, peak=hbm, unit="GB/s", frac=ach / hbm)
        classes[k].update(share=shares[k], launches=v["count"], avg_us=1e3 * v["ms"] / v["count"],
                          per_launch_bytes=v["bytes"] / v["count"], per_launch_flops=v["flops"] / v["count"])
    dom = max((k for k in classes if k != "allreduce"), key=lambda k: shares[k], default=None)
    roof = None
    traffic = {}
    try:   # dram bytes per launch of each kernel class from the committed `ncu --set full` capture
        with open(os.path.join(ROOT, "profiles", "traffic.json")) as f:
            traffic = json.load(f)
    except Exception:
        pass
    if dom:
        c = classes[dom]
        roof = {"kernel": dom, "bound": c["bound"], "achieved": round(c["achieved"], 2), "peak": c["peak"],
                "unit": c["unit"], "frac": round(c["frac"], 4),
                "traffic": traffic.get(dom, {}).get("dram_bytes_per_launch"),
                "traffic_algorithmic_bytes": traffic.get(dom, {}).get("algorithmic_bytes_per_launch"),
                "traffic_source": traffic.get(dom, {}).get("source"), "peak_source": peak_src,
                "share_of_kernel_time": round(c["share"], 4)}

    # ---- in-situ decode pass (no per-launch events): device time of a pass of the whole
    # decode path, from a batch with n_new generated tokens minus one with a single one,
    # against the bytes a pass must stream (this rank's weights + the KV cache it reads)
    decode_pass = None
    if not gen:
        bsz, slen = 8, 256
        ids_d = torch.from_numpy(np.random.default_rng(3).integers(0, cfg.vocab, size=bsz * slen)
                                 .astype(np.int32)).cuda()

        def batch_ms(n_new, k=1):
            best = 1e30
            for _ in range(2):
                group.barrier()
                a, z = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                a.record()
                for _ in range(k):
                    eng.submit(None, bsz, slen, n_new, 0.0, device_tokens=ids_d)
                eng.drain()
                z.record()
                z.synchronize()
                best = min(best, group.max(a.elapsed_time(z)))
            return best
        t1, tn = batch_ms(1), batch_ms(args.n_new)
        pass_us = (tn - t1) / (args.n_new - 1) * 1e3
        h, f, t = cfg.hidden, cfg.ffn, world
        w_bytes = cfg.n_layers * (4 * h * h + 2 * h * f) / t * 2 + cfg.vocab / t * h * 2
        ctx_avg = slen + args.n_new / 2
        kv_bytes = cfg.n_layers * bsz * ctx_avg * 2 * (h / t) * 2
        gbs = (w_bytes + kv_bytes) / (pass_us * 1e-6) / 1e9
        decode_pass = {"batch": bsz, "prompt": slen, "us": round(pass_us, 1),
                       "bytes": round(w_bytes + kv_bytes), "achieved": round(gbs, 1), "peak": hbm,
                       "unit": "GB/s", "frac": round(gbs / hbm, 4),
                       "note": "whole decode pass (all kernels, PDL chain intact), CUDA events around "
                               "batches with n_new and 1 generated tokens; bytes = weights + KV read"}
        if args.inflight >= 2 and args.mode == "interleaved":
            # the same with two such batches served together: what the schedule that ran
            # streams while both batches decode (at t = 1 their passes run concurrently on
            # the two streams, R31), per pass of one batch
            t1b, tnb = batch_ms(1, 2), batch_ms(args.n_new, 2)
            pass2 = (tnb - t1b) / (2 * (args.n_new - 1)) * 1e3
            gbs2 = (w_bytes + kv_bytes) / (pass2 * 1e-6) / 1e9
            decode_pass["two_batches"] = {"us_per_pass_per_batch": round(pass2, 1), "achieved": round(gbs2, 1),
                                          "frac": round(gbs2 / hbm, 4),
                                          "note": "two equal batches served together (both decode "
                                                  "concurrently); aggregate weight + KV stream"}

    # (the in-kernel trace buffer is per process: not with loopback ranks sharing one)
    gemm_situ = decode_gemm_in_situ(eng, cfg, world, torch) if not gen and not args.loopback else None
    if roof is not None and gemm_situ is not None and roof["kernel"] == "gemm_decode":
        gemm_situ["peak"] = hbm
        gemm_situ["frac"] = round(gemm_situ["achieved"] / hbm, 4)
        roof["in_situ_pdl"] = gemm_situ

    # ---- where the GPU time goes in the schedule that ran (N = 1: one traced run of 4 batches)
    cap_trace = None
    if world == 1 and not gen and not args.quick:
        cap_trace = capacity_trace(eng, make_trace(4, float("inf"), seed=args.seed, vocab=cfg.vocab,
                                                   n_decode=args.n_new), torch)

    # ---- NVLink all-reduce sweep (N > 1)
    ar_sweep = allreduce_sweep(eng, group, torch, F=args.F) if world > 1 and not args.quick else None
    scheduler = eng.scheduler_name()
    eng.close()

    # ---- the BASELINE metric: operating points of serial TP vs the interleaved mode
    ops = None
    if not args.no_latency:
        modes = ["serial", "interleaved"] + (["pipeline"] if world > 1 and not args.quick else [])
        n_b = max(8, min(args.steps, 16))
        cap_batches = len(timed) / dev_s
        fracs = (0.3, 0.5, 0.8) if args.quick else (0.2, 0.35, 0.5, 0.65, 0.8, 0.95)
        sweep = {}
        for mode in modes:
            ekw["nccl_uid"] = new_uid()
            e = LigerEngine(cfg, mode=mode, **ekw)
            e.profile([8, 64, 256, 512, 1024, 2048, 4096])
            for r in warm[:2]:
                e.submit(r["tokens"], r["batch"], r["seq_len"], r["n_decode"], 0.0)
            e.drain()
            pts = []
            for fr in fracs:
                tr = make_trace(n_b, fr * cap_batches, seed=args.seed + 1, vocab=cfg.vocab, n_decode=args.n_new,
                                **trace_kw)
                p = serve_poisson(e, group, tr)
                p["rate_req_s"] = fr * cap_batches * float(np.mean([r["batch"] for r in tr]))
                p["rate_frac_of_capacity"] = fr
                pts.append(p)
            sweep[mode] = {"scheduler": e.scheduler_name(), "points": pts}
            e.close()
        ser = sweep["serial"]["points"]
        L_star = 1.5 * ser[0]["mean_s"]
        # serial saturation: the highest swept rate it still keeps up with (completed >= 0.95 lambda)
        sat = max((p["rate_req_s"] for p in ser if p["req_s"] >= 0.95 * p["rate_req_s"]),
                  default=ser[0]["rate_req_s"])
        ops = {"L_star_s": round(L_star, 4), "serial_saturation_req_s": round(sat, 3),
               "req_s_at_L_star": {m: (round(v, 3) if v else None) for m, v in
                                   ((m, req_s_at_latency(sweep[m]["points"], L_star)) for m in sweep)},
               "sweep": {m: {"scheduler": sweep[m]["scheduler"],
                             "points": [{k: round(v, 4) for k, v in p.items()} for p in sweep[m]["points"]]}
                         for m in sweep},
               "trace": f"Poisson, {n_b} batches per point, seed {args.seed + 1}, rates = fractions of the "
                        f"measured capacity ({', '.join(str(f) for f in fracs)})"}

    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        cpu = cpu_oracle_sample(cfg)
        cpu.pop("per_batch_s", None)

    w_rank_gb = (cfg.n_layers * (4 * cfg.hidden ** 2 + 2 * cfg.hidden * cfg.ffn) + cfg.vocab * cfg.hidden) * 2 \
        / world / 1e9
    if rank == 0:
        t1_note = ("t = 1: no all-reduce to interleave (P:149); the interleaved mode runs the in-flight "
                   "batches' kernel lists concurrently on its two streams (reading R31); Algorithm 1, the "
                   "decomposition factor and the contention factor are inactive")
        result["line"] = {
            "metric": METRIC, "value": round(value, 3), "unit": "req/s", "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": round(1e3 * dev_s / len(timed), 3), "higher_is_better": True,
            "scaling": "strong", "vs_baseline": None, "dtype": "bf16", "data": "synthetic",
            "config": {"workload": (f"{cfg.name} random-init bf16, TP={world}, " +
                                    (f"generative (P:316): batches of 32 x start length 16, one sampling "
                                     f"iteration (+ the conditioning pass)" if gen else
                                     f"batches of 2/4/8 x prompt U[128,512], {args.n_new} generated tokens") +
                                    f", all {len(timed)} batches offered at once (capacity)"),
                       "model": cfg.name, "tp": world, "mode": args.mode, "scheduler": scheduler,
                       "loopback": bool(args.loopback), "sync": args.sync, "fused_ar": args.fused_ar,
                       "max_inflight": args.inflight,
                       "decomp_factor": args.F if world > 1 else None,
                       "contention_factor": (args.cf if args.cf > 0 else cf_cal) if world > 1 else None,
                       "note": t1_note if world == 1 else None,
                       "contention_factor_calibrated": round(cf_cal, 4),
                       "contention_factor_vs_gemm_sm_reserve": {str(k): v for k, v in sorted(cf_reserve.items())},
                       "sequences": seqs, "batches": len(timed),
                       "l2": f"inputs larger than L2 (weights {w_rank_gb:.1f} GB per rank)"},
            "operating_points": ops,
            "e2e": {"value": round(seqs / e2e_s, 3), "unit": "req/s", "h2d_bytes_per_step": int(h2d),
                    "d2h_bytes_per_step": int(d2h)},
            "roofline": roof,
            "allreduce": classes.get("allreduce"),
            "allreduce_sweep": ar_sweep,
            "decode_pass_in_situ": decode_pass,
            "capacity_trace": cap_trace,
            "kernel_classes": {k: {kk: (round(vv, 4) if isinstance(vv, float) else vv) for kk, vv in v.items()}
                               for k, v in classes.items()},
            "cpu_baseline": cpu,
            "clocks": clk,
            "gpu_launches": int(st["gpu_launches"]),
            "host": {"wall_s": round(wall_s, 3), "host_us": round(st["host_us"], 1),
                     "wait_us": round(st["wait_us"], 1), "rounds": st["rounds"], "kernels": st["kernels"],
                     "comm_host_us": round(st["comm_host_us"], 1),
                     "host_us_per_round_excl_wait": round((st["host_us"] - st["wait_us"]) / max(1, st["rounds"]),
                                                          2),
                     "host_us_per_round_excl_wait_and_comm": round(
                         (st["host_us"] - st["wait_us"] - st["comm_host_us"]) / max(1, st["rounds"]), 2)},
        }


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _watchdog(seconds):
    """Fail loudly instead of hanging: a rank still running after `seconds` (e.g. a peer
    lost in a collective) prints why and exits non-zero, so torchrun ends the job."""
    if seconds <= 0:
        return

    def fire():
        print(f"bench.py: rank {os.environ.get('RANK', '0')} still running after {seconds:.0f} s "
              f"(LIGER_BENCH_TIMEOUT_S); exiting", file=sys.stderr, flush=True)
        os._exit(3)
    t = threading.Timer(seconds, fire)
    t.daemon = True
    t.start()


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=12)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--config", default="opt-13b")
    ap.add_argument("--layers", type=int, default=None, help="debug only: fewer layers (invalid for reporting)")
    ap.add_argument("--mode", default="interleaved", choices=["interleaved", "serial", "pipeline", "pipeline_th"],
                    help="Liger (interleaved), Intra-Op (serial TP) or Inter-Op (pipeline) baseline")
    ap.add_argument("--inflight", type=int, default=2)
    ap.add_argument("--F", type=int, default=8)
    ap.add_argument("--cf", type=float, default=1.1, help="contention factor; <= 0: use the calibrated one")
    ap.add_argument("--n-new", type=int, default=32)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-latency", action="store_true")
    ap.add_argument("--quick", action="store_true", help="fewer operating points, no SM-reserve / AR sweeps")
    ap.add_argument("--loopback", action="store_true",
                    help="run the --gpus N ranks as threads sharing one GPU (loopback communicator dry run)")
    ap.add_argument("--seed", type=int, default=0)
    ap.add_argument("--fused-ar", action="store_true",
                    help="serial TP competitor: row-parallel GEMM + all-reduce fused over peer memory "
                         "(LIGER_FUSED_AR=1 with the one-shot peer backend; use with --mode serial)")
    ap.add_argument("--sync", default="hybrid", choices=["hybrid", "cpu_gpu", "inter_stream"],
                    help="Algorithm 1 round synchronisation (§3.4 Fig. 8; ablation §4.5)")
    ap.add_argument("--workload", default="mixed", choices=["mixed", "generative"],
                    help="mixed: batches of 2/4/8 x prompt U[128,512] + n_new generated tokens (BASELINE.json "
                         "configs[1]); generative: the paper's sampling-phase task (P:316, Fig. 11) -- batches of "
                         "32 sequences at start length 16, one sampling iteration each (the 16-token conditioning "
                         "pass that fills the KV cache is included in the step)")
    args = ap.parse_args()
    if args.workload == "generative":
        args.n_new = 2
    if args.fused_ar:
        if args.loopback:   # loopback ranks share one GPU: no peer-memory kernels there
            ap.error("--fused-ar needs one GPU per rank (not --loopback)")
        os.environ["LIGER_FUSED_AR"] = "1"
        os.environ["LIGER_ONESHOT_AR"] = "1"
    # N > 1 without torchrun: re-launch under torch.distributed.run, one process per GPU
    if (args.impl == "ours" and args.gpus > 1 and not args.loopback and "WORLD_SIZE" not in os.environ):
        cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={args.gpus}",
               "--master-addr=127.0.0.1", f"--master-port={_free_port()}", os.path.abspath(__file__)] + sys.argv[1:]
        return subprocess.call(cmd)
    _redirect_stdout()
    if args.impl == "reference":
        return run_reference(args)
    _watchdog(float(os.environ.get("LIGER_BENCH_TIMEOUT_S", "1800")))

    import torch
    result = {}
    if args.loopback:
        from paper_conf_ppopp_duwjchcl24_b200.engine import LigerEngine
        world = args.gpus
        shared = ThreadShared(world)
        errs = []

        def th(r):
            try:
                g = ThreadGroup(shared, r)
                rank_main(args, g, 0, uid_factory(g, LigerEngine.loopback_id), result)
            except Exception as e:
                import traceback
                errs.append(f"rank {r}: {e!r}\n{traceback.format_exc()}")
                shared.bar.abort()
        ths = [threading.Thread(target=th, args=(r,), daemon=True) for r in range(world)]
        for t in ths:
            t.start()
        for t in ths:
            t.join()
        if errs:
            print("\n".join(errs), file=sys.stderr)
            return 1
    else:
        import torch.distributed as dist
        world = int(os.environ.get("WORLD_SIZE", "1"))
        rank = int(os.environ.get("RANK", "0"))
        local = int(os.environ.get("LOCAL_RANK", "0"))
        if world != args.gpus:
            print(f"bench.py: WORLD_SIZE={world} but --gpus {args.gpus}", file=sys.stderr)
            return 2
        torch.cuda.set_device(local)
        if world > 1:
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
        group = DistGroup(world, rank)
        from paper_conf_ppopp_duwjchcl24_b200.engine import LigerEngine
        rank_main(args, group, local, uid_factory(group, LigerEngine.unique_id), result)
        if world > 1:
            dist.destroy_process_group()
    if "line" in result:
        emit(result["line"])
    return 0


if __name__ == "__main__":
    sys.exit(main())
