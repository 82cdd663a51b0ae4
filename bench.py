"""Benchmark of the Liger hot path (driver contract).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference]

Workload (BASELINE.json configs[1]): OPT-13B random-init bf16, Poisson-shaped
request batches (batch 2/4/8, prompt U[128, 512], 32 generated tokens), served
through the C ABI (liger_submit / liger_step / liger_poll).  One "step" = one
request batch through the whole hot path (prefill pass + 31 decode passes over
all 40 layers).  N GPUs = tensor parallel degree N (one process per GPU).

value    = requests (sequences) per second of the whole job with the prompts
           already resident in HBM, all K batches offered at once (capacity;
           device time between two synchronised barriers, max over ranks).
e2e      = the same with host prompts copied in and generated tokens copied
           out through the public API inside the timed region.
latency  = mean / p99 request latency (pending + execution) of a
           Poisson trace at a fixed rate of 0.5 x the measured capacity.
roofline = the dominant kernel class (by device time) in a timed replay with
           per-launch CUDA events inside the library.
"""
import argparse
import json
import math
import os
import subprocess
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)
# stdout carries exactly one JSON line: NCCL prints a version banner at NCCL_DEBUG=WARN/VERSION
os.environ["NCCL_DEBUG"] = "NONE"
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


# ----------------------------------------------------------------------------- CPU oracle baseline
def cpu_oracle_sample(cfg, b=2, s=256, n_new=32, budget_s=20.0):
    """Time the fp64 oracle on a bounded sample of the workload: one decoder
    layer's prefill over a [b, s] batch and one decode step at ctx s+16, then
    extrapolate to L layers and n_new passes (labelled as such)."""
    from oracle import model as om
    rng = np.random.default_rng(0)
    h, f = cfg.hidden, cfg.ffn
    # weights are inputs: a cheap normal generator (the oracle's arithmetic is what is timed)
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
    while True:
        om.decoder_layer(cfg, w, xd, k, v, start_pos=s)
        reps += 1
        if time.perf_counter() - t0 > min(5.0, budget_s / 4) or reps >= 8:
            break
    t_dc = (time.perf_counter() - t0) / reps
    per_batch = cfg.n_layers * (t_pf + (n_new - 1) * t_dc)
    cores = os.cpu_count()
    return {"value": b / per_batch, "unit": "req/s", "cores": cores, "kind": "oracle",
            "sample": (f"fp64 numpy oracle, one {cfg.name} layer: prefill b={b} s={s} ({t_pf:.2f}s) + "
                       f"{reps} decode steps at ctx {s + 1} ({t_dc * 1e3:.1f} ms each); extrapolated x{cfg.n_layers} "
                       f"layers x {n_new} passes"),
            "per_batch_s": per_batch}


def run_reference(args):
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return 0
    cfg = get_config(args.config)
    vals = []
    for i in range(args.warmup + args.steps):
        r = cpu_oracle_sample(cfg, budget_s=8.0)
        if i >= args.warmup:
            vals.append(r["value"])
    v = float(np.mean(vals))
    line = {"impl": "reference", "metric": METRIC, "value": v, "unit": "req/s", "n_gpus": args.gpus,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * 2 / v, "higher_is_better": True,
            "scaling": "strong", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "config": {"workload": f"{args.config} TP={args.gpus}: one layer prefill+decode sample, extrapolated",
                       "model": args.config},
            "cpu_baseline": {**{k: r[k] for k in ("unit", "cores", "kind", "sample")}, "value": v},
            "e2e": {"value": v, "unit": "req/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    emit(line)
    return 0


# ----------------------------------------------------------------------------- GPU arm
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
        os.environ["LIGER_FUSED_AR"] = "1"
        os.environ["LIGER_ONESHOT_AR"] = "1"
    _redirect_stdout()
    if args.impl == "reference":
        return run_reference(args)

    import torch
    import torch.distributed as dist
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    torch.cuda.set_device(local)
    if world > 1:
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
        gloo = dist.new_group(backend="gloo")
    from paper_conf_ppopp_duwjchcl24_b200.engine import LigerEngine
    cfg = get_config(args.config, args.layers)
    uid = None
    if world > 1:
        obj = [LigerEngine.unique_id() if rank == 0 else None]
        dist.broadcast_object_list(obj, src=0, group=gloo)
        uid = obj[0]
    gen = args.workload == "generative"
    trace_kw = (dict(batch_sizes=(32,), prompt_range=(16, 16)) if gen else {})
    eng = LigerEngine(cfg, world=world, rank=rank, nccl_uid=uid, mode=args.mode, max_batch=32 if gen else 8,
                      max_seq=16 if gen else 512, max_new=args.n_new, max_inflight=args.inflight, decomp_factor=args.F,
                      contention_factor=args.cf, seed=args.seed, sync=args.sync)
    eng.profile([8, 64, 256, 512, 1024, 2048, 4096])
    # contention factor: measured GEMM || all-reduce slowdown (1-rank proxy at N=1)
    cf_cal, _ = eng.calibrate_cf([8, 256, 1024], set_cf=args.cf <= 0)
    # contention control: the same calibration with the GEMM grid
    # leaving SMs to the communication kernel
    cf_reserve = {}
    for rsv in (8, 16, 32):
        eng.set_gemm_sm_reserve(rsv)
        cf_reserve[rsv] = round(eng.calibrate_cf([8, 256, 1024], set_cf=False)[0], 4)
    eng.set_gemm_sm_reserve(int(os.environ.get("LIGER_GEMM_SM_RESERVE", "0")))
    cf_reserve[0] = round(cf_cal, 4)

    def barrier():
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()

    def max_over_ranks(x):
        if world == 1:
            return x
        t = torch.tensor([x], dtype=torch.float64, device="cuda")
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        return float(t.item())

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
        barrier()
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
        toks = []
        eng.drain()
        if host_io:
            for bid in ids:
                toks.append(eng.poll(bid, want_tokens=True)[1])
        torch.cuda.nvtx.range_pop()
        torch.cuda.synchronize()
        e1.record()
        e1.synchronize()
        wall = time.perf_counter() - t_host0
        dev_s = max_over_ranks(e0.elapsed_time(e1) * 1e-3)
        return dev_s, wall, eng.stats(), toks

    clocks = ClockSampler(local)
    clocks.start()
    dev_s, wall_s, st, _ = timed_run(False)
    clk = clocks.stop()
    value = seqs / dev_s

    e2e_s, _, _, toks = timed_run(True)
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
        if k in ("gemm_prefill",):
            ach = v["flops"] / (v["ms"] * 1e-3) / 1e12
            classes[k] = dict(bound="tensor", achieved=ach, peak=tc_sus, unit="TFLOP/s", frac=ach / tc_sus)
        elif k == "allreduce":
            continue
        else:
            ach = v["bytes"] / (v["ms"] * 1e-3) / 1e9
            classes[k] = dict(bound="hbm", achieved=ach, peak=hbm, unit="GB/s", frac=ach / hbm)
        classes[k].update(share=shares[k], launches=v["count"], avg_us=1e3 * v["ms"] / v["count"],
                          per_launch_bytes=v["bytes"] / v["count"], per_launch_flops=v["flops"] / v["count"])
    dom = max(classes, key=lambda k: shares[k]) if classes else None
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

        def batch_ms(n_new):
            best = 1e30
            for _ in range(2):
                barrier()
                a, z = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                a.record()
                eng.submit(None, bsz, slen, n_new, 0.0, device_tokens=ids_d)
                eng.drain()
                z.record()
                z.synchronize()
                best = min(best, max_over_ranks(a.elapsed_time(z)))
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

    # ---- latency at a fixed request rate (Poisson, 0.5 x capacity)
    lat = None
    if not args.no_latency:
        cap_batches = len(timed) / dev_s
        rate = 0.5 * cap_batches
        tr = make_trace(len(timed), rate, seed=args.seed + 1, vocab=cfg.vocab, n_decode=args.n_new, **trace_kw)
        barrier()
        t0 = time.monotonic()
        ids, arr = [], []
        i = 0
        while i < len(tr) or eng_pending(eng, ids):
            now = time.monotonic() - t0
            # all ranks must submit identically: rank 0 decides how many arrivals are due
            due = sum(1 for r in tr[i:] if r["arrival_s"] <= now)
            if world > 1 and i < len(tr):   # i advances identically on every rank; afterwards no collective
                obj = [due]
                dist.broadcast_object_list(obj, src=0, group=gloo)
                due = obj[0]
            for r in tr[i:i + due]:
                ids.append(eng.submit(r["tokens"], r["batch"], r["seq_len"], r["n_decode"], t0 + r["arrival_s"]))
                arr.append(r["batch"])
            i += due
            rc = eng.step()
            if rc == 2 and i < len(tr):       # idle: wait for the next arrival
                time.sleep(max(0.0, min(0.001, tr[i]["arrival_s"] - (time.monotonic() - t0))))
        eng.drain()
        lats, wts = [], []
        for bid, bsz in zip(ids, arr):
            res, _ = eng.poll(bid)
            lats += [res.finish_s - res.arrival_s] * bsz
        lats.sort()
        lat = {"rate_req_s": rate * float(np.mean([r["batch"] for r in tr])),
               "mean_s": float(np.mean(lats)), "p99_s": float(lats[max(0, math.ceil(0.99 * len(lats)) - 1)])}

    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        cpu = cpu_oracle_sample(cfg)
        cpu.pop("per_batch_s", None)

    if rank == 0:
        line = {
            "metric": METRIC, "value": round(value, 3), "unit": "req/s", "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": round(1e3 * dev_s / len(timed), 3), "higher_is_better": True,
            "scaling": "strong", "vs_baseline": None, "dtype": "bf16", "data": "synthetic",
            "config": {"workload": (f"{cfg.name} random-init bf16, TP={world}, " +
                                    (f"generative (P:316): batches of 32 x start length 16, one sampling "
                                     f"iteration (+ the conditioning pass)" if gen else
                                     f"batches of 2/4/8 x prompt U[128,512], {args.n_new} generated tokens") +
                                    f", all {len(timed)} batches offered at once (capacity)"),
                       "model": cfg.name, "tp": world,
                       "mode": args.mode, "sync": args.sync, "fused_ar": args.fused_ar, "max_inflight": args.inflight, "decomp_factor": args.F,
                       "contention_factor": args.cf if args.cf > 0 else cf_cal,
                       "contention_factor_calibrated": round(cf_cal, 4),
                       "contention_factor_vs_gemm_sm_reserve": {str(k): v for k, v in sorted(cf_reserve.items())},
                       "sequences": seqs, "batches": len(timed),
                       "l2": "inputs larger than L2 (weights 26 GB per TP=1 rank)"},
            "latency": lat,
            "e2e": {"value": round(seqs / e2e_s, 3), "unit": "req/s", "h2d_bytes_per_step": int(h2d),
                    "d2h_bytes_per_step": int(d2h)},
            "roofline": roof,
            "decode_pass_in_situ": decode_pass,
            "kernel_classes": {k: {kk: (round(vv, 4) if isinstance(vv, float) else vv) for kk, vv in v.items()}
                               for k, v in classes.items()},
            "cpu_baseline": cpu,
            "clocks": clk,
            "gpu_launches": int(st["gpu_launches"]),
            "host": {"wall_s": round(wall_s, 3), "host_us": round(st["host_us"], 1),
                     "rounds": st["rounds"], "kernels": st["kernels"]},
        }
        emit(line)
    eng.close()
    if world > 1:
        dist.destroy_process_group()
    return 0


def eng_pending(eng, ids):
    for bid in ids:
        if eng.poll(bid) is None:
            return True
    return False


if __name__ == "__main__":
    sys.exit(main())
