"""The peer-memory all-reduce kernels (csrc/peer_ar.cu one-shot; the fused row-parallel
GEMM + all-reduce of serial TP, csrc/gemm.cu fixup producer + csrc/norm.cu add + LN
consumer) element-wise against the oracle, on ONE GPU.

The ranks of these tests share the box's single GPU, where kernels that wait on each
other must not run concurrently (nothing guarantees they are co-scheduled;
B200_PROFILING.md).  Every test therefore runs each kernel phase by phase through the
C-ABI: all ranks' staging / publishing launches first, a host synchronisation, then all
ranks' waiting / summing launches, whose waits are already satisfied.  The kernels are the
ones the serving path launches with both phases in one launch per rank (one rank per GPU).
The one-shot protocol with the ranks truly concurrent (spinning on each other) runs as ONE
cooperative launch holding every rank's blocks (liger_op_oneshot_allreduce_emulated), the
emulation B200_PROFILING.md prescribes when there are fewer GPUs than ranks.

Oracle: oracle.model.allreduce_decomposed (the per-layer all-reduce of P:286 as a
sum of the ranks' bf16 partials) and oracle.model.layer_norm (C2)."""
import numpy as np
import pytest
import torch

from gpu_helpers import bf16_dev, errs, to_np64, workspace
from liger_inputs import bf16_rne, c0_values
from oracle import model as om

pytestmark = pytest.mark.gpu

CAP = 1 << 20


@pytest.fixture(scope="module")
def L():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    torch.cuda.set_device(0)
    from paper_conf_ppopp_duwjchcl24_b200 import liger
    return liger


def _regions(L, world):
    return [L.ipc_region_create(CAP)[0] for _ in range(world)]


def _free(L, regions):
    torch.cuda.synchronize()
    for r in regions:
        L.lib().liger_ipc_region_free(r)


def _part(q, n, seed=77):
    # C0 values with magnitudes clipped to [2^-10, 2^-3] (exponent gap <= 7): a sum of up
    # to 8 of them needs <= 18 significant bits, exact in fp32, so the rank-ordered fp32 sum
    # rounded once must equal bf16_rne(oracle) bit for bit
    v = c0_values(seed, 100 + q, np.arange(n, dtype=np.uint64), -3)
    return np.where(np.abs(v) < 2.0 ** -10, np.where(v < 0, -(2.0 ** -10), 2.0 ** -10), v).astype(np.float32)


def _bits(t):
    return t.view(torch.int16).cpu().numpy()


@pytest.mark.parametrize("world", [2, 4, 8])
def test_oneshot_allreduce_phased_vs_oracle(L, world):
    """a6 / a10 / a13: the one-shot kernel (stage + epoch publish, then wait + rank-ordered
    fp32 sum) on seeded bf16 partials, whole and as decomposed contiguous pieces (one epoch
    per piece, as the engine issues them), equals bf16_rne(oracle sum) bit for bit on every
    rank; epochs alternate the two staging buffers."""
    F = 8
    regions = _regions(L, world)
    epoch = 0
    try:
        for n in (8 * 5120, 16 * 1024 + 8, 256):
            parts = [_part(q, n) for q in range(world)]
            for ks in ([8], [2, 3, 3], [1] * 8):
                bufs = [bf16_dev(parts[q]) for q in range(world)]
                u = 0
                for k in ks:
                    e0, e1 = n * u // F, n * (u + k) // F
                    e0, e1 = e0 // 8 * 8, (e1 // 8 * 8 if u + k < F else n)   # 16-byte pieces
                    u += k
                    if e1 <= e0:
                        continue
                    epoch += 1
                    for q in range(world):
                        L.oneshot_allreduce(bufs[q][e0:e1], regions, q, CAP, epoch, phases=L.AR_PHASE_STAGE)
                    torch.cuda.synchronize()
                    for q in range(world):
                        L.oneshot_allreduce(bufs[q][e0:e1], regions, q, CAP, epoch, phases=L.AR_PHASE_REDUCE)
                    torch.cuda.synchronize()
                ref = om.allreduce_decomposed([p.astype(np.float64) for p in parts], F, ks)
                want = bf16_rne(ref.astype(np.float32))
                want_bits = (want.view(np.uint32) >> 16).astype(np.uint16).view(np.int16)
                for q in range(world):
                    assert np.array_equal(_bits(bufs[q]), want_bits), (world, n, ks, q)
    finally:
        _free(L, regions)


@pytest.mark.parametrize("world", [2, 4, 8])
def test_oneshot_allreduce_concurrent_ranks_vs_oracle(L, world):
    """The same kernel code with the ranks truly concurrent: every rank's one-shot all-reduce
    of a call as ONE cooperative launch (block group q = rank q: stage, publish its epoch,
    spin until all t flags arrive, rank-ordered fp32 sum), 6 consecutive calls alternating
    the staging buffers and reusing the flags and counters -- what ranks on t GPUs do, run
    with every block co-resident.  Every rank ends with bf16_rne(oracle sum), bit for bit."""
    regions = _regions(L, world)
    try:
        for epoch, n in enumerate((8 * 5120, 16 * 1024 + 8, 256, 8 * 5120, 40, 4096), start=1):
            parts = [_part(q, n, seed=90 + epoch) for q in range(world)]
            bufs = [bf16_dev(parts[q]) for q in range(world)]
            L.oneshot_allreduce_emulated(bufs, regions, CAP, epoch)
            torch.cuda.synchronize()
            ref = om.allreduce_decomposed([p.astype(np.float64) for p in parts], 1, [1])
            want = bf16_rne(ref.astype(np.float32))
            want_bits = (want.view(np.uint32) >> 16).astype(np.uint16).view(np.int16)
            for q in range(world):
                assert np.array_equal(_bits(bufs[q]), want_bits), (world, epoch, n, q)
    finally:
        _free(L, regions)


def test_oneshot_rejects_bad_phases(L):
    regions = _regions(L, 2)
    try:
        buf = torch.zeros(64, dtype=torch.bfloat16, device="cuda")
        for ph in (0, 4):
            with pytest.raises(L.LigerError):
                L.oneshot_allreduce(buf, regions, 0, CAP, 1, phases=ph)
        with pytest.raises(L.LigerError):   # epoch numbers start at 1
            L.oneshot_allreduce(buf, regions, 0, CAP, 0)
    finally:
        _free(L, regions)


@pytest.mark.parametrize("world", [2, 4])
def test_fused_gemm_allreduce_phased_vs_oracle(L, world):
    """§8(f) next row 4, the fused row-parallel GEMM + all-reduce: every rank's split-K
    GEMM fixup stages bf16(x_q W_q^T) and publishes its epoch; every rank's add + LN then
    sums the staged rows in rank order, adds the residual and the bias and normalises.
    Bit-identical to the unfused kernels (GEMM -> one-shot all-reduce -> add + LN) on every
    rank, and the oracle element-wise (C2 of x + sum_q bf16(x_q W_q^T) + b, R16 bounds)."""
    M, h, ffn = 3, 1024, 4096
    K = ffn // world
    plan = L.gemm_plan(M, h, K)
    assert plan["splits"] > 1   # the fixup kernel is the producer
    xs = [c0_values(5, 10 + q, np.arange(M * K, dtype=np.uint64), -1).reshape(M, K) for q in range(world)]
    ws_ = [c0_values(5, 20 + q, np.arange(h * K, dtype=np.uint64), -6).reshape(h, K) for q in range(world)]
    res = c0_values(5, 30, np.arange(M * h, dtype=np.uint64), -2).reshape(M, h)
    bias = c0_values(5, 31, np.arange(h, dtype=np.uint64), -6)
    g = 1 + c0_values(5, 32, np.arange(h, dtype=np.uint64), -4)
    be = c0_values(5, 33, np.arange(h, dtype=np.uint64), -4)
    xd = [bf16_dev(x) for x in xs]
    wt = []
    for w in ws_:
        t = torch.empty(L.tiled_numel(h, K), dtype=torch.bfloat16, device="cuda")
        L.tile_weight(bf16_dev(w), t)
        wt.append(t)
    gd, bed, bd = bf16_dev(g), bf16_dev(be), bf16_dev(bias)
    wss = [workspace(L.gemm_workspace_bytes(M, h, K)) for _ in range(world)]
    regions = _regions(L, world)
    try:
        # fused: producers (every rank), sync, consumers (every rank)
        xo_f = [bf16_dev(res) for _ in range(world)]
        y_f = [torch.empty(M, h, dtype=torch.bfloat16, device="cuda") for _ in range(world)]
        for q in range(world):
            L.gemm_fused_ar_stage(xd[q], wt[q], M, h, K, regions, q, CAP, 1, wss[q])
        torch.cuda.synchronize()
        for q in range(world):
            L.add_layernorm_fused_ar(regions, q, CAP, 1, xo_f[q], bd, xo_f[q], y_f[q], gd, bed)
        torch.cuda.synchronize()
        # unfused: GEMM partials, one-shot all-reduce (phased), add + LN
        parts = [torch.empty(M, h, dtype=torch.bfloat16, device="cuda") for _ in range(world)]
        for q in range(world):
            L.gemm_tiled(xd[q], wt[q], parts[q], N=h, workspace=wss[q])
        torch.cuda.synchronize()
        part_np = [to_np64(p) for p in parts]
        for q in range(world):
            L.oneshot_allreduce(parts[q], regions, q, CAP, 2, phases=L.AR_PHASE_STAGE)
        torch.cuda.synchronize()
        for q in range(world):
            L.oneshot_allreduce(parts[q], regions, q, CAP, 2, phases=L.AR_PHASE_REDUCE)
        torch.cuda.synchronize()
        xo_u, y_u = [], []
        for q in range(world):
            xo = bf16_dev(res)
            y = torch.empty(M, h, dtype=torch.bfloat16, device="cuda")
            L.add_layernorm(xo, gd, bed, y, add=parts[q], add_bias=bd, x_out=xo)
            xo_u.append(xo)
            y_u.append(y)
        torch.cuda.synchronize()
        for q in range(world):
            assert np.array_equal(_bits(xo_f[q]), _bits(xo_u[0])), q
            assert np.array_equal(_bits(y_f[q]), _bits(y_u[0])), q
        # oracle: the GEMM partials (fp64 products of the bf16 operands), their sum, C2
        P = [to_np64(xd[q]) @ to_np64(bf16_dev(ws_[q])).T for q in range(world)]
        for q in range(world):   # each rank's partial (before the sum) vs the oracle's
            rel, mae = errs(part_np[q], P[q])
            assert rel <= 2e-2 and mae <= 1e-3, (q, rel, mae)
        r = res.astype(np.float64) + sum(P) + bias
        rel, mae = errs(to_np64(xo_f[0]), r)
        assert rel <= 2e-2 and mae <= 1e-3, (rel, mae)
        ref = om.layer_norm(r, g.astype(np.float64), be.astype(np.float64), 1e-5)
        rel, mae = errs(to_np64(y_f[0]), ref)
        assert rel <= 2e-2 and mae <= 1e-2, (rel, mae)
    finally:
        _free(L, regions)
