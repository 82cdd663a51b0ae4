"""Quick GPU sanity check of the kernel entry points against torch (dev tool)."""
import sys, time, torch
sys.path.insert(0, __file__.rsplit('/tools/', 1)[0])
from paper_conf_ppopp_duwjchcl24_b200 import liger as L
L.lib()
dev = 'cuda'
torch.manual_seed(0)

def rel(a, b):
    return ((a.float() - b.float()).abs().max() / b.float().abs().max().clamp_min(1e-30)).item()

ok = True
for (M, N, K) in [(2, 384, 256), (16, 256, 128), (64, 512, 256), (300, 640, 1024), (256, 5120, 5120), (8, 15360, 5120), (1000, 2048, 4096), (33, 1000, 3000)]:
    x = (torch.randn(M, K, device=dev) * 0.5).bfloat16()
    w = (torch.randn(N, K, device=dev) / K ** 0.5).bfloat16()
    b = (torch.randn(N, device=dev) * 0.1).bfloat16()
    out = torch.zeros(M, N, device=dev, dtype=torch.bfloat16)
    ws = torch.zeros(max(L.gemm_workspace_bytes(M, N, K), 16384) // 4 + 1, device=dev, dtype=torch.int32)
    L.gemm(x, w, out, bias=b, act="gelu_tanh", scale_cols=N // 3, scale=0.125, workspace=ws)
    torch.cuda.synchronize()
    ref = x.float() @ w.float().T + b.float()
    ref[:, :N // 3] *= 0.125
    ref = torch.nn.functional.gelu(ref, approximate='tanh')
    r = rel(out, ref)
    # slices must be bit-identical
    out2 = torch.zeros_like(out)
    step = max(16, (N // 8) // 16 * 16)
    c = 0
    while c < N:
        L.gemm(x, w, out2, n0=c, n1=min(N, c + step), bias=b, act="gelu_tanh", scale_cols=N // 3, scale=0.125, workspace=ws)
        c += step
    torch.cuda.synchronize()
    same = torch.equal(out, out2)
    print(f"gemm M={M} N={N} K={K}: rel={r:.3e} slices_bitexact={same}")
    ok &= r < 2e-2 and same

# timing of a decode-like and prefill-like gemm
for (M, N, K) in [(8, 15360, 5120), (2, 20480, 5120), (4096, 15360, 5120), (256, 5120, 5120)]:
    x = torch.randn(M, K, device=dev).bfloat16(); w = (torch.randn(N, K, device=dev) / K ** 0.5).bfloat16()
    out = torch.empty(M, N, device=dev, dtype=torch.bfloat16)
    ws = torch.zeros(max(L.gemm_workspace_bytes(M, N, K), 16384) // 4 + 1, device=dev, dtype=torch.int32)
    for _ in range(3): L.gemm(x, w, out, workspace=ws)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(); n = 20
    for _ in range(n): L.gemm(x, w, out, workspace=ws)
    e1.record(); torch.cuda.synchronize()
    t = e0.elapsed_time(e1) / n * 1e-3
    print(f"time M={M} N={N} K={K}: {t*1e6:.1f} us  {2*M*N*K/t/1e12:.1f} TFLOP/s  {(N*K*2+M*K*2+M*N*2)/t/1e9:.0f} GB/s")

# layernorm
for (R, h) in [(5, 256), (64, 5120), (3, 12288)]:
    x = torch.randn(R, h, device=dev).bfloat16(); a = torch.randn(R, h, device=dev).bfloat16(); ab = torch.randn(h, device=dev).bfloat16()
    g = torch.randn(h, device=dev).bfloat16(); be = torch.randn(h, device=dev).bfloat16()
    y = torch.empty_like(x); xo = torch.empty_like(x)
    L.add_layernorm(x, g, be, y, add=a, add_bias=ab, x_out=xo)
    torch.cuda.synchronize()
    r_ = (x.float() + a.float() + ab.float()).bfloat16().float()
    ref = torch.nn.functional.layer_norm(r_, (h,), g.float(), be.float(), 1e-5)
    print(f"ln R={R} h={h}: rel={rel(y, ref):.3e} xo_exact={torch.equal(xo.float(), r_)}")

# attention prefill + decode vs SDPA
for (b, s, heads, d) in [(2, 32, 2, 64), (2, 100, 3, 128), (1, 300, 2, 128)]:
    qkv = (torch.randn(b * s, 3 * heads * d, device=dev) * 0.5).bfloat16()
    qkv[:, :heads * d] *= d ** -0.5
    o = torch.empty(b * s, heads * d, device=dev, dtype=torch.bfloat16)
    maxp = (s + 64) // 16 + 1
    pt = torch.arange(b * maxp, device=dev, dtype=torch.int32).reshape(b, maxp)
    pool = torch.zeros(b * maxp, 2, heads, 16, d, device=dev, dtype=torch.bfloat16)
    L.attn_prefill(qkv, o, pool, pt, b=b, s=s, heads=heads, d=d)
    torch.cuda.synchronize()
    q = qkv[:, :heads*d].float().reshape(b, s, heads, d).transpose(1, 2)
    k = qkv[:, heads*d:2*heads*d].float().reshape(b, s, heads, d).transpose(1, 2)
    v = qkv[:, 2*heads*d:].float().reshape(b, s, heads, d).transpose(1, 2)
    ref = torch.nn.functional.scaled_dot_product_attention(q, k, v, is_causal=True, scale=1.0).transpose(1, 2).reshape(b * s, heads * d)
    print(f"prefill b={b} s={s} h={heads} d={d}: rel={rel(o, ref):.3e}")
    # cache content check
    kc = pool[:, 0].permute(0, 2, 1, 3)  # page, tok, head, d
    kk = torch.stack([kc[pt[bi, p // 16], p % 16] for bi in range(b) for p in range(s)]).reshape(b, s, heads, d)
    print("  cache K exact:", torch.equal(kk.transpose(1, 2).float(), k))
    # decode one step at pos = s
    qkv1 = (torch.randn(b, 3 * heads * d, device=dev) * 0.5).bfloat16()
    qkv1[:, :heads * d] *= d ** -0.5
    o1 = torch.empty(b, heads * d, device=dev, dtype=torch.bfloat16)
    ws = torch.zeros(L.attn_decode_workspace_bytes(b, heads, d, s + 1) // 4 + 1, device=dev, dtype=torch.int32)
    L.attn_decode(qkv1, o1, pool, pt, b=b, pos=s, heads=heads, d=d, workspace=ws)
    torch.cuda.synchronize()
    q1 = qkv1[:, :heads*d].float().reshape(b, 1, heads, d).transpose(1, 2)
    k1 = torch.cat([k, qkv1[:, heads*d:2*heads*d].float().reshape(b, 1, heads, d).transpose(1, 2)], 2)
    v1 = torch.cat([v, qkv1[:, 2*heads*d:].float().reshape(b, 1, heads, d).transpose(1, 2)], 2)
    ref1 = torch.nn.functional.scaled_dot_product_attention(q1, k1, v1, scale=1.0).transpose(1, 2).reshape(b, heads * d)
    print(f"decode pos={s}: rel={rel(o1, ref1):.3e}")
print("OK" if ok else "GEMM FAILED")
