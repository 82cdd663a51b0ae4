"""Dev experiment: spacing of dependent back-to-back kernels (PDL on/off)."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_ppopp_duwjchcl24_b200 import liger as L
h = 5120
x = torch.randn(8, h, device="cuda").bfloat16(); g = torch.randn(h, device="cuda").bfloat16(); y = torch.empty_like(x)
def chain(n):
    for _ in range(n):
        L.add_layernorm(x, g, g, y)
        L.add_layernorm(y, g, g, x)
for _ in range(3): chain(10)
torch.cuda.synchronize()
a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
a.record(); chain(200); b.record(); torch.cuda.synchronize()
print(f"LN chain: {a.elapsed_time(b) / 400 * 1e3:.2f} us per dependent kernel (PDL {'off' if os.environ.get('LIGER_NO_PDL') else 'on'})")
