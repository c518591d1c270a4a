"""Probe: seastar_adam vs torch's fused Adam and a plain copy on a 213.7M-parameter buffer (bgs V1 size)."""
import torch, time, sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_eurosys_wumcjlzcy21_b200 import _lib as L
n = 333845 * 640
p, g, m, v = (torch.rand(n, device="cuda") for _ in range(4))
step = torch.ones(1, dtype=torch.int32, device="cuda")
def t(f, k=10):
    f(); torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    for _ in range(k): f()
    b.record(); b.synchronize()
    return a.elapsed_time(b) / k
ms = t(lambda: L.seastar_adam(p, g, m, v, n, 0.01, 0.9, 0.999, 1e-8, step))
print(f"seastar_adam {ms:.3f} ms  {7*4*n/ms/1e6:.0f} GB/s")
y = torch.empty_like(p)
ms = t(lambda: y.copy_(p))
print(f"copy {ms:.3f} ms  {2*4*n/ms/1e6:.0f} GB/s")
ms = t(lambda: torch.add(p, g, out=y))
print(f"add (2r1w) {ms:.3f} ms  {3*4*n/ms/1e6:.0f} GB/s")
ps, gs, ms_, vs = [p], [g], [m], [v]
st = [torch.tensor(1.0, device="cuda")]
ms2 = t(lambda: torch._fused_adam_(ps, gs, ms_, vs, [], st, lr=0.01, beta1=0.9, beta2=0.999, weight_decay=0.0, eps=1e-8, amsgrad=False, maximize=False))
print(f"torch fused adam {ms2:.3f} ms  {7*4*n/ms2/1e6:.0f} GB/s")
