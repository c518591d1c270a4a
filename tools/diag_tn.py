"""Debug the tcgen05 dW kernel: compare with fp64 numpy on a few shapes."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
from paper_conf_eurosys_wumcjlzcy21_b200 import _lib as L
for (M, K, N) in [(256, 32, 1), (256, 32, 32), (256, 128, 32), (1024, 128, 64), (1000, 602, 16), (5003, 602, 64)]:
    rng = np.random.default_rng(0)
    X = rng.standard_normal((M, K)).astype(np.float32)
    dY = rng.standard_normal((M, N)).astype(np.float32)
    ldx = (K + 3) // 4 * 4 + 4
    ldy = (N + 3) // 4 * 4
    Xp = np.zeros((M, ldx), np.float32); Xp[:, :K] = X
    Yp = np.zeros((M, ldy), np.float32); Yp[:, :N] = dY
    wsb = L.seastar_linear_bwd_weight_workspace(M, K, N)
    ws = torch.zeros(wsb, dtype=torch.uint8, device="cuda")
    dW = torch.full((K, N), float("nan"), device="cuda")
    L.seastar_linear_bwd_weight(torch.from_numpy(Xp).cuda(), M, K, ldx, torch.from_numpy(Yp).cuda(), N, ldy, dW, None, ws, wsb)
    torch.cuda.synchronize()
    got = dW.cpu().numpy()
    ref = X.astype(np.float64).T @ dY.astype(np.float64)
    err = np.abs(got - ref).max() / np.abs(ref).max()
    print(M, K, N, "err", err, "zeros", (got == 0).mean(), "nan", np.isnan(got).mean())
    if err > 1e-5:
        # which structure? compare with transposed / partial products
        print("  got[:4,:4]", got[:4, :4]); print("  ref[:4,:4]", ref[:4, :4])
        part = ws[: K * N * 4].view(torch.float32).cpu().numpy().reshape(K, N) if True else None
        print("  part0[:2,:4]", part[:2, :4])
