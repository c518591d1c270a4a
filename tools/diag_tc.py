import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
from paper_conf_eurosys_wumcjlzcy21_b200 import _lib as L
torch.manual_seed(0)
for (M, K, N) in [(128, 32, 16), (128, 64, 16), (256, 32, 16), (128, 32, 64), (777, 1433, 16)]:
    X = torch.randn(M, K, dtype=torch.float64)
    W = torch.randn(K, N, dtype=torch.float64)
    ref = (X @ W).numpy()
    Xd = X.float().cuda().contiguous(); Wd = W.float().cuda().contiguous()
    Y = torch.zeros(M, N, device="cuda")
    L.seastar_linear_fwd(Xd, M, K, K, Wd, N, None, None, "none", Y, N)
    torch.cuda.synchronize()
    y = Y.cpu().double().numpy()
    err = np.abs(y - ref)
    print(M, K, N, "max rel", err.max() / np.abs(ref).max())
    if err.max() / np.abs(ref).max() > 1e-4:
        print("  rows bad:", np.where(err.max(1) > 1e-3 * np.abs(ref).max())[0][:20])
        print("  cols bad:", np.where(err.max(0) > 1e-3 * np.abs(ref).max())[0][:20])
        print("  y[0,:8]", y[0, :8]); print("  r[0,:8]", ref[0, :8])
        # hypothesis checks
        for name, alt in [("X only first 8 k", X[:, :8] @ W[:8]), ("transposed B?", None)]:
            if alt is not None:
                print("  ", name, np.abs(y - alt.numpy()).max() / np.abs(ref).max())
