import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
from paper_conf_eurosys_wumcjlzcy21_b200 import _lib as L
torch.manual_seed(0)
for (M, K, N, ldx) in [(128, 128, 16, 128), (128, 160, 16, 160), (128, 256, 16, 256), (128, 96, 16, 96),
                       (128, 1433, 16, 1436), (128, 100, 16, 100), (128, 100, 16, 104), (777, 1433, 16, 1436)]:
    X = torch.randn(M, K, dtype=torch.float64)
    W = torch.randn(K, N, dtype=torch.float64)
    ref = (X @ W).numpy()
    Xp = torch.full((M, ldx), float("nan"))
    Xp[:, :K] = X.float()
    Xd = Xp.cuda(); Wd = W.float().cuda().contiguous()
    Y = torch.zeros(M, N, device="cuda")
    L.seastar_linear_fwd(Xd, M, K, ldx, Wd, N, None, None, "none", Y, N)
    torch.cuda.synchronize()
    y = Y.cpu().double().numpy()
    err = np.abs(y - ref)
    print(M, K, N, ldx, "max rel", err.max() / np.abs(ref).max(), "nan" if np.isnan(y).any() else "")
