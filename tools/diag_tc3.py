import sys, os
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT); sys.path.insert(0, os.path.join(ROOT, "tests"))
import numpy as np, torch
import oracle
from helpers import padded, rnd
from paper_conf_eurosys_wumcjlzcy21_b200 import _lib as L
M, K, N = 777, 1433, 16
X, W, b = rnd(1, (M, K)), rnd(2, (K, N)), rnd(3, (N,))
rs = rnd(4, (M,), 0.5, 2.0)
for (ldx, ldy, use_b, use_rs, act) in [(1436, 21, True, True, "relu"), (1436, 16, False, False, "none"),
                                        (1436, 21, False, False, "none"), (1436, 16, True, False, "none"),
                                        (1436, 16, False, True, "none"), (1436, 16, False, False, "relu")]:
    Y = torch.full((M, ldy), float("nan"), device="cuda")
    L.seastar_linear_fwd(torch.from_numpy(padded(X, ldx)).cuda(), M, K, ldx, torch.from_numpy(W).cuda(), N,
                         torch.from_numpy(b).cuda() if use_b else None, torch.from_numpy(rs).cuda() if use_rs else None,
                         act, Y, ldy)
    torch.cuda.synchronize()
    ref = oracle.linear_fwd(X, W, b if use_b else None)
    ref = oracle.act_fwd(act, ref) * (rs.astype(np.float64)[:, None] if use_rs else 1)
    y = Y.cpu().numpy()[:, :N].astype(np.float64)
    err = np.abs(y - ref)
    print(ldx, ldy, use_b, use_rs, act, "max rel", err.max() / np.abs(ref).max(), "bad rows", np.where(err.max(1) > 1e-3)[0][:10])
