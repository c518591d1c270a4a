import os, sys, torch, numpy as np
sys.path.insert(0, os.getcwd())
from paper_conf_eurosys_wumcjlzcy21_b200 import _lib as L
torch.manual_seed(0)
for (M, K, N, ldx, ldy) in [(5003, 602, 64, 604, 64), (20000, 602, 64, 604, 64), (60000, 602, 64, 604, 64), (232965, 602, 64, 604, 64), (232965, 602, 16, 604, 16), (19793, 8710, 64, 8712, 64), (60000, 602, 32, 604, 32)]:
    X = torch.randn(M, ldx, device="cuda"); dY = torch.randn(M, ldy, device="cuda")
    ref = (X[:, :K].double().T @ dY[:, :N].double())
    ws_b = L.seastar_linear_bwd_weight_workspace(M, K, N)
    ws = torch.empty(ws_b, dtype=torch.uint8, device="cuda")
    dW = torch.full((K, N), float("nan"), device="cuda"); db = torch.empty(N, device="cuda")
    L.seastar_linear_bwd_weight(X, M, K, ldx, dY, N, ldy, dW, db, ws, ws_b)
    torch.cuda.synchronize()
    err = ((dW.double() - ref).abs().max() / ref.abs().max()).item()
    bad = ((dW.double() - ref).abs() > 1e-4 * ref.abs().max()).nonzero()
    print(M, K, N, "err", err, "bad", bad.shape[0], bad[:5].tolist() if bad.shape[0] else "")
