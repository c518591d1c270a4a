"""Time the dense / row kernels of a Reddit-shaped step in isolation (CUDA events, 10 reps after warm-up).

    python tools/bench_dense.py
Shapes: M = 232,965 vertices, F_in = 602 (ld 604), GCN hidden 16, GAT 8 heads x 8, 41 classes.
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_eurosys_wumcjlzcy21_b200 import _lib as L  # noqa: E402

M, K, LDX = 232965, 602, 604
dev = "cuda"
torch.manual_seed(0)
X = torch.randn(M, LDX, device=dev)


def timeit(name, fn, bytes_=None, reps=10):
    for _ in range(3):
        fn()
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    for _ in range(reps):
        fn()
    b.record()
    torch.cuda.synchronize()
    ms = a.elapsed_time(b) / reps
    extra = f"  {bytes_ / ms / 1e6:8.0f} GB/s" if bytes_ else ""
    print(f"{name:40s} {ms:8.4f} ms{extra}", flush=True)
    return ms


for N in (16, 64):
    W = torch.randn(K, N, device=dev) * 0.05
    ldy = (N + 3) // 4 * 4
    Y = torch.empty(M, ldy, device=dev)
    wsb = L.seastar_linear_fwd_workspace(K, N)
    ws = torch.empty(wsb, dtype=torch.uint8, device=dev)
    timeit(f"linear_fwd tc   M x {K} x {N}", lambda: L.seastar_linear_fwd(X, M, K, LDX, W, N, None, None, "none", Y, ldy,
                                                                           ws, wsb), M * LDX * 4 + M * ldy * 4)
    dY = torch.randn(M, ldy, device=dev)
    dW = torch.empty(K, N, device=dev)
    db = torch.empty(N, device=dev)
    wsb2 = L.seastar_linear_bwd_weight_workspace(M, K, N)
    ws2 = torch.empty(wsb2, dtype=torch.uint8, device=dev)
    timeit(f"linear_bwd_weight M x {K} x {N}", lambda: L.seastar_linear_bwd_weight(X, M, K, LDX, dY, N, ldy, dW, db, ws2,
                                                                                  wsb2), M * LDX * 4 + M * ldy * 4)

# layer-2 shapes
for (K2, N2) in ((16, 41), (64, 41)):
    H1 = torch.randn(M, K2, device=dev)
    W2 = torch.randn(K2, N2, device=dev)
    Z = torch.empty(M, 44, device=dev)
    wsb = L.seastar_linear_fwd_workspace(K2, N2)
    ws = torch.empty(wsb, dtype=torch.uint8, device=dev)
    timeit(f"linear_fwd      M x {K2} x {N2}", lambda: L.seastar_linear_fwd(H1, M, K2, K2, W2, N2, None, None, "none", Z,
                                                                           44, ws, wsb), M * (K2 + 44) * 4)
    dZ = torch.randn(M, 44, device=dev)
    dH = torch.empty(M, K2, device=dev)
    timeit(f"linear_bwd_data M x {N2} -> {K2}", lambda: L.seastar_linear_bwd_data(dZ, M, N2, 44, W2, K2, None, H1, "elu",
                                                                                  dH, K2), M * (44 + 2 * K2) * 4)
    dW2 = torch.empty(K2, N2, device=dev)
    db2 = torch.empty(N2, device=dev)
    wsb2 = L.seastar_linear_bwd_weight_workspace(M, K2, N2)
    ws2 = torch.empty(wsb2, dtype=torch.uint8, device=dev)
    timeit(f"linear_bwd_weight M x {K2} x {N2}", lambda: L.seastar_linear_bwd_weight(H1, M, K2, K2, dZ, N2, 44, dW2, db2,
                                                                                    ws2, wsb2), M * (K2 + 44) * 4)

# softmax / colsum
C = 41
Zs = torch.randn(M, 44, device=dev)
lab = torch.randint(0, C, (M,), device=dev)
loss = torch.empty(1, device=dev)
dZs = torch.empty(M, 44, device=dev)
wsb = L.seastar_softmax_xent_workspace(M)
ws = torch.empty(wsb, dtype=torch.uint8, device=dev)
timeit("softmax_xent", lambda: L.seastar_softmax_xent(Zs, M, M, C, 44, lab, loss, dZs, 44, ws, wsb), M * 88 * 4)
out = torch.empty(64, device=dev)
wsb = L.seastar_colsum_workspace(M, 64)
ws = torch.empty(wsb, dtype=torch.uint8, device=dev)
T64 = torch.randn(M, 64, device=dev)
timeit("colsum M x 64", lambda: L.seastar_colsum(T64, M, 64, 64, out, ws, wsb), M * 64 * 4)
