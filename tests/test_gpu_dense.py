"""a4 / a11 and the training glue on the GPU vs the oracle: dense transform fwd/bwd, softmax
cross-entropy, column sums, Adam."""
import numpy as np
import pytest

import oracle
from conftest import rel_err
from helpers import padded, rnd

pytestmark = pytest.mark.gpu
TOL = 1e-5


@pytest.fixture(scope="module")
def env():
    import torch
    assert torch.cuda.is_available()
    from paper_conf_eurosys_wumcjlzcy21_b200 import _lib as L
    return dict(torch=torch, L=L)


def dev(env, a):
    return env["torch"].from_numpy(np.ascontiguousarray(a)).cuda()


SHAPES = [(1, 1, 1), (5, 3, 7), (1000, 602, 16), (3001, 64, 41), (777, 1433, 16), (2000, 70, 64), (513, 16, 70),
          (300, 8710, 8)]


@pytest.mark.parametrize("M,K,N", SHAPES)
def test_linear_fwd(env, M, K, N):
    torch, L = env["torch"], env["L"]
    X, W, b = rnd(1, (M, K)), rnd(2, (K, N)), rnd(3, (N,))
    rs = rnd(4, (M,), 0.5, 2.0)
    ldx = K + 3
    ldy = N + 5
    Y = torch.full((M, ldy), float("nan"), device="cuda")
    L.seastar_linear_fwd(dev(env, padded(X, ldx)), M, K, ldx, dev(env, W), N, dev(env, b), dev(env, rs), "relu",
                         Y, ldy)
    ref = oracle.act_fwd("relu", oracle.linear_fwd(X, W, b)) * rs.astype(np.float64)[:, None]
    assert rel_err(Y.cpu().numpy()[:, :N], ref) <= TOL
    assert np.isnan(Y.cpu().numpy()[:, N:]).all()


TC_SHAPES = [(128, 32, 16), (1000, 602, 16), (5003, 602, 64), (777, 64, 41), (3001, 1433, 70), (300, 8710, 8),
             (2048, 100, 128), (129, 33, 1),
             (60000, 602, 64),   # many chunks per CTA: the raw-tile ring wraps many times (r2: a WAR race showed here)
             (5000, 2048, 64), (19793, 8710, 64), (2708, 1433, 16)]   # K splits (few row tiles, long K)


@pytest.mark.parametrize("M,K,N", TC_SHAPES)
def test_linear_fwd_tcgen05(env, M, K, N):
    """ldx % 4 == 0 and 16-B aligned X -> the tcgen05 3xTF32 kernel (TMA + TMEM); must meet the fp32 tolerance."""
    torch, L = env["torch"], env["L"]
    X, W, b = rnd(41, (M, K)), rnd(42, (K, N)), rnd(43, (N,))
    rs = rnd(44, (M,), 0.5, 2.0)
    ldx = (K + 3) // 4 * 4 + 4
    ldy = (N + 3) // 4 * 4
    Y = torch.full((M, ldy), float("nan"), device="cuda")
    ws_b = L.seastar_linear_fwd_workspace(K, N)
    ws = torch.empty(ws_b, dtype=torch.uint8, device="cuda")
    L.seastar_linear_fwd(dev(env, padded(X, ldx)), M, K, ldx, dev(env, W), N, dev(env, b), dev(env, rs), "relu",
                         Y, ldy, ws, ws_b)
    ref = oracle.act_fwd("relu", oracle.linear_fwd(X, W, b)) * rs.astype(np.float64)[:, None]
    assert rel_err(Y.cpu().numpy()[:, :N], ref) <= TOL
    if ldy > N:
        assert np.isnan(Y.cpu().numpy()[:, N:]).all()
    # large-magnitude inputs: the hi/lo split keeps fp32 accuracy (1xTF32 would miss by ~1e-3)
    X2 = (X.astype(np.float64) * 1e3 + 0.123456789).astype(np.float32)
    L.seastar_linear_fwd(dev(env, padded(X2, ldx)), M, K, ldx, dev(env, W), N, None, None, "none", Y, ldy, ws, ws_b)
    assert rel_err(Y.cpu().numpy()[:, :N], oracle.linear_fwd(X2, W)) <= TOL


@pytest.mark.parametrize("M,K,N", SHAPES)
def test_linear_bwd(env, M, K, N):
    torch, L = env["torch"], env["L"]
    X, W, dY = rnd(5, (M, K)), rnd(6, (K, N)), rnd(7, (M, N))
    rs = rnd(8, (M,), 0.5, 2.0)
    dX = torch.empty((M, K), device="cuda")
    Z = rnd(9, (M, K)).astype(np.float64)
    Yact = oracle.act_fwd("elu", Z).astype(np.float32)
    L.seastar_linear_bwd_data(dev(env, dY), M, N, N, dev(env, W), K, dev(env, rs), dev(env, Yact), "elu", dX, K)
    rdX, rdW, rdb = oracle.linear_bwd(X, W, dY)
    assert rel_err(dX.cpu().numpy(), oracle.act_bwd("elu", Z, rdX * rs.astype(np.float64)[:, None])) <= TOL
    ws_b = L.seastar_linear_bwd_weight_workspace(M, K, N)
    ws = torch.empty(ws_b, dtype=torch.uint8, device="cuda")
    dW = torch.empty((K, N), device="cuda")
    db = torch.empty((N,), device="cuda")
    L.seastar_linear_bwd_weight(dev(env, X), M, K, K, dev(env, dY), N, N, dW, db, ws, ws_b)
    assert rel_err(dW.cpu().numpy(), rdW) <= TOL
    assert rel_err(db.cpu().numpy(), rdb) <= TOL


@pytest.mark.parametrize("M,C", [(1, 1), (100, 7), (5000, 41), (3000, 70)])
def test_softmax_xent(env, M, C):
    torch, L = env["torch"], env["L"]
    Z = rnd(9, (M, C), -3, 3)
    lab = (rnd(10, (M,), 0, 1).astype(np.float64) * C).astype(np.int64).clip(0, C - 1)
    ws_b = L.seastar_softmax_xent_workspace(M)
    ws = torch.empty(ws_b, dtype=torch.uint8, device="cuda")
    loss = torch.empty((1,), device="cuda")
    dZ = torch.empty((M, C), device="cuda")
    L.seastar_softmax_xent(dev(env, Z), M, M, C, C, dev(env, lab), loss, dZ, C, ws, ws_b)
    rl, rd = oracle.softmax_xent(Z, lab)
    assert abs(loss.item() - rl) <= TOL * abs(rl)
    assert rel_err(dZ.cpu().numpy(), rd) <= TOL
    # a rank holding M of n_total rows scales by the global count
    L.seastar_softmax_xent(dev(env, Z), M, 3 * M, C, C, dev(env, lab), loss, dZ, C, ws, ws_b)
    assert abs(loss.item() - rl / 3) <= TOL * abs(rl)
    assert rel_err(dZ.cpu().numpy(), rd / 3) <= TOL


def test_colsum_axpby_adam(env):
    torch, L = env["torch"], env["L"]
    M, F = 12345, 37
    X = rnd(11, (M, F))
    ws_b = L.seastar_colsum_workspace(M, F)
    ws = torch.empty(ws_b, dtype=torch.uint8, device="cuda")
    out = torch.empty((F,), device="cuda")
    L.seastar_colsum(dev(env, padded(X, 40)), M, F, 40, out, ws, ws_b)
    assert rel_err(out.cpu().numpy(), X.astype(np.float64).sum(0)) <= TOL
    x, y = rnd(12, (1000,)), rnd(13, (1000,))
    yd = dev(env, y.copy())
    L.seastar_axpby(1000, 0.5, dev(env, x), -2.0, yd)
    assert rel_err(yd.cpu().numpy(), 0.5 * x.astype(np.float64) - 2.0 * y) <= TOL
    n = 4097
    p, g = rnd(14, (n,)), rnd(15, (n,))
    pd, md, vd = dev(env, p.copy()), torch.zeros(n, device="cuda"), torch.zeros(n, device="cuda")
    step = torch.zeros(1, dtype=torch.int32, device="cuda")
    pr, mr, vr = p.astype(np.float64), np.zeros(n), np.zeros(n)
    for t in (1, 2, 3):
        L.seastar_step_inc(step)
        L.seastar_adam(pd, dev(env, g), md, vd, n, 0.01, 0.9, 0.999, 1e-8, step)
        oracle.adam(pr, g, mr, vr, 0.01, t)
    assert rel_err(pd.cpu().numpy() - p, pr - p) <= 1e-4   # update magnitude ~lr; compare the deltas


TC_TN_SHAPES = [(256, 32, 1), (1000, 602, 16), (5003, 602, 64), (3001, 64, 41), (300, 8710, 8), (4099, 100, 33),
                (20000, 128, 32), (233, 602, 16), (2000, 64, 70), (3000, 100, 130), (300, 40, 200),
                (60000, 602, 64), (60000, 602, 32)]   # >= 16 chunks per CTA (r2: the raw-ring WAR race of tc_tn2)


@pytest.mark.parametrize("M,K,N", TC_TN_SHAPES)
def test_linear_bwd_weight_tcgen05(env, M, K, N):
    """ldx % 4 == ldy % 4 == 0 (16-B aligned rows) -> the tcgen05 MN-major 3xTF32 dW kernel (M >= 256)."""
    torch, L = env["torch"], env["L"]
    X, dY = rnd(51, (M, K)), rnd(52, (M, N))
    ldx = (K + 3) // 4 * 4 + 4
    ldy = (N + 3) // 4 * 4
    ws_b = L.seastar_linear_bwd_weight_workspace(M, K, N)
    ws = torch.empty(ws_b, dtype=torch.uint8, device="cuda")
    dW = torch.full((K, N), float("nan"), device="cuda")
    db = torch.empty((N,), device="cuda")
    L.seastar_linear_bwd_weight(dev(env, padded(X, ldx)), M, K, ldx, dev(env, padded(dY, ldy)), N, ldy, dW, db, ws,
                                ws_b)
    _, rdW, rdb = oracle.linear_bwd(X, np.zeros((K, N), np.float32), dY)
    assert rel_err(dW.cpu().numpy(), rdW) <= TOL
    assert rel_err(db.cpu().numpy(), rdb) <= TOL
    # large-magnitude rows: the hi/lo split keeps fp32 accuracy
    X2 = (X.astype(np.float64) * 1e3 + 0.123456789).astype(np.float32)
    L.seastar_linear_bwd_weight(dev(env, padded(X2, ldx)), M, K, ldx, dev(env, padded(dY, ldy)), N, ldy, dW, db, ws,
                                ws_b)
    _, rdW2, _ = oracle.linear_bwd(X2, np.zeros((K, N), np.float32), dY)
    assert rel_err(dW.cpu().numpy(), rdW2) <= TOL


def test_row_scale():
    """seastar_row_scale (APPNP's n (.) pre-scaling): Y[i] = s[i] X[i], strided and in place."""
    import torch
    from paper_conf_eurosys_wumcjlzcy21_b200 import _lib as L
    import synth
    M, F, ld = 1000, 5, 8
    X = synth.uniform(1, (M, ld))
    s = synth.uniform(2, (M,), 0.1, 2.0)
    Xd, sd = torch.from_numpy(X).cuda(), torch.from_numpy(s).cuda()
    Y = torch.full((M, ld), float("nan"), device="cuda")
    L.seastar_row_scale(Xd, M, F, ld, sd, Y, ld)
    np.testing.assert_array_equal(Y.cpu().numpy()[:, :F], (s[:, None] * X[:, :F]).astype(np.float32))
    L.seastar_row_scale(Xd, M, F, ld, sd, Xd, ld)
    np.testing.assert_array_equal(Xd.cpu().numpy()[:, :F], Y.cpu().numpy()[:, :F])
