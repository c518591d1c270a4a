"""NEXT-2 parity: featureless R-GCN layer with basis decomposition (seastar_rgcn_basis_fwd/bwd) and the dense
basis combination (seastar_basis_combine/_bwd) vs the fp64 oracle (tests/test_oracle_rgcn_basis.py pins it)."""
import numpy as np
import pytest

import oracle
import synth
from conftest import rel_err
from helpers import rnd

pytestmark = pytest.mark.gpu
TOL = 1e-5


@pytest.fixture(scope="module")
def env():
    import torch
    assert torch.cuda.is_available()
    from paper_conf_eurosys_wumcjlzcy21_b200 import _lib as L
    from paper_conf_eurosys_wumcjlzcy21_b200.graph import Graph
    N, R = 3000, 45
    ip, ix, et = synth.powerlaw_directed_typed(N, 24000, 0.6, 0.6, R, 1.0, 23)
    # a typed in-hub (1300 in-edges over 5 types) and an out-hub (vertex 3 sends 1100 edges): several 32-edge
    # chunks per row on both sides; 9 isolated vertices at the end
    dst = np.repeat(np.arange(N), np.diff(ip))
    hs = (rnd(5, (1300,), 0, 1).astype(np.float64) * N).astype(np.int64).clip(0, N - 1)
    ht = (rnd(6, (1300,), 0, 1).astype(np.float64) * 5).astype(np.int64).clip(0, 4)
    od = (rnd(7, (1100,), 0, 1).astype(np.float64) * N).astype(np.int64).clip(0, N - 1)
    ot = (rnd(8, (1100,), 0, 1).astype(np.float64) * R).astype(np.int64).clip(0, R - 1)
    ip, ix, et = synth.csr_from_edges(N + 9, np.concatenate([ix, hs, np.full(1100, 3)]),
                                      np.concatenate([dst, np.full(1300, 11), od]), np.concatenate([et, ht, ot]))
    g = Graph(ip, ix, et, num_etypes=R, rgcn_norm=True)
    return dict(torch=torch, L=L, g=g, ip=ip, ix=ix, et=et, N=N + 9, R=R)


def dev(env, a):
    return env["torch"].from_numpy(np.ascontiguousarray(a, np.float32)).cuda()


SHAPES = [(8, 16), (30, 16), (45, 16), (3, 4), (5, 32), (2, 128), (40, 8)]


@pytest.mark.parametrize("B,F", SHAPES)
def test_basis_fwd(env, B, F):
    torch, L, g, N, R = env["torch"], env["L"], env["g"], env["N"], env["R"]
    ldv = B * F + 4                      # padded rows: the pad must never be read into a result
    V = rnd(1, (N, B, F))
    Vp = np.full((N, ldv), np.nan, np.float32)
    Vp[:, :B * F] = V.reshape(N, B * F)
    a, b, loop = rnd(2, (R, B)), rnd(3, (F,)), rnd(4, (N, F))
    Y = torch.full((N, F), float("nan"), device="cuda")
    L.seastar_rgcn_basis_fwd(g.handle, dev(env, Vp), B, F, ldv, dev(env, a), None, dev(env, loop), F, dev(env, b),
                             "relu", Y, F)
    ref = oracle.act_fwd("relu", oracle.rgcn_basis_fwd(env["ip"], env["ix"], env["et"], V, a) + loop + b)
    assert rel_err(Y.cpu().numpy(), ref) <= TOL
    # without loop / bias / act, user norm; bitwise deterministic
    nu = rnd(9, (len(env["ix"]),), 0.1, 1.0)
    Y1, Y2 = torch.empty((N, F), device="cuda"), torch.empty((N, F), device="cuda")
    for Yk in (Y1, Y2):
        L.seastar_rgcn_basis_fwd(g.handle, dev(env, Vp), B, F, ldv, dev(env, a), dev(env, nu), None, 0, None, "none",
                                 Yk, F)
    assert torch.equal(Y1, Y2)
    assert rel_err(Y1.cpu().numpy(), oracle.rgcn_basis_fwd(env["ip"], env["ix"], env["et"], V, a, nu)) <= TOL


@pytest.mark.parametrize("B,F", SHAPES)
def test_basis_bwd(env, B, F):
    torch, L, g, N, R = env["torch"], env["L"], env["g"], env["N"], env["R"]
    V, a, dA = rnd(11, (N, B, F)), rnd(12, (R, B)), rnd(13, (N, F))
    ldv = B * F
    dV = torch.full((N, ldv), float("nan"), device="cuda")
    da = torch.full((R, B), float("nan"), device="cuda")
    ws_b = L.seastar_rgcn_basis_bwd_workspace(g.handle, B)
    ws = torch.empty(ws_b, dtype=torch.uint8, device="cuda")
    Vd = dev(env, V.reshape(N, ldv))
    L.seastar_rgcn_basis_bwd(g.handle, Vd, B, F, ldv, dev(env, a), None, dev(env, dA), F, dV, da, ws, ws_b)
    rdV, rda = oracle.rgcn_basis_bwd(env["ip"], env["ix"], env["et"], V, a, dA)
    assert rel_err(dV.cpu().numpy(), rdV.reshape(N, ldv)) <= TOL
    assert rel_err(da.cpu().numpy(), rda) <= TOL
    # bitwise deterministic, and each half alone gives the same numbers
    dV2, da2 = torch.empty_like(dV), torch.empty_like(da)
    L.seastar_rgcn_basis_bwd(g.handle, Vd, B, F, ldv, dev(env, a), None, dev(env, dA), F, dV2, None, None, 0)
    L.seastar_rgcn_basis_bwd(g.handle, Vd, B, F, ldv, dev(env, a), None, dev(env, dA), F, None, da2, ws, ws_b)
    assert torch.equal(dV, dV2) and torch.equal(da, da2)


def test_basis_reduces_to_featureless_rgcn(env):
    """B = R, a = I: the featureless lookup W_r[u] (NEXT-2 special case of the a7 layer)."""
    torch, L, g, N, R = env["torch"], env["L"], env["g"], env["N"], env["R"]
    F = 4
    V = rnd(21, (N, R, F))
    Y = torch.empty((N, F), device="cuda")
    L.seastar_rgcn_basis_fwd(g.handle, dev(env, V.reshape(N, R * F)), R, F, R * F, dev(env, np.eye(R)), None, None, 0,
                             None, "none", Y, F)
    ref = oracle.rgcn_fwd(env["ip"], env["ix"], env["et"], np.eye(N), np.transpose(V, (1, 0, 2)))
    assert rel_err(Y.cpu().numpy(), ref) <= TOL


@pytest.mark.parametrize("R,B,K", [(45, 8, 16 * 16), (90, 90, 16 * 4), (1, 1, 3), (207, 40, 16 * 2)])
def test_basis_combine(env, R, B, K):
    torch, L = env["torch"], env["L"]
    a, Vb, dW = rnd(31, (R, B)), rnd(32, (B, K)), rnd(33, (R, K))
    W = torch.empty((R, K), device="cuda")
    L.seastar_basis_combine(dev(env, a), dev(env, Vb), R, B, K, W)
    assert rel_err(W.cpu().numpy(), oracle.basis_combine(a, Vb.reshape(B, K, 1))[:, :, 0]) <= TOL
    da, dVb = torch.empty((R, B), device="cuda"), torch.empty((B, K), device="cuda")
    L.seastar_basis_combine_bwd(dev(env, a), dev(env, Vb), dev(env, dW), R, B, K, da, dVb)
    rda, rdVb = oracle.basis_combine_bwd(a, Vb.reshape(B, K, 1), dW.reshape(R, K, 1))
    assert rel_err(da.cpu().numpy(), rda) <= TOL
    assert rel_err(dVb.cpu().numpy(), rdVb[:, :, 0]) <= TOL


def test_basis_bad_args(env):
    L, g = env["L"], env["g"]
    torch = env["torch"]
    x = torch.zeros(64, device="cuda")
    with pytest.raises(L.SeastarError):
        L.seastar_rgcn_basis_fwd(g.handle, x, 2, 12, 24, x, None, None, 0, None, "none", x, 12)   # F not pow2
    with pytest.raises(L.SeastarError):
        L.seastar_rgcn_basis_fwd(g.handle, x, 200, 16, 3200, x, None, None, 0, None, "none", x, 16)  # B*F > 2048
