"""Degree-border rows (PAPER.md L439-L441, L1253 CTA + Warp): GCN and GAT forward and backward on
a graph whose destinations and sources have in- / out-degree exactly 0, 1, 31, 32, 33, 1023, 1024, 1025, 4096, so
every bucket boundary of a3 -- sub-warp rows (< 32), warp rows (32..1023) and the multi-warp hub CTAs (>= 1024) --
is crossed on both the forward (in-degree) and the reverse (out-degree) side, vs the fp64 oracle."""
import numpy as np
import pytest

import oracle
from conftest import rel_err
from helpers import BORDER_DEGREES, border_graph, padded, rnd

pytestmark = pytest.mark.gpu
TOL = 1e-5


@pytest.fixture(scope="module")
def env():
    import torch
    assert torch.cuda.is_available()
    from paper_conf_eurosys_wumcjlzcy21_b200 import _lib as L
    from paper_conf_eurosys_wumcjlzcy21_b200.graph import Graph
    ip, ix = border_graph()
    g = Graph(ip, ix)
    info = g.info
    assert info["max_in_degree"] == 4096 and info["max_out_degree"] == 4096
    assert info["fwd_bucket_rows"][0] == 3 and info["rev_bucket_rows"][0] == 3     # degrees 1024, 1025, 4096
    return dict(torch=torch, L=L, g=g, ip=ip, ix=ix, N=len(ip) - 1)


def dev(env, a):
    return env["torch"].from_numpy(np.ascontiguousarray(a)).cuda()


def test_border_degrees_exact(env):
    indeg = np.diff(env["ip"])
    outdeg = np.bincount(env["ix"], minlength=env["N"])
    nb = len(BORDER_DEGREES)
    assert indeg[:nb].tolist() == list(BORDER_DEGREES)
    assert outdeg[nb:2 * nb].tolist() == list(BORDER_DEGREES)


@pytest.mark.parametrize("F", [16, 41, 64])
def test_gcn_borders(env, F):
    torch, L, g, N, ip, ix = env["torch"], env["L"], env["g"], env["N"], env["ip"], env["ix"]
    ld = (F + 3) // 4 * 4
    T, b = rnd(1, (N, F)), rnd(2, (F,))
    sn, dn = oracle.degree_norms(ip, ix)[::-1]
    Y = torch.full((N, ld), float("nan"), device="cuda")
    L.seastar_gcn_fwd(g.handle, dev(env, padded(T, ld)), F, ld, dev(env, dn.astype(np.float32)), dev(env, b), "relu",
                      0.0, None, Y)
    ref = oracle.act_fwd("relu", oracle.gcn_aggregate(ip, ix, T, None, dn.astype(np.float32)) + b)
    assert rel_err(Y.cpu().numpy()[:, :F], ref) <= TOL
    G = rnd(3, (N, F))
    dT = torch.full((N, ld), float("nan"), device="cuda")
    L.seastar_gcn_bwd(g.handle, dev(env, padded(G, ld)), F, ld, dev(env, sn.astype(np.float32)), 1.0, None, "none",
                      None, dT, None)
    ref = oracle.gcn_aggregate_T(ip, ix, G, sn.astype(np.float32), None)
    assert rel_err(dT.cpu().numpy()[:, :F], ref) <= TOL


@pytest.mark.parametrize("H,F", [(8, 8), (1, 41), (4, 16)])
def test_gat_borders(env, H, F):
    torch, L, g, N, ip, ix = env["torch"], env["L"], env["g"], env["N"], env["ip"], env["ix"]
    W = H * F
    ld = (W + 3) // 4 * 4
    T, el, er = rnd(11, (N, W)), rnd(12, (N, H), -2, 2), rnd(13, (N, H), -2, 2)
    A = torch.full((N, ld), float("nan"), device="cuda")
    Y = torch.full((N, ld), float("nan"), device="cuda")
    lse = torch.empty((N, H), device="cuda")
    Td = dev(env, padded(T, ld))
    L.seastar_gat_fwd(g.handle, Td, dev(env, el), dev(env, er), H, F, ld, 0.2, None, "none", A, Y, lse)
    Ar, _, _ = oracle.gat_fwd(ip, ix, T.reshape(N, H, F), el, er, 0.2)
    assert rel_err(A.cpu().numpy()[:, :W], Ar.reshape(N, W)) <= TOL
    dY = rnd(14, (N, W))
    D = torch.zeros((N, L.seastar_gat_record_ld(H, F)), device="cuda")
    L.seastar_gat_bwd_prep(g.handle, dev(env, padded(dY, ld)), Y, "none", A, dev(env, er), lse, H, F, ld, D)
    dT = torch.full((N, ld), float("nan"), device="cuda")
    dl = torch.empty((N, H), device="cuda")
    dr = torch.empty((N, H), device="cuda")
    L.seastar_gat_bwd(g.handle, Td, dev(env, el), D, H, F, ld, 0.2, dT, dl)
    L.seastar_gat_der(g.handle, Td, dev(env, el), D, H, F, ld, 0.2, dr)
    dTr, dlr, drr = oracle.gat_bwd(ip, ix, T.reshape(N, H, F), el, er, dY.reshape(N, H, F), 0.2)
    assert rel_err(dT.cpu().numpy()[:, :W], dTr.reshape(N, W)) <= TOL
    assert rel_err(dl.cpu().numpy(), dlr) <= TOL
    assert rel_err(dr.cpu().numpy(), drr) <= TOL
