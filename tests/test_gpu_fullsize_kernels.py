"""Kernel parity at the bench's full size: every graph kernel of the Reddit-shaped step (configs[4],
114.6 M edges), launched exactly as bench.py launches it (same graph handle, same kernel variants:
GCN F = 16; GAT head-per-lane 8 x 8 and single-head 1 x 41, forward-saved der factors), on seeded
synthetic inputs shared with the oracle, compared on sampled output rows the oracle computes one
by one (and on whole tensors where the oracle produces them anyway).

Row sample: 2,000 seeded-random vertices + the 64 largest and 64 smallest in- and out-degree
vertices (the hub rows take the CTA / multi-warp paths, the smallest the sub-warp paths).
Tolerance: north_star's 1e-5, max-abs normalised per tensor.
"""
import numpy as np
import pytest

import oracle
import synth
from conftest import rel_err
from helpers import padded, rnd

pytestmark = pytest.mark.gpu
TOL = 1e-5


@pytest.fixture(scope="module")
def R():
    import torch
    assert torch.cuda.is_available()
    from paper_conf_eurosys_wumcjlzcy21_b200 import _lib as L
    from paper_conf_eurosys_wumcjlzcy21_b200.graph import Graph
    cfg = synth.CONFIGS["reddit"]
    ip, ix = synth.make_graph(cfg)
    N = cfg.N
    indeg = np.diff(ip)
    outdeg = np.bincount(ix, minlength=N)
    pick = (synth.uniform(77, (2000,), 0, 1).astype(np.float64) * N).astype(np.int64).clip(0, N - 1)
    o_in, o_out = np.argsort(indeg, kind="stable"), np.argsort(outdeg, kind="stable")
    rows = np.unique(np.concatenate([pick, o_in[:64], o_in[-64:], o_out[:64], o_out[-64:]]))
    return dict(torch=torch, L=L, g=Graph(ip, ix), ip=ip, ix=ix, N=N, rows=rows)


def dev(R, a):
    return R["torch"].from_numpy(np.ascontiguousarray(a)).cuda()


def test_gcn_fwd_bwd_reddit(R):
    """gcn_fwd (layer 1 of the bench: relu, dst norm, bias, src-norm-scaled second output) and gcn_bwd
    (layer 2 backward: relu' from the saved activation, post-scale), F = 16."""
    torch, L, g, N, rows = R["torch"], R["L"], R["g"], R["N"], R["rows"]
    F = 16
    sn, dn = g.degree_norms("both")
    sn_h, dn_h = sn.cpu().numpy(), dn.cpu().numpy()
    T = rnd(101, (N, F))
    b = rnd(102, (F,), -0.1, 0.1)
    Y = torch.empty((N, F), device="cuda")
    Ys = torch.empty((N, F), device="cuda")
    L.seastar_gcn_fwd(g.handle, dev(R, T), F, F, dn, dev(R, b), "relu", 0.0, None, Y, sn, Ys)
    agg = oracle.gcn_aggregate(R["ip"], R["ix"], T, None, dn_h, rows)
    ref = oracle.act_fwd("relu", agg + b.astype(np.float64))
    assert rel_err(Y.cpu().numpy()[rows], ref) <= TOL
    assert rel_err(Ys.cpu().numpy()[rows], ref * sn_h[rows, None].astype(np.float64)) <= TOL
    # backward on the reverse CSR
    dP = rnd(103, (N, F))
    Z = rnd(104, (N, F)).astype(np.float64)
    Yact = oracle.act_fwd("relu", Z).astype(np.float32)
    dA = torch.empty((N, F), device="cuda")
    dPo = torch.empty((N, F), device="cuda")
    L.seastar_gcn_bwd(g.handle, dev(R, dP), F, F, sn, 1.0, dev(R, Yact), "relu", dn, dA, dPo)
    gref = oracle.gcn_aggregate_T(R["ip"], R["ix"], dP, sn_h, None, rows)
    ref = oracle.act_bwd("relu", Z[rows], gref)
    assert rel_err(dA.cpu().numpy()[rows], ref) <= TOL
    assert rel_err(dPo.cpu().numpy()[rows], ref * dn_h[rows, None].astype(np.float64)) <= TOL


@pytest.mark.parametrize("H,F,act", [(8, 8, "elu"), (1, 41, "none")])
def test_gat_layer_reddit(R, H, F, act):
    """gat_fwd (+ der factors) -> gat_bwd_prep (record D, der) -> gat_bwd (dT, del) for one GAT layer of
    the bench, all rows on the GPU; oracle: forward on the sampled rows, explicit-Jacobian backward
    (der for every vertex, dT / del on the sampled source rows)."""
    torch, L, g, N, rows = R["torch"], R["L"], R["g"], R["N"], R["rows"]
    ip, ix = R["ip"], R["ix"]
    W = H * F
    ld = (W + 3) // 4 * 4
    T = rnd(200 + H, (N, W))
    a_l, a_r = rnd(210 + H, (H, F), -0.5, 0.5), rnd(220 + H, (H, F), -0.5, 0.5)
    el, er = oracle.gat_attn_proj(T.reshape(N, H, F), a_l, a_r)
    el32, er32 = el.astype(np.float32), er.astype(np.float32)
    b = rnd(230 + H, (W,), -0.1, 0.1)
    Td = dev(R, padded(T, ld))
    eld, erd = dev(R, el32), dev(R, er32)
    A = torch.empty((N, ld), device="cuda")
    Y = torch.empty((N, ld), device="cuda")
    lse = torch.empty((N, H), device="cuda")
    B = torch.empty((N, ld), device="cuda")
    bs = torch.empty((N, H), device="cuda")
    L.seastar_gat_fwd(g.handle, Td, eld, erd, H, F, ld, 0.2, dev(R, b), act, A, Y, lse, B, bs)
    Ar, lr, _ = oracle.gat_fwd(ip, ix, T.reshape(N, H, F), el32, er32, 0.2)
    Ar = Ar.reshape(N, W)
    assert rel_err(A.cpu().numpy()[rows, :W], Ar[rows]) <= TOL
    assert rel_err(Y.cpu().numpy()[rows, :W], oracle.act_fwd(act, Ar[rows] + b)) <= TOL
    assert rel_err(lse.cpu().numpy()[rows], lr[rows]) <= TOL
    # backward
    dY = rnd(240 + H, (N, W), -1e-3, 1e-3)
    ldd = L.seastar_gat_record_ld(H, F)
    D = torch.empty((N, ldd), device="cuda")
    der = torch.empty((N, H), device="cuda")
    L.seastar_gat_bwd_prep(g.handle, dev(R, padded(dY, ld)), Y, act, A, erd, lse, H, F, ld, D, B, bs, der)
    dT = torch.empty((N, ld), device="cuda")
    dl = torch.empty((N, H), device="cuda")
    L.seastar_gat_bwd(g.handle, Td, eld, D, H, F, ld, 0.2, dT, dl)
    dA = oracle.act_bwd(act, Ar + b, dY)
    dTr, dlr, drr = oracle.gat_bwd(ip, ix, T.reshape(N, H, F), el32, er32, dA.reshape(N, H, F), 0.2, rows)
    assert rel_err(der.cpu().numpy(), drr) <= TOL
    assert rel_err(dl.cpu().numpy()[rows], dlr) <= TOL
    assert rel_err(dT.cpu().numpy()[rows, :W], dTr.reshape(len(rows), W)) <= TOL
