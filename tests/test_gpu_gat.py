"""a6 / a9 parity: fused GAT forward (online softmax) and source-major backward vs the fp64 oracle
(explicit softmax Jacobian, no c_v trick)."""
import numpy as np
import pytest

import oracle
import synth
from conftest import rel_err
from helpers import hub_graph, padded, rnd

pytestmark = pytest.mark.gpu
TOL = 1e-5


@pytest.fixture(scope="module")
def env():
    import torch
    assert torch.cuda.is_available()
    from paper_conf_eurosys_wumcjlzcy21_b200 import _lib as L
    from paper_conf_eurosys_wumcjlzcy21_b200.graph import Graph
    ip, ix = hub_graph(N=2500, E_dir=25000, hub_deg=1200, isolated=5)
    return dict(torch=torch, L=L, g=Graph(ip, ix), ip=ip, ix=ix, N=len(ip) - 1, Graph=Graph)


def dev(env, a):
    return env["torch"].from_numpy(np.ascontiguousarray(a)).cuda()


def run_fwd(env, g, N, H, F, ld, T, el, er, b, act, slope=0.2, save_B=False):
    torch, L = env["torch"], env["L"]
    A = torch.full((N, ld), float("nan"), device="cuda")
    Y = torch.full((N, ld), float("nan"), device="cuda")
    lse = torch.empty((N, H), device="cuda")
    B = torch.full((N, ld), float("nan"), device="cuda") if save_B else None
    bs = torch.empty((N, H), device="cuda") if save_B else None
    L.seastar_gat_fwd(g.handle, dev(env, padded(T, ld)), dev(env, el), dev(env, er), H, F, ld, slope,
                      None if b is None else dev(env, b), act, A, Y, lse, B, bs)
    if save_B:
        return A, Y, lse, B, bs
    return A, Y, lse


# covers: head-per-lane (H | 32, F % 4 == 0), single-head multi-chunk (H = 1, VPL 1..8), generic chunked
CASES = [(1, 3), (1, 4), (1, 16), (1, 33), (1, 41), (1, 70), (1, 128), (2, 3), (2, 4), (8, 8), (4, 16), (8, 4),
         (3, 5), (2, 32), (16, 4),
         (8, 32), (16, 16), (32, 8)]   # rows of 256 floats: head-per-lane kernels (the chunked ones stop at 128)


@pytest.mark.parametrize("H,F", CASES)
def test_gat_fwd(env, H, F):
    N, W = env["N"], H * F
    ld = ((W + 3) // 4) * 4
    T, el, er, b = rnd(1, (N, W)), rnd(2, (N, H), -2, 2), rnd(3, (N, H), -2, 2), rnd(4, (W,))
    A, Y, lse = run_fwd(env, env["g"], N, H, F, ld, T, el, er, b, "elu")
    Ar, lr, _ = oracle.gat_fwd(env["ip"], env["ix"], T.reshape(N, H, F), el, er, 0.2)
    Ar = Ar.reshape(N, W)
    assert rel_err(A.cpu().numpy()[:, :W], Ar) <= TOL
    assert rel_err(Y.cpu().numpy()[:, :W], oracle.act_fwd("elu", Ar + b)) <= TOL
    l = lse.cpu().numpy()
    fin = np.isfinite(lr)
    assert np.array_equal(np.isfinite(l), fin)           # -inf exactly for empty rows
    assert rel_err(l[fin], lr[fin]) <= TOL


def test_gat_special_cases(env):
    torch, L, N = env["torch"], env["L"], env["N"]
    H, F = 2, 4
    deg = np.diff(env["ip"])
    # constant T -> A == c on non-empty rows, 0 on empty rows
    A, _, _ = run_fwd(env, env["g"], N, H, F, 8, np.full((N, 8), 2.5, np.float32), rnd(1, (N, H)), rnd(2, (N, H)),
                      None, "none")
    a = A.cpu().numpy()
    assert np.abs(a[deg > 0] - 2.5).max() <= 2.5 * TOL and (a[deg == 0] == 0).all()
    # el = er = 0 -> uniform attention = mean aggregation
    T = rnd(5, (N, 8))
    A, _, _ = run_fwd(env, env["g"], N, H, F, 8, T, np.zeros((N, H), np.float32), np.zeros((N, H), np.float32),
                      None, "none")
    mean = oracle.gcn_aggregate(env["ip"], env["ix"], T, None, 1.0 / np.maximum(deg, 1))
    assert rel_err(A.cpu().numpy(), mean) <= TOL
    # huge logits stay finite (max-subtracted online softmax)
    A, _, lse = run_fwd(env, env["g"], N, H, F, 8, T, np.full((N, H), 1e4, np.float32),
                        np.full((N, H), 1e4, np.float32), None, "none")
    assert np.isfinite(A.cpu().numpy()).all()


@pytest.mark.parametrize("H,F", CASES)
def test_gat_bwd_chain(env, H, F):
    """dY -> prep (dA, c) -> src-major bwd (dT, del, ds) -> der segment sum -> attn-proj bwd."""
    torch, L, g, N = env["torch"], env["L"], env["g"], env["N"]
    W = H * F
    ld = ((W + 3) // 4) * 4
    T = rnd(11, (N, W))
    a_l, a_r = rnd(12, (H, F)), rnd(13, (H, F))
    el, er = oracle.gat_attn_proj(T.reshape(N, H, F), a_l, a_r)
    el32, er32 = el.astype(np.float32), er.astype(np.float32)
    b = rnd(14, (W,))
    act = "elu"
    A, Y, lse = run_fwd(env, g, N, H, F, ld, T, el32, er32, b, act)
    dY = rnd(15, (N, W))
    ldd = L.seastar_gat_record_ld(H, F)
    D = torch.empty((N, ldd), device="cuda")
    # forward-saved der factors (B, b) -> the row pass emits der; must agree with the dst-major pass
    A_b, Y_b, lse_b, Bf, bsf = run_fwd(env, g, N, H, F, ld, T, el32, er32, b, act, save_B=True)
    assert torch.equal(A_b[:, :W], A[:, :W]) and torch.equal(lse_b, lse)   # saving B does not perturb the forward
    dr_b = torch.empty((N, H), device="cuda")
    L.seastar_gat_bwd_prep(g.handle, dev(env, padded(dY, ld)), Y, act, A, dev(env, er32), lse, H, F, ld, D, Bf, bsf,
                           dr_b)
    dT = torch.full((N, ld), float("nan"), device="cuda")
    dl = torch.empty((N, H), device="cuda")
    Td = dev(env, padded(T, ld))
    L.seastar_gat_bwd(g.handle, Td, dev(env, el32), D, H, F, ld, 0.2, dT, dl)
    dr = torch.empty((N, H), device="cuda")
    L.seastar_gat_der(g.handle, Td, dev(env, el32), D, H, F, ld, 0.2, dr)
    # oracle: plain Jacobian on the same fp32 inputs
    Ar, _, _ = oracle.gat_fwd(env["ip"], env["ix"], T.reshape(N, H, F), el32, er32, 0.2)
    dA = oracle.act_bwd(act, Ar.reshape(N, W) + b, dY)
    dTr, dlr, drr = oracle.gat_bwd(env["ip"], env["ix"], T.reshape(N, H, F), el32, er32, dA.reshape(N, H, F), 0.2)
    assert rel_err(dT.cpu().numpy()[:, :W], dTr.reshape(N, W)) <= TOL
    assert rel_err(dl.cpu().numpy(), dlr) <= TOL
    assert rel_err(dr.cpu().numpy(), drr) <= TOL
    assert rel_err(dr_b.cpu().numpy(), drr) <= TOL
    # projection backward: dT += del a_l + der a_r ; da_l, da_r
    ws_b = L.seastar_gat_attn_proj_bwd_workspace(N, H, F)
    ws = torch.empty(ws_b, dtype=torch.uint8, device="cuda")
    dal = torch.empty((H, F), device="cuda")
    dar = torch.empty((H, F), device="cuda")
    L.seastar_gat_attn_proj_bwd(Td, N, H, F, ld, dev(env, a_l), dev(env, a_r), dl, dr, dT, dal, dar, ws, ws_b)
    dTp, dalr, darr = oracle.gat_attn_proj_bwd(T.reshape(N, H, F), a_l, a_r, dlr, drr)
    assert rel_err(dT.cpu().numpy()[:, :W], (dTr + dTp).reshape(N, W)) <= TOL
    assert rel_err(dal.cpu().numpy(), dalr) <= TOL
    assert rel_err(dar.cpu().numpy(), darr) <= TOL


def test_gat_attn_proj(env):
    torch, L = env["torch"], env["L"]
    N, H, F = 1000, 8, 8
    T, a_l, a_r = rnd(1, (N, H * F)), rnd(2, (H, F)), rnd(3, (H, F))
    el = torch.empty((N, H), device="cuda")
    er = torch.empty((N, H), device="cuda")
    L.seastar_gat_attn_proj(dev(env, T), N, H, F, H * F, dev(env, a_l), dev(env, a_r), el, er)
    elr, err = oracle.gat_attn_proj(T.reshape(N, H, F), a_l, a_r)
    assert rel_err(el.cpu().numpy(), elr) <= TOL and rel_err(er.cpu().numpy(), err) <= TOL


def test_gat_fwd_deterministic(env):
    N, H, F = env["N"], 8, 8
    T, el, er = rnd(1, (N, 64)), rnd(2, (N, H)), rnd(3, (N, H))
    A1, _, l1 = run_fwd(env, env["g"], N, H, F, 64, T, el, er, None, "none")
    A2, _, l2 = run_fwd(env, env["g"], N, H, F, 64, T, el, er, None, "none")
    assert env["torch"].equal(A1, A2) and env["torch"].equal(l1, l2)
