"""a5 / a8 parity: fused GCN / APPNP aggregation kernels (C ABI) vs the fp64 oracle.

Tolerance (north_star): max|gpu - ref| / max|ref| <= 1e-5 per tensor."""
import numpy as np
import pytest

import oracle
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
    ip, ix = hub_graph()
    return dict(torch=torch, L=L, g=Graph(ip, ix), ip=ip, ix=ix, N=len(ip) - 1)


def dev(env, a):
    return env["torch"].from_numpy(np.ascontiguousarray(a)).cuda()


def act_np(act, z):
    return oracle.act_fwd(act, z)


@pytest.mark.parametrize("F", [1, 3, 4, 5, 7, 8, 16, 41, 64, 70, 128, 200])
@pytest.mark.parametrize("padld", [False, True])
def test_gcn_fwd(env, F, padld):
    torch, L, g, N = env["torch"], env["L"], env["g"], env["N"]
    ld = ((F + 3) // 4) * 4 + (4 if padld else 0) if padld or F % 4 == 0 else F
    T = rnd(10 + F, (N, F))
    dn = rnd(20, (N,), 0.1, 1.0)
    b = rnd(30 + F, (F,))
    Td = dev(env, padded(T, ld))
    Y = torch.full((N, ld), float("nan"), device="cuda")
    Ys = torch.full((N, ld), float("nan"), device="cuda")
    osc = dev(env, rnd(40, (N,), 0.5, 2.0))
    L.seastar_gcn_fwd(g.handle, Td, F, ld, dev(env, dn), dev(env, b), "relu", 0.0, None, Y, osc, Ys)
    agg = oracle.gcn_aggregate(env["ip"], env["ix"], T, None, dn)
    ref = act_np("relu", agg + b.astype(np.float64))
    got = Y.cpu().numpy()[:, :F]
    assert rel_err(got, ref) <= TOL
    assert rel_err(Ys.cpu().numpy()[:, :F], ref * osc.cpu().numpy()[:, None].astype(np.float64)) <= TOL
    if ld > F:   # padding columns of the outputs are never written
        assert np.isnan(Y.cpu().numpy()[:, F:]).all()


@pytest.mark.parametrize("F", [5, 16, 64])
def test_appnp_step_and_activations(env, F):
    torch, L, g, N = env["torch"], env["L"], env["g"], env["N"]
    ld = ((F + 3) // 4) * 4
    T, H0 = rnd(1, (N, F)), rnd(2, (N, F))
    n = rnd(3, (N,), 0.1, 1.0)
    Y = torch.empty((N, ld), device="cuda")
    L.seastar_gcn_fwd(g.handle, dev(env, padded(T, ld)), F, ld, dev(env, n), None, "none", 0.1,
                      dev(env, padded(H0, ld)), Y)
    ref = 0.9 * oracle.gcn_aggregate(env["ip"], env["ix"], T, None, n) + 0.1 * H0
    assert rel_err(Y.cpu().numpy()[:, :F], ref) <= TOL
    for act in ("elu", "sigmoid", "none"):
        L.seastar_gcn_fwd(g.handle, dev(env, padded(T, ld)), F, ld, None, None, act, 0.0, None, Y)
        ref = act_np(act, oracle.gcn_aggregate(env["ip"], env["ix"], T))
        assert rel_err(Y.cpu().numpy()[:, :F], ref) <= TOL, act


@pytest.mark.parametrize("F", [1, 3, 8, 16, 41, 64, 128])
@pytest.mark.parametrize("act", ["none", "relu", "elu"])
def test_gcn_bwd(env, F, act):
    torch, L, g, N = env["torch"], env["L"], env["g"], env["N"]
    ld = ((F + 3) // 4) * 4
    dP = rnd(50 + F, (N, F))
    sn = rnd(51, (N,), 0.1, 1.0)
    ps = rnd(52, (N,), 0.5, 1.5)
    Z = rnd(53, (N, F)).astype(np.float64)
    Yact = oracle.act_fwd(act, Z).astype(np.float32)
    dA = torch.full((N, ld), float("nan"), device="cuda")
    dPo = torch.full((N, ld), float("nan"), device="cuda")
    L.seastar_gcn_bwd(g.handle, dev(env, padded(dP, ld)), F, ld, dev(env, sn), 0.75, dev(env, padded(Yact, ld)),
                      act, dev(env, ps), dA, dPo)
    g_ref = 0.75 * oracle.gcn_aggregate_T(env["ip"], env["ix"], dP, sn, None)
    ref = oracle.act_bwd(act, Z, g_ref) if act != "none" else g_ref
    assert rel_err(dA.cpu().numpy()[:, :F], ref) <= TOL
    assert rel_err(dPo.cpu().numpy()[:, :F], ref * ps.astype(np.float64)[:, None]) <= TOL


def test_adjoint_identity_and_determinism(env):
    torch, L, g, N = env["torch"], env["L"], env["g"], env["N"]
    F = 16
    T, G = rnd(7, (N, F)), rnd(8, (N, F))
    sn, dn = g.degree_norms("both")
    Td, Gd = dev(env, T), dev(env, G)
    Td_s = Td * sn[:, None]          # src-scaled table (what the dense transform's epilogue writes)
    Y = torch.empty((N, F), device="cuda")
    L.seastar_gcn_fwd(g.handle, Td_s, F, F, dn, None, "none", 0.0, None, Y)
    Gs = Gd * dn[:, None]
    dT = torch.empty((N, F), device="cuda")
    L.seastar_gcn_bwd(g.handle, Gs, F, F, sn, 1.0, None, "none", None, dT, None)
    lhs = (Gd.double() * Y.double()).sum().item()
    rhs = (dT.double() * Td.double()).sum().item()
    assert abs(lhs - rhs) <= 1e-5 * max(abs(lhs), 1.0)
    Y2 = torch.empty_like(Y)
    L.seastar_gcn_fwd(g.handle, Td_s, F, F, dn, None, "none", 0.0, None, Y2)
    assert torch.equal(Y, Y2)        # forward is bitwise deterministic (no atomics)


def test_errors_are_loud(env):
    torch, L, g = env["torch"], env["L"], env["g"]
    from paper_conf_eurosys_wumcjlzcy21_b200 import SeastarError
    with pytest.raises(SeastarError, match="INVALID_ARGUMENT"):
        L.seastar_gcn_fwd(g.handle, None, 16, 16, None, None, "none", 0.0, None, None)
    with pytest.raises(SeastarError, match="INVALID_ARGUMENT"):
        Y = torch.empty((env["N"], 8), device="cuda")
        L.seastar_gcn_fwd(g.handle, Y, 16, 8, None, None, "none", 0.0, None, Y)
