"""NEXT-3 parity: seastar_dropout (counter-based inverted dropout) against the oracle's mask -- identical keep
decisions (bit-exact, integer work), values within fp32 rounding -- and the dropout-composed GCN2 / GAT2
training steps (single GPU and row-partitioned) against the oracle compositions."""
import numpy as np
import pytest

import oracle
import synth
from conftest import rel_err
from oracle import model_ref

pytestmark = pytest.mark.gpu
TOL = 1e-5


@pytest.fixture(scope="module")
def env():
    import torch
    assert torch.cuda.is_available()
    from paper_conf_eurosys_wumcjlzcy21_b200 import _lib as L
    from paper_conf_eurosys_wumcjlzcy21_b200 import models, partition
    from paper_conf_eurosys_wumcjlzcy21_b200.graph import Graph
    return dict(torch=torch, L=L, models=models, part=partition, Graph=Graph)


@pytest.mark.parametrize("M,F,ld,p,row0,step", [(1000, 16, 16, 0.5, 0, 0), (777, 602, 604, 0.6, 123, 7),
                                                (5, 3, 4, 0.1, 0, 1), (2048, 41, 44, 0.9, 4096, 123456),
                                                (300, 64, 64, 0.0, 0, 3)])
def test_dropout_kernel(env, M, F, ld, p, row0, step):
    torch, L = env["torch"], env["L"]
    X = synth.uniform(1, (M, F), 0.5, 1.5)                      # nonzero, so Y == 0 <=> dropped
    Xp = np.full((M, ld), np.nan, np.float32)
    Xp[:, :F] = X
    Xd = torch.from_numpy(Xp).cuda()
    Y = torch.full((M, ld), float("nan"), device="cuda")
    st = torch.tensor([step], dtype=torch.int32, device="cuda")
    L.seastar_dropout(Xd, M, F, ld, row0, p, 0xABCDEF12345, 3, st, Y, ld)
    mask = oracle.dropout_mask(0xABCDEF12345, 3, step, M, F, p, row0=row0)
    y = Y.cpu().numpy()
    assert np.array_equal(y[:, :F] != 0, mask > 0)              # identical keep decisions
    assert rel_err(y[:, :F], X * mask) <= 1e-6
    assert np.isnan(y[:, F:]).all()                             # padding never written
    # in place, and the backward is the same call
    L.seastar_dropout(Xd, M, F, ld, row0, p, 0xABCDEF12345, 3, st, Xd, ld)
    assert torch.equal(Xd[:, :F], Y[:, :F])


def test_dropout_fresh_mask_per_step_under_graph_replay(env):
    torch, L = env["torch"], env["L"]
    M, F = 512, 16
    X = torch.ones((M, F), device="cuda")
    Y = torch.empty_like(X)
    st = torch.zeros(1, dtype=torch.int32, device="cuda")
    g = torch.cuda.CUDAGraph()
    s = torch.cuda.Stream()
    s.wait_stream(torch.cuda.current_stream())
    with torch.cuda.graph(g, stream=s):
        L.seastar_dropout(X, M, F, F, 0, 0.5, 42, 1, st, Y, F)
        L.seastar_step_inc(st)
    torch.cuda.current_stream().wait_stream(s)
    for step in range(3):
        g.replay()
        torch.cuda.synchronize()
        assert np.array_equal(Y.cpu().numpy() != 0, oracle.dropout_mask(42, 1, step, M, F, 0.5) > 0)


def _check(m, loss_ref, grads_ref):
    loss = m.forward()
    m.backward()
    assert abs(loss.item() - loss_ref) <= TOL * abs(loss_ref)
    for k, ref in grads_ref.items():
        got = m.P.g(k).cpu().numpy()
        assert rel_err(got, ref.reshape(got.shape)) <= TOL, k


def test_gcn2_dropout(env):
    torch, models, Graph = env["torch"], env["models"], env["Graph"]
    ip, ix = synth.powerlaw_sym(2000, 16000, 0.6, 61)
    N, Fin, H, C = 2000, 120, 16, 7
    X, lab = synth.uniform(1, (N, Fin)), synth.labels(2, N, C)
    p = {"W1": synth.glorot(3, Fin, H), "b1": synth.uniform(4, (H,), -0.1, 0.1),
         "W2": synth.glorot(5, H, C), "b2": synth.uniform(6, (C,), -0.1, 0.1)}
    m = models.GCN2(Graph(ip, ix), torch.from_numpy(X).cuda(), torch.from_numpy(lab).cuda(), p, dropout=0.5, seed=99)
    _check(m, *model_ref.gcn2(ip, ix, X, lab, {k: v.astype(np.float64) for k, v in p.items()},
                              drop={"p": 0.5, "seed": 99, "step": 0}))


def test_gat2_dropout(env):
    torch, models, Graph = env["torch"], env["models"], env["Graph"]
    ip, ix = synth.powerlaw_sym(1500, 12000, 0.6, 62)
    N, Fin, heads, hid, C = 1500, 100, 8, 8, 41
    X, lab = synth.uniform(11, (N, Fin)), synth.labels(12, N, C)
    p = {"W1": synth.glorot(13, Fin, heads * hid), "al1": synth.uniform(14, (heads, hid), -0.5, 0.5),
         "ar1": synth.uniform(15, (heads, hid), -0.5, 0.5), "b1": synth.uniform(16, (heads * hid,), -0.1, 0.1),
         "W2": synth.glorot(17, heads * hid, C), "al2": synth.uniform(18, (1, C), -0.5, 0.5),
         "ar2": synth.uniform(19, (1, C), -0.5, 0.5), "b2": synth.uniform(20, (C,), -0.1, 0.1)}
    Xp = torch.zeros((N, 100), device="cuda")
    Xp.copy_(torch.from_numpy(X))
    m = models.GAT2(Graph(ip, ix), Xp, torch.from_numpy(lab).cuda(), p, heads, hid, dropout=0.6, seed=7)
    _check(m, *model_ref.gat2(ip, ix, X, lab, {k: v.astype(np.float64) for k, v in p.items()}, heads, hid,
                              drop={"p": 0.6, "seed": 7, "step": 0}))


def test_gcn2_dropout_partitioned(env):
    """Masks are keyed by the global element index: P = 2 ranks reproduce the single-GPU step."""
    from test_gpu_partition import run_ranks
    torch, models, part, Graph = env["torch"], env["models"], env["part"], env["Graph"]
    P, N, Fin, H, C = 2, 1801, 60, 16, 5
    ip, ix = synth.powerlaw_sym(N, 14000, 0.5, 63)
    X, lab = synth.uniform(21, (N, Fin)), synth.labels(22, N, C)
    p = {"W1": synth.glorot(23, Fin, H), "b1": synth.uniform(24, (H,), -0.1, 0.1),
         "W2": synth.glorot(25, H, C), "b2": synth.uniform(26, (C,), -0.1, 0.1)}

    def build(r, comm):
        torch.cuda.set_device(0)
        rb, re = part.row_range(N, P, r)
        m = models.GCN2(Graph(ip, ix, row_begin=rb, row_end=re), torch.from_numpy(X[rb:re]).cuda(),
                        torch.from_numpy(lab[rb:re]).cuda(), p, comm=comm, n_pad_rows=part.gathered_rows(N, P),
                        dropout=0.5, seed=5)
        l = m.forward().item()
        m.backward()
        torch.cuda.synchronize()
        return l, {k: m.P.g(k).cpu().numpy().copy() for k in p}

    res = run_ranks(P, build)
    rl, rg = model_ref.gcn2(ip, ix, X, lab, {k: v.astype(np.float64) for k, v in p.items()},
                            drop={"p": 0.5, "seed": 5, "step": 0})
    assert abs(sum(r[0] for r in res) - rl) <= TOL * abs(rl)
    for k in rg:
        assert rel_err(res[0][1][k], rg[k].reshape(res[0][1][k].shape)) <= TOL, k


@pytest.mark.parametrize("H,F", [(8, 8), (1, 41), (4, 16)])
def test_gat_fwd_attn_dropout(env, H, F):
    """NEXT-3 attention dropout in the fused forward: A = sum_e a_e m_e T_u with m_e keyed by (user edge id, head);
    the softmax statistics (lse) are not masked."""
    torch, L, Graph = env["torch"], env["L"], env["Graph"]
    from helpers import hub_graph
    ip, ix = hub_graph(N=2500, E_dir=20000, seed=64)
    N, E = len(ip) - 1, len(ix)
    g = Graph(ip, ix)
    T = synth.uniform(1, (N, H, F))
    el, er = synth.uniform(2, (N, H)), synth.uniform(3, (N, H))
    ld = (H * F + 3) // 4 * 4
    Tp = np.zeros((N, ld), np.float32)
    Tp[:, :H * F] = T.reshape(N, H * F)
    st = torch.tensor([4], dtype=torch.int32, device="cuda")
    spec = L.dropout_spec(0.5, 3, 77, st)
    d = lambda a: torch.from_numpy(np.ascontiguousarray(a, np.float32)).cuda()
    A = torch.zeros((N, ld), device="cuda")
    Y = torch.zeros((N, ld), device="cuda")
    lse = torch.zeros((N, H), device="cuda")
    L.seastar_gat_fwd(g.handle, d(Tp), d(el), d(er), H, F, ld, 0.2, None, "none", A, Y, lse, attn_drop=spec)
    mask = oracle.dropout_mask(77, 3, 4, E, H, 0.5)
    rA, rl, _ = oracle.gat_fwd(ip, ix, T, el, er, 0.2, mask=mask)
    assert rel_err(A.cpu().numpy()[:, :H * F], rA.reshape(N, H * F)) <= TOL
    lg = lse.cpu().numpy()
    fin = np.isfinite(rl)
    assert np.array_equal(np.isfinite(lg), fin) and rel_err(lg[fin], rl[fin]) <= TOL


@pytest.mark.parametrize("save_B", [True, False])
def test_gat2_attn_dropout(env, save_B):
    """DGL's GAT defaults: feat_drop 0.6 on both layer inputs and attn_drop 0.6 on both layers' attention."""
    torch, models, Graph = env["torch"], env["models"], env["Graph"]
    ip, ix = synth.powerlaw_sym(1500, 12000, 0.6, 65)
    N, Fin, heads, hid, C = 1500, 100, 8, 8, 41
    X, lab = synth.uniform(11, (N, Fin)), synth.labels(12, N, C)
    p = {"W1": synth.glorot(13, Fin, heads * hid), "al1": synth.uniform(14, (heads, hid), -0.5, 0.5),
         "ar1": synth.uniform(15, (heads, hid), -0.5, 0.5), "b1": synth.uniform(16, (heads * hid,), -0.1, 0.1),
         "W2": synth.glorot(17, heads * hid, C), "al2": synth.uniform(18, (1, C), -0.5, 0.5),
         "ar2": synth.uniform(19, (1, C), -0.5, 0.5), "b2": synth.uniform(20, (C,), -0.1, 0.1)}
    m = models.GAT2(Graph(ip, ix), torch.from_numpy(X).cuda(), torch.from_numpy(lab).cuda(), p, heads, hid,
                    dropout=0.6, attn_dropout=0.6, seed=8, save_der_factors=save_B)
    _check(m, *model_ref.gat2(ip, ix, X, lab, {k: v.astype(np.float64) for k, v in p.items()}, heads, hid,
                              drop={"p": 0.6, "attn_p": 0.6, "seed": 8, "step": 0}))


def test_appnp_edge_dropout(env):
    """DGL APPNPConv's edge_drop: a fresh edge mask per propagation step, fused into the aggregation kernels."""
    torch, models, Graph = env["torch"], env["models"], env["Graph"]
    ip, ix = synth.powerlaw_sym(1800, 15000, 0.5, 66)
    N, Fin, Hd, C, K = 1800, 150, 64, 5, 10
    X, lab = synth.uniform(21, (N, Fin)), synth.labels(22, N, C)
    p = {"W1": synth.glorot(23, Fin, Hd), "b1": synth.uniform(24, (Hd,), -0.1, 0.1),
         "W2": synth.glorot(25, Hd, C), "b2": synth.uniform(26, (C,), -0.1, 0.1)}
    m = models.APPNPNet(Graph(ip, ix), torch.from_numpy(X).cuda(), torch.from_numpy(lab).cuda(), p, K=K, alpha=0.1,
                        edge_dropout=0.5, seed=12)
    _check(m, *model_ref.appnp(ip, ix, X, lab, {k: v.astype(np.float64) for k, v in p.items()}, K, 0.1,
                               drop={"edge_p": 0.5, "seed": 12, "step": 0}))


@pytest.mark.parametrize("F", [16, 5, 64])
def test_gcn_edge_dropout_kernels(env, F):
    """seastar_gcn_fwd / _bwd with edge dropout vs the weighted oracle aggregation (both degree buckets)."""
    torch, L, Graph = env["torch"], env["L"], env["Graph"]
    from helpers import hub_graph
    ip, ix = hub_graph(N=2500, E_dir=20000, seed=67)
    N, E = len(ip) - 1, len(ix)
    g = Graph(ip, ix)
    ld = (F + 3) // 4 * 4
    T = synth.uniform(1, (N, F))
    Tp = np.zeros((N, ld), np.float32)
    Tp[:, :F] = T
    st = torch.tensor([2], dtype=torch.int32, device="cuda")
    spec = L.dropout_spec(0.3, 16, 5, st)
    w = oracle.dropout_mask(5, 16, 2, E, 1, 0.3)[:, 0]
    Y = torch.zeros((N, ld), device="cuda")
    L.seastar_gcn_fwd(g.handle, torch.from_numpy(Tp).cuda(), F, ld, None, None, "none", 0.0, None, Y, edge_drop=spec)
    assert rel_err(Y.cpu().numpy()[:, :F], oracle.gcn_aggregate(ip, ix, T, edge_w=w)) <= TOL
    dA = torch.zeros((N, ld), device="cuda")
    L.seastar_gcn_bwd(g.handle, torch.from_numpy(Tp).cuda(), F, ld, None, 1.0, None, "none", None, dA, None,
                      edge_drop=spec)
    assert rel_err(dA.cpu().numpy()[:, :F], oracle.gcn_aggregate_T(ip, ix, T, edge_w=w)) <= TOL
