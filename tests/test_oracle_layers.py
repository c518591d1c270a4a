"""Pins for the oracle's layer definitions (rows a4-a11, SURVEY.md §8(c) "What pins each part").

Every pin is something other than the oracle itself:
  * dense NumPy brute force on tiny graphs (adjacency-matrix products, dense masked softmax) --
    a textbook SpMM / softmax, independent of the oracle's edge loops;
  * closed forms and special cases (star graph, uniform attention, alpha = 1, K -> inf solve,
    R = 1 mean aggregation, featureless X = I, ln C for uniform logits, Adam's first step);
  * invariants (softmax rows sum to 1, adjoint identity, permutation equivariance);
  * central finite differences in fp64 for every backward.
"""
import numpy as np
import pytest

import oracle
import synth
from conftest import rel_err


def dense_adj(indptr, indices):
    """A[v,u] = number of edges u->v."""
    N = len(indptr) - 1
    A = np.zeros((N, N))
    for v in range(N):
        for e in range(indptr[v], indptr[v + 1]):
            A[v, indices[e]] += 1
    return A


def small_graph(seed=0, N=12, E=60, R=0):
    if R:
        return synth.random_graph(N, E, seed, R)
    return synth.random_graph(N, E, seed)


def rnd(seed, *shape):
    return synth.uniform(seed, shape, -1.0, 1.0).astype(np.float64)


def fd_grad(f, x, h=1e-6):
    """Central differences of scalar f w.r.t. every entry of x (fp64)."""
    g = np.zeros_like(x)
    flat = x.reshape(-1)
    gf = g.reshape(-1)
    for i in range(flat.size):
        old = flat[i]
        flat[i] = old + h
        fp = f()
        flat[i] = old - h
        fm = f()
        flat[i] = old
        gf[i] = (fp - fm) / (2 * h)
    return g


# ------------------------------------------------------------------ linear
def test_linear_matches_matmul_and_fd():
    X, W, b, dY = rnd(1, 9, 7), rnd(2, 7, 5), rnd(3, 5), rnd(4, 9, 5)
    np.testing.assert_allclose(oracle.linear_fwd(X, W, b), X @ W + b, rtol=1e-13, atol=1e-13)
    dX, dW, db = oracle.linear_bwd(X, W, dY)
    np.testing.assert_allclose(dX, dY @ W.T, rtol=1e-13, atol=1e-13)
    np.testing.assert_allclose(dW, X.T @ dY, rtol=1e-13, atol=1e-13)
    np.testing.assert_allclose(db, dY.sum(0), rtol=1e-13, atol=1e-13)


@pytest.mark.parametrize("act", ["none", "relu", "elu", "sigmoid"])
def test_activations(act):
    z = np.array([-2.0, -0.5, 0.0, 0.3, 4.0])
    ref = {"none": z, "relu": np.maximum(z, 0), "elu": np.where(z > 0, z, np.exp(z) - 1),
           "sigmoid": 1 / (1 + np.exp(-z))}[act]
    np.testing.assert_allclose(oracle.act_fwd(act, z), ref, rtol=1e-14, atol=1e-15)
    zz = np.array([-1.3, -0.2, 0.7, 2.1])  # away from the ReLU kink
    g = np.ones_like(zz)
    num = (oracle.act_fwd(act, zz + 1e-6) - oracle.act_fwd(act, zz - 1e-6)) / 2e-6
    np.testing.assert_allclose(oracle.act_bwd(act, zz, g), num, rtol=1e-7, atol=1e-9)


# ------------------------------------------------------------------ GCN (Fig. 1)
@pytest.mark.parametrize("seed", [0, 1, 2])
def test_gcn_aggregate_vs_dense(seed):
    indptr, indices = small_graph(seed)
    N = len(indptr) - 1
    A = dense_adj(indptr, indices)
    H = rnd(10 + seed, N, 5)
    sn, dn = rnd(20 + seed, N), rnd(30 + seed, N)
    ref = np.diag(dn) @ A @ np.diag(sn) @ H
    assert rel_err(oracle.gcn_aggregate(indptr, indices, H, sn, dn), ref) < 1e-13
    # adjoint = transposed dense product
    G = rnd(40 + seed, N, 5)
    refT = np.diag(sn) @ A.T @ np.diag(dn) @ G
    assert rel_err(oracle.gcn_aggregate_T(indptr, indices, G, sn, dn), refT) < 1e-13
    # sampled rows agree with the full evaluation
    rows = np.array([N - 1, 0, 3])
    np.testing.assert_array_equal(oracle.gcn_aggregate(indptr, indices, H, sn, dn, rows),
                                  oracle.gcn_aggregate(indptr, indices, H, sn, dn)[rows])


def test_gcn_star_closed_form():
    # star: leaves 1..n point at centre 0; T == 1 gives Y[0] = sum of src_norm
    n = 9
    indptr, indices = synth.csr_from_edges(n + 1, list(range(1, n + 1)), [0] * n)
    sn = np.arange(1, n + 2, dtype=np.float64)
    Y = oracle.gcn_aggregate(indptr, indices, np.ones((n + 1, 3)), sn, None)
    np.testing.assert_allclose(Y[0], np.full(3, sn[1:].sum()))
    assert (Y[1:] == 0).all()   # empty in-neighbourhood -> 0 (reading #8)


def test_gcn_adjoint_identity():
    indptr, indices = small_graph(5, N=30, E=200)
    N = 30
    H, G = rnd(1, N, 4), rnd(2, N, 4)
    sn, dn = oracle.degree_norms(indptr, indices)[::-1]
    lhs = (G * oracle.gcn_aggregate(indptr, indices, H, sn, dn)).sum()
    rhs = (oracle.gcn_aggregate_T(indptr, indices, G, sn, dn) * H).sum()
    assert abs(lhs - rhs) < 1e-12 * max(1, abs(lhs))


@pytest.mark.parametrize("Fin,Fout,act", [(6, 3, "relu"), (3, 6, "sigmoid"), (4, 4, "none")])
def test_gcn_layer_fd(Fin, Fout, act):
    indptr, indices = small_graph(7, N=8, E=30)
    N = 8
    in_n, out_n = oracle.degree_norms(indptr, indices)
    X, W, b, R = rnd(1, N, Fin), rnd(2, Fin, Fout), rnd(3, Fout), rnd(4, N, Fout)

    def loss():
        return (oracle.gcn_layer_fwd(indptr, indices, X, W, b, act, out_n, in_n)[0] * R).sum()

    Y, Z = oracle.gcn_layer_fwd(indptr, indices, X, W, b, act, out_n, in_n)
    # forward vs dense definition act(b + D_in A D_out X W)
    A = dense_adj(indptr, indices)
    Zd = np.diag(in_n) @ A @ np.diag(out_n) @ X @ W + b
    assert rel_err(Z, Zd) < 1e-13
    dX, dW, db = oracle.gcn_layer_bwd(indptr, indices, X, W, Z, act, out_n, in_n, R)
    assert rel_err(dX, fd_grad(loss, X)) < 1e-7
    assert rel_err(dW, fd_grad(loss, W)) < 1e-7
    assert rel_err(db, fd_grad(loss, b)) < 1e-7


# ------------------------------------------------------------------ APPNP
def appnp_dense(indptr, indices, H0, K, alpha):
    n = 1 / np.sqrt(np.maximum(np.diff(indptr), 1))
    Ahat = np.diag(n) @ dense_adj(indptr, indices) @ np.diag(n)
    Z = H0.copy()
    for _ in range(K):
        Z = (1 - alpha) * Ahat @ Z + alpha * H0
    return Z, Ahat


def test_appnp_special_cases_and_fd():
    indptr, indices = small_graph(3, N=10, E=40)
    H0 = rnd(5, 10, 3)
    np.testing.assert_array_equal(oracle.appnp_fwd(indptr, indices, H0, 0, 0.1), H0)      # K = 0
    np.testing.assert_allclose(oracle.appnp_fwd(indptr, indices, H0, 5, 1.0), H0)         # alpha = 1
    Z, Ahat = appnp_dense(indptr, indices, H0, 3, 0.1)
    assert rel_err(oracle.appnp_fwd(indptr, indices, H0, 3, 0.1), Z) < 1e-13
    # fixed point for K -> inf: alpha (I - (1-alpha) Ahat)^-1 H0 (symmetric graph => |eig| <= 1)
    sym_ip, sym_ix = synth.powerlaw_sym(10, 30, 0.5, 77)
    Zinf = oracle.appnp_fwd(sym_ip, sym_ix, H0, 400, 0.1)
    _, Ah = appnp_dense(sym_ip, sym_ix, H0, 0, 0.1)
    assert rel_err(Zinf, 0.1 * np.linalg.solve(np.eye(10) - 0.9 * Ah, H0)) < 1e-12
    R = rnd(6, 10, 3)
    dH0 = oracle.appnp_bwd(indptr, indices, R, 2, 0.1)
    num = fd_grad(lambda: (oracle.appnp_fwd(indptr, indices, H0, 2, 0.1) * R).sum(), H0)
    assert rel_err(dH0, num) < 1e-7


# ------------------------------------------------------------------ GAT (Fig. 2)
def gat_dense(indptr, indices, T, el, er, slope):
    N, H, F = T.shape
    A = dense_adj(indptr, indices)
    out = np.zeros((N, H, F))
    lse = np.full((N, H), -np.inf)
    for h in range(H):
        s = el[None, :, h] + er[:, None, h]                  # s[v,u]
        z = np.where(s > 0, s, slope * s)
        w = A * np.exp(z)                                    # multiplicity-weighted exp
        den = w.sum(1)
        nz = den > 0
        out[nz, h, :] = (w[nz] / den[nz, None]) @ T[:, h, :]
        lse[nz, h] = np.log(den[nz])
    return out, lse


@pytest.mark.parametrize("H,F", [(1, 4), (2, 3), (8, 8)])
def test_gat_fwd_vs_dense_and_softmax_rows(H, F):
    indptr, indices = small_graph(9, N=14, E=80)
    N = 14
    T, el, er = rnd(1, N, H, F), rnd(2, N, H), rnd(3, N, H)
    A, lse, alpha = oracle.gat_fwd(indptr, indices, T, el, er, 0.2, want_alpha=True)
    Ad, lsed = gat_dense(indptr, indices, T, el, er, 0.2)
    assert rel_err(A, Ad) < 1e-13
    nz = np.isfinite(lsed)
    np.testing.assert_allclose(lse[nz], lsed[nz], rtol=1e-13, atol=1e-13)
    assert np.array_equal(np.isinf(lse), ~nz)
    # sum_e alpha_e = 1 per (v,h) with in-edges
    dst = np.repeat(np.arange(N), np.diff(indptr))
    sums = np.zeros((N, H))
    np.add.at(sums, dst, alpha)
    deg = np.diff(indptr)
    np.testing.assert_allclose(sums[deg > 0], 1.0, rtol=0, atol=1e-14)


def test_gat_special_cases():
    indptr, indices = small_graph(4, N=10, E=50)
    N, H, F = 10, 2, 3
    deg = np.diff(indptr)
    # constant T -> A == c
    A, _, _ = oracle.gat_fwd(indptr, indices, np.full((N, H, F), 2.5), rnd(1, N, H), rnd(2, N, H))
    np.testing.assert_allclose(A[deg > 0], 2.5, rtol=1e-14)
    # a_l = a_r = 0 -> el = er = 0 -> uniform alpha -> mean aggregation = GCN with dst_norm 1/indeg
    T = rnd(3, N, H, F)
    el, er = oracle.gat_attn_proj(T, np.zeros((H, F)), np.zeros((H, F)))
    A, _, _ = oracle.gat_fwd(indptr, indices, T, el, er)
    mean = oracle.gcn_aggregate(indptr, indices, T.reshape(N, H * F), None, 1.0 / np.maximum(deg, 1))
    assert rel_err(A.reshape(N, H * F), mean) < 1e-13
    # two in-edges: alpha_1 = sigmoid(z1 - z2)
    ip, ix = synth.csr_from_edges(3, [1, 2], [0, 0])
    T3 = rnd(4, 3, 1, 2)
    el3, er3 = np.array([[0.0], [0.7], [-1.9]]), np.array([[0.3], [0.0], [0.0]])
    _, _, al = oracle.gat_fwd(ip, ix, T3, el3, er3, 0.2, want_alpha=True)
    lr = lambda x: x if x > 0 else 0.2 * x
    z1, z2 = lr(0.7 + 0.3), lr(-1.9 + 0.3)
    np.testing.assert_allclose(al[0, 0], 1 / (1 + np.exp(-(z1 - z2))), rtol=1e-14)
    # single in-edge: A = T_u ; huge logits stay finite
    ip, ix = synth.csr_from_edges(2, [1], [0])
    A, lse, _ = oracle.gat_fwd(ip, ix, rnd(5, 2, 1, 4), np.array([[0.0], [1e4]]), np.array([[1e4], [0.0]]))
    np.testing.assert_allclose(A[0, 0], rnd(5, 2, 1, 4)[1, 0])
    assert np.isfinite(lse[0]).all() and np.isfinite(A).all()


def test_gat_permutation_equivariance():
    indptr, indices = small_graph(8, N=9, E=40)
    N, H, F = 9, 2, 2
    T, el, er = rnd(1, N, H, F), rnd(2, N, H), rnd(3, N, H)
    A, _, _ = oracle.gat_fwd(indptr, indices, T, el, er)
    pi = np.array([3, 8, 0, 5, 1, 7, 2, 6, 4])       # new id of old vertex i
    dst = np.repeat(np.arange(N), np.diff(indptr))
    ip2, ix2 = synth.csr_from_edges(N, pi[indices], pi[dst])
    inv = np.argsort(pi)
    A2, _, _ = oracle.gat_fwd(ip2, ix2, T[inv], el[inv], er[inv])
    assert rel_err(A2[pi], A) < 1e-13


@pytest.mark.parametrize("H,F", [(1, 3), (2, 2)])
def test_gat_bwd_fd(H, F):
    indptr, indices = small_graph(12, N=7, E=25)
    N = 7
    T, el, er, Rw = rnd(1, N, H, F), rnd(2, N, H), rnd(3, N, H), rnd(4, N, H, F)
    f = lambda: (oracle.gat_fwd(indptr, indices, T, el, er, 0.2)[0] * Rw).sum()
    dT, dl, dr = oracle.gat_bwd(indptr, indices, T, el, er, Rw, 0.2)
    assert rel_err(dT, fd_grad(f, T)) < 1e-7
    assert rel_err(dl, fd_grad(f, el)) < 1e-7
    assert rel_err(dr, fd_grad(f, er)) < 1e-7
    rows = np.array([4, 0])
    dTs, dls, _ = oracle.gat_bwd(indptr, indices, T, el, er, Rw, 0.2, rows=rows)
    np.testing.assert_array_equal(dTs, dT[rows])
    np.testing.assert_array_equal(dls, dl[rows])


def test_gat_attn_proj_and_bwd_fd():
    N, H, F = 5, 2, 3
    T, al, ar = rnd(1, N, H, F), rnd(2, H, F), rnd(3, H, F)
    el, er = oracle.gat_attn_proj(T, al, ar)
    np.testing.assert_allclose(el, np.einsum("nhf,hf->nh", T, al), rtol=1e-14)
    np.testing.assert_allclose(er, np.einsum("nhf,hf->nh", T, ar), rtol=1e-14)
    gl, gr = rnd(4, N, H), rnd(5, N, H)
    f = lambda: (oracle.gat_attn_proj(T, al, ar)[0] * gl).sum() + (oracle.gat_attn_proj(T, al, ar)[1] * gr).sum()
    dT, dal, dar = oracle.gat_attn_proj_bwd(T, al, ar, gl, gr)
    assert rel_err(dT, fd_grad(f, T)) < 1e-8
    assert rel_err(dal, fd_grad(f, al)) < 1e-8
    assert rel_err(dar, fd_grad(f, ar)) < 1e-8


# ------------------------------------------------------------------ R-GCN
def test_rgcn_R1_is_mean_gcn():
    indptr, indices = small_graph(2, N=11, E=50)
    N = 11
    et = np.zeros(50, np.int32)
    X, W = rnd(1, N, 4), rnd(2, 1, 4, 3)
    Y = oracle.rgcn_fwd(indptr, indices, et, X, W)
    deg = np.maximum(np.diff(indptr), 1)
    ref = np.diag(1.0 / deg) @ dense_adj(indptr, indices) @ X @ W[0]
    assert rel_err(Y, ref) < 1e-13


def test_rgcn_norm_equal_weights_featureless_relabel():
    indptr, indices, et = small_graph(3, N=10, E=60, R=4)
    N, R = 10, 4
    norm = oracle.rgcn_norm(indptr, et, R)
    # per-(v,r) norms sum to 1 over each present type
    dst = np.repeat(np.arange(N), np.diff(indptr))
    for v in range(N):
        for r in range(R):
            m = (dst == v) & (et == r)
            if m.any():
                np.testing.assert_allclose(norm[m].sum(), 1.0)
    # all W_r equal -> a GCN with per-edge weights norm_e
    X, W0 = rnd(1, N, 3), rnd(2, 3, 2)
    Y = oracle.rgcn_fwd(indptr, indices, et, X, np.stack([W0] * R))
    Aw = np.zeros((N, N))
    np.add.at(Aw, (dst, indices), norm)
    assert rel_err(Y, Aw @ X @ W0) < 1e-13
    # featureless X = I -> lookup W_r[u]
    W = rnd(3, R, N, 2)
    Yf = oracle.rgcn_fwd(indptr, indices, et, np.eye(N), W)
    ref = np.zeros((N, 2))
    for e in range(60):
        ref[dst[e]] += norm[e] * W[et[e], indices[e]]
    assert rel_err(Yf, ref) < 1e-13
    # relabel types with the matching permutation of W_r -> same output
    perm = np.array([2, 0, 3, 1])
    W4 = rnd(4, R, 3, 2)
    W4p = np.empty_like(W4)
    W4p[perm] = W4
    Yp = oracle.rgcn_fwd(indptr, indices, perm[et].astype(np.int32), X, W4p)
    assert rel_err(Yp, oracle.rgcn_fwd(indptr, indices, et, X, W4)) < 1e-14


def test_rgcn_bwd_fd():
    indptr, indices, et = small_graph(5, N=6, E=20, R=3)
    N = 6
    X, W, Rw = rnd(1, N, 3), rnd(2, 3, 3, 2), rnd(3, N, 2)
    norm = oracle.rgcn_norm(indptr, et, 3)
    f = lambda: (oracle.rgcn_fwd(indptr, indices, et, X, W, norm) * Rw).sum()
    dX, dW = oracle.rgcn_bwd(indptr, indices, et, X, W, Rw, norm)
    assert rel_err(dX, fd_grad(f, X)) < 1e-8
    assert rel_err(dW, fd_grad(f, W)) < 1e-8


# ------------------------------------------------------------------ loss / optimiser
def test_softmax_xent():
    C = 7
    loss, d = oracle.softmax_xent(np.zeros((4, C)), np.array([0, 3, 6, 2]))
    np.testing.assert_allclose(loss, np.log(C), rtol=1e-15)        # uniform logits -> ln C
    np.testing.assert_allclose(d.sum(1), 0.0, atol=1e-16)
    Z, lab = rnd(1, 5, C), np.array([1, 0, 6, 2, 2])
    _, d = oracle.softmax_xent(Z, lab)
    assert rel_err(d, fd_grad(lambda: oracle.softmax_xent(Z, lab, False)[0], Z)) < 1e-8


def test_adam_closed_form():
    g = np.array([0.5, -2.0, 1e-3])
    p, m, v = np.zeros(3), np.zeros(3), np.zeros(3)
    oracle.adam(p, g, m, v, lr=0.01, t=1)
    # first step: m_hat = g, v_hat = g^2 -> update = lr * g / (|g| + eps)
    np.testing.assert_allclose(p, -0.01 * g / (np.abs(g) + 1e-8), rtol=1e-12)
    # second step with the same gradient: m_hat = g, v_hat = g^2 again
    oracle.adam(p, g, m, v, lr=0.01, t=2)
    np.testing.assert_allclose(p, -0.02 * g / (np.abs(g) + 1e-8), rtol=1e-12)


def test_marshalling_independent_of_input_dtype():
    """fp32 / int32 inputs are converted by the wrapper; results must equal the fp64 inputs' (guards
    against passing pointers to temporaries across the C call)."""
    indptr, indices = small_graph(4, N=40, E=300)
    H = rnd(1, 40, 6)
    sn, dn = rnd(2, 40), rnd(3, 40)
    ref = oracle.gcn_aggregate(indptr, indices, H, sn, dn)
    import gc
    for _ in range(3):
        got = oracle.gcn_aggregate(indptr.astype(np.int32), indices.astype(np.int32), H.astype(np.float32),
                                   sn.astype(np.float32), dn.astype(np.float32))
        gc.collect()
        ref32 = np.diag(dn.astype(np.float32).astype(np.float64)) @ dense_adj(indptr, indices) @ \
            np.diag(sn.astype(np.float32).astype(np.float64)) @ H.astype(np.float32).astype(np.float64)
        assert rel_err(got, ref32) < 1e-13
        gotT = oracle.gcn_aggregate_T(indptr, indices, H.astype(np.float32), sn.astype(np.float32),
                                      dn.astype(np.float32))
        assert rel_err(gotT, oracle.gcn_aggregate_T(indptr, indices, H.astype(np.float32).astype(np.float64),
                                                    sn.astype(np.float32).astype(np.float64),
                                                    dn.astype(np.float32).astype(np.float64))) == 0.0
    assert rel_err(ref, ref) == 0.0


def test_aggregate_T_prebuilt_adjacency_identical():
    """oracle.out_adjacency (hoisted out of bench.py's timed sample) changes nothing: bitwise equal output."""
    indptr, indices = small_graph(11, N=30, E=200)
    G = rnd(3, 30, 5)
    sn, dn = oracle.degree_norms(indptr, indices)[::-1]
    rows = np.array([4, 0, 17, 29])
    adj = oracle.out_adjacency(indptr, indices)
    np.testing.assert_array_equal(oracle.gcn_aggregate_T(indptr, indices, G, sn, dn, rows, adj=adj),
                                  oracle.gcn_aggregate_T(indptr, indices, G, sn, dn, rows))
    dst, optr, oeid = adj
    assert optr[-1] == 200 and sorted(oeid.tolist()) == list(range(200))
    np.testing.assert_array_equal(np.repeat(np.arange(30), np.diff(optr)), indices[oeid])   # row u lists out(u)
