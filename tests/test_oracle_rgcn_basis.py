"""Pins for the NEXT-2 oracle functions (reading #27): the featureless R-GCN input
layer with basis decomposition, W_r = sum_b a[r,b] V_b, h_u = one-hot(u)  =>  h_u W_r = sum_b a[r,b] V[u,b,:].

Pinned by: a dense adjacency-matrix formulation (sum_r A_r W_r with A_r the normalised per-type adjacency -- a
textbook SpMM, independent of the oracle's edge loops); the B = R, a = I special case, which is the featureless
lookup W_r[u] of the already-pinned R-GCN layer; type relabelling invariance; central finite differences."""
import numpy as np

import oracle
from conftest import rel_err
from test_oracle_layers import fd_grad, rnd, small_graph


def per_type_adj(indptr, indices, et, norm, R):
    N = len(indptr) - 1
    dst = np.repeat(np.arange(N), np.diff(indptr))
    A = np.zeros((R, N, N))
    np.add.at(A, (et, dst, indices), norm)
    return A


def test_basis_fwd_dense():
    indptr, indices, et = small_graph(11, N=13, E=70, R=5)
    N, R, B, F = 13, 5, 3, 4
    V, a = rnd(1, N, B, F), rnd(2, R, B)
    norm = oracle.rgcn_norm(indptr, et, R)
    Y = oracle.rgcn_basis_fwd(indptr, indices, et, V, a)
    A = per_type_adj(indptr, indices, et, norm, R)
    W = np.einsum("rb,ubf->ruf", a, V)                  # W_r as an N x F matrix (featureless input)
    ref = sum(A[r] @ W[r] for r in range(R))
    assert rel_err(Y, ref) < 1e-13
    # sampled rows
    rows = np.array([12, 0, 5])
    assert rel_err(oracle.rgcn_basis_fwd(indptr, indices, et, V, a, rows=rows), ref[rows]) < 1e-13
    # user-supplied norm (all ones) -> plain per-type sum
    ones = np.ones(70)
    ref1 = sum(per_type_adj(indptr, indices, et, ones, R)[r] @ W[r] for r in range(R))
    assert rel_err(oracle.rgcn_basis_fwd(indptr, indices, et, V, a, norm=ones), ref1) < 1e-13


def test_basis_identity_is_featureless_rgcn():
    indptr, indices, et = small_graph(12, N=9, E=40, R=4)
    N, R, F = 9, 4, 3
    V = rnd(3, N, R, F)
    Y = oracle.rgcn_basis_fwd(indptr, indices, et, V, np.eye(R))
    Wr = np.transpose(V, (1, 0, 2))                     # W_r[u,:] = V[u,r,:]
    assert rel_err(Y, oracle.rgcn_fwd(indptr, indices, et, np.eye(N), Wr)) < 1e-13


def test_basis_relabel_types():
    indptr, indices, et = small_graph(13, N=10, E=50, R=4)
    N, R, B, F = 10, 4, 2, 4
    V, a = rnd(4, N, B, F), rnd(5, R, B)
    perm = np.array([3, 1, 0, 2])
    ap = np.empty_like(a)
    ap[perm] = a
    Yp = oracle.rgcn_basis_fwd(indptr, indices, perm[et].astype(np.int32), V, ap)
    assert rel_err(Yp, oracle.rgcn_basis_fwd(indptr, indices, et, V, a)) < 1e-14


def test_basis_bwd_fd():
    indptr, indices, et = small_graph(14, N=7, E=25, R=3)
    N, R, B, F = 7, 3, 2, 3
    V, a, Rw = rnd(6, N, B, F), rnd(7, R, B), rnd(8, N, F)
    norm = oracle.rgcn_norm(indptr, et, R)
    f = lambda: (oracle.rgcn_basis_fwd(indptr, indices, et, V, a, norm) * Rw).sum()
    dV, da = oracle.rgcn_basis_bwd(indptr, indices, et, V, a, Rw, norm)
    assert rel_err(dV, fd_grad(f, V)) < 1e-8
    assert rel_err(da, fd_grad(f, a)) < 1e-8
    # the two halves are independent
    assert oracle.rgcn_basis_bwd(indptr, indices, et, V, a, Rw, norm, need_dV=False)[0] is None
    np.testing.assert_array_equal(oracle.rgcn_basis_bwd(indptr, indices, et, V, a, Rw, norm, need_da=False)[0], dV)


def test_basis_combine():
    R, B, Fi, Fo = 4, 4, 3, 2
    Vb = rnd(9, B, Fi, Fo)
    np.testing.assert_array_equal(oracle.basis_combine(np.eye(R), Vb), Vb)     # a = I: W_r = V_r
    a = np.zeros((R, B))
    a[:, 1] = np.arange(1, R + 1)                                                 # rank-1: W_r = (r+1) V_1
    W = oracle.basis_combine(a, Vb)
    for r in range(R):
        assert rel_err(W[r], (r + 1) * Vb[1]) < 1e-15
    a, dW = rnd(10, R, B), rnd(11, R, Fi, Fo)
    da, dVb = oracle.basis_combine_bwd(a, Vb, dW)
    f = lambda: (oracle.basis_combine(a, Vb) * dW).sum()
    assert rel_err(da, fd_grad(f, a)) < 1e-8
    assert rel_err(dVb, fd_grad(f, Vb)) < 1e-8


def test_rgcnb2_model_fd():
    """The NEXT-2 model composition (oracle/model_ref.rgcnb2): every gradient against central differences
    of its loss."""
    from oracle import model_ref
    import synth
    indptr, indices, et = small_graph(15, N=9, E=30, R=3)
    N, R, B1, B2, Hd, C = 9, 3, 2, 2, 3, 2
    lab = synth.labels(1, N, C)
    p = {"V1": rnd(20, N, B1, Hd), "a1": rnd(21, R, B1), "b1": rnd(22, Hd) * 0.1, "V2": rnd(23, B2, Hd, C),
         "a2": rnd(24, R, B2), "b2": rnd(25, C) * 0.1}
    acts = {}
    loss, grads = model_ref.rgcnb2(indptr, indices, et, lab, p, acts)
    assert np.abs(acts["Z1"]).min() > 1e-4          # no ReLU kink within the FD step
    for k in p:
        fd = fd_grad(lambda: model_ref.rgcnb2(indptr, indices, et, lab, p)[0], p[k])
        assert rel_err(grads[k], fd) < 1e-7, k
