"""Pins for the oracle's degree normalisation and the R-GCN model composition (VERDICT r1 "What's weak" 1).

`orc_degree_norms` (oracle/seastar_oracle.c) is pinned here by facts of linear algebra and by hand-computed
values, never by restating its formula:

* DESIGN.md reading #1 (Fig. 1 L85-L93 "1/norm", DGL norm='both'): for a SYMMETRIC graph with a
  self-loop on every vertex, the operator Â = D_in^-1/2 A D_out^-1/2 is the symmetric normalised adjacency.
  Its spectral radius is exactly 1 with the Perron eigenvector D^1/2·1 (Â D^1/2 1 = D^-1/2 A 1 = D^1/2 1).
  A wrong exponent (deg^-1 or deg^-1/4), a dropped clamp or an off-by-one degree moves the top eigenvalue
  off 1; numpy's eigensolver supplies the eigenvector independently.
* Directed hand graphs where in- and out-degree differ (stars, a chain), so swapping the two norms or
  counting the wrong endpoint changes the printed values.
* DESIGN.md reading #23 (APPNP, [38]): with H0 equal to that Perron eigenvector, Z = H0 is the fixed point
  of Z <- (1-a) Â Z + a H0 for every K and a.
* The whole `model_ref.rgcn2` composition (R-GCN, [53] / PAPER.md §6.3.5) against central
  differences of its loss.
"""
import numpy as np

import oracle
import synth
from conftest import rel_err
from test_oracle_layers import dense_adj, fd_grad, rnd, small_graph


def _connected_sym_graph(N, chords, seed):
    """Symmetric multigraph: a ring (so it is connected and the Perron eigenvalue is simple), random chords
    in both directions, and one self-loop per vertex."""
    a = (synth.uniform(seed, (chords,), 0.0, 1.0) * N).astype(np.int64).clip(0, N - 1)
    b = (synth.uniform(seed + 1, (chords,), 0.0, 1.0) * N).astype(np.int64).clip(0, N - 1)
    ring = np.arange(N)
    src = np.concatenate([ring, (ring + 1) % N, a, b, ring])
    dst = np.concatenate([(ring + 1) % N, ring, b, a, ring])
    return synth.csr_from_edges(N, src, dst)


def _sym_norm_operator(indptr, indices):
    in_n, out_n = oracle.degree_norms(indptr, indices)
    return np.diag(in_n) @ dense_adj(indptr, indices) @ np.diag(out_n), in_n, out_n


def test_symmetric_selfloop_graph_spectral_radius_one():
    indptr, indices = _connected_sym_graph(60, 200, 5)
    Ahat, in_n, out_n = _sym_norm_operator(indptr, indices)
    assert np.allclose(Ahat, Ahat.T, rtol=0, atol=1e-15)        # in == out degree on a symmetric graph
    w, V = np.linalg.eigh(Ahat)
    assert abs(w[-1] - 1.0) < 1e-12, w[-1]
    assert np.all(np.abs(w) <= 1.0 + 1e-12)
    v = np.abs(V[:, -1])                                      # Perron vector, from the eigensolver
    # it is proportional to sqrt(deg) = 1 / in_norm (and to 1 / out_norm)
    ref = 1.0 / in_n
    assert rel_err(v / np.linalg.norm(v), ref / np.linalg.norm(ref)) < 1e-10
    ref = 1.0 / out_n
    assert rel_err(v / np.linalg.norm(v), ref / np.linalg.norm(ref)) < 1e-10


def test_appnp_fixed_point_of_perron_vector():
    indptr, indices = _connected_sym_graph(40, 130, 9)
    Ahat, _, _ = _sym_norm_operator(indptr, indices)
    w, V = np.linalg.eigh(Ahat)
    H0 = np.stack([V[:, -1], 3.0 * V[:, -1]], axis=1)
    for K, alpha in ((1, 0.1), (10, 0.1), (7, 0.5)):
        Z = oracle.appnp_fwd(indptr, indices, H0, K, alpha)
        assert rel_err(Z, H0) < 1e-12, (K, alpha)


def test_directed_in_star_hand_values():
    # 9 leaves -> centre 0.  indeg(0) = 9, outdeg(0) = 0 (clamped to 1); leaves: indeg 0 (clamped), outdeg 1.
    k = 9
    indptr = np.array([0, k] + [k] * k)
    indices = np.arange(1, k + 1)
    in_n, out_n = oracle.degree_norms(indptr, indices)
    assert in_n[0] == 1.0 / 3.0 and out_n[0] == 1.0
    assert np.all(in_n[1:] == 1.0) and np.all(out_n[1:] == 1.0)
    Y = oracle.gcn_aggregate(indptr, indices, np.ones((k + 1, 1)), out_n, in_n)
    # Y[centre] = (1/sqrt 9) * sum over 9 leaves of (1/sqrt 1) * 1 = 3; leaves receive nothing
    assert Y[0, 0] == 3.0 and np.all(Y[1:] == 0.0)


def test_directed_out_star_hand_values():
    # centre 0 -> 4 leaves.  outdeg(0) = 4, indeg(0) = 0; every leaf has indeg 1, outdeg 0.
    k = 4
    indptr = np.array([0, 0] + list(range(1, k + 1)))
    indices = np.zeros(k, np.int64)
    in_n, out_n = oracle.degree_norms(indptr, indices)
    assert out_n[0] == 0.5 and in_n[0] == 1.0
    Y = oracle.gcn_aggregate(indptr, indices, np.ones((k + 1, 1)), out_n, in_n)
    # each leaf: (1/sqrt 1) * (1/sqrt 4) * 1 = 0.5; a swapped norm would give 1 (src) and 1/2 (dst) -> 1/2 vs
    # the in-star's 1/3 above, so the two stars together catch a swap in either direction
    assert Y[0, 0] == 0.0 and np.all(Y[1:, 0] == 0.5)


def test_directed_chain_with_hub_hand_values():
    # edges (src -> dst): 1->0, 2->0, 3->0, 4->0, 0->1, 1->2
    # indeg: 0:4 1:1 2:1 3:0 4:0   outdeg: 0:1 1:2 2:1 3:1 4:1
    src = np.array([1, 2, 3, 4, 0, 1])
    dst = np.array([0, 0, 0, 0, 1, 2])
    indptr, indices = synth.csr_from_edges(5, src, dst)[:2]
    in_n, out_n = oracle.degree_norms(indptr, indices)
    np.testing.assert_array_equal(in_n, [0.5, 1.0, 1.0, 1.0, 1.0])
    np.testing.assert_array_equal(out_n, [1.0, 1 / np.sqrt(2.0), 1.0, 1.0, 1.0])
    x = np.array([[1.0], [2.0], [3.0], [5.0], [7.0]])
    Y = oracle.gcn_aggregate(indptr, indices, x, out_n, in_n)
    # Y0 = 1/2 (2/sqrt2 + 3 + 5 + 7);  Y1 = 1 * 1;  Y2 = 2/sqrt2
    np.testing.assert_allclose(Y[:, 0], [0.5 * (np.sqrt(2.0) + 15.0), 1.0, np.sqrt(2.0), 0.0, 0.0], rtol=1e-15)


def test_rgcn2_model_fd():
    """model_ref.rgcn2 (dense-feature R-GCN, configs[3]): every gradient against central differences."""
    from oracle import model_ref
    indptr, indices, et = small_graph(17, N=9, E=34, R=3)
    N, R, Fin, Hd, C = 9, 3, 4, 3, 2
    X = rnd(30, N, Fin)
    lab = synth.labels(3, N, C)
    p = {"W1": rnd(31, R, Fin, Hd), "b1": rnd(32, Hd) * 0.1, "W2": rnd(33, R, Hd, C), "b2": rnd(34, C) * 0.1}
    acts = {}
    _, grads = model_ref.rgcn2(indptr, indices, et, X, lab, p, acts)
    assert np.abs(acts["Z1"]).min() > 1e-4                  # no ReLU kink within the FD step
    for k in p:
        fd = fd_grad(lambda: model_ref.rgcn2(indptr, indices, et, X, lab, p)[0], p[k])
        assert rel_err(grads[k], fd) < 1e-7, k
