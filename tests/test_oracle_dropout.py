"""Pins for the NEXT-3 dropout mask (reading #27; "Dropout layer", DGL defaults).

The generator is Vigna's splitmix64 output function, pinned by its published reference outputs for state 0
(0xe220a8397b1dcdaf, 0x6e789e6aa1b965f4, 0x06c45d188009454f -- successive states are multiples of the golden
gamma); the mask by its defining statistics (keep rate 1 - p within 6 sigma, inverted scaling 1/(1-p) so the
expectation is preserved, no correlation between sites / steps / neighbouring indices), its boundary cases
(p = 0 keeps everything), and by being a pure function of the element's global index (row offsets reproduce
slices of the full mask: the partitioned case)."""
import numpy as np

import oracle

G = 0x9E3779B97F4A7C15


def test_splitmix64_reference_outputs():
    assert oracle.sm64(0) == 0xE220A8397B1DCDAF
    assert oracle.sm64(G) == 0x6E789E6AA1B965F4
    assert oracle.sm64((2 * G) & 0xFFFFFFFFFFFFFFFF) == 0x06C45D188009454F


def test_keep_rate_and_scale():
    M, F = 3000, 40
    for p in (0.1, 0.5, 0.6, 0.9):
        m = oracle.dropout_mask(7, 1, 3, M, F, p)
        p32 = float(np.float32(p))
        vals = np.unique(m)
        assert set(vals.tolist()) <= {0.0, 1.0 / (1.0 - p32)}
        kept = (m > 0).mean()
        sigma = np.sqrt(p * (1 - p) / m.size)
        assert abs(kept - (1 - p)) < 6 * sigma, (p, kept)
        assert abs(m.mean() - 1.0) < 6 * sigma / (1 - p)          # inverted dropout keeps the expectation


def test_p0_keeps_everything_and_determinism():
    assert np.all(oracle.dropout_mask(1, 2, 3, 50, 7, 0.0) == 1.0)
    a = oracle.dropout_mask(11, 2, 5, 200, 16, 0.5)
    np.testing.assert_array_equal(a, oracle.dropout_mask(11, 2, 5, 200, 16, 0.5))


def test_independent_streams():
    M, F, p = 2000, 32, 0.5
    base = oracle.dropout_mask(3, 1, 0, M, F, p) > 0
    for other in (oracle.dropout_mask(3, 2, 0, M, F, p), oracle.dropout_mask(3, 1, 1, M, F, p),
                  oracle.dropout_mask(4, 1, 0, M, F, p)):
        agree = (base == (other > 0)).mean()
        assert abs(agree - 0.5) < 6 * np.sqrt(0.25 / base.size), agree
    flat = base.ravel().astype(np.float64)
    c = np.corrcoef(flat[:-1], flat[1:])[0, 1]                  # neighbouring indices uncorrelated
    assert abs(c) < 6 / np.sqrt(flat.size)


def test_global_index_slices():
    full = oracle.dropout_mask(9, 1, 2, 100, 12, 0.3)
    np.testing.assert_array_equal(oracle.dropout_mask(9, 1, 2, 40, 12, 0.3, row0=37), full[37:77])


def test_gcn2_and_gat2_with_dropout_fd():
    """The dropout-composed model references (oracle/model_ref.py): every gradient vs central differences
    with the masks held fixed (they are a function of (seed, site, step), not of the parameters)."""
    import synth
    from oracle import model_ref
    from conftest import rel_err
    from test_oracle_layers import fd_grad, small_graph
    ip, ix = small_graph(21, N=10, E=40)
    N, Fin, H, C = 10, 5, 6, 3
    X = synth.uniform(1, (N, Fin)).astype(np.float64)
    lab = synth.labels(2, N, C)
    drop = {"p": 0.5, "seed": 5, "step": 2}
    pg = {"W1": synth.uniform(3, (Fin, H)).astype(np.float64), "b1": synth.uniform(4, (H,)).astype(np.float64) * .1,
          "W2": synth.uniform(5, (H, C)).astype(np.float64), "b2": synth.uniform(6, (C,)).astype(np.float64) * .1}
    acts = {}
    _, g = model_ref.gcn2(ip, ix, X, lab, pg, acts, drop)
    assert np.abs(acts["Z1"]).min() > 1e-4
    for k in pg:
        assert rel_err(g[k], fd_grad(lambda: model_ref.gcn2(ip, ix, X, lab, pg, None, drop)[0], pg[k])) < 1e-7, k
    heads, hid = 2, 3
    pa = {"W1": synth.uniform(13, (Fin, heads * hid)).astype(np.float64),
          "al1": synth.uniform(14, (heads, hid)).astype(np.float64), "ar1": synth.uniform(15, (heads, hid)).astype(np.float64),
          "b1": synth.uniform(16, (heads * hid,)).astype(np.float64) * .1,
          "W2": synth.uniform(17, (heads * hid, C)).astype(np.float64),
          "al2": synth.uniform(18, (1, C)).astype(np.float64), "ar2": synth.uniform(19, (1, C)).astype(np.float64),
          "b2": synth.uniform(20, (C,)).astype(np.float64) * .1}
    for d in (drop, dict(drop, attn_p=0.4), dict(drop, p=0.0, attn_p=0.6)):
        _, g = model_ref.gat2(ip, ix, X, lab, pa, heads, hid, None, d)
        for k in pa:
            fd = fd_grad(lambda: model_ref.gat2(ip, ix, X, lab, pa, heads, hid, None, d)[0], pa[k])
            assert rel_err(g[k], fd) < 1e-6, (d, k)


def test_gat_attention_mask_layer():
    """gat_fwd / gat_bwd with an attention mask: all-ones is the unmasked layer, all-zeros gives A = 0 and no T
    gradient, and the masked layer's gradients match central differences."""
    import synth
    from conftest import rel_err
    from test_oracle_layers import fd_grad, small_graph
    ip, ix = small_graph(22, N=9, E=36)
    N, H, F, E = 9, 2, 3, 36
    T = synth.uniform(1, (N, H, F)).astype(np.float64)
    el, er = synth.uniform(2, (N, H)).astype(np.float64), synth.uniform(3, (N, H)).astype(np.float64)
    A0, l0, _ = oracle.gat_fwd(ip, ix, T, el, er)
    A1, l1, _ = oracle.gat_fwd(ip, ix, T, el, er, mask=np.ones((E, H)))
    np.testing.assert_array_equal(A0, A1)
    np.testing.assert_array_equal(l0, l1)
    Az, lz, _ = oracle.gat_fwd(ip, ix, T, el, er, mask=np.zeros((E, H)))
    assert np.all(Az == 0) and np.array_equal(lz, l0)           # the softmax itself is not masked
    mask = oracle.dropout_mask(9, 3, 0, E, H, 0.5)
    R = synth.uniform(4, (N, H, F)).astype(np.float64)
    f = lambda: (oracle.gat_fwd(ip, ix, T, el, er, mask=mask)[0] * R).sum()
    dT, dl, dr = oracle.gat_bwd(ip, ix, T, el, er, R, mask=mask)
    assert rel_err(dT, fd_grad(f, T)) < 1e-8
    # del / der are the gradients w.r.t. el (source side) and er (destination side)
    assert rel_err(dl, fd_grad(f, el)) < 1e-8
    assert rel_err(dr, fd_grad(f, er)) < 1e-8


def test_appnp_edge_dropout_fd():
    """APPNP with a fresh edge-dropout mask per propagation step: the model's gradients vs central differences,
    and all-ones masks reduce to the plain propagation."""
    import synth
    from oracle import model_ref
    from conftest import rel_err
    from test_oracle_layers import fd_grad, small_graph
    ip, ix = small_graph(23, N=10, E=44)
    N, Fin, Hd, C, K = 10, 4, 5, 3, 3
    X = synth.uniform(1, (N, Fin)).astype(np.float64)
    lab = synth.labels(2, N, C)
    p = {"W1": synth.uniform(3, (Fin, Hd)).astype(np.float64), "b1": synth.uniform(4, (Hd,)).astype(np.float64) * .1,
         "W2": synth.uniform(5, (Hd, C)).astype(np.float64), "b2": synth.uniform(6, (C,)).astype(np.float64) * .1}
    H0 = synth.uniform(7, (N, C)).astype(np.float64)
    np.testing.assert_array_equal(oracle.appnp_fwd(ip, ix, H0, K, 0.1),
                                  oracle.appnp_fwd(ip, ix, H0, K, 0.1, edge_masks=[np.ones(44)] * K))
    drop = {"edge_p": 0.5, "seed": 3, "step": 1}
    acts = {}
    _, g = model_ref.appnp(ip, ix, X, lab, p, K, 0.1, acts, drop)
    assert np.abs(acts["Z1"]).min() > 1e-4
    for k in p:
        fd = fd_grad(lambda: model_ref.appnp(ip, ix, X, lab, p, K, 0.1, None, drop)[0], p[k])
        assert rel_err(g[k], fd) < 1e-7, k
