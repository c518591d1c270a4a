"""Pins of the kink envelopes (tests/kinks.py) on CPU: flipping one ambiguous ReLU decision by hand in
the oracle composition changes the first-layer gradients by exactly what the envelope bounds."""
import numpy as np

import oracle
import synth
import kinks


def _gcn_grads_with_mask(ip, ix, X, W1, dH1, mask):
    in_n, out_n = oracle.degree_norms(ip, ix)
    dZ1 = dH1 * mask
    dT = oracle.gcn_aggregate_T(ip, ix, dZ1, out_n, in_n)
    _, dW1, _ = oracle.linear_bwd(X, W1, dT, need_dX=False, need_db=False)
    return dW1, dZ1.sum(0)


def test_relu_gcn_envelope_covers_a_flip():
    ip, ix = synth.powerlaw_sym(300, 2000, 0.6, 3)
    N, Fin, H = 300, 20, 8
    X = synth.uniform(1, (N, Fin)).astype(np.float64)
    W1 = synth.glorot(2, Fin, H).astype(np.float64)
    in_n, out_n = oracle.degree_norms(ip, ix)
    Z1 = oracle.gcn_aggregate(ip, ix, oracle.linear_fwd(X, W1), out_n, in_n)
    dH1 = synth.uniform(3, (N, H)).astype(np.float64)
    r, j = np.unravel_index(np.argmin(np.abs(Z1)), Z1.shape)
    band = 1.01 * abs(Z1[r, j]) / np.abs(Z1).max()
    old = kinks.BAND
    kinks.BAND = band
    try:
        env, n = kinks.relu_gcn(ip, ix, X, Z1, dH1, {"W1": (Fin, H), "b1": (H,)})
    finally:
        kinks.BAND = old
    assert n >= 1
    mask = (Z1 > 0).astype(np.float64)
    dW1, db1 = _gcn_grads_with_mask(ip, ix, X, W1, dH1, mask)
    mask[r, j] = 1.0 - mask[r, j]
    dW1f, db1f = _gcn_grads_with_mask(ip, ix, X, W1, dH1, mask)
    assert np.all(np.abs(dW1f - dW1) <= env["W1"] * (1 + 1e-12) + 1e-15)
    assert np.all(np.abs(db1f - db1) <= env["b1"] * (1 + 1e-12) + 1e-15)
    assert np.abs(dW1f - dW1).max() > 0.5 * env["W1"].max()      # tight for a single flip


def test_relu_mlp_envelope_covers_a_flip():
    N, Fin, H = 200, 12, 6
    X = synth.uniform(4, (N, Fin)).astype(np.float64)
    W1 = synth.glorot(5, Fin, H).astype(np.float64)
    Z1 = X @ W1
    dH1 = synth.uniform(6, (N, H)).astype(np.float64)
    r, j = np.unravel_index(np.argmin(np.abs(Z1)), Z1.shape)
    old = kinks.BAND
    kinks.BAND = 1.01 * abs(Z1[r, j]) / np.abs(Z1).max()
    try:
        env, n = kinks.relu_mlp(X, Z1, dH1, {"W1": (Fin, H), "b1": (H,)})
    finally:
        kinks.BAND = old
    mask = (Z1 > 0).astype(np.float64)
    g0 = X.T @ (dH1 * mask)
    mask[r, j] = 1.0 - mask[r, j]
    g1 = X.T @ (dH1 * mask)
    assert n >= 1 and np.all(np.abs(g1 - g0) <= env["W1"] + 1e-15)
    assert np.allclose(np.abs(g1 - g0)[:, j], env["W1"][:, j]) if n == 1 else True
