"""Kink-aware gradient envelopes for the whole-model parity tests (test infrastructure, numpy).

The models' gradients are discontinuous where an activation's derivative jumps: ReLU'(z) at z = 0 and
LeakyReLU'(s) at s = 0 (Fig. 2, the GAT edge score; reading #6).  A GPU forward that
agrees with the oracle to 1e-6 can take the other branch for a pre-activation whose oracle value lies
within that distance of 0 -- both decisions are correct answers for the inputs (the several-correct-
results case of DESIGN.md §3).  The tests therefore compare each gradient within

    tol * max|ref|  +  envelope

where the envelope is a rigorous bound on what flipping any subset of the AMBIGUOUS decisions (oracle
pre-activation within band * its max-abs of the kink) can change, computed from oracle quantities only:

* ReLU hidden layer Z1 (GCN2 / APPNP / R-GCN): flipping (r, j) changes dZ1[r, j] by dH1[r, j]; that adds
  dH1[r, j] to db1[j] and dH1[r, j] * (d Z1[r, j] / d W1[:, j]) to dW1[:, j] -- (A_hat X)[r, :] for GCN
  (transform first), X[r, :] for APPNP's MLP, sum_{e in in(r), type t} norm_e X[src_e] for R-GCN's W1[t].
* LeakyReLU edge score s_e,h of a GAT layer: flipping it changes ds_e,h by
  (1 - slope) a_e,h |g_e,h - c_v,h| (a = attention, g = <dA_v, T_u>, c = <dA_v, A_v>), which reaches
  da_l[h] through T_u, da_r[h] through T_v and dW[:, head h] through Xin_u (x) a_l[h] and Xin_v (x) a_r[h].
  (The flipped layer's terms; the effect on the layers below is not bounded here and must stay within
  tol on its own.)

Every function returns {param name: envelope array} (zeros where nothing is ambiguous) and the count
of ambiguous decisions.
"""
import numpy as np

import oracle

BAND = 1e-5          # the forward tolerance: a GPU pre-activation may sit this far (x max-abs) from the oracle's


def _ambiguous(Z, empty_rows=None):
    """(rows, cols) of pre-activations within BAND * max|Z| of the kink.  Rows of vertices without
    in-edges are structural: both sides compute exactly the bias there, so their decisions agree."""
    amb = np.abs(Z) <= BAND * np.abs(Z).max()
    if empty_rows is not None:
        amb[empty_rows] = False
    return np.nonzero(amb)


def relu_gcn(ip, ix, X, Z1, dH1, shapes):
    r, j = _ambiguous(Z1, np.diff(ip) == 0)
    env = {k: np.zeros(s) for k, s in shapes.items()}
    if r.size:
        in_n, out_n = oracle.degree_norms(ip, ix)
        rows, inv = np.unique(r, return_inverse=True)
        AX = np.abs(oracle.gcn_aggregate(ip, ix, X, out_n, in_n, rows))        # (A_hat X)[r, :]
        w = np.abs(dH1[r, j])
        np.add.at(env["b1"], j, w)
        for k in range(r.size):
            env["W1"][:, j[k]] += w[k] * AX[inv[k]]
    return env, int(r.size)


def relu_mlp(X, Z1, dH1, shapes):
    r, j = _ambiguous(Z1)
    env = {k: np.zeros(s) for k, s in shapes.items()}
    if r.size:
        w = np.abs(dH1[r, j])
        np.add.at(env["b1"], j, w)
        for k in range(r.size):
            env["W1"][:, j[k]] += w[k] * np.abs(X[r[k]].astype(np.float64))
    return env, int(r.size)


def relu_rgcn(ip, ix, et, R, X, Z1, dH1, shapes):
    r, j = _ambiguous(Z1, np.diff(ip) == 0)
    env = {k: np.zeros(s) for k, s in shapes.items()}
    if r.size:
        norm = oracle.rgcn_norm(ip, et, R)
        w = np.abs(dH1[r, j])
        np.add.at(env["b1"], j, w)
        for k in range(r.size):
            for e in range(ip[r[k]], ip[r[k] + 1]):
                env["W1"][et[e], :, j[k]] += w[k] * norm[e] * np.abs(X[ix[e]].astype(np.float64))
    return env, int(r.size)


def relu_rgcnb(ip, ix, et, R, V1, a1, Z1, dH1, shapes):
    """NEXT-2 featureless basis layer: flipping (r, j) adds dH1[r, j] * norm_e * a1[t_e, b] to dV1[src_e, b, j]
    and dH1[r, j] * norm_e * V1[src_e, b, j] to da1[t_e, b] for every in-edge e of r."""
    r, j = _ambiguous(Z1, np.diff(ip) == 0)
    env = {k: np.zeros(s) for k, s in shapes.items()}
    if r.size:
        norm = oracle.rgcn_norm(ip, et, R)
        w = np.abs(dH1[r, j])
        np.add.at(env["b1"], j, w)
        for k in range(r.size):
            for e in range(ip[r[k]], ip[r[k] + 1]):
                env["V1"][ix[e], :, j[k]] += w[k] * norm[e] * np.abs(a1[et[e]])
                env["a1"][et[e], :] += w[k] * norm[e] * np.abs(V1[ix[e], :, j[k]])
    return env, int(r.size)


def gat_layer(ip, ix, L, H, F, slope=0.2, chunk=8_000_000):
    """Envelope for the flipped layer's own parameters (W, al, ar) from ambiguous edge scores."""
    el, er = L["el"], L["er"]
    N = el.shape[0]
    tau = BAND * (np.abs(el).max(0) + np.abs(er).max(0))            # per head
    T = L["T"].reshape(N, H, F)
    A = L["A"].reshape(N, H, F)
    dZ = L["dZ"].reshape(N, H, F)
    Xin = np.abs(np.asarray(L["Xin"], np.float64))
    env = {"W": np.zeros((Xin.shape[1], H * F)), "al": np.zeros((H, F)), "ar": np.zeros((H, F))}
    count = 0
    E = len(ix)
    for e0 in range(0, E, chunk):
        e1 = min(E, e0 + chunk)
        dst = np.searchsorted(ip, np.arange(e0, e1), side="right") - 1
        src = ix[e0:e1]
        s = el[src] + er[dst]                                           # [n, H]
        ei, hh = np.nonzero(np.abs(s) <= tau)
        for k in range(ei.size):
            u, v, h = int(src[ei[k]]), int(dst[ei[k]]), int(hh[k])
            sv = s[ei[k], h]
            z = sv if sv > 0 else slope * sv
            a = np.exp(z - L["lse"][v, h])
            g = float(dZ[v, h] @ T[u, h])
            c = float(dZ[v, h] @ A[v, h])
            d = (1.0 - slope) * a * abs(g - c)
            env["al"][h] += d * np.abs(T[u, h])
            env["ar"][h] += d * np.abs(T[v, h])
            env["W"][:, h * F:(h + 1) * F] += np.outer(Xin[u], d * np.abs(L["al"][h])) + \
                np.outer(Xin[v], d * np.abs(L["ar"][h]))
        count += ei.size
    return env, count
