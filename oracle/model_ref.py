"""Whole-model references composed from the pinned oracle functions (test infrastructure).

Each function returns (loss, grads) for one forward + backward of the paper's models with the
readings of DESIGN.md §3; the GPU models in paper_conf_eurosys_wumcjlzcy21_b200.models must match
them parameter by parameter."""
import numpy as np

import oracle  # noqa: F401  (package of the oracle functions composed here)


def _mask(drop, site, M, F):
    """NEXT-3 inverted-dropout multiplier for one dropout site (all ones when drop is None or p = 0).
    drop = dict(p=..., seed=..., step=...[, attn_p=...]); sites: GCN 1 = hidden; GAT 1 = X, 2 = hidden, 3 / 4 =
    layer-1 / layer-2 attention (E x H, by user edge id)."""
    if not drop or drop["p"] == 0.0:
        return None
    return oracle.dropout_mask(drop["seed"], site, drop["step"], M, F, drop["p"])


def gcn2(ip, ix, X, lab, p, acts=None, drop=None):
    in_n, out_n = oracle.degree_norms(ip, ix)
    T = oracle.linear_fwd(X, p["W1"])
    Z1 = oracle.gcn_aggregate(ip, ix, T, out_n, in_n) + p["b1"]
    H1 = oracle.act_fwd("relu", Z1)
    m1 = _mask(drop, 1, *H1.shape)
    P2 = oracle.gcn_aggregate(ip, ix, H1 if m1 is None else H1 * m1, out_n, in_n)
    logits = oracle.linear_fwd(P2, p["W2"], p["b2"])
    loss, dlog = oracle.softmax_xent(logits, lab)
    dP2, dW2, db2 = oracle.linear_bwd(P2, p["W2"], dlog)
    dH1 = oracle.gcn_aggregate_T(ip, ix, dP2, out_n, in_n)
    if m1 is not None:
        dH1 = dH1 * m1
    dZ1 = oracle.act_bwd("relu", Z1, dH1)
    db1 = dZ1.sum(0)
    dT = oracle.gcn_aggregate_T(ip, ix, dZ1, out_n, in_n)
    _, dW1, _ = oracle.linear_bwd(X, p["W1"], dT, need_dX=False, need_db=False)
    if acts is not None:
        acts.update(H1=H1, logits=logits, Z1=Z1, dH1=dH1)
    return loss, {"W1": dW1, "b1": db1, "W2": dW2, "b2": db2}


def _gat_layer_fwd(ip, ix, Xin, W, al, ar, b, act, H, F, mask=None):
    N = Xin.shape[0]
    T = oracle.linear_fwd(Xin, W).reshape(N, H, F)
    el, er = oracle.gat_attn_proj(T, al, ar)
    A, lse, _ = oracle.gat_fwd(ip, ix, T, el, er, 0.2, mask=mask)
    Z = A.reshape(N, H * F) + b
    _gat_layer_fwd.lse = lse          # exposed to callers that want it (acts); not part of the return value
    return T, el, er, Z, oracle.act_fwd(act, Z)


def _gat_layer_bwd(ip, ix, Xin, W, al, ar, T, el, er, Z, act, dY, H, F, need_dX, mask=None):
    N = Xin.shape[0]
    dZ = oracle.act_bwd(act, Z, dY)
    db = dZ.sum(0)
    dT, dl, dr = oracle.gat_bwd(ip, ix, T, el, er, dZ.reshape(N, H, F), 0.2, mask=mask)
    dTp, dal, dar = oracle.gat_attn_proj_bwd(T, al, ar, dl, dr)
    dTt = (dT + dTp).reshape(N, H * F)
    dX, dW, _ = oracle.linear_bwd(Xin, W, dTt, need_dX=need_dX, need_db=False)
    _gat_layer_bwd.dZ = dZ
    return dX, dW, dal, dar, db


def gat2(ip, ix, X, lab, p, heads, hidden, acts=None, drop=None):
    C = p["W2"].shape[1]
    m0 = _mask(drop, 1, *X.shape)                    # feat_drop on the layer-1 input
    Xd = X if m0 is None else X * m0
    E = int(ip[-1])
    ad = {"p": drop["attn_p"], "seed": drop["seed"], "step": drop["step"]} if drop and drop.get("attn_p") else None
    a1, a2 = _mask(ad, 3, E, heads), _mask(ad, 4, E, 1)   # attn_drop, by (user edge id, head)
    T1, el1, er1, Z1, Y1 = _gat_layer_fwd(ip, ix, Xd, p["W1"], p["al1"], p["ar1"], p["b1"], "elu", heads, hidden,
                                          a1)
    lse1 = _gat_layer_fwd.lse
    m1 = _mask(drop, 2, *Y1.shape)                   # feat_drop on the layer-2 input
    Y1d = Y1 if m1 is None else Y1 * m1
    T2, el2, er2, Z2, Y2 = _gat_layer_fwd(ip, ix, Y1d, p["W2"], p["al2"], p["ar2"], p["b2"], "none", 1, C, a2)
    lse2 = _gat_layer_fwd.lse
    loss, dY2 = oracle.softmax_xent(Y2, lab)
    dY1, dW2, dal2, dar2, db2 = _gat_layer_bwd(ip, ix, Y1d, p["W2"], p["al2"], p["ar2"], T2, el2, er2, Z2, "none",
                                               dY2, 1, C, True, a2)
    if m1 is not None:
        dY1 = dY1 * m1
    dZ2 = _gat_layer_bwd.dZ
    _, dW1, dal1, dar1, db1 = _gat_layer_bwd(ip, ix, Xd, p["W1"], p["al1"], p["ar1"], T1, el1, er1, Z1, "elu", dY1,
                                             heads, hidden, False, a1)
    dZ1 = _gat_layer_bwd.dZ
    if acts is not None:
        acts.update(Y1=Y1, Y2=Y2,
                    layers=[dict(Xin=Xd, T=T1, el=el1, er=er1, A=Z1 - p["b1"], lse=lse1, dZ=dZ1, al=p["al1"],
                                 ar=p["ar1"]),
                            dict(Xin=Y1d, T=T2, el=el2, er=er2, A=Z2 - p["b2"], lse=lse2, dZ=dZ2, al=p["al2"],
                                 ar=p["ar2"])])
    return loss, {"W1": dW1, "al1": dal1, "ar1": dar1, "b1": db1, "W2": dW2, "al2": dal2, "ar2": dar2, "b2": db2}


def appnp(ip, ix, X, lab, p, K, alpha, acts=None, drop=None):
    """drop: dict(edge_p=..., seed=..., step=...): DGL APPNPConv's edge_drop, a fresh [E] mask per propagation
    step k (site 16 + k, by user edge id)."""
    Z1 = oracle.linear_fwd(X, p["W1"], p["b1"])
    Hh = oracle.act_fwd("relu", Z1)
    H0 = oracle.linear_fwd(Hh, p["W2"], p["b2"])
    masks = None
    if drop and drop.get("edge_p"):
        E = int(ip[-1])
        masks = [oracle.dropout_mask(drop["seed"], 16 + k, drop["step"], E, 1, drop["edge_p"])[:, 0] for k in range(K)]
    Z = oracle.appnp_fwd(ip, ix, H0, K, alpha, edge_masks=masks)
    loss, dZ = oracle.softmax_xent(Z, lab)
    dH0 = oracle.appnp_bwd(ip, ix, dZ, K, alpha, edge_masks=masks)
    dHh, dW2, db2 = oracle.linear_bwd(Hh, p["W2"], dH0)
    dZ1 = oracle.act_bwd("relu", Z1, dHh)
    _, dW1, db1 = oracle.linear_bwd(X, p["W1"], dZ1, need_dX=False)
    if acts is not None:
        acts.update(Z=Z, Z1=Z1, dH1=dHh)
    return loss, {"W1": dW1, "b1": db1, "W2": dW2, "b2": db2}


def rgcn2(ip, ix, et, X, lab, p, acts=None):
    Z1 = oracle.rgcn_fwd(ip, ix, et, X, p["W1"]) + p["b1"]
    H1 = oracle.act_fwd("relu", Z1)
    Z2 = oracle.rgcn_fwd(ip, ix, et, H1, p["W2"]) + p["b2"]
    loss, dZ2 = oracle.softmax_xent(Z2, lab)
    dH1, dW2 = oracle.rgcn_bwd(ip, ix, et, H1, p["W2"], dZ2)
    db2 = dZ2.sum(0)
    dZ1 = oracle.act_bwd("relu", Z1, dH1)
    _, dW1 = oracle.rgcn_bwd(ip, ix, et, X, p["W1"], dZ1, need_dX=False)
    if acts is not None:
        acts.update(H1=H1, logits=Z2, Z1=Z1, dH1=dH1)
    return loss, {"W1": dW1, "b1": dZ1.sum(0), "W2": dW2, "b2": db2}


def rgcnb2(ip, ix, et, lab, p, acts=None):
    """NEXT-2 R-GCN (featureless input layer with bases, dense basis output layer; reading #26)."""
    Z1 = oracle.rgcn_basis_fwd(ip, ix, et, p["V1"], p["a1"]) + p["b1"]
    H1 = oracle.act_fwd("relu", Z1)
    W2 = oracle.basis_combine(p["a2"], p["V2"])
    Z2 = oracle.rgcn_fwd(ip, ix, et, H1, W2) + p["b2"]
    loss, dZ2 = oracle.softmax_xent(Z2, lab)
    dH1, dW2 = oracle.rgcn_bwd(ip, ix, et, H1, W2, dZ2)
    da2, dV2 = oracle.basis_combine_bwd(p["a2"], p["V2"], dW2)
    dZ1 = oracle.act_bwd("relu", Z1, dH1)
    dV1, da1 = oracle.rgcn_basis_bwd(ip, ix, et, p["V1"], p["a1"], dZ1)
    if acts is not None:
        acts.update(H1=H1, logits=Z2, Z1=Z1, dH1=dH1)
    return loss, {"V1": dV1, "a1": da1, "b1": dZ1.sum(0), "V2": dV2, "a2": da2, "b2": dZ2.sum(0)}
