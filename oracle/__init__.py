"""CPU oracle for Seastar's hot path -- TEST INFRASTRUCTURE ONLY.

Plain, slow, obviously-correct fp64 implementation of what the fused kernels compute, written
from the paper (/root/reference/PAPER.md; Wu et al., EuroSys'21) before any kernel.  Only
``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline`` / ``--impl reference``
legs may import this package.  It shares no code with ``paper_conf_eurosys_wumcjlzcy21_b200``
and never imports it; both consume the seeded inputs of ``synth``.

The edge loops live in ``seastar_oracle.c`` (compiled with gcc on first use); this module only
marshals numpy arrays and composes the per-layer definitions:

=========================  ===================================================  ==================
function                   definition                                           paper passage
=========================  ===================================================  ==================
preprocess                 degree-sorted CSR / reverse CSR / edge-id carry      L301, Fig.7
degree_norms               deg^-1/2, deg clamped >= 1                            Fig.1 "1/norm" (reading #1)
linear_fwd/bwd             T = X W (+b) and its VJP                              L289, Fig.2 f = W h
gcn_aggregate(_T)          dst_n * sum_in src_n * H   and its adjoint           Fig.1, Fig.3
gcn_layer_fwd/bwd          act(b + sum 1/norm h_u W)                             Fig.1 L85-93
appnp_fwd/bwd              Z <- (1-a) n A n Z + a H0, K steps                   [38] (L79, L481), reading #1
gat_attn_proj(_bwd)        e_u = f_u^T attn_u                                    Fig.2 L95-107
gat_fwd / gat_bwd          LeakyReLU -> edge softmax -> weighted sum            Fig.2, Fig.3
rgcn_norm/fwd/bwd          sum_r sum_{u in N_r(v)} 1/c_{v,r} h_u W_r           L465-475, [53]
rgcn_basis_fwd/bwd         featureless input, W_r = sum_b a_rb V_b (NEXT-2)      L485, L1219-1227, [53]
basis_combine(_bwd)        W_r = sum_b a_rb V_b for a dense layer (NEXT-2)       [53] (reading #26)
dropout_mask               counter-based keep mask x 1/(1-p) (NEXT-3)            L361, L481 (reading #27)
softmax_xent, adam         DGL default training loop                             L481
=========================  ===================================================  ==================

``oracle/model_ref.py`` composes these functions into whole training steps of the four models (the
reference the GPU models are compared with, and the CPU baseline ``bench.py`` times for configs[0..3]).

Every pin of these functions (hand fixtures, closed forms, dense brute force, finite differences)
is in ``tests/test_oracle_*.py``.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "seastar_oracle.c")
_SO = os.path.join(_HERE, "liboracle.so")

ACT = {"none": 0, "relu": 1, "elu": 2, "sigmoid": 3}


def build(force: bool = False) -> str:
    if force or not os.path.exists(_SO) or os.path.getmtime(_SO) < os.path.getmtime(_SRC):
        tmp = _SO + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-fopenmp", "-fPIC", "-shared", _SRC, "-o", tmp, "-lm"])
        os.replace(tmp, _SO)
    return _SO


_lib = None
_P = ctypes.c_void_p
_I = ctypes.c_int64
_D = ctypes.c_double


def _L():
    global _lib
    if _lib is None:
        lib = ctypes.CDLL(build())
        sig = {
            "orc_preprocess": ([_I, _I, _P, _P, _P, _I, _I] + [_P] * 12, ctypes.c_int),
            "orc_degree_norms": ([_I, _I, _P, _P, _P, _P], None),
            "orc_act_fwd": ([ctypes.c_int, _I, _P, _P], None),
            "orc_act_bwd": ([ctypes.c_int, _I, _P, _P, _P], None),
            "orc_linear_fwd": ([_I, _I, _I, _P, _P, _P, _P], None),
            "orc_linear_bwd": ([_I, _I, _I, _P, _P, _P, _P, _P, _P], None),
            "orc_gcn_aggregate": ([_I, _I, _P, _P, _I, _P, _P, _P, _P, _I, _P, _P], None),
            "orc_gcn_aggregate_T": ([_I, _I, _P, _P, _I, _P, _P, _P, _P, _I, _P, _P, _P, _P, _P], None),
            "orc_out_adjacency": ([_I, _I, _P, _P, _P, _P, _P], None),
            "orc_set_num_threads": ([ctypes.c_int], None),
            "orc_gat_attn_proj": ([_I, _I, _I, _P, _P, _P, _P, _P], None),
            "orc_gat_fwd": ([_I, _I, _P, _P, _I, _I, _P, _P, _P, _D, _P, _I, _P, _P, _P, _P], None),
            "orc_gat_bwd": ([_I, _I, _P, _P, _I, _I, _P, _P, _P, _D, _P, _P, _I, _P, _P, _P, _P, _P, _P, _P], None),
            "orc_rgcn_norm": ([_I, _I, _P, _P, ctypes.c_int32, _P], None),
            "orc_rgcn_fwd": ([_I, _I, _P, _P, _P, _I, _I, _P, _P, _P, _P, _I, _P], None),
            "orc_rgcn_bwd": ([_I, _I, _P, _P, _P, ctypes.c_int32, _I, _I, _P, _P, _P, _P, _P, _P], None),
            "orc_rgcn_basis_fwd": ([_I, _I, _P, _P, _P, _I, _I, _P, _P, _P, _P, _I, _P], None),
            "orc_rgcn_basis_bwd": ([_I, _I, _P, _P, _P, ctypes.c_int32, _I, _I, _P, _P, _P, _P, _P, _P], None),
            "orc_sm64": ([ctypes.c_uint64], ctypes.c_uint64),
            "orc_dropout_keep": ([ctypes.c_uint64, ctypes.c_uint32, ctypes.c_int32, _I, _I, ctypes.c_float, _P], None),
            "orc_softmax_xent": ([_I, _I, _P, _P, _P], _D),
            "orc_adam": ([_I, _P, _P, _P, _P, _D, _D, _D, _D, _I], None),
        }
        for name, (args, res) in sig.items():
            fn = getattr(lib, name)
            fn.argtypes = args
            fn.restype = res
        _lib = lib
    return _lib


def _p(a):
    if a is None:
        return None
    assert a.flags["C_CONTIGUOUS"], "oracle arrays must be C-contiguous"
    return a.ctypes.data


def _f64(a):
    return None if a is None else np.ascontiguousarray(a, dtype=np.float64)


def _i64(a):
    return None if a is None else np.ascontiguousarray(a, dtype=np.int64)


def _i32(a):
    return None if a is None else np.ascontiguousarray(a, dtype=np.int32)


def _act_id(act):
    return ACT[act] if isinstance(act, str) else int(act)


# ------------------------------------------------------------------------------------------
# a1-a3 graph representation
# ------------------------------------------------------------------------------------------
def preprocess(indptr, indices, etypes=None, row_begin=0, row_end=None):
    """Degree-sorted forward CSR + reverse CSR (+ LSF for partial ranges); all int64 arrays."""
    indptr, indices, etypes = _i64(indptr), _i64(indices), _i32(etypes)
    N = indptr.size - 1
    E = int(indptr[-1])
    row_end = N if row_end is None else row_end
    n_loc = row_end - row_begin
    E_fwd = int(indptr[row_end] - indptr[row_begin])
    E_rev = int(((indices >= row_begin) & (indices < row_end)).sum())
    o = {k: np.empty(n, np.int64) for k, n in [
        ("fwd_perm", n_loc), ("fwd_off", n_loc + 1), ("fwd_src", E_fwd), ("fwd_eid", E_fwd), ("fwd_type", E_fwd),
        ("rev_perm", n_loc), ("rev_off", n_loc + 1), ("rev_dst", E_rev), ("rev_eid", E_rev), ("rev_pos", E_rev),
        ("rev_type", E_rev), ("lsf_off", N + 1), ("lsf_eid", E_rev)]}
    rc = _L().orc_preprocess(N, E, _p(indptr), _p(indices), _p(etypes), row_begin, row_end,
                             *[_p(o[k]) for k in ("fwd_perm", "fwd_off", "fwd_src", "fwd_eid", "fwd_type",
                                                  "rev_perm", "rev_off", "rev_dst", "rev_eid", "rev_pos",
                                                  "rev_type", "lsf_off", "lsf_eid")])
    assert rc == 0
    if row_begin == 0 and row_end == N:
        del o["lsf_off"], o["lsf_eid"]
    return o


def degree_norms(indptr, indices):
    """(in_norm, out_norm) = max(deg,1)^-1/2 per vertex."""
    indptr, indices = _i64(indptr), _i64(indices)
    N = indptr.size - 1
    a, b = np.empty(N), np.empty(N)
    _L().orc_degree_norms(N, int(indptr[-1]), _p(indptr), _p(indices), _p(a), _p(b))
    return a, b


# ------------------------------------------------------------------------------------------
# activations, dense transform
# ------------------------------------------------------------------------------------------
def act_fwd(act, Z):
    Z = _f64(Z)
    Y = np.empty_like(Z)
    _L().orc_act_fwd(_act_id(act), Z.size, _p(Z), _p(Y))
    return Y


def act_bwd(act, Z, dY):
    Z, dY = _f64(Z), _f64(dY)
    dZ = np.empty_like(Z)
    _L().orc_act_bwd(_act_id(act), Z.size, _p(Z), _p(dY), _p(dZ))
    return dZ


def linear_fwd(X, W, b=None):
    X, W, b = _f64(X), _f64(W), _f64(b)
    M, K = X.shape
    Y = np.empty((M, W.shape[1]))
    _L().orc_linear_fwd(M, K, W.shape[1], _p(X), _p(W), _p(b), _p(Y))
    return Y


def linear_bwd(X, W, dY, need_dX=True, need_dW=True, need_db=True):
    X, W, dY = _f64(X), _f64(W), _f64(dY)
    M, K = X.shape
    Nout = W.shape[1]
    dX = np.empty((M, K)) if need_dX else None
    dW = np.empty((K, Nout)) if need_dW else None
    db = np.empty(Nout) if need_db else None
    _L().orc_linear_bwd(M, K, Nout, _p(X), _p(W), _p(dY), _p(dX), _p(dW), _p(db))
    return dX, dW, db


# ------------------------------------------------------------------------------------------
# GCN / APPNP
# ------------------------------------------------------------------------------------------
def gcn_aggregate(indptr, indices, H, src_norm=None, dst_norm=None, rows=None, edge_w=None):
    indptr, indices, H, edge_w = _i64(indptr), _i64(indices), _f64(H), _f64(edge_w)
    N = indptr.size - 1
    F = H.shape[1]
    rows = _i64(rows)
    nrows = N if rows is None else rows.size
    out = np.empty((nrows, F))
    sn, dn = _f64(src_norm), _f64(dst_norm)     # keep the converted arrays alive across the C call
    _L().orc_gcn_aggregate(N, int(indptr[-1]), _p(indptr), _p(indices), F, _p(H), _p(sn), _p(dn), _p(rows), nrows,
                           _p(out), _p(edge_w))
    return out


def out_adjacency(indptr, indices):
    """(dst[E], optr[N+1], oeid[E]): the graph's out-adjacency, a pure function of the graph.  Pass it as
    ``adj=`` to gcn_aggregate_T to keep its O(E) construction out of a timed row sample."""
    indptr, indices = _i64(indptr), _i64(indices)
    N, E = indptr.size - 1, int(indptr[-1])
    dst, optr, oeid = np.empty(E, np.int64), np.empty(N + 1, np.int64), np.empty(E, np.int64)
    _L().orc_out_adjacency(N, E, _p(indptr), _p(indices), _p(dst), _p(optr), _p(oeid))
    return dst, optr, oeid


def set_num_threads(n):
    _L().orc_set_num_threads(int(n))


def gcn_aggregate_T(indptr, indices, G, src_norm=None, dst_norm=None, rows=None, edge_w=None, adj=None):
    indptr, indices, G, edge_w = _i64(indptr), _i64(indices), _f64(G), _f64(edge_w)
    N = indptr.size - 1
    F = G.shape[1]
    rows = _i64(rows)
    nrows = N if rows is None else rows.size
    out = np.empty((nrows, F))
    sn, dn = _f64(src_norm), _f64(dst_norm)     # keep the converted arrays alive across the C call
    ad = (None, None, None) if adj is None else tuple(_i64(a) for a in adj)
    _L().orc_gcn_aggregate_T(N, int(indptr[-1]), _p(indptr), _p(indices), F, _p(G), _p(sn), _p(dn), _p(rows),
                             nrows, _p(out), _p(edge_w), *(_p(a) for a in ad))
    return out


def gcn_layer_fwd(indptr, indices, X, W, b, act, src_norm, dst_norm):
    """Fig. 1: Y = act(b + dst_n * sum_in src_n * X_u W).  Returns (Y, Zpre).

    Transform first iff F_in > F_out (reading #20); both orders are the same linear map."""
    if W.shape[0] > W.shape[1]:
        Z = gcn_aggregate(indptr, indices, linear_fwd(X, W), src_norm, dst_norm)
    else:
        Z = linear_fwd(gcn_aggregate(indptr, indices, X, src_norm, dst_norm), W)
    if b is not None:
        Z = Z + _f64(b)[None, :]
    return act_fwd(act, Z), Z


def gcn_layer_bwd(indptr, indices, X, W, Zpre, act, src_norm, dst_norm, dY, need_dX=True):
    """VJP of gcn_layer_fwd: returns (dX, dW, db)."""
    dZ = act_bwd(act, Zpre, dY)
    db = dZ.sum(axis=0)
    P = gcn_aggregate(indptr, indices, X, src_norm, dst_norm)     # Â X  (so that Z = Â X W + b)
    _, dW, _ = linear_bwd(P, W, dZ, need_dX=False, need_db=False)
    dX = None
    if need_dX:
        dP, _, _ = linear_bwd(P, W, dZ, need_dW=False, need_db=False)
        dX = gcn_aggregate_T(indptr, indices, dP, src_norm, dst_norm)
    return dX, dW, db


def appnp_fwd(indptr, indices, H0, K, alpha, norm=None, edge_masks=None):
    """APPNP propagation [38]: Z^0 = H0, Z^{k+1} = (1-a) * n * sum_in n_u Z^k_u + a * H0.
    norm defaults to in-degree^-1/2 on both sides (DGL APPNPConv; reading in DESIGN.md).
    edge_masks: optional list of K [E] edge-dropout multipliers (by user edge id), one per step (NEXT-3)."""
    H0 = _f64(H0)
    if norm is None:
        norm, _ = degree_norms(indptr, indices)
    Z = H0.copy()
    for k in range(K):
        w = None if edge_masks is None else edge_masks[k]
        Z = (1.0 - alpha) * gcn_aggregate(indptr, indices, Z, norm, norm, edge_w=w) + alpha * H0
    return Z


def appnp_bwd(indptr, indices, dZ, K, alpha, norm=None, edge_masks=None):
    """VJP of appnp_fwd w.r.t. H0 (reversing the recurrence; step k's edge mask in reverse order)."""
    dZ = _f64(dZ)
    if norm is None:
        norm, _ = degree_norms(indptr, indices)
    G = dZ.copy()
    dH0 = np.zeros_like(dZ)
    for k in reversed(range(K)):
        dH0 += alpha * G
        w = None if edge_masks is None else edge_masks[k]
        G = (1.0 - alpha) * gcn_aggregate_T(indptr, indices, G, norm, norm, edge_w=w)
    return dH0 + G


# ------------------------------------------------------------------------------------------
# GAT
# ------------------------------------------------------------------------------------------
def gat_attn_proj(T, a_l, a_r):
    """T [N,H,F] -> (el, er) [N,H]."""
    T, a_l, a_r = _f64(T), _f64(a_l), _f64(a_r)
    N, H, F = T.shape
    el, er = np.empty((N, H)), np.empty((N, H))
    _L().orc_gat_attn_proj(N, H, F, _p(T), _p(a_l), _p(a_r), _p(el), _p(er))
    return el, er


def gat_attn_proj_bwd(T, a_l, a_r, del_, der):
    """VJP of gat_attn_proj: (dT contribution [N,H,F], da_l [H,F], da_r [H,F])."""
    T, a_l, a_r, del_, der = map(_f64, (T, a_l, a_r, del_, der))
    dT = del_[:, :, None] * a_l[None] + der[:, :, None] * a_r[None]
    da_l = np.einsum("uh,uhf->hf", del_, T)
    da_r = np.einsum("uh,uhf->hf", der, T)
    return dT, da_l, da_r


def gat_fwd(indptr, indices, T, el, er, slope=0.2, rows=None, want_alpha=False, mask=None):
    """Returns (A [nrows,H,F], lse [nrows,H], alpha [E,H] or None).  mask: [E,H] attention-dropout
    multiplier by user edge id (NEXT-3), A = sum_e alpha_e mask_e T_u."""
    indptr, indices, T, el, er, mask = _i64(indptr), _i64(indices), _f64(T), _f64(el), _f64(er), _f64(mask)
    N = indptr.size - 1
    E = int(indptr[-1])
    _, H, F = T.shape
    rows = _i64(rows)
    nrows = N if rows is None else rows.size
    A = np.empty((nrows, H, F))
    lse = np.empty((nrows, H))
    alpha = np.empty((E, H)) if want_alpha else None
    _L().orc_gat_fwd(N, E, _p(indptr), _p(indices), H, F, _p(T), _p(el), _p(er), slope, _p(rows), nrows,
                     _p(A), _p(lse), _p(alpha), _p(mask))
    return A, lse, alpha


def gat_bwd(indptr, indices, T, el, er, dA, slope=0.2, rows=None, mask=None, adj=None):
    """Returns (dT [nrows,H,F], del [nrows,H], der [N,H]).  mask: as in gat_fwd; adj: out_adjacency() or None."""
    indptr, indices, T, el, er, dA = _i64(indptr), _i64(indices), _f64(T), _f64(el), _f64(er), _f64(dA)
    mask = _f64(mask)
    N = indptr.size - 1
    _, H, F = T.shape
    rows = _i64(rows)
    nrows = N if rows is None else rows.size
    dT = np.empty((nrows, H, F))
    dl = np.empty((nrows, H))
    dr = np.empty((N, H))
    ad = (None, None, None) if adj is None else tuple(_i64(a) for a in adj)
    _L().orc_gat_bwd(N, int(indptr[-1]), _p(indptr), _p(indices), H, F, _p(T), _p(el), _p(er), slope, _p(dA),
                     _p(rows), nrows, _p(dT), _p(dl), _p(dr), _p(mask), *(_p(a) for a in ad))
    return dT, dl, dr


# ------------------------------------------------------------------------------------------
# R-GCN
# ------------------------------------------------------------------------------------------
def rgcn_norm(indptr, etypes, R):
    indptr, etypes = _i64(indptr), _i32(etypes)
    N = indptr.size - 1
    out = np.empty(int(indptr[-1]))
    _L().orc_rgcn_norm(N, int(indptr[-1]), _p(indptr), _p(etypes), R, _p(out))
    return out


def rgcn_fwd(indptr, indices, etypes, X, W, norm=None, rows=None):
    """sum_{e in in(v)} norm_e X[src] W[type] ; norm=None => 1/c_{v,r}.  W is [R,Fin,Fout]."""
    indptr, indices, etypes, X, W = _i64(indptr), _i64(indices), _i32(etypes), _f64(X), _f64(W)
    N = indptr.size - 1
    R, Fin, Fout = W.shape
    norm = rgcn_norm(indptr, etypes, R) if norm is None else _f64(norm)
    rows = _i64(rows)
    nrows = N if rows is None else rows.size
    out = np.empty((nrows, Fout))
    _L().orc_rgcn_fwd(N, int(indptr[-1]), _p(indptr), _p(indices), _p(etypes), Fin, Fout, _p(X), _p(W),
                      _p(norm), _p(rows), nrows, _p(out))
    return out


def rgcn_bwd(indptr, indices, etypes, X, W, dA, norm=None, need_dX=True, need_dW=True):
    indptr, indices, etypes, X, W, dA = _i64(indptr), _i64(indices), _i32(etypes), _f64(X), _f64(W), _f64(dA)
    N = indptr.size - 1
    R, Fin, Fout = W.shape
    norm = rgcn_norm(indptr, etypes, R) if norm is None else _f64(norm)
    dX = np.empty((N, Fin)) if need_dX else None
    dW = np.empty((R, Fin, Fout)) if need_dW else None
    _L().orc_rgcn_bwd(N, int(indptr[-1]), _p(indptr), _p(indices), _p(etypes), R, Fin, Fout, _p(X), _p(W),
                      _p(norm), _p(dA), _p(dX), _p(dW))
    return dX, dW


# ------------------------------------------------------------------------------------------
# NEXT-2: R-GCN with featureless input and basis decomposition (reading #27)
# ------------------------------------------------------------------------------------------
def rgcn_basis_fwd(indptr, indices, etypes, V, a, norm=None, rows=None):
    """sum_{e in in(v)} norm_e sum_b a[type_e, b] V[src_e, b, :] ; V is [N, B, F], a is [R, B]."""
    indptr, indices, etypes, V, a = _i64(indptr), _i64(indices), _i32(etypes), _f64(V), _f64(a)
    N = indptr.size - 1
    R, B = a.shape
    assert V.shape[:2] == (N, B), V.shape
    F = V.shape[2]
    norm = rgcn_norm(indptr, etypes, R) if norm is None else _f64(norm)
    rows = _i64(rows)
    nrows = N if rows is None else rows.size
    out = np.empty((nrows, F))
    _L().orc_rgcn_basis_fwd(N, int(indptr[-1]), _p(indptr), _p(indices), _p(etypes), B, F, _p(V), _p(a),
                            _p(norm), _p(rows), nrows, _p(out))
    return out


def rgcn_basis_bwd(indptr, indices, etypes, V, a, dA, norm=None, need_dV=True, need_da=True):
    indptr, indices, etypes, V, a, dA = (_i64(indptr), _i64(indices), _i32(etypes), _f64(V), _f64(a),
                                         _f64(dA))
    N = indptr.size - 1
    R, B = a.shape
    F = V.shape[2]
    norm = rgcn_norm(indptr, etypes, R) if norm is None else _f64(norm)
    dV = np.empty((N, B, F)) if need_dV else None
    da = np.empty((R, B)) if need_da else None
    _L().orc_rgcn_basis_bwd(N, int(indptr[-1]), _p(indptr), _p(indices), _p(etypes), R, B, F, _p(V), _p(a),
                            _p(norm), _p(dA), _p(dV), _p(da))
    return dV, da


def basis_combine(a, Vb):
    """W[r] = sum_b a[r,b] Vb[b]   (a [R,B], Vb [B,Fin,Fout] -> W [R,Fin,Fout]); [53] Eq. 3."""
    a, Vb = _f64(a), _f64(Vb)
    R, B = a.shape
    W = np.zeros((R,) + Vb.shape[1:])
    for r in range(R):
        for b in range(B):
            W[r] += a[r, b] * Vb[b]
    return W


def basis_combine_bwd(a, Vb, dW):
    """VJP of basis_combine: da[r,b] = <dW[r], Vb[b]>, dVb[b] = sum_r a[r,b] dW[r]."""
    a, Vb, dW = _f64(a), _f64(Vb), _f64(dW)
    R, B = a.shape
    da = np.array([[float((dW[r] * Vb[b]).sum()) for b in range(B)] for r in range(R)])
    dVb = np.zeros_like(Vb)
    for b in range(B):
        for r in range(R):
            dVb[b] += a[r, b] * dW[r]
    return da, dVb


# ------------------------------------------------------------------------------------------
# NEXT-3: reproducible dropout (reading #27)
# ------------------------------------------------------------------------------------------
def sm64(z):
    return int(_L().orc_sm64(int(z) & 0xFFFFFFFFFFFFFFFF))


def dropout_mask(seed, site, step, M, F, p, row0=0):
    """[M, F] fp64 inverted-dropout multiplier: keep(seed, site, step, (row0 + r) * F + f) / (1 - p), else 0."""
    p32 = float(np.float32(p))
    keep = np.empty(M * F, np.uint8)
    _L().orc_dropout_keep(int(seed), int(site), int(step), int(row0) * int(F), M * F, p32, _p(keep))
    return keep.reshape(M, F).astype(np.float64) / (1.0 - p32)


# ------------------------------------------------------------------------------------------
# loss, optimiser
# ------------------------------------------------------------------------------------------
def softmax_xent(logits, labels, want_grad=True):
    logits, labels = _f64(logits), _i64(labels)
    M, C = logits.shape
    d = np.empty((M, C)) if want_grad else None
    loss = _L().orc_softmax_xent(M, C, _p(logits), _p(labels), _p(d))
    return loss, d


def adam(param, grad, m, v, lr, t, b1=0.9, b2=0.999, eps=1e-8):
    """In-place Adam step on fp64 arrays (param, m, v are updated)."""
    for a in (param, m, v):
        assert a.dtype == np.float64 and a.flags["C_CONTIGUOUS"]
    grad = _f64(grad)
    _L().orc_adam(param.size, _p(param), _p(grad), _p(m), _p(v), lr, b1, b2, eps, t)
