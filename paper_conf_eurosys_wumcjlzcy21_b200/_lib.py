"""Thin ctypes binding of ``include/seastar.h`` -- argument marshalling only.

Every function here has the name of the C entry point it calls and does nothing but turn torch
tensors into device pointers, pick the current CUDA stream and raise on a non-zero status.  All
work happens in ``libseastar.so`` (the hand-written sm_100a kernels); there is no CPU fallback:
importing this module on a machine without the built library, or calling into it without a B200,
raises.
"""
from __future__ import annotations

import ctypes
import os

import torch

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libseastar.so")

ACT = {"none": 0, "relu": 1, "elu": 2, "sigmoid": 3}
GRAPH_RGCN_NORM = 1
FWD, REV, LSF = 0, 1, 2
NORM_BOTH, NORM_IN = 0, 1
NUM_BUCKETS = 4
STATUS = {0: "OK", 1: "INVALID_ARGUMENT", 2: "INVALID_GRAPH", 3: "OUT_OF_MEMORY", 4: "CUDA", 5: "UNSUPPORTED"}


class SeastarError(RuntimeError):
    def __init__(self, fn: str, status: int, msg: str):
        super().__init__(f"{fn} failed with SEASTAR_ERR_{STATUS.get(status, status)}: {msg}")
        self.status = status


class seastar_graph_info_t(ctypes.Structure):
    _fields_ = [
        ("num_nodes", ctypes.c_int64), ("num_edges", ctypes.c_int64),
        ("row_begin", ctypes.c_int64), ("row_end", ctypes.c_int64),
        ("num_fwd_edges", ctypes.c_int64), ("num_rev_edges", ctypes.c_int64),
        ("max_in_degree", ctypes.c_int64), ("max_out_degree", ctypes.c_int64),
        ("num_etypes", ctypes.c_int32), ("partitioned", ctypes.c_int32),
        ("fwd_bucket_rows", ctypes.c_int64 * NUM_BUCKETS), ("rev_bucket_rows", ctypes.c_int64 * NUM_BUCKETS),
    ]


_P = ctypes.c_void_p
_I64 = ctypes.c_int64
_I32 = ctypes.c_int32
_F = ctypes.c_float
_SZ = ctypes.c_size_t
_ST = ctypes.c_int

# name -> (argtypes, restype)
_SIGS = {
    "seastar_last_error": ([], ctypes.c_char_p),
    "seastar_abi_version": ([], _I32),
    "seastar_device_check": ([], _ST),
    "seastar_graph_create": ([_I64, _I64, _P, _P, _P, _I32, _I64, _I64, ctypes.c_uint32, _P,
                              ctypes.POINTER(_P)], _ST),
    "seastar_graph_destroy": ([_P], _ST),
    "seastar_graph_info": ([_P, ctypes.POINTER(seastar_graph_info_t)], _ST),
    "seastar_graph_export": ([_P, _I32, _P, _P, _P, _P, _P, _P, _P, _P], _ST),
    "seastar_graph_degree_norms": ([_P, _I32, _P, _P, _P], _ST),
    "seastar_linear_fwd": ([_P, _I64, _I64, _I64, _P, _I64, _P, _P, _I32, _P, _I64, _P, _SZ, _P], _ST),
    "seastar_linear_fwd_workspace": ([_I64, _I64], _SZ),
    "seastar_linear_bwd_data": ([_P, _I64, _I64, _I64, _P, _I64, _P, _P, _I32, _P, _I64, _P], _ST),
    "seastar_linear_bwd_weight": ([_P, _I64, _I64, _I64, _P, _I64, _I64, _P, _P, _P, _SZ, _P], _ST),
    "seastar_linear_bwd_weight_workspace": ([_I64, _I64, _I64], _SZ),
    "seastar_gcn_fwd": ([_P, _P, _I64, _I64, _P, _P, _I32, _F, _P, _P, _P, _P, _P, _P], _ST),
    "seastar_gcn_bwd": ([_P, _P, _I64, _I64, _P, _F, _P, _I32, _P, _P, _P, _P, _P], _ST),
    "seastar_gcn_fwd_split": ([_P, _I32, _P, _I64, _P, _I64, _I64, _P, _P, _I32, _F, _P, _P, _P, _P, _P, _I64, _P, _P],
                              _ST),
    "seastar_gcn_bwd_split": ([_P, _I32, _P, _I64, _P, _I64, _I64, _P, _F, _P, _I32, _P, _P, _P, _P, _I64, _P, _P],
                              _ST),
    "seastar_gat_attn_proj": ([_P, _I64, _I32, _I32, _I64, _P, _P, _P, _P, _P], _ST),
    "seastar_gat_fwd": ([_P, _P, _P, _P, _I32, _I32, _I64, _F, _P, _I32, _P, _P, _P, _P, _P, _P, _P], _ST),
    "seastar_gat_record_ld": ([_I32, _I32], _I64),
    "seastar_gat_bwd_prep": ([_P, _P, _P, _I32, _P, _P, _P, _I32, _I32, _I64, _P, _P, _P, _P, _P], _ST),
    "seastar_gat_bwd": ([_P, _P, _P, _P, _I32, _I32, _I64, _F, _P, _P, _P, _P], _ST),
    "seastar_gat_der": ([_P, _P, _P, _P, _I32, _I32, _I64, _F, _P, _P, _P], _ST),
    "seastar_gat_attn_proj_bwd": ([_P, _I64, _I32, _I32, _I64, _P, _P, _P, _P, _P, _P, _P, _P, _SZ, _P], _ST),
    "seastar_gat_attn_proj_bwd_workspace": ([_I64, _I32, _I32], _SZ),
    "seastar_rgcn_fwd": ([_P, _P, _I64, _I64, _P, _I64, _P, _P, _I32, _P, _I64, _P, _SZ, _P], _ST),
    "seastar_rgcn_fwd_workspace": ([_P, _I64, _I64], _SZ),
    "seastar_rgcn_bwd": ([_P, _P, _I64, _I64, _P, _I64, _I64, _P, _P, _P, _I32, _P, _P, _P, _SZ, _P], _ST),
    "seastar_rgcn_bwd_workspace": ([_P, _I64, _I64], _SZ),
    "seastar_rgcn_basis_fwd": ([_P, _P, _I64, _I64, _I64, _P, _P, _P, _I64, _P, _I32, _P, _I64, _P], _ST),
    "seastar_rgcn_basis_bwd": ([_P, _P, _I64, _I64, _I64, _P, _P, _P, _I64, _P, _P, _P, _SZ, _P], _ST),
    "seastar_rgcn_basis_bwd_workspace": ([_P, _I64], _SZ),
    "seastar_dropout": ([_P, _I64, _I64, _I64, _I64, _F, ctypes.c_uint64, ctypes.c_uint32, _P, _P, _I64, _P], _ST),
    "seastar_basis_combine": ([_P, _P, _I32, _I32, _I64, _P, _P], _ST),
    "seastar_basis_combine_bwd": ([_P, _P, _P, _I32, _I32, _I64, _P, _P, _P], _ST),
    "seastar_softmax_xent": ([_P, _I64, _I64, _I32, _I64, _P, _P, _P, _I64, _P, _SZ, _P], _ST),
    "seastar_softmax_xent_workspace": ([_I64], _SZ),
    "seastar_colsum": ([_P, _I64, _I64, _I64, _P, _P, _SZ, _P], _ST),
    "seastar_colsum_workspace": ([_I64, _I64], _SZ),
    "seastar_axpby": ([_I64, _F, _P, _F, _P, _P], _ST),
    "seastar_row_scale": ([_P, _I64, _I64, _I64, _P, _P, _I64, _P], _ST),
    "seastar_adam": ([_P, _P, _P, _P, _I64, _F, _F, _F, _F, _P, _P], _ST),
    "seastar_step_inc": ([_P, _P], _ST),
}

_lib = None


def load() -> ctypes.CDLL:
    """Load libseastar.so (raises if it has not been built: there is no fallback)."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise ImportError(f"{LIB_PATH} is missing; build it with "
                              "`python -m paper_conf_eurosys_wumcjlzcy21_b200.build` (nvcc, sm_100a)")
        lib = ctypes.CDLL(LIB_PATH)
        for name, (args, res) in _SIGS.items():
            fn = getattr(lib, name)
            fn.argtypes = args
            fn.restype = res
        _lib = lib
    return _lib


def exported_symbols():
    return list(_SIGS)


def _ptr(x):
    if x is None:
        return None
    if isinstance(x, int):
        return x
    if isinstance(x, torch.Tensor):
        return x.data_ptr() if x.numel() else None
    raise TypeError(f"cannot pass {type(x)} as a pointer")


def _dptr(x, what):
    """device pointer of a CUDA tensor (checked)."""
    if x is None:
        return None
    if isinstance(x, torch.Tensor):
        if not x.is_cuda:
            raise ValueError(f"{what} must be a CUDA tensor")
        return x.data_ptr() if x.numel() else None
    return _ptr(x)


def _stream(stream):
    if stream is None:
        return torch.cuda.current_stream().cuda_stream
    if isinstance(stream, torch.cuda.Stream):
        return stream.cuda_stream
    return int(stream)


def _call(name, *args):
    st = getattr(load(), name)(*args)
    if st != 0:
        msg = load().seastar_last_error()
        raise SeastarError(name, st, msg.decode() if msg else "")


def _act(a):
    return ACT[a] if isinstance(a, str) else int(a)


# ----------------------------------------------------------------------------------- library
def seastar_abi_version() -> int:
    return int(load().seastar_abi_version())


def seastar_device_check() -> None:
    _call("seastar_device_check")


def seastar_last_error() -> str:
    m = load().seastar_last_error()
    return m.decode() if m else ""


# ----------------------------------------------------------------------------------- graph
def seastar_graph_create(N, E, indptr, indices, etypes=None, num_etypes=0, row_begin=0, row_end=None, flags=0,
                         stream=None) -> int:
    out = _P()
    row_end = N if row_end is None else row_end
    _call("seastar_graph_create", N, E, _dptr(indptr, "indptr"), _dptr(indices, "indices"), _dptr(etypes, "etypes"),
          num_etypes, row_begin, row_end, flags, _stream(stream), ctypes.byref(out))
    return out.value


def seastar_graph_destroy(g) -> None:
    _call("seastar_graph_destroy", g)


def seastar_graph_info(g) -> dict:
    info = seastar_graph_info_t()
    _call("seastar_graph_info", g, ctypes.byref(info))
    d = {k: getattr(info, k) for k, _ in seastar_graph_info_t._fields_}
    d["fwd_bucket_rows"] = list(info.fwd_bucket_rows)
    d["rev_bucket_rows"] = list(info.rev_bucket_rows)
    return d


def seastar_graph_export(g, which, perm=None, off=None, nbr=None, eid=None, pos=None, etype=None, norm=None,
                         stream=None) -> None:
    _call("seastar_graph_export", g, which, *[_dptr(x, "export buffer") for x in (perm, off, nbr, eid, pos, etype,
                                                                                  norm)], _stream(stream))


def seastar_graph_degree_norms(g, mode, src_norm_loc=None, dst_norm_loc=None, stream=None) -> None:
    _call("seastar_graph_degree_norms", g, mode, _dptr(src_norm_loc, "src_norm"), _dptr(dst_norm_loc, "dst_norm"),
          _stream(stream))


# ----------------------------------------------------------------------------------- dense
def seastar_linear_fwd_workspace(K, Nout) -> int:
    return int(load().seastar_linear_fwd_workspace(K, Nout))


def seastar_linear_fwd(X, M, K, ldx, W, Nout, bias, row_scale, act, Y, ldy, workspace=None, ws_bytes=0,
                       stream=None) -> None:
    _call("seastar_linear_fwd", _dptr(X, "X"), M, K, ldx, _dptr(W, "W"), Nout, _dptr(bias, "bias"),
          _dptr(row_scale, "row_scale"), _act(act), _dptr(Y, "Y"), ldy, _dptr(workspace, "workspace"), ws_bytes,
          _stream(stream))


def seastar_linear_bwd_data(dY, M, Nout, ldy, W, K, row_scale, Yact, act, dX, ldx, stream=None) -> None:
    _call("seastar_linear_bwd_data", _dptr(dY, "dY"), M, Nout, ldy, _dptr(W, "W"), K, _dptr(row_scale, "row_scale"),
          _dptr(Yact, "Yact"), _act(act), _dptr(dX, "dX"), ldx, _stream(stream))


def seastar_linear_bwd_weight_workspace(M, K, Nout) -> int:
    return int(load().seastar_linear_bwd_weight_workspace(M, K, Nout))


def seastar_linear_bwd_weight(X, M, K, ldx, dY, Nout, ldy, dW, db, workspace, ws_bytes, stream=None) -> None:
    _call("seastar_linear_bwd_weight", _dptr(X, "X"), M, K, ldx, _dptr(dY, "dY"), Nout, ldy, _dptr(dW, "dW"),
          _dptr(db, "db"), _dptr(workspace, "workspace"), ws_bytes, _stream(stream))


# ----------------------------------------------------------------------------------- GCN / APPNP
def seastar_gcn_fwd(g, T_all, F, ld, dst_norm, bias, act, alpha, H0_loc, Y_loc, out_scale=None, Ys_loc=None,
                    stream=None, edge_drop=None) -> None:
    _call("seastar_gcn_fwd", g, _dptr(T_all, "T_all"), F, ld, _dptr(dst_norm, "dst_norm"), _dptr(bias, "bias"),
          _act(act), float(alpha), _dptr(H0_loc, "H0"), _dptr(Y_loc, "Y"), _dptr(out_scale, "out_scale"),
          _dptr(Ys_loc, "Ys"), _spec(edge_drop), _stream(stream))


def seastar_gcn_bwd(g, dP_all, F, ld, src_norm, scale, Yact_loc, act, post_scale, dA_loc, dP_loc,
                    stream=None, edge_drop=None) -> None:
    _call("seastar_gcn_bwd", g, _dptr(dP_all, "dP_all"), F, ld, _dptr(src_norm, "src_norm"), float(scale),
          _dptr(Yact_loc, "Yact"), _act(act), _dptr(post_scale, "post_scale"), _dptr(dA_loc, "dA"),
          _dptr(dP_loc, "dP"), _spec(edge_drop), _stream(stream))


def seastar_gcn_fwd_split(g, phase, T_loc, ldloc, T_all, F, ld, dst_norm, bias, act, alpha, H0_loc, Y_loc,
                          out_scale, Ys_loc, part, ldp, stream=None, edge_drop=None) -> None:
    _call("seastar_gcn_fwd_split", g, int(phase), _dptr(T_loc, "T_loc"), ldloc, _dptr(T_all, "T_all"), F, ld,
          _dptr(dst_norm, "dst_norm"), _dptr(bias, "bias"), _act(act), float(alpha), _dptr(H0_loc, "H0"),
          _dptr(Y_loc, "Y"), _dptr(out_scale, "out_scale"), _dptr(Ys_loc, "Ys"), _dptr(part, "part"), ldp,
          _spec(edge_drop), _stream(stream))


def seastar_gcn_bwd_split(g, phase, dP_loc_in, ldloc, dP_all, F, ld, src_norm, scale, Yact_loc, act, post_scale,
                          dA_loc, dP_loc, part, ldp, stream=None, edge_drop=None) -> None:
    _call("seastar_gcn_bwd_split", g, int(phase), _dptr(dP_loc_in, "dP_loc_in"), ldloc, _dptr(dP_all, "dP_all"), F,
          ld, _dptr(src_norm, "src_norm"), float(scale), _dptr(Yact_loc, "Yact"), _act(act),
          _dptr(post_scale, "post_scale"), _dptr(dA_loc, "dA"), _dptr(dP_loc, "dP"), _dptr(part, "part"), ldp,
          _spec(edge_drop), _stream(stream))


# ----------------------------------------------------------------------------------- GAT
def seastar_gat_attn_proj(T, M, H, F, ldt, a_l, a_r, el, er, stream=None) -> None:
    _call("seastar_gat_attn_proj", _dptr(T, "T"), M, H, F, ldt, _dptr(a_l, "a_l"), _dptr(a_r, "a_r"),
          _dptr(el, "el"), _dptr(er, "er"), _stream(stream))


class seastar_dropout_spec(ctypes.Structure):
    """NEXT-3 dropout descriptor (include/seastar.h): p, site, seed, device step counter (or NULL)."""
    _fields_ = [("p", ctypes.c_float), ("site", ctypes.c_uint32), ("seed", ctypes.c_uint64), ("step", ctypes.c_void_p)]


def dropout_spec(p, site, seed, step=None):
    """A seastar_dropout_spec (None when p == 0); step: a device int32 tensor (e.g. the Adam step counter)."""
    if not p:
        return None
    return seastar_dropout_spec(float(p), int(site), int(seed), _dptr(step, "step"))


def _spec(d):
    return ctypes.addressof(d) if d is not None else None


def seastar_gat_fwd(g, T_all, el_all, er_loc, H, F, ldt, slope, bias, act, A_loc, Y_loc, lse_loc, B_loc=None,
                    b_loc=None, stream=None, attn_drop=None) -> None:
    _call("seastar_gat_fwd", g, _dptr(T_all, "T"), _dptr(el_all, "el"), _dptr(er_loc, "er"), H, F, ldt,
          float(slope), _dptr(bias, "bias"), _act(act), _dptr(A_loc, "A"), _dptr(Y_loc, "Y"), _dptr(lse_loc, "lse"),
          _dptr(B_loc, "B"), _dptr(b_loc, "b"), _spec(attn_drop), _stream(stream))


def seastar_gat_record_ld(H, F) -> int:
    return int(load().seastar_gat_record_ld(H, F))


def seastar_gat_bwd_prep(g, dY_loc, Y_loc, act, A_loc, er_loc, lse_loc, H, F, ldt, D_loc, B_loc=None, b_loc=None,
                         der_loc=None, stream=None) -> None:
    _call("seastar_gat_bwd_prep", g, _dptr(dY_loc, "dY"), _dptr(Y_loc, "Y"), _act(act), _dptr(A_loc, "A"),
          _dptr(er_loc, "er"), _dptr(lse_loc, "lse"), H, F, ldt, _dptr(D_loc, "D"), _dptr(B_loc, "B"),
          _dptr(b_loc, "b"), _dptr(der_loc, "der"), _stream(stream))


def seastar_gat_bwd(g, T_loc, el_loc, D_all, H, F, ldt, slope, dT_loc, del_loc, stream=None, attn_drop=None) -> None:
    _call("seastar_gat_bwd", g, _dptr(T_loc, "T"), _dptr(el_loc, "el"), _dptr(D_all, "D"), H, F, ldt, float(slope),
          _dptr(dT_loc, "dT"), _dptr(del_loc, "del"), _spec(attn_drop), _stream(stream))


def seastar_gat_der(g, T_all, el_all, D_loc, H, F, ldt, slope, der_loc, stream=None, attn_drop=None) -> None:
    _call("seastar_gat_der", g, _dptr(T_all, "T"), _dptr(el_all, "el"), _dptr(D_loc, "D"), H, F, ldt, float(slope),
          _dptr(der_loc, "der"), _spec(attn_drop), _stream(stream))


def seastar_gat_attn_proj_bwd_workspace(M, H, F) -> int:
    return int(load().seastar_gat_attn_proj_bwd_workspace(M, H, F))


def seastar_gat_attn_proj_bwd(T, M, H, F, ldt, a_l, a_r, del_, der, dT, da_l, da_r, workspace, ws_bytes,
                              stream=None) -> None:
    _call("seastar_gat_attn_proj_bwd", _dptr(T, "T"), M, H, F, ldt, _dptr(a_l, "a_l"), _dptr(a_r, "a_r"),
          _dptr(del_, "del"), _dptr(der, "der"), _dptr(dT, "dT"), _dptr(da_l, "da_l"), _dptr(da_r, "da_r"),
          _dptr(workspace, "workspace"), ws_bytes, _stream(stream))


# ----------------------------------------------------------------------------------- R-GCN
def seastar_rgcn_fwd_workspace(g, F_in, F_out) -> int:
    return int(load().seastar_rgcn_fwd_workspace(g, F_in, F_out))


def seastar_rgcn_fwd(g, X_all, F_in, ldx, W, F_out, norm_user, bias, act, Y_loc, ldy, workspace=None, ws_bytes=None,
                     stream=None) -> None:
    """workspace=None: a device buffer of seastar_rgcn_fwd_workspace() bytes is allocated here (memory plumbing
    only; the models pass their own)."""
    if workspace is None:
        need = seastar_rgcn_fwd_workspace(g, F_in, F_out)
        if need:
            import torch
            workspace = torch.empty(need, dtype=torch.uint8, device=Y_loc.device)
    if ws_bytes is None:
        ws_bytes = 0 if workspace is None else workspace.numel() * workspace.element_size()
    _call("seastar_rgcn_fwd", g, _dptr(X_all, "X"), F_in, ldx, _dptr(W, "W"), F_out, _dptr(norm_user, "norm"),
          _dptr(bias, "bias"), _act(act), _dptr(Y_loc, "Y"), ldy, _dptr(workspace, "workspace"), ws_bytes,
          _stream(stream))


def seastar_rgcn_bwd_workspace(g, F_in, F_out) -> int:
    return int(load().seastar_rgcn_bwd_workspace(g, F_in, F_out))


def seastar_rgcn_bwd(g, X_all, F_in, ldx, dA_all, F_out, ldd, W, norm_user, Yact_loc, act, dX_loc, dW, workspace,
                     ws_bytes, stream=None) -> None:
    _call("seastar_rgcn_bwd", g, _dptr(X_all, "X"), F_in, ldx, _dptr(dA_all, "dA"), F_out, ldd, _dptr(W, "W"),
          _dptr(norm_user, "norm"), _dptr(Yact_loc, "Yact"), _act(act), _dptr(dX_loc, "dX"), _dptr(dW, "dW"),
          _dptr(workspace, "workspace"), ws_bytes, _stream(stream))


# ----------------------------------------------------------------------------------- R-GCN, featureless + bases (NEXT-2)
def seastar_rgcn_basis_fwd(g, V_all, B, F, ldv, a, norm_user, loop_loc, ldl, bias, act, Y_loc, ldy,
                           stream=None) -> None:
    _call("seastar_rgcn_basis_fwd", g, _dptr(V_all, "V"), B, F, ldv, _dptr(a, "a"), _dptr(norm_user, "norm"),
          _dptr(loop_loc, "loop"), ldl, _dptr(bias, "bias"), _act(act), _dptr(Y_loc, "Y"), ldy, _stream(stream))


def seastar_rgcn_basis_bwd_workspace(g, B) -> int:
    return int(load().seastar_rgcn_basis_bwd_workspace(g, B))


def seastar_rgcn_basis_bwd(g, V_all, B, F, ldv, a, norm_user, dA_all, ldd, dV_loc, da, workspace, ws_bytes,
                           stream=None) -> None:
    _call("seastar_rgcn_basis_bwd", g, _dptr(V_all, "V"), B, F, ldv, _dptr(a, "a"), _dptr(norm_user, "norm"),
          _dptr(dA_all, "dA"), ldd, _dptr(dV_loc, "dV"), _dptr(da, "da"), _dptr(workspace, "workspace"), ws_bytes,
          _stream(stream))


def seastar_basis_combine(a, Vb, R, B, K, W, stream=None) -> None:
    _call("seastar_basis_combine", _dptr(a, "a"), _dptr(Vb, "Vb"), R, B, K, _dptr(W, "W"), _stream(stream))


def seastar_basis_combine_bwd(a, Vb, dW, R, B, K, da, dVb, stream=None) -> None:
    _call("seastar_basis_combine_bwd", _dptr(a, "a"), _dptr(Vb, "Vb"), _dptr(dW, "dW"), R, B, K, _dptr(da, "da"),
          _dptr(dVb, "dVb"), _stream(stream))


# ----------------------------------------------------------------------------------- dropout (NEXT-3)
def seastar_dropout(X, M, F, ldx, row0, p, seed, site, step, Y, ldy, stream=None) -> None:
    _call("seastar_dropout", _dptr(X, "X"), M, F, ldx, row0, p, seed, site, _dptr(step, "step"), _dptr(Y, "Y"), ldy,
          _stream(stream))


# ----------------------------------------------------------------------------------- glue
def seastar_softmax_xent_workspace(M) -> int:
    return int(load().seastar_softmax_xent_workspace(M))


def seastar_softmax_xent(Z, M, n_total, C, ldz, labels, loss, dZ, lddz, workspace, ws_bytes, stream=None) -> None:
    _call("seastar_softmax_xent", _dptr(Z, "Z"), M, n_total, C, ldz, _dptr(labels, "labels"), _dptr(loss, "loss"),
          _dptr(dZ, "dZ"), lddz, _dptr(workspace, "workspace"), ws_bytes, _stream(stream))


def seastar_colsum_workspace(M, F) -> int:
    return int(load().seastar_colsum_workspace(M, F))


def seastar_colsum(X, M, F, ld, out, workspace, ws_bytes, stream=None) -> None:
    _call("seastar_colsum", _dptr(X, "X"), M, F, ld, _dptr(out, "out"), _dptr(workspace, "workspace"), ws_bytes,
          _stream(stream))


def seastar_row_scale(X, M, F, ldx, scale, Y, ldy, stream=None) -> None:
    _call("seastar_row_scale", _dptr(X, "X"), M, F, ldx, _dptr(scale, "scale"), _dptr(Y, "Y"), ldy, _stream(stream))


def seastar_axpby(n, a, x, b, y, stream=None) -> None:
    _call("seastar_axpby", n, float(a), _dptr(x, "x"), float(b), _dptr(y, "y"), _stream(stream))


def seastar_adam(param, grad, m, v, n, lr, beta1, beta2, eps, step, stream=None) -> None:
    _call("seastar_adam", _dptr(param, "param"), _dptr(grad, "grad"), _dptr(m, "m"), _dptr(v, "v"), n, float(lr),
          float(beta1), float(beta2), float(eps), _dptr(step, "step"), _stream(stream))


def seastar_step_inc(counter, stream=None) -> None:
    _call("seastar_step_inc", _dptr(counter, "counter"), _stream(stream))
