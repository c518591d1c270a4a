"""Whole training epochs of the paper's models, every step in libseastar.so kernels.

PAPER.md §7 (L477-L481) trains GCN [37], GAT [58], APPNP [38] and R-GCN [53] with DGL's default
configurations.  Each class below owns its buffers (allocated once, so an epoch launches kernels
only -- capturable in a CUDA graph) and exposes ``epoch()`` = forward + softmax cross-entropy +
backward + Adam, all through the C ABI.  PyTorch only allocates memory and, when the graph is
row-partitioned over several GPUs, moves rows between ranks with NCCL collectives
(``torch.distributed``): all-gather of the per-layer source rows, all-gather of the packed
backward records, reduce-scatter of GAT's partial ``der``, and one all-reduce of the flat gradient
buffer.

Readings of the paper used here: dropout p = 0; ReLU hidden / identity output for
GCN; ELU hidden (heads concatenated) / 1-head identity output for GAT; LeakyReLU slope 0.2; bias
inside the activation; DGL "both" degree normalisation for GCN, in-degree^-1/2 for APPNP.
"""
from __future__ import annotations

import numpy as np
import torch

from . import _lib as L
from .graph import Graph


def _ld(F: int) -> int:
    return (F + 3) // 4 * 4


def _local_rows(m) -> int:
    """Rows of the per-rank buffers: the owned rows on one GPU; ceil(N/P) when partitioned, so every
    rank contributes an equal chunk to the all-gathers (rows past n_loc are never written)."""
    if m.comm.world == 1:
        return m.n
    assert m.rows_all % m.comm.world == 0 and m.rows_all // m.comm.world >= m.n
    return m.rows_all // m.comm.world


class Comm:
    """Row-partition plumbing.  P = 1: every gather is the identity (no copies).

    The collectives are NCCL's (``torch.distributed`` with the nccl backend).  When the process group
    is gloo (``staged=True``; used to run the partitioned path with several ranks on ONE GPU, e.g. on a
    single-GPU test box) the same calls are staged through host memory with identical shapes."""

    def __init__(self, world: int = 1, rank: int = 0, group=None, staged: bool | None = None):
        self.world, self.rank, self.group = world, rank, group
        if staged is None:
            staged = world > 1 and torch.distributed.get_backend(group) == "gloo"
        self.staged = staged

    @staticmethod
    def _rows(t: torch.Tensor) -> torch.Tensor:
        """A column slice [:, :F] of a row-padded buffer -> the full padded rows (same storage)."""
        if t.is_contiguous():
            return t
        assert t.dim() == 2 and t.stride(1) == 1, "gathered tables are row-major"
        return torch.as_strided(t, (t.shape[0], t.stride(0)), (t.stride(0), 1))

    def all_gather(self, out_all: torch.Tensor, loc: torch.Tensor):
        if self.world == 1:
            return loc
        loc = self._rows(loc)
        assert out_all.is_contiguous() and out_all.numel() == loc.numel() * self.world, (out_all.shape, loc.shape)
        if self.staged:
            parts = [torch.empty(loc.shape, dtype=loc.dtype) for _ in range(self.world)]
            torch.distributed.all_gather(parts, loc.cpu(), group=self.group)
            out_all.view(self.world, *loc.shape).copy_(torch.stack(parts))
        else:
            torch.distributed.all_gather_into_tensor(out_all, loc, group=self.group)
        return out_all

    class _Done:
        def wait(self):
            return None

    def all_gather_async(self, out_all: torch.Tensor, loc: torch.Tensor):
        """NEXT-1: start the all-gather and return a handle whose wait() makes the current stream wait for it; the
        caller launches the owned-neighbour phase of the aggregation in between (NCCL runs on its own stream).
        The staged gloo path is synchronous (the handle is already complete)."""
        if self.world == 1 or self.staged:
            self.all_gather(out_all, loc)
            return Comm._Done()
        loc = self._rows(loc)
        assert out_all.is_contiguous() and out_all.numel() == loc.numel() * self.world, (out_all.shape, loc.shape)
        return torch.distributed.all_gather_into_tensor(out_all, loc, group=self.group, async_op=True)

    def all_reduce(self, flat: torch.Tensor):
        if self.world > 1:
            if self.staged:
                h = flat.cpu()
                torch.distributed.all_reduce(h, group=self.group)
                flat.copy_(h)
            else:
                torch.distributed.all_reduce(flat, group=self.group)


class _Params:
    """One flat fp32 buffer for parameters, gradients and Adam moments (one all-reduce, one Adam launch)."""

    def __init__(self, shapes: dict, init: dict, device):
        self.offsets = {}
        n = 0
        for k, s in shapes.items():
            self.offsets[k] = (n, s)
            n += int(np.prod(s))
        self.n = n
        self.flat = torch.zeros(n, device=device)
        self.grad = torch.zeros(n, device=device)
        self.m = torch.zeros(n, device=device)
        self.v = torch.zeros(n, device=device)
        self.step = torch.zeros(1, dtype=torch.int32, device=device)
        for k, a in init.items():
            self.p(k).copy_(torch.from_numpy(np.ascontiguousarray(a, np.float32)).reshape(self.offsets[k][1]))

    def _view(self, buf, k):
        o, s = self.offsets[k]
        return buf[o:o + int(np.prod(s))].view(*s)

    def p(self, k):
        return self._view(self.flat, k)

    def g(self, k):
        return self._view(self.grad, k)

    def adam(self, lr, b1=0.9, b2=0.999, eps=1e-8):
        L.seastar_step_inc(self.step)
        L.seastar_adam(self.flat, self.grad, self.m, self.v, self.n, lr, b1, b2, eps, self.step)


def _linear(ws, X, M, K, ldx, W, N, bias, row_scale, act, Y, ldy):
    """seastar_linear_fwd with its workspace (tensor-core path: W is split into tf32 hi/lo tiles there)."""
    buf = ws.need(L.seastar_linear_fwd_workspace(K, N))
    L.seastar_linear_fwd(X, M, K, ldx, W, N, bias, row_scale, act, Y, ldy, buf, buf.numel())


class _Ws:
    """Grow-only byte workspace shared by the deterministic reductions."""

    def __init__(self, device):
        self.device = device
        self.buf = torch.empty(256, dtype=torch.uint8, device=device)

    def need(self, nbytes: int) -> torch.Tensor:
        if nbytes > self.buf.numel():
            self.buf = torch.empty(nbytes, dtype=torch.uint8, device=self.device)
        return self.buf


class GCN2:
    """2-layer GCN (Fig. 1 / Fig. 3): F_in -> hidden (ReLU) -> C (identity), softmax-xent.

    Layer 1 transforms first (F_in > hidden), layer 2 aggregates first (hidden < C)
    (reading #20).  The src-side norm is folded into the producing kernel's epilogue, the dst-side
    norm, bias and activation into the aggregation's epilogue, and the activation derivative and
    next-layer norm into the backward aggregation's epilogue."""

    def __init__(self, g: Graph, X_loc: torch.Tensor, labels_loc: torch.Tensor, params: dict, lr=0.01,
                 comm: Comm | None = None, n_pad_rows: int | None = None, dropout: float = 0.0, seed: int = 0,
                 overlap: bool | None = None):
        self.g, self.X, self.lab, self.lr = g, X_loc, labels_loc, lr
        self.drop_p, self.drop_seed = float(dropout), int(seed)     # NEXT-3: dropout on the hidden layer (DGL: 0.5)
        self.comm = comm or Comm()
        dev = X_loc.device
        self.n = g.n_loc
        self.N = g.N
        self.rows_all = n_pad_rows if n_pad_rows is not None else g.N      # all-gather height (P * n_per)
        self.Fin = X_loc.shape[1]
        self.H = params["W1"].shape[1]
        self.C = params["W2"].shape[1]
        self.P = _Params({"W1": params["W1"].shape, "b1": (self.H,), "W2": params["W2"].shape, "b2": (self.C,)},
                         params, dev)
        self.src_n, self.dst_n = g.degree_norms("both")
        H, C, n = self.H, self.C, _local_rows(self)
        e = lambda r, c: torch.zeros((r, c), device=dev)
        self.T1 = e(n, H)          # src_norm * (X W1), local rows
        self.H1 = e(n, H)          # relu(dst_norm * sum T1 + b1)
        self.H1s = e(n, H)         # src_norm * H1 (layer-2 table)
        self.P2 = e(n, H)          # dst_norm * sum H1s
        self.ldc = _ld(C)
        self.logits = e(n, self.ldc)
        self.dlogits = e(n, self.ldc)
        self.dP2 = e(n, H)         # dst_norm * (dlogits W2^T)
        self.dA1 = e(n, H)
        self.dP1 = e(n, H)
        self.dT1 = e(n, H)
        self.loss = torch.zeros(1, device=dev)
        self.ws = _Ws(dev)
        P = self.comm.world
        self.T1_all = e(self.rows_all, H) if P > 1 else None
        self.H1s_all = e(self.rows_all, H) if P > 1 else None
        self.dP2_all = e(self.rows_all, H) if P > 1 else None
        self.dP1_all = e(self.rows_all, H) if P > 1 else None
        # NEXT-1: partitioned aggregations in two phases around each all-gather (owned-neighbour edges first)
        self.overlap = (P > 1) if overlap is None else (bool(overlap) and P > 1)
        self.part = e(n, H) if self.overlap else None
        self.timer = None

    def _agg_fwd(self, loc, tab_all_buf, dst_norm, bias, act, out, out_scale=None, outs=None):
        """forward aggregation of the gathered `loc` rows (one phase, or NEXT-1's two phases around the gather)"""
        g, H = self.g, self.H
        if not self.overlap:
            tab = self.comm.all_gather(tab_all_buf, loc)
            L.seastar_gcn_fwd(g.handle, tab, H, H, dst_norm, bias, act, 0.0, None, out, out_scale, outs)
            return
        h = self.comm.all_gather_async(tab_all_buf, loc)
        L.seastar_gcn_fwd_split(g.handle, 1, loc, H, None, H, H, None, None, "none", 0.0, None, None, None, None,
                                self.part, H)
        h.wait()
        L.seastar_gcn_fwd_split(g.handle, 2, None, 0, tab_all_buf, H, H, dst_norm, bias, act, 0.0, None, out,
                                out_scale, outs, self.part, H)

    def _agg_bwd(self, loc, tab_all_buf, Yact, act, post_scale, dA, dP):
        g, H = self.g, self.H
        if not self.overlap:
            tab = self.comm.all_gather(tab_all_buf, loc)
            L.seastar_gcn_bwd(g.handle, tab, H, H, self.src_n, 1.0, Yact, act, post_scale, dA, dP)
            return
        h = self.comm.all_gather_async(tab_all_buf, loc)
        L.seastar_gcn_bwd_split(g.handle, 1, loc, H, None, H, H, None, 1.0, None, "none", None, None, None,
                                self.part, H)
        h.wait()
        L.seastar_gcn_bwd_split(g.handle, 2, None, 0, tab_all_buf, H, H, self.src_n, 1.0, Yact, act, post_scale, dA,
                                dP, self.part, H)

    def _t(self, name):
        if self.timer is not None:
            self.timer(name)

    def forward(self):
        g, p, H, C, n = self.g, self.P, self.H, self.C, self.n
        _linear(self.ws, self.X, n, self.Fin, self.X.stride(0), p.p("W1"), H, None, self.src_n, "none",
                             self.T1, H)
        self._t("gcn_fwd1")
        self._agg_fwd(self.T1, self.T1_all, self.dst_n, p.p("b1"), "relu", self.H1, self.src_n, self.H1s)
        self._t("gcn_fwd1_end")
        if self.drop_p > 0:      # layer-2 input src_n * drop(H1): the mask commutes with the row scale
            L.seastar_dropout(self.H1s, n, H, H, g.row_begin, self.drop_p, self.drop_seed, 1, p.step, self.H1s, H)
        self._agg_fwd(self.H1s, self.H1s_all, self.dst_n, None, "none", self.P2)
        _linear(self.ws, self.P2, n, H, H, p.p("W2"), C, p.p("b2"), None, "none", self.logits, self.ldc)
        ws = self.ws.need(L.seastar_softmax_xent_workspace(n))
        L.seastar_softmax_xent(self.logits, n, self.g.N, C, self.ldc, self.lab, self.loss, self.dlogits, self.ldc,
                               ws, ws.numel())
        return self.loss

    def backward(self):
        g, p, H, C, n = self.g, self.P, self.H, self.C, self.n
        ws = self.ws.need(max(L.seastar_linear_bwd_weight_workspace(n, H, C),
                              L.seastar_linear_bwd_weight_workspace(n, self.Fin, H),
                              L.seastar_colsum_workspace(n, H)))
        L.seastar_linear_bwd_weight(self.P2, n, H, H, self.dlogits, C, self.ldc, p.g("W2"), p.g("b2"), ws,
                                    ws.numel())
        L.seastar_linear_bwd_data(self.dlogits, n, C, self.ldc, p.p("W2"), H, self.dst_n, None, "none", self.dP2, H)
        self._t("gcn_bwd2")
        self._agg_bwd(self.dP2, self.dP2_all, self.H1, "relu", self.dst_n, self.dA1, self.dP1)
        self._t("gcn_bwd2_end")
        if self.drop_p > 0:      # d drop(H1) -> dH1: the same mask, commuting with relu' and the dst_n scale
            for t in (self.dA1, self.dP1):
                L.seastar_dropout(t, n, H, H, g.row_begin, self.drop_p, self.drop_seed, 1, p.step, t, H)
        L.seastar_colsum(self.dA1, n, H, H, p.g("b1"), ws, ws.numel())
        self._agg_bwd(self.dP1, self.dP1_all, None, "none", None, self.dT1, None)
        L.seastar_linear_bwd_weight(self.X, n, self.Fin, self.X.stride(0), self.dT1, H, H, p.g("W1"), None, ws,
                                    ws.numel())
        self.comm.all_reduce(self.P.grad)

    def epoch(self):
        loss = self.forward()
        self.backward()
        self.P.adam(self.lr)
        return loss


class GAT2:
    """2-layer GAT (Fig. 2 / Fig. 3): F_in -> heads x hidden (ELU, concat) -> 1 x C, softmax-xent.
    LeakyReLU slope 0.2, attention vectors a_l (source) / a_r (destination) per head.

    save_der_factors=True (default): the forward also writes B_v, b_v so the backward row pass emits der
    directly (one edge pass per layer backward instead of two); False uses the dst-major
    seastar_gat_der pass instead (less memory)."""

    def __init__(self, g: Graph, X_loc: torch.Tensor, labels_loc: torch.Tensor, params: dict, heads: int,
                 hidden: int, lr=0.005, slope=0.2, comm: Comm | None = None, n_pad_rows: int | None = None,
                 save_der_factors: bool = True, dropout: float = 0.0, seed: int = 0, attn_dropout: float = 0.0):
        self.g, self.X, self.lab, self.lr, self.slope = g, X_loc, labels_loc, lr, slope
        self.drop_p, self.drop_seed = float(dropout), int(seed)     # NEXT-3: feat_drop on both layer inputs
        self.save_B = save_der_factors
        self.comm = comm or Comm()
        dev = X_loc.device
        self.n, self.N = g.n_loc, g.N
        self.rows_all = n_pad_rows if n_pad_rows is not None else g.N
        self.Fin = X_loc.shape[1]
        self.H1, self.F1 = heads, hidden
        self.W1w = heads * hidden
        self.C = params["W2"].shape[1]
        shapes = {"W1": (self.Fin, self.W1w), "al1": (heads, hidden), "ar1": (heads, hidden), "b1": (self.W1w,),
                  "W2": (self.W1w, self.C), "al2": (1, self.C), "ar2": (1, self.C), "b2": (self.C,)}
        self.P = _Params(shapes, params, dev)
        # NEXT-3 attn_drop (sites 3 / 4, by user edge id and head; the generic chunked GAT kernels run)
        self.ad = {"1": L.dropout_spec(attn_dropout, 3, seed, self.P.step),
                   "2": L.dropout_spec(attn_dropout, 4, seed, self.P.step)}
        n, W1w, C = _local_rows(self), self.W1w, self.C
        # layer 2 (one head): el2 lives in T2's first padding column (seastar_gat_fwd: el_all == T_all + H*F) and the
        # row stride is a whole number of 32-byte sectors, so a gathered T2 row brings its el2 along -- 6 sectors per
        # edge on Reddit (C = 41, ld 48) instead of 6.5 + 1 for a separate el table
        self.ld1, self.ld2 = _ld(W1w), (C + 1 + 7) // 8 * 8
        e = lambda r, c: torch.zeros((r, c), device=dev)
        self.T1, self.A1, self.Y1 = e(n, self.ld1), e(n, self.ld1), e(n, self.ld1)
        self.el1, self.er1, self.lse1 = e(n, heads), e(n, heads), e(n, heads)
        self.T2, self.A2, self.Y2 = e(n, self.ld2), e(n, self.ld2), e(n, self.ld2)
        self.el2 = self.T2[:, C:C + 1]
        self.er2, self.lse2 = e(n, 1), e(n, 1)
        self.dY2 = e(n, self.ld2)
        self.ldd1, self.ldd2 = L.seastar_gat_record_ld(heads, hidden), L.seastar_gat_record_ld(1, C)
        self.D1, self.D2 = e(n, self.ldd1), e(n, self.ldd2)
        self.dT1, self.dT2 = e(n, self.ld1), e(n, self.ld2)
        self.del1, self.del2 = e(n, heads), e(n, 1)
        self.der1, self.der2 = e(n, heads), e(n, 1)
        self.dY1 = e(n, self.ld1)
        if self.drop_p > 0:      # dropped layer inputs (kept for the weight gradients)
            self.Xd = e(n, X_loc.stride(0))[:, :self.Fin]
            self.Y1d = e(n, self.ld1)
        else:
            self.Xd, self.Y1d = X_loc, self.Y1
        self.B1, self.bs1 = (e(n, self.ld1), e(n, heads)) if self.save_B else (None, None)
        self.B2, self.bs2 = (e(n, self.ld2), e(n, 1)) if self.save_B else (None, None)
        self.loss = torch.zeros(1, device=dev)
        self.ws = _Ws(dev)
        P = self.comm.world
        R = self.rows_all
        self.T1_all = e(R, self.ld1) if P > 1 else None
        self.el1_all = e(R, heads) if P > 1 else None
        self.T2_all = e(R, self.ld2) if P > 1 else None
        self.el2_all = None                                   # packed into T2_all's rows
        self.D1_all = e(R, self.ldd1) if P > 1 else None
        self.D2_all = e(R, self.ldd2) if P > 1 else None
        self.timer = None

    def _t(self, name):
        if self.timer is not None:
            self.timer(name)

    def forward(self):
        g, p, n = self.g, self.P, self.n
        H, F, W, C = self.H1, self.F1, self.W1w, self.C
        if self.drop_p > 0:
            L.seastar_dropout(self.X, n, self.Fin, self.X.stride(0), g.row_begin, self.drop_p, self.drop_seed, 1,
                              p.step, self.Xd, self.Xd.stride(0))
        _linear(self.ws, self.Xd, n, self.Fin, self.Xd.stride(0), p.p("W1"), W, None, None, "none", self.T1,
                             self.ld1)
        L.seastar_gat_attn_proj(self.T1, n, H, F, self.ld1, p.p("al1"), p.p("ar1"), self.el1, self.er1)
        T1_all = self.comm.all_gather(self.T1_all, self.T1)
        el1_all = self.comm.all_gather(self.el1_all, self.el1)
        self._gathered1 = (T1_all, el1_all)
        self._t("gat_fwd1")
        L.seastar_gat_fwd(g.handle, T1_all, el1_all, self.er1, H, F, self.ld1, self.slope, p.p("b1"), "elu", self.A1,
                          self.Y1, self.lse1, self.B1, self.bs1, attn_drop=self.ad["1"])
        self._t("gat_fwd1_end")
        if self.drop_p > 0:
            L.seastar_dropout(self.Y1, n, W, self.ld1, g.row_begin, self.drop_p, self.drop_seed, 2, p.step, self.Y1d,
                              self.ld1)
        _linear(self.ws, self.Y1d, n, W, self.ld1, p.p("W2"), C, None, None, "none", self.T2, self.ld2)
        L.seastar_gat_attn_proj(self.T2, n, 1, C, self.ld2, p.p("al2"), p.p("ar2"), self.el2, self.er2)
        T2_all = self.comm.all_gather(self.T2_all, self.T2)
        el2_all = T2_all[:, C:C + 1]                          # el2 travels inside the gathered T2 rows
        self._gathered2 = (T2_all, el2_all)
        self._t("gat_fwd2")
        L.seastar_gat_fwd(g.handle, T2_all, el2_all, self.er2, 1, C, self.ld2, self.slope, p.p("b2"), "none", self.A2,
                          self.Y2, self.lse2, self.B2, self.bs2, attn_drop=self.ad["2"])
        self._t("gat_fwd2_end")
        ws = self.ws.need(L.seastar_softmax_xent_workspace(n))
        L.seastar_softmax_xent(self.Y2, n, self.g.N, C, self.ld2, self.lab, self.loss, self.dY2, self.ld2, ws,
                               ws.numel())
        return self.loss

    def _layer_bwd(self, T, T_loc_ld, el, er, A, Y, lse, dY, act, H, F, D, D_all_buf, dT, del_, der, gathered,
                   al, ar, dal, dar, db, tag, B, bs):
        g, n = self.g, self.n
        L.seastar_gat_bwd_prep(g.handle, dY, Y, act, A, er, lse, H, F, T_loc_ld, D, B, bs, der if B is not None else None)
        ldd = L.seastar_gat_record_ld(H, F)
        ws = self.ws.need(max(L.seastar_colsum_workspace(n, H * F), L.seastar_gat_attn_proj_bwd_workspace(n, H, F)))
        L.seastar_colsum(D, n, H * F, ldd, db, ws, ws.numel())       # db = sum_v dA[v] (dA = first H*F columns)
        D_all = self.comm.all_gather(D_all_buf, D)
        self._t(f"gat_bwd{tag}")
        L.seastar_gat_bwd(g.handle, T, el, D_all, H, F, T_loc_ld, self.slope, dT, del_, attn_drop=self.ad[tag])
        self._t(f"gat_bwd{tag}_end")
        if B is None:
            self._t(f"gat_der{tag}")
            L.seastar_gat_der(g.handle, gathered[0], gathered[1], D, H, F, T_loc_ld, self.slope, der,
                              attn_drop=self.ad[tag])
            self._t(f"gat_der{tag}_end")
        L.seastar_gat_attn_proj_bwd(T, n, H, F, T_loc_ld, al, ar, del_, der, dT, dal, dar, ws, ws.numel())

    def backward(self):
        p, n = self.P, self.n
        H, F, W, C = self.H1, self.F1, self.W1w, self.C
        self._layer_bwd(self.T2, self.ld2, self.el2, self.er2, self.A2, self.Y2, self.lse2, self.dY2, "none", 1, C,
                        self.D2, self.D2_all, self.dT2, self.del2, self.der2, self._gathered2, p.p("al2"),
                        p.p("ar2"), p.g("al2"), p.g("ar2"), p.g("b2"), "2", self.B2, self.bs2)
        ws = self.ws.need(max(L.seastar_linear_bwd_weight_workspace(n, W, C),
                              L.seastar_linear_bwd_weight_workspace(n, self.Fin, W)))
        L.seastar_linear_bwd_weight(self.Y1d, n, W, self.ld1, self.dT2, C, self.ld2, p.g("W2"), None, ws, ws.numel())
        L.seastar_linear_bwd_data(self.dT2, n, C, self.ld2, p.p("W2"), W, None, None, "none", self.dY1, self.ld1)
        if self.drop_p > 0:
            L.seastar_dropout(self.dY1, n, W, self.ld1, self.g.row_begin, self.drop_p, self.drop_seed, 2, p.step,
                              self.dY1, self.ld1)
        self._layer_bwd(self.T1, self.ld1, self.el1, self.er1, self.A1, self.Y1, self.lse1, self.dY1, "elu", H, F,
                        self.D1, self.D1_all, self.dT1, self.del1, self.der1, self._gathered1, p.p("al1"),
                        p.p("ar1"), p.g("al1"), p.g("ar1"), p.g("b1"), "1", self.B1, self.bs1)
        ws = self.ws.need(L.seastar_linear_bwd_weight_workspace(n, self.Fin, W))
        L.seastar_linear_bwd_weight(self.Xd, n, self.Fin, self.Xd.stride(0), self.dT1, W, self.ld1, p.g("W1"), None,
                                    ws, ws.numel())
        self.comm.all_reduce(self.P.grad)

    def epoch(self):
        loss = self.forward()
        self.backward()
        self.P.adam(self.lr)
        return loss


class APPNPNet:
    """APPNP [38]: H0 = MLP(X) (Linear -> ReLU -> Linear), K steps Z <- (1-a) n A n Z + a H0, softmax-xent.
    Each propagation step is one fused gcn_fwd (APPNP epilogue, writes Z and n*Z for the next step)."""

    def __init__(self, g: Graph, X_loc, labels_loc, params: dict, K=10, alpha=0.1, lr=0.01, comm: Comm | None = None,
                 n_pad_rows: int | None = None, edge_dropout: float = 0.0, seed: int = 0, overlap: bool | None = None):
        self.g, self.X, self.lab, self.K, self.alpha, self.lr = g, X_loc, labels_loc, K, alpha, lr
        self.comm = comm or Comm()
        dev = X_loc.device
        self.n = g.n_loc
        self.rows_all = n_pad_rows if n_pad_rows is not None else g.N
        self.Fin = X_loc.shape[1]
        self.Hd = params["W1"].shape[1]
        self.C = params["W2"].shape[1]
        self.P = _Params({"W1": params["W1"].shape, "b1": (self.Hd,), "W2": params["W2"].shape, "b2": (self.C,)},
                         params, dev)
        _, self.nrm = g.degree_norms("in")
        n, Hd, C = _local_rows(self), self.Hd, self.C
        self.ldc = _ld(C)
        e = lambda r, c: torch.zeros((r, c), device=dev)
        self.Hh = e(n, Hd)
        self.H0 = e(n, self.ldc)
        self.Z = [e(n, self.ldc) for _ in range(K + 1)]       # Z[0] aliases H0's values (copied by linear)
        self.Zs = [e(n, self.ldc) for _ in range(K + 1)]      # n * Z[k]
        self.G = e(n, self.ldc)
        self.Gs = [e(n, self.ldc), e(n, self.ldc)]
        self.Gtmp = e(n, self.ldc)
        self.dH0 = e(n, self.ldc)
        self.dHh = e(n, Hd)
        self.loss = torch.zeros(1, device=dev)
        self.ws = _Ws(dev)
        # NEXT-3 edge_drop (DGL APPNPConv): a fresh mask per propagation step k (site 16 + k, by user edge id)
        self.ed = [L.dropout_spec(edge_dropout, 16 + k, seed, self.P.step) for k in range(K)]
        P = self.comm.world
        self.Zs_all = e(self.rows_all, self.ldc) if P > 1 else None
        self.Gs_all = e(self.rows_all, self.ldc) if P > 1 else None
        # NEXT-1: each propagation step's aggregation in two phases around its all-gather (see GCN2)
        self.overlap = (P > 1) if overlap is None else (bool(overlap) and P > 1)
        self.part = e(n, self.ldc) if self.overlap else None
        self.timer = None

    def _t(self, name):
        if self.timer is not None:
            self.timer(name)

    def forward(self):
        g, p, n, Hd, C, ld = self.g, self.P, self.n, self.Hd, self.C, self.ldc
        _linear(self.ws, self.X, n, self.Fin, self.X.stride(0), p.p("W1"), Hd, p.p("b1"), None, "relu", self.Hh,
                             Hd)
        _linear(self.ws, self.Hh, n, Hd, Hd, p.p("W2"), C, p.p("b2"), None, "none", self.H0, ld)
        L.seastar_row_scale(self.H0, n, C, ld, self.nrm, self.Zs[0], ld)           # Z^0 = H0, pre-scaled by n
        for k in range(self.K):
            self._t("appnp_fwd") if k == 0 else None
            if self.overlap:
                h = self.comm.all_gather_async(self.Zs_all, self.Zs[k])
                L.seastar_gcn_fwd_split(g.handle, 1, self.Zs[k], ld, None, C, ld, None, None, "none", 0.0, None, None,
                                        None, None, self.part, ld, edge_drop=self.ed[k])
                h.wait()
                L.seastar_gcn_fwd_split(g.handle, 2, None, 0, self.Zs_all, C, ld, self.nrm, None, "none", self.alpha,
                                        self.H0, self.Z[k + 1], self.nrm, self.Zs[k + 1], self.part, ld,
                                        edge_drop=self.ed[k])
            else:
                Zs_all = self.comm.all_gather(self.Zs_all, self.Zs[k])
                L.seastar_gcn_fwd(g.handle, Zs_all, C, ld, self.nrm, None, "none", self.alpha, self.H0, self.Z[k + 1],
                                  self.nrm, self.Zs[k + 1], edge_drop=self.ed[k])
            self._t("appnp_fwd_end") if k == 0 else None
        out = self.Z[self.K] if self.K > 0 else self.H0
        ws = self.ws.need(L.seastar_softmax_xent_workspace(n))
        L.seastar_softmax_xent(out, n, self.g.N, C, ld, self.lab, self.loss, self.G, ld, ws, ws.numel())
        return self.loss

    def backward(self):
        g, p, n, Hd, C, ld, a = self.g, self.P, self.n, self.Hd, self.C, self.ldc, self.alpha
        # G = dL/dZ^K ; for k = K-1..0: dH0 += a G ; G <- (1-a) n sum_out n G
        self.dH0.zero_()
        if self.K > 0:
            L.seastar_row_scale(self.G, n, C, ld, self.nrm, self.Gs[0], ld)
        cur = 0
        G = self.G
        for k in range(self.K):
            L.seastar_axpby(n * ld, a, G, 1.0, self.dH0)
            nxt = self.Gtmp if G is self.G else self.G
            self._t("appnp_bwd") if k == 0 else None
            ed = self.ed[self.K - 1 - k]
            if self.overlap:
                h = self.comm.all_gather_async(self.Gs_all, self.Gs[cur])
                L.seastar_gcn_bwd_split(g.handle, 1, self.Gs[cur], ld, None, C, ld, None, 1.0, None, "none", None, None,
                                        None, self.part, ld, edge_drop=ed)
                h.wait()
                L.seastar_gcn_bwd_split(g.handle, 2, None, 0, self.Gs_all, C, ld, self.nrm, 1.0 - a, None, "none",
                                        self.nrm, nxt, self.Gs[1 - cur], self.part, ld, edge_drop=ed)
            else:
                Gs_all = self.comm.all_gather(self.Gs_all, self.Gs[cur])
                L.seastar_gcn_bwd(g.handle, Gs_all, C, ld, self.nrm, 1.0 - a, None, "none", self.nrm, nxt,
                                  self.Gs[1 - cur], edge_drop=ed)
            self._t("appnp_bwd_end") if k == 0 else None
            G = nxt
            cur = 1 - cur
        L.seastar_axpby(n * ld, 1.0, G, 1.0, self.dH0)
        ws = self.ws.need(max(L.seastar_linear_bwd_weight_workspace(n, Hd, C),
                              L.seastar_linear_bwd_weight_workspace(n, self.Fin, Hd)))
        L.seastar_linear_bwd_weight(self.Hh, n, Hd, Hd, self.dH0, C, ld, p.g("W2"), p.g("b2"), ws, ws.numel())
        L.seastar_linear_bwd_data(self.dH0, n, C, ld, p.p("W2"), Hd, None, self.Hh, "relu", self.dHh, Hd)
        L.seastar_linear_bwd_weight(self.X, n, self.Fin, self.X.stride(0), self.dHh, Hd, Hd, p.g("W1"), p.g("b1"), ws,
                                    ws.numel())
        self.comm.all_reduce(self.P.grad)

    def epoch(self):
        loss = self.forward()
        self.backward()
        self.P.adam(self.lr)
        return loss


class RGCN2:
    """2-layer R-GCN [53] (§6.3.5): F_in -> hidden (ReLU) -> C, one weight matrix per
    relation, normaliser 1/c_{v,r} (graph built with rgcn_norm=True), softmax-xent."""

    def __init__(self, g: Graph, X_loc, labels_loc, params: dict, lr=0.01, comm: Comm | None = None,
                 n_pad_rows: int | None = None):
        self.g, self.X, self.lab, self.lr = g, X_loc, labels_loc, lr
        self.comm = comm or Comm()
        dev = X_loc.device
        self.n = g.n_loc
        self.rows_all = n_pad_rows if n_pad_rows is not None else g.N
        R, self.Fin, self.Hd = params["W1"].shape
        self.C = params["W2"].shape[2]
        assert X_loc.stride(0) % 4 == 0, "R-GCN input rows need a leading dimension that is a multiple of 4"
        self.P = _Params({"W1": params["W1"].shape, "b1": (self.Hd,), "W2": params["W2"].shape, "b2": (self.C,)},
                         params, dev)
        n = _local_rows(self)
        if X_loc.shape[0] < n:      # the input rows are all-gathered too: pad this rank's chunk
            Xp = torch.zeros((n, X_loc.stride(0)), device=dev)
            Xp[:X_loc.shape[0], :X_loc.shape[1]] = X_loc
            self.X = Xp[:, :X_loc.shape[1]]
        self.ldh, self.ldc = _ld(self.Hd), _ld(self.C)
        e = lambda r, c: torch.zeros((r, c), device=dev)
        self.H1, self.dZ1 = e(n, self.ldh), e(n, self.ldh)
        self.logits, self.dlog = e(n, self.ldc), e(n, self.ldc)
        self.loss = torch.zeros(1, device=dev)
        self.ws = _Ws(dev)
        P, Ra = self.comm.world, self.rows_all
        self.X_all = e(Ra, X_loc.stride(0)) if P > 1 else None
        self.H1_all = e(Ra, self.ldh) if P > 1 else None
        self.dlog_all = e(Ra, self.ldc) if P > 1 else None
        self.dZ1_all = e(Ra, self.ldh) if P > 1 else None
        self.timer = None

    def _t(self, name):
        if self.timer is not None:
            self.timer(name)

    def forward(self):
        g, p, n = self.g, self.P, self.n
        ws = self.ws.need(max(L.seastar_rgcn_fwd_workspace(g.handle, self.Fin, self.Hd),
                              L.seastar_rgcn_fwd_workspace(g.handle, self.Hd, self.C), 256))
        self._X_all = self.comm.all_gather(self.X_all, self.X)
        self._t("rgcn_fwd1")
        L.seastar_rgcn_fwd(g.handle, self._X_all, self.Fin, self.X.stride(0), p.p("W1"), self.Hd, None, p.p("b1"),
                           "relu", self.H1, self.ldh, ws, ws.numel())
        self._t("rgcn_fwd1_end")
        self._H1_all = self.comm.all_gather(self.H1_all, self.H1)
        L.seastar_rgcn_fwd(g.handle, self._H1_all, self.Hd, self.ldh, p.p("W2"), self.C, None, p.p("b2"), "none",
                           self.logits, self.ldc, ws, ws.numel())
        ws = self.ws.need(L.seastar_softmax_xent_workspace(n))
        L.seastar_softmax_xent(self.logits, n, self.g.N, self.C, self.ldc, self.lab, self.loss, self.dlog, self.ldc,
                               ws, ws.numel())
        return self.loss

    def backward(self):
        g, p, n = self.g, self.P, self.n
        ws = self.ws.need(max(L.seastar_rgcn_bwd_workspace(g.handle, self.Hd, self.C),
                              L.seastar_rgcn_bwd_workspace(g.handle, self.Fin, self.Hd),
                              L.seastar_colsum_workspace(n, max(self.C, self.Hd))))
        L.seastar_colsum(self.dlog, n, self.C, self.ldc, p.g("b2"), ws, ws.numel())
        dlog_all = self.comm.all_gather(self.dlog_all, self.dlog)
        self._t("rgcn_bwd2")
        L.seastar_rgcn_bwd(g.handle, self._H1_all, self.Hd, self.ldh, dlog_all, self.C, self.ldc, p.p("W2"), None,
                           self.H1, "relu", self.dZ1, p.g("W2"), ws, ws.numel())
        self._t("rgcn_bwd2_end")
        L.seastar_colsum(self.dZ1, n, self.Hd, self.ldh, p.g("b1"), ws, ws.numel())
        dZ1_all = self.comm.all_gather(self.dZ1_all, self.dZ1)
        L.seastar_rgcn_bwd(g.handle, self._X_all, self.Fin, self.X.stride(0), dZ1_all, self.Hd, self.ldh, p.p("W1"),
                           None, None, "none", None, p.g("W1"), ws, ws.numel())
        self.comm.all_reduce(self.P.grad)

    def epoch(self):
        loss = self.forward()
        self.backward()
        self.P.adam(self.lr)
        return loss


class RGCNBasis2:
    """2-layer R-GCN as the paper trained it on aifb / mutag / bgs (Table 2, Table 3
    L1219-L1227; DGL's entity-classification defaults): a featureless input layer
    h_u W_r = sum_b a1[r,b] V1[u,b,:] (ReLU), a dense output layer W2_r = sum_b a2[r,b] V2[b] (identity),
    normaliser 1/c_{v,r}, no self-loop, softmax cross-entropy.  SURVEY.md §8(f) NEXT-2, reading #26.

    Parameters: V1 [N, B1, Hd] (row-partitioned like the vertices: each rank owns and updates the rows of
    its vertices, gathered for the forward; never all-reduced), a1 [R, B1], b1 [Hd], V2 [B2, Hd, C],
    a2 [R, B2], b2 [C] (replicated, one flat all-reduced buffer)."""

    def __init__(self, g: Graph, labels_loc, params: dict, lr=0.01, comm: Comm | None = None,
                 n_pad_rows: int | None = None):
        self.g, self.lab, self.lr = g, labels_loc, lr
        self.comm = comm or Comm()
        dev = labels_loc.device
        self.n = g.n_loc
        self.rows_all = n_pad_rows if n_pad_rows is not None else g.N
        self.R, self.B1 = params["a1"].shape
        self.B2, self.Hd, self.C = params["V2"].shape
        Vn = params["V1"]
        assert Vn.shape[1:] == (self.B1, self.Hd)
        n = _local_rows(self)
        self.ldv = self.B1 * self.Hd
        V1_loc = np.zeros((n, self.B1, self.Hd), np.float32)     # padded rows stay 0 (never read)
        if Vn.shape[0] == g.N:                                    # whole table given: take the owned rows
            Vn = Vn[g.row_begin:g.row_begin + self.n]
        assert Vn.shape[0] == self.n, "V1 must cover all N vertices or exactly the owned rows"
        V1_loc[:self.n] = Vn
        self.E = _Params({"V1": (n, self.ldv)}, {"V1": V1_loc.reshape(n, self.ldv)}, dev)
        shp = {"a1": params["a1"].shape, "b1": (self.Hd,), "V2": params["V2"].shape, "a2": params["a2"].shape,
               "b2": (self.C,)}
        self.P = _Params(shp, {k: params[k] for k in shp}, dev)
        self.ldh, self.ldc = _ld(self.Hd), _ld(self.C)
        e = lambda r, c: torch.zeros((r, c), device=dev)
        self.H1, self.dZ1 = e(n, self.ldh), e(n, self.ldh)
        self.logits, self.dlog = e(n, self.ldc), e(n, self.ldc)
        self.W2 = torch.zeros((self.R, self.Hd, self.C), device=dev)
        self.dW2 = torch.zeros_like(self.W2)
        self.loss = torch.zeros(1, device=dev)
        self.ws = _Ws(dev)
        P, Ra = self.comm.world, self.rows_all
        self.V1_all = e(Ra, self.ldv) if P > 1 else None
        self.H1_all = e(Ra, self.ldh) if P > 1 else None
        self.dlog_all = e(Ra, self.ldc) if P > 1 else None
        self.dZ1_all = e(Ra, self.ldh) if P > 1 else None
        self.timer = None

    def _t(self, name):
        if self.timer is not None:
            self.timer(name)

    def grad(self, k):
        return self.E.g(k)[:self.n].reshape(self.n, self.B1, self.Hd) if k == "V1" else self.P.g(k)

    def param(self, k):
        return self.E.p(k)[:self.n].reshape(self.n, self.B1, self.Hd) if k == "V1" else self.P.p(k)

    def forward(self):
        g, p, n = self.g, self.P, self.n
        self._V1_all = self.comm.all_gather(self.V1_all, self.E.p("V1"))
        self._t("rgcnb_fwd1")
        L.seastar_rgcn_basis_fwd(g.handle, self._V1_all, self.B1, self.Hd, self.ldv, p.p("a1"), None, None, 0,
                                 p.p("b1"), "relu", self.H1, self.ldh)
        self._t("rgcnb_fwd1_end")
        L.seastar_basis_combine(p.p("a2"), p.p("V2"), self.R, self.B2, self.Hd * self.C, self.W2)
        self._H1_all = self.comm.all_gather(self.H1_all, self.H1)
        ws = self.ws.need(max(L.seastar_rgcn_fwd_workspace(g.handle, self.Hd, self.C), 256))
        L.seastar_rgcn_fwd(g.handle, self._H1_all, self.Hd, self.ldh, self.W2, self.C, None, p.p("b2"), "none",
                           self.logits, self.ldc, ws, ws.numel())
        ws = self.ws.need(L.seastar_softmax_xent_workspace(n))
        L.seastar_softmax_xent(self.logits, n, self.g.N, self.C, self.ldc, self.lab, self.loss, self.dlog, self.ldc,
                               ws, ws.numel())
        return self.loss

    def backward(self):
        g, p, n = self.g, self.P, self.n
        ws = self.ws.need(max(L.seastar_rgcn_bwd_workspace(g.handle, self.Hd, self.C),
                              L.seastar_rgcn_basis_bwd_workspace(g.handle, self.B1),
                              L.seastar_colsum_workspace(n, max(self.C, self.Hd))))
        L.seastar_colsum(self.dlog, n, self.C, self.ldc, p.g("b2"), ws, ws.numel())
        dlog_all = self.comm.all_gather(self.dlog_all, self.dlog)
        L.seastar_rgcn_bwd(g.handle, self._H1_all, self.Hd, self.ldh, dlog_all, self.C, self.ldc, self.W2, None,
                           self.H1, "relu", self.dZ1, self.dW2, ws, ws.numel())
        L.seastar_basis_combine_bwd(p.p("a2"), p.p("V2"), self.dW2, self.R, self.B2, self.Hd * self.C, p.g("a2"),
                                    p.g("V2"))
        L.seastar_colsum(self.dZ1, n, self.Hd, self.ldh, p.g("b1"), ws, ws.numel())
        dZ1_all = self.comm.all_gather(self.dZ1_all, self.dZ1)
        self._t("rgcnb_bwd1")
        L.seastar_rgcn_basis_bwd(g.handle, self._V1_all, self.B1, self.Hd, self.ldv, p.p("a1"), None, dZ1_all,
                                 self.ldh, self.E.g("V1"), p.g("a1"), ws, ws.numel())
        self._t("rgcnb_bwd1_end")
        self.comm.all_reduce(self.P.grad)      # V1's gradient rows are owned: no reduction

    def epoch(self):
        loss = self.forward()
        self.backward()
        self.P.adam(self.lr)
        self.E.adam(self.lr)
        return loss


class CapturedEpoch:
    """One model's training epoch captured once in a CUDA graph and replayed (the launch-bound small
    configs spend more time issuing ~20 C-ABI calls from Python than in the kernels).  Every call of an
    epoch is stream-ordered and allocation-free once the model's buffers exist (seastar.h conventions),
    so the captured graph is exactly the eager epoch; ``epoch()`` replays it and returns the model's
    (static) loss tensor.  Run the eager epoch at least once before capturing (it sizes the workspaces)."""

    def __init__(self, model):
        self.model = model
        self.graph = torch.cuda.CUDAGraph(keep_graph=True)      # kept for kernel_names()
        s = torch.cuda.Stream()
        s.wait_stream(torch.cuda.current_stream())
        with torch.cuda.graph(self.graph, stream=s):
            self.loss = model.epoch()
        torch.cuda.current_stream().wait_stream(s)

    def epoch(self):
        self.graph.replay()
        return self.loss

    def kernel_names(self) -> list:
        """Names of the kernel nodes one replay launches (read back from the captured cudaGraph_t through
        the driver API): the measured per-epoch launch list behind bench.py's ``gpu_launches``."""
        from cuda.bindings import driver as cu
        g = cu.CUgraph(int(self.graph.raw_cuda_graph()))
        err, _, n = cu.cuGraphGetNodes(g, 0)
        err, nodes, n = cu.cuGraphGetNodes(g, n)
        assert err == cu.CUresult.CUDA_SUCCESS, err
        names = []
        for nd in nodes[:n]:
            err, t = cu.cuGraphNodeGetType(nd)
            if t != cu.CUgraphNodeType.CU_GRAPH_NODE_TYPE_KERNEL:
                continue
            err, prm = cu.cuGraphKernelNodeGetParams(nd)
            name = None
            if int(prm.func):
                err, name = cu.cuFuncGetName(prm.func)
            if not name and int(prm.kern):
                err, name = cu.cuKernelGetName(prm.kern)
            names.append(name.decode() if isinstance(name, bytes) else str(name))
        return names


class PrefetchedInput:
    """A step's input rows streamed host -> device one step ahead (a DataLoader-style prefetch): the pinned
    host rows are copied into a device staging buffer on a side stream while the previous step's kernels
    run, and moved into the model's input buffer (a device-to-device copy) at the start of the step that
    consumes them.  ``prefetch()`` issues the next copy, ``consume()`` makes the current stream wait for it."""

    def __init__(self, host_pinned: torch.Tensor, dest: torch.Tensor):
        assert host_pinned.is_pinned() and dest.is_cuda and host_pinned.shape == dest.shape
        self.h, self.dest = host_pinned, dest
        self.stage = torch.empty(host_pinned.shape, dtype=host_pinned.dtype, device=dest.device)
        self.cs = torch.cuda.Stream(device=dest.device)
        self.ready = torch.cuda.Event()
        self.free = torch.cuda.Event()
        self.free.record(torch.cuda.current_stream())

    def prefetch(self):
        self.cs.wait_event(self.free)                 # the staging buffer has been consumed
        with torch.cuda.stream(self.cs):
            self.stage.copy_(self.h, non_blocking=True)
            self.ready.record(self.cs)

    def consume(self):
        cur = torch.cuda.current_stream()
        cur.wait_event(self.ready)
        self.dest.copy_(self.stage)
        self.free.record(cur)
