"""Graph handle: owns a ``seastar_graph`` built on the GPU by ``seastar_graph_create``."""
from __future__ import annotations

import numpy as np
import torch

from . import _lib as L


def _dev_i64(x, device):
    if isinstance(x, torch.Tensor):
        return x.to(device=device, dtype=torch.int64).contiguous()
    return torch.from_numpy(np.ascontiguousarray(x, dtype=np.int64)).to(device)


class Graph:
    """Degree-sorted CSR / reverse CSR of a user in-CSR graph (§6.1, Fig. 7).

    ``indptr``/``indices`` are the user's in-CSR (numpy or torch); they are copied to the device,
    preprocessed by the library's kernels and released.  ``row_begin/row_end`` select the owned
    destination range for multi-GPU partitions.
    """

    def __init__(self, indptr, indices, etypes=None, num_etypes=0, row_begin=0, row_end=None,
                 rgcn_norm=False, device=None, stream=None):
        device = torch.device(device) if device is not None else torch.device("cuda", torch.cuda.current_device())
        ip = _dev_i64(indptr, device)
        ix = _dev_i64(indices, device)
        et = None
        if etypes is not None:
            et = (etypes.to(device=device, dtype=torch.int32) if isinstance(etypes, torch.Tensor)
                  else torch.from_numpy(np.ascontiguousarray(etypes, dtype=np.int32)).to(device)).contiguous()
            if num_etypes <= 0:
                num_etypes = int(et.max().item()) + 1 if et.numel() else 1
        self.N = ip.numel() - 1
        self.E = ix.numel()
        self.device = device
        self.handle = None
        with torch.cuda.device(device):
            self.handle = L.seastar_graph_create(self.N, self.E, ip, ix, et, num_etypes, row_begin,
                                                 self.N if row_end is None else row_end,
                                                 L.GRAPH_RGCN_NORM if rgcn_norm else 0, stream)
        self.info = L.seastar_graph_info(self.handle)
        self.row_begin = self.info["row_begin"]
        self.row_end = self.info["row_end"]
        self.n_loc = self.row_end - self.row_begin
        self.num_etypes = self.info["num_etypes"]
        self.typed = etypes is not None
        self.rgcn_norm = rgcn_norm

    def close(self):
        if self.handle:
            L.seastar_graph_destroy(self.handle)
            self.handle = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    # -------------------------------------------------------------------------------------------
    def export(self, which: str = "fwd") -> dict:
        """Copy an index set to fresh int32 device tensors (for bit-exact tests)."""
        w = {"fwd": L.FWD, "rev": L.REV, "lsf": L.LSF}[which]
        i32 = dict(dtype=torch.int32, device=self.device)
        if which == "lsf":
            n_rows, n_e = self.N, self.info["num_rev_edges"]
        else:
            n_rows = self.n_loc
            n_e = self.info["num_fwd_edges"] if which == "fwd" else self.info["num_rev_edges"]
        out = {"off": torch.empty(n_rows + 1, **i32), "eid": torch.empty(n_e, **i32)}
        if which != "lsf":
            out["perm"] = torch.empty(n_rows, **i32)
            out["nbr"] = torch.empty(n_e, **i32)
        if which == "rev":
            out["pos"] = torch.empty(n_e, **i32)
        if self.typed and which != "lsf":
            out["type"] = torch.empty(n_e, **i32)
        if self.rgcn_norm and which != "lsf":
            out["norm"] = torch.empty(n_e, dtype=torch.float32, device=self.device)
        L.seastar_graph_export(self.handle, w, out.get("perm"), out["off"], out.get("nbr"), out["eid"],
                               out.get("pos"), out.get("type"), out.get("norm"))
        return out

    def degree_norms(self, mode: str = "both"):
        """(src_norm, dst_norm) per owned vertex, deg^-1/2 with deg clamped >= 1."""
        m = {"both": L.NORM_BOTH, "in": L.NORM_IN}[mode]
        s = torch.empty(self.n_loc, dtype=torch.float32, device=self.device)
        d = torch.empty(self.n_loc, dtype=torch.float32, device=self.device)
        L.seastar_graph_degree_norms(self.handle, m, s, d)
        return s, d
