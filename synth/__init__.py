"""Seeded synthetic inputs shared by the oracle tests and the GPU path.

This module holds none of the Seastar method's arithmetic: it draws graphs shaped like the
paper's datasets (Table 2) and dense tensors (features, Glorot weights,
labels) with the counter-based recipe of SURVEY.md §8(d).  The heavy lifting is in
``synth.c`` (compiled on first use with gcc, or by ``__graft_entry__.build()``).

Both sides of every parity test (``oracle/`` and ``paper_conf_eurosys_wumcjlzcy21_b200``)
consume exactly these arrays; neither imports the other.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from dataclasses import dataclass, field

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SO = os.path.join(_HERE, "libsynth.so")
_SRC = os.path.join(_HERE, "synth.c")

_i64 = ctypes.c_int64
_u64 = ctypes.c_uint64
_dbl = ctypes.c_double
_p = ctypes.c_void_p


def build(force: bool = False) -> str:
    """Compile libsynth.so next to synth.c (gcc -O2 -fopenmp)."""
    if force or not os.path.exists(_SO) or os.path.getmtime(_SO) < os.path.getmtime(_SRC):
        tmp = _SO + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-fopenmp", "-fPIC", "-shared", _SRC, "-o", tmp, "-lm"])
        os.replace(tmp, _SO)
    return _SO


_lib = None


def _L():
    global _lib
    if _lib is None:
        _lib = ctypes.CDLL(build())
        _lib.synth_powerlaw_sym.argtypes = [_i64, _i64, _dbl, _u64, ctypes.c_int, _p, _p]
        _lib.synth_powerlaw_sym.restype = ctypes.c_int
        _lib.synth_powerlaw_directed_typed.argtypes = [_i64, _i64, _dbl, _dbl, ctypes.c_int32, _dbl,
                                                       _u64, _p, _p, _p]
        _lib.synth_powerlaw_directed_typed.restype = ctypes.c_int
        _lib.synth_uniform_f32.argtypes = [_u64, _i64, _dbl, _dbl, _p]
        _lib.synth_uniform_f32.restype = None
        _lib.synth_labels.argtypes = [_u64, _i64, ctypes.c_int32, _p]
        _lib.synth_labels.restype = None
        _lib.synth_u64.argtypes = [_u64, _u64]
        _lib.synth_u64.restype = _u64
    return _lib


def _ptr(a: np.ndarray) -> int:
    assert a.flags["C_CONTIGUOUS"]
    return a.ctypes.data


def powerlaw_sym(N: int, E_dir: int, s: float, seed: int, self_loops: bool = True):
    """Symmetric Chung-Lu graph as a user in-CSR (indptr[N+1] int64, indices[E] int64 src ids)."""
    E = E_dir + (N if self_loops else 0)
    indptr = np.empty(N + 1, np.int64)
    indices = np.empty(E, np.int64)
    rc = _L().synth_powerlaw_sym(N, E_dir, s, seed, int(self_loops), _ptr(indptr), _ptr(indices))
    if rc:
        raise ValueError("synth_powerlaw_sym: bad arguments")
    return indptr, indices


def powerlaw_directed_typed(N: int, E: int, s_in: float, s_out: float, R: int, zipf_a: float, seed: int):
    """Directed typed Chung-Lu graph: (indptr, indices, etypes int32)."""
    indptr = np.empty(N + 1, np.int64)
    indices = np.empty(E, np.int64)
    etypes = np.empty(E, np.int32)
    rc = _L().synth_powerlaw_directed_typed(N, E, s_in, s_out, R, zipf_a, seed, _ptr(indptr),
                                            _ptr(indices), _ptr(etypes))
    if rc:
        raise ValueError("synth_powerlaw_directed_typed: bad arguments")
    return indptr, indices, etypes


def uniform(seed: int, shape, lo: float = -1.0, hi: float = 1.0) -> np.ndarray:
    out = np.empty(int(np.prod(shape)), np.float32)
    _L().synth_uniform_f32(seed, out.size, lo, hi, _ptr(out))
    return out.reshape(shape)


def glorot(seed: int, fan_in: int, fan_out: int, shape=None) -> np.ndarray:
    """Glorot-uniform U[-l, l], l = sqrt(6 / (fan_in + fan_out))."""
    lim = float(np.sqrt(6.0 / (fan_in + fan_out)))
    return uniform(seed, shape if shape is not None else (fan_in, fan_out), -lim, lim)


def labels(seed: int, n: int, C: int) -> np.ndarray:
    out = np.empty(n, np.int64)
    _L().synth_labels(seed, n, C, _ptr(out))
    return out


def u64(seed: int, i: int) -> int:
    return int(_L().synth_u64(seed, i))


def csr_from_edges(N: int, src, dst, etype=None):
    """User in-CSR from an edge list; edge id = position after a stable sort by dst."""
    src = np.asarray(src, np.int64)
    dst = np.asarray(dst, np.int64)
    order = np.argsort(dst, kind="stable")
    indptr = np.zeros(N + 1, np.int64)
    np.add.at(indptr, dst + 1, 1)
    indptr = np.cumsum(indptr)
    out = (indptr, src[order].copy())
    if etype is not None:
        out = out + (np.asarray(etype, np.int32)[order].copy(),)
    return out


def random_graph(N: int, E: int, seed: int, R: int = 0):
    """Uniform random multigraph (self-loops and duplicate edges allowed) for edge-case tests."""
    src = (uniform(seed, (E,), 0.0, 1.0).astype(np.float64) * N).astype(np.int64).clip(0, N - 1)
    dst = (uniform(seed + 7, (E,), 0.0, 1.0).astype(np.float64) * N).astype(np.int64).clip(0, N - 1)
    if R:
        typ = (uniform(seed + 13, (E,), 0.0, 1.0).astype(np.float64) * R).astype(np.int64).clip(0, R - 1)
        return csr_from_edges(N, src, dst, typ)
    return csr_from_edges(N, src, dst)


# ---------------------------------------------------------------------------------------------
# The five BASELINE.json configurations as concrete synthetic workloads.
# ---------------------------------------------------------------------------------------------
@dataclass
class Config:
    name: str
    N: int
    E_dir: int            # directed non-loop edges (symmetric graphs) or all edges (typed graph)
    s: float
    F_in: int
    hidden: int
    classes: int
    model: str
    heads: int = 1
    self_loops: bool = True
    typed: bool = False
    R: int = 1
    zipf_a: float = 1.0
    K: int = 0
    alpha: float = 0.0
    cfg_id: int = 0
    extra: dict = field(default_factory=dict)

    @property
    def graph_seed(self) -> int:
        return 1000 + self.cfg_id

    @property
    def feat_seed(self) -> int:
        return 2000 + self.cfg_id

    def weight_seed(self, layer: int) -> int:
        return 3000 + 10 * self.cfg_id + layer

    @property
    def label_seed(self) -> int:
        return 4000 + self.cfg_id

    @property
    def E(self) -> int:
        return self.E_dir + (self.N if (self.self_loops and not self.typed) else 0)


CONFIGS = {
    # configs[0]: 2-layer GCN, hidden 16, Cora-shaped (2,708 V, 10,556 E, 1,433 feats, 7 classes)
    "cora_gcn": Config("cora_gcn", 2708, 10556, 0.60, 1433, 16, 7, "gcn", cfg_id=1),
    # configs[1]: 2-layer GAT 8 heads x 8 hidden, CoraFull-shaped (19,793 V, 126,842 E, 8,710 feats, 70 cls)
    "corafull_gat": Config("corafull_gat", 19793, 126842, 0.50, 8710, 8, 70, "gat", heads=8, cfg_id=2),
    # configs[2]: APPNP K=10, alpha=0.1, Coauthor-Physics-shaped (34,493 V, 495,924 E, 8,415 feats, 5 cls)
    "physics_appnp": Config("physics_appnp", 34493, 495924, 0.50, 8415, 64, 5, "appnp", K=10, alpha=0.1,
                            cfg_id=3),
    # configs[3]: R-GCN, AM-shaped (1.9M V, 5.7M E, 133 relations), dense synthetic X 16 -> 16 -> 11
    "am_rgcn": Config("am_rgcn", 1_900_000, 5_700_000, 0.60, 16, 16, 11, "rgcn", self_loops=False,
                      typed=True, R=133, zipf_a=1.0, cfg_id=4),
    # NEXT-2: R-GCN as the paper ran it, Table 2 L485 shapes (aifb 8,285 V / 58,086 E /
    # 90 relations; mutag 23,644 / 148,454 / 46; bgs 333,845 / 1,832,398 / 206), featureless input, hidden 16,
    # DGL entity-classification defaults: bases = R (aifb), 30 (mutag), 40 (bgs); classes 4 / 2 / 2
    "aifb_rgcnb": Config("aifb_rgcnb", 8285, 58086, 0.60, 0, 16, 4, "rgcnb", self_loops=False, typed=True, R=90,
                         cfg_id=6, extra={"bases": 90}),
    "mutag_rgcnb": Config("mutag_rgcnb", 23644, 148454, 0.60, 0, 16, 2, "rgcnb", self_loops=False, typed=True,
                          R=46, cfg_id=7, extra={"bases": 30}),
    "bgs_rgcnb": Config("bgs_rgcnb", 333845, 1832398, 0.60, 0, 16, 2, "rgcnb", self_loops=False, typed=True,
                        R=206, cfg_id=8, extra={"bases": 40}),
    # configs[4]: GCN and GAT full-graph training, Reddit-shaped (232,965 V, 114,615,892 E incl. self-loops)
    "reddit": Config("reddit", 232_965, 114_615_892 - 232_965, 0.35, 602, 16, 41, "gcn+gat", heads=8,
                     cfg_id=5, extra={"gat_hidden": 8}),
}


def make_graph(cfg: Config):
    """(indptr, indices[, etypes]) for a config, deterministic in cfg.graph_seed."""
    if cfg.typed:
        return powerlaw_directed_typed(cfg.N, cfg.E_dir, cfg.s, cfg.s, cfg.R, cfg.zipf_a, cfg.graph_seed)
    return powerlaw_sym(cfg.N, cfg.E_dir, cfg.s, cfg.graph_seed, cfg.self_loops)


def _gcn_params(cfg: Config, fin: int, hid: int, C: int, base: int = 0) -> dict:
    return {"W1": glorot(cfg.weight_seed(base + 1), fin, hid), "b1": np.zeros(hid, np.float32),
            "W2": glorot(cfg.weight_seed(base + 2), hid, C), "b2": np.zeros(C, np.float32)}


def _gat_params(cfg: Config, heads: int, hid: int) -> dict:
    Wd, C = heads * hid, cfg.classes
    return {"W1": glorot(cfg.weight_seed(11), cfg.F_in, Wd),
            "al1": glorot(cfg.weight_seed(12), hid, 1, (heads, hid)),
            "ar1": glorot(cfg.weight_seed(13), hid, 1, (heads, hid)),
            "b1": np.zeros(Wd, np.float32),
            "W2": glorot(cfg.weight_seed(14), Wd, C),
            "al2": glorot(cfg.weight_seed(15), C, 1, (1, C)),
            "ar2": glorot(cfg.weight_seed(16), C, 1, (1, C)),
            "b2": np.zeros(C, np.float32)}


def workload(name: str) -> dict:
    """The complete seeded input set of one BASELINE config: graph, features, labels and the initial
    parameters of every model the config trains (biases 0, as in DGL's init; Glorot weights).
    Keys: cfg, indptr, indices, etypes (typed only), X [N, F_in] f32, labels [N] i64, and one
    parameter dict per model name ("gcn", "gat", "appnp", "rgcn")."""
    cfg = CONFIGS[name]
    g = make_graph(cfg)
    out = {"cfg": cfg, "indptr": g[0], "indices": g[1], "etypes": g[2] if cfg.typed else None,
           "X": uniform(cfg.feat_seed, (cfg.N, cfg.F_in), -1.0, 1.0),
           "labels": labels(cfg.label_seed, cfg.N, cfg.classes)}
    models = cfg.model.split("+")
    if "gcn" in models or "appnp" in models:
        out[models[0] if "appnp" in models else "gcn"] = _gcn_params(cfg, cfg.F_in, cfg.hidden, cfg.classes)
    if "gat" in models:
        out["gat"] = _gat_params(cfg, cfg.heads, cfg.extra.get("gat_hidden", cfg.hidden))
    if "rgcn" in models:
        R, fin, hid, C = cfg.R, cfg.F_in, cfg.hidden, cfg.classes
        out["rgcn"] = {"W1": glorot(cfg.weight_seed(1), fin, hid, (R, fin, hid)), "b1": np.zeros(hid, np.float32),
                       "W2": glorot(cfg.weight_seed(2), hid, C, (R, hid, C)), "b2": np.zeros(C, np.float32)}
    if "rgcnb" in models:
        R, hid, C, B = cfg.R, cfg.hidden, cfg.classes, cfg.extra["bases"]
        out["rgcnb"] = {"V1": glorot(cfg.weight_seed(1), cfg.N, hid, (cfg.N, B, hid)),
                        "a1": glorot(cfg.weight_seed(2), R, B, (R, B)), "b1": np.zeros(hid, np.float32),
                        "V2": glorot(cfg.weight_seed(3), hid, C, (B, hid, C)),
                        "a2": glorot(cfg.weight_seed(4), R, B, (R, B)), "b2": np.zeros(C, np.float32)}
    return out
