"""Tiny-graph pass over every kernel family of libseastar.so, run under compute-sanitizer:

    compute-sanitizer --tool {memcheck,racecheck,synccheck,initcheck} python tools/sanitize_driver.py

Graph creation (untyped, typed with R-GCN norms, row-partitioned), GCN2 (with hidden dropout), GAT2 at the
head-per-lane 8x8 shape, a generic 3x5 shape and with attention dropout, APPNP (edge dropout), R-GCN2,
R-GCN with bases, the tcgen05 and SIMT dense transforms, softmax cross-entropy and Adam: one epoch each.
The graphs include a hub row (in-degree >= 1024, the hub bucket) and isolated vertices.  No results are
checked here (parity is the GPU test suite's job); the sanitizer's exit code is the verdict."""
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import synth  # noqa: E402
from paper_conf_eurosys_wumcjlzcy21_b200 import _lib as L  # noqa: E402
from paper_conf_eurosys_wumcjlzcy21_b200.graph import Graph  # noqa: E402
from paper_conf_eurosys_wumcjlzcy21_b200 import models as M  # noqa: E402


def hub_graph(N, E, seed, R=0):
    """Random multigraph plus one hub destination with 1,100 in-edges and a few isolated vertices."""
    rng = np.random.default_rng(seed)
    src = rng.integers(0, N - 3, E)
    dst = rng.integers(0, N - 3, E)
    src = np.concatenate([src, rng.integers(0, N - 3, 1100)])
    dst = np.concatenate([dst, np.full(1100, 5)])
    et = rng.integers(0, R, src.size) if R else None
    return synth.csr_from_edges(N, src, dst, et)


def main():
    dev = torch.device("cuda", 0)
    torch.cuda.set_device(0)
    L.seastar_device_check()
    N = 1500
    ip, ix = hub_graph(N, 9000, 1)
    X = torch.from_numpy(synth.uniform(1, (N, 40))).to(dev)
    Xw = torch.zeros((N, 64), device=dev)          # 16-B row stride, TMA-fed transform
    Xw[:, :40] = X
    lab = torch.from_numpy(synth.labels(2, N, 5)).to(dev)
    g = Graph(ip, ix, device=dev)
    gcn = {"W1": synth.glorot(3, 40, 16), "b1": np.zeros(16, np.float32), "W2": synth.glorot(4, 16, 5),
           "b2": np.zeros(5, np.float32)}
    for m in (M.GCN2(g, Xw[:, :40], lab, gcn), M.GCN2(g, Xw[:, :40], lab, gcn, dropout=0.5, seed=3)):
        m.epoch()
    for heads, hid, ad in ((8, 8, 0.0), (3, 5, 0.0), (8, 8, 0.3)):
        Wd = heads * hid
        gp = {"W1": synth.glorot(5, 40, Wd), "al1": synth.uniform(6, (heads, hid)), "ar1": synth.uniform(7, (heads, hid)),
              "b1": np.zeros(Wd, np.float32), "W2": synth.glorot(8, Wd, 5), "al2": synth.uniform(9, (1, 5)),
              "ar2": synth.uniform(10, (1, 5)), "b2": np.zeros(5, np.float32)}
        for save_B in (True, False):
            M.GAT2(g, Xw[:, :40], lab, gp, heads, hid, save_der_factors=save_B, attn_dropout=ad, seed=1).epoch()
    ap = {"W1": synth.glorot(11, 40, 16), "b1": np.zeros(16, np.float32), "W2": synth.glorot(12, 16, 5),
          "b2": np.zeros(5, np.float32)}
    M.APPNPNet(g, Xw[:, :40], lab, ap, K=3, alpha=0.1).epoch()
    M.APPNPNet(g, Xw[:, :40], lab, ap, K=3, alpha=0.1, edge_dropout=0.2, seed=2).epoch()
    g.close()

    # partitioned graph (rows [500, 1000) of 3 ranks; the LSF index)
    gp3 = Graph(ip, ix, row_begin=500, row_end=1000, device=dev)
    T_all = torch.from_numpy(synth.uniform(20, (N, 16))).to(dev)
    Y = torch.empty((500, 16), device=dev)
    L.seastar_gcn_fwd(gp3.handle, T_all, 16, 16, None, None, "relu", 0.0, None, Y)
    L.seastar_gcn_bwd(gp3.handle, T_all, 16, 16, None, 1.0, None, "none", None, Y, None)
    gp3.close()

    # typed graphs: R-GCN (dense X) and R-GCN with bases
    R = 7
    ip, ix, et = hub_graph(N, 9000, 3, R)
    gt = Graph(ip, ix, et, num_etypes=R, rgcn_norm=True, device=dev)
    X16 = torch.from_numpy(synth.uniform(13, (N, 16))).to(dev)
    rp = {"W1": synth.glorot(14, 16, 16, (R, 16, 16)), "b1": np.zeros(16, np.float32),
          "W2": synth.glorot(15, 16, 5, (R, 16, 5)), "b2": np.zeros(5, np.float32)}
    M.RGCN2(gt, X16, lab, rp).epoch()
    B = 3
    bp = {"V1": synth.glorot(16, N, 16, (N, B, 16)), "a1": synth.glorot(17, R, B, (R, B)),
          "b1": np.zeros(16, np.float32), "V2": synth.glorot(18, 16, 5, (B, 16, 5)),
          "a2": synth.glorot(19, R, B, (R, B)), "b2": np.zeros(5, np.float32)}
    M.RGCNBasis2(gt, lab, bp).epoch()
    gt.close()
    torch.cuda.synchronize()
    print("sanitize driver OK")


if __name__ == "__main__":
    main()
