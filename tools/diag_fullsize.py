"""Diagnostics (not a test): per-intermediate max-abs-normalised errors of one training step at a
BASELINE config's full size, GPU (C ABI) vs the fp64 oracle.  python tools/diag_fullsize.py physics_appnp"""
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import oracle  # noqa: E402
import synth  # noqa: E402
from paper_conf_eurosys_wumcjlzcy21_b200 import models  # noqa: E402
from paper_conf_eurosys_wumcjlzcy21_b200.graph import Graph  # noqa: E402


def rel(got, ref):
    got = np.asarray(got, np.float64).reshape(np.shape(ref))
    return float(np.abs(got - ref).max() / (np.abs(ref).max() or 1.0))


def devX(X):
    N, F = X.shape
    Xp = torch.zeros((N, (F + 3) // 4 * 4), device="cuda")
    Xp[:, :F].copy_(torch.from_numpy(X))
    return Xp[:, :F]


def appnp(w):
    cfg = w["cfg"]
    ip, ix, X, lab = w["indptr"], w["indices"], w["X"], w["labels"]
    p = {k: np.asarray(v, np.float64) for k, v in w["appnp"].items()}
    m = models.APPNPNet(Graph(ip, ix), devX(X), torch.from_numpy(lab).cuda(), w["appnp"], K=cfg.K, alpha=cfg.alpha)
    m.forward()
    m.backward()
    torch.cuda.synchronize()
    C = cfg.classes
    Z1 = oracle.linear_fwd(X, p["W1"], p["b1"])
    Hh = oracle.act_fwd("relu", Z1)
    H0 = oracle.linear_fwd(Hh, p["W2"], p["b2"])
    print("Hh", rel(m.Hh.cpu().numpy(), Hh), "H0", rel(m.H0[:, :C].cpu().numpy(), H0))
    Z = H0
    for k in range(cfg.K):
        Z = oracle.appnp_fwd(ip, ix, Z, 1, cfg.alpha) if False else Z
    Zk = oracle.appnp_fwd(ip, ix, H0, cfg.K, cfg.alpha)
    print("Z_K", rel(m.Z[cfg.K][:, :C].cpu().numpy(), Zk))
    loss, dZ = oracle.softmax_xent(Zk, lab)
    dH0 = oracle.appnp_bwd(ip, ix, dZ, cfg.K, cfg.alpha)
    print("dH0", rel(m.dH0[:, :C].cpu().numpy(), dH0))
    dHh, dW2, db2 = oracle.linear_bwd(Hh, p["W2"], dH0)
    dZ1 = oracle.act_bwd("relu", Z1, dHh)
    print("dZ1 (dHh after relu')", rel(m.dHh.cpu().numpy(), dZ1))
    _, dW1, db1 = oracle.linear_bwd(X, p["W1"], dZ1, need_dX=False)
    print("dW1", rel(m.P.g("W1").cpu().numpy(), dW1), "db1", rel(m.P.g("b1").cpu().numpy(), db1))
    # isolate the dense dW: oracle dW1 from the GPU's own dZ1 (diagnostic only)
    _, dW1g, db1g = oracle.linear_bwd(X, p["W1"], m.dHh.cpu().numpy().astype(np.float64), need_dX=False)
    print("dW1 vs X^T(gpu dZ1) [dense kernel alone]", rel(m.P.g("W1").cpu().numpy(), dW1g),
          "db1 alone", rel(m.P.g("b1").cpu().numpy(), db1g))
    print("|dW1| max", np.abs(dW1).max(), "sum|terms| max", (np.abs(X).T @ np.abs(dZ1)).max())


def gat(w):
    cfg = w["cfg"]
    ip, ix, X, lab = w["indptr"], w["indices"], w["X"], w["labels"]
    heads, hid = cfg.heads, cfg.extra.get("gat_hidden", cfg.hidden)
    p = {k: np.asarray(v, np.float64) for k, v in w["gat"].items()}
    m = models.GAT2(Graph(ip, ix), devX(X), torch.from_numpy(lab).cuda(), w["gat"], heads, hid)
    m.forward()
    m.backward()
    torch.cuda.synchronize()
    from oracle import model_ref as M
    N, C = X.shape[0], cfg.classes
    T1, el1, er1, Z1, Y1 = M._gat_layer_fwd(ip, ix, X, p["W1"], p["al1"], p["ar1"], p["b1"], "elu", heads, hid)
    print("T1", rel(m.T1[:, :heads * hid].cpu().numpy(), T1.reshape(N, -1)), "el1", rel(m.el1.cpu().numpy(), el1),
          "Y1", rel(m.Y1[:, :heads * hid].cpu().numpy(), Y1))
    T2, el2, er2, Z2, Y2 = M._gat_layer_fwd(ip, ix, Y1, p["W2"], p["al2"], p["ar2"], p["b2"], "none", 1, C)
    print("T2", rel(m.T2[:, :C].cpu().numpy(), T2.reshape(N, -1)), "el2", rel(m.el2.cpu().numpy(), el2),
          "er2", rel(m.er2.cpu().numpy(), er2), "Y2", rel(m.Y2[:, :C].cpu().numpy(), Y2))
    loss, dY2 = oracle.softmax_xent(Y2, lab)
    dT, dl, dr = oracle.gat_bwd(ip, ix, T2, el2, er2, dY2.reshape(N, 1, C), 0.2)
    print("del2", rel(m.del2.cpu().numpy(), dl), "der2", rel(m.der2.cpu().numpy(), dr))
    dar = (dr[:, 0:1] * T2.reshape(N, C)).sum(0)
    dal = (dl[:, 0:1] * T2.reshape(N, C)).sum(0)
    print("dal2", rel(m.P.g("al2").cpu().numpy(), dal), "dar2", rel(m.P.g("ar2").cpu().numpy(), dar))
    der_g = m.der2.cpu().numpy().astype(np.float64)
    T2g = m.T2[:, :C].cpu().numpy().astype(np.float64)
    print("dar2 vs sum(gpu der * gpu T) [reduction alone]",
          rel(m.P.g("ar2").cpu().numpy(), (der_g[:, 0:1] * T2g).sum(0)))


if __name__ == "__main__":
    name = sys.argv[1]
    w = synth.workload(name)
    {"physics_appnp": appnp, "reddit": gat, "corafull_gat": gat}[name](w)
