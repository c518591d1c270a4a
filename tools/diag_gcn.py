import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "tests"))
import numpy as np, torch
import oracle
from helpers import hub_graph, padded, rnd
from paper_conf_eurosys_wumcjlzcy21_b200 import _lib as L
from paper_conf_eurosys_wumcjlzcy21_b200.graph import Graph
ip, ix = hub_graph()
N = len(ip) - 1
g = Graph(ip, ix)
print(g.info)
deg = np.diff(ip)
for F, ld in [(16, 16), (16, 20), (1, 4), (41, 44)]:
    T = rnd(10 + F, (N, F))
    Y = torch.full((N, ld), float("nan"), device="cuda")
    L.seastar_gcn_fwd(g.handle, torch.from_numpy(padded(T, ld)).cuda(), F, ld, None, None, "none", 0.0, None, Y)
    torch.cuda.synchronize()
    got = Y.cpu().numpy()[:, :F]
    ref = oracle.gcn_aggregate(ip, ix, T)
    err = np.abs(got - ref).max(1)
    bad = np.argsort(-err)[:8]
    print(F, ld, "max err", err.max(), "n bad rows", (err > 1e-4).sum())
    for v in bad:
        print("   v", v, "deg", deg[v], "err", err[v], "got", got[v][:3], "ref", ref[v][:3])
