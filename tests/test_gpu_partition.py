"""Partitioned kernels on one GPU: P "ranks" as threads, each with its own row-range graph
(seastar_graph_create(row_begin,row_end)), buffers and models.GCN2 / GAT2 / RGCN2 instance, and a
lockstep in-process communicator in place of NCCL.  Loss and all-reduced gradients must match the
oracle composition of the unpartitioned model (SURVEY.md §4 item 8a on the device)."""
import threading

import numpy as np
import pytest

from oracle import model_ref
import synth
from conftest import rel_err

pytestmark = pytest.mark.gpu
TOL = 1e-5


class ThreadComm:
    """all_gather / all_reduce between P threads sharing one device (ordered, deterministic)."""

    def __init__(self, world, rank, shared, barrier):
        self.world, self.rank, self.shared, self.barrier = world, rank, shared, barrier

    def _exchange(self, t):
        import torch
        torch.cuda.synchronize()
        self.shared[self.rank] = t.clone()
        self.barrier.wait()
        parts = [self.shared[r] for r in range(self.world)]
        self.barrier.wait()
        return parts

    def all_gather(self, out_all, loc):
        import torch
        out_all.copy_(torch.cat(self._exchange(loc), 0))
        return out_all

    def all_gather_async(self, out_all, loc):
        """NEXT-1 interface: the lockstep exchange completes here; the handle's wait() is a no-op"""
        self.all_gather(out_all, loc)

        class _Done:
            def wait(self):
                return None
        return _Done()

    def reduce_scatter(self, out_loc, part_all):
        raise AssertionError("the partitioned models never reduce-scatter")

    def all_reduce(self, flat):
        parts = self._exchange(flat)
        tot = parts[0].clone()
        for p in parts[1:]:
            tot += p
        flat.copy_(tot)


def run_ranks(P, build):
    shared = {}
    barrier = threading.Barrier(P)
    out, errs = [None] * P, []

    def body(r):
        try:
            out[r] = build(r, ThreadComm(P, r, shared, barrier))
        except BaseException as e:  # noqa: BLE001
            errs.append(e)
            barrier.abort()

    th = [threading.Thread(target=body, args=(r,)) for r in range(P)]
    for t in th:
        t.start()
    for t in th:
        t.join()
    if errs:
        raise errs[0]
    return out


@pytest.fixture(scope="module")
def env():
    import torch
    assert torch.cuda.is_available()
    from paper_conf_eurosys_wumcjlzcy21_b200 import models, partition
    from paper_conf_eurosys_wumcjlzcy21_b200.graph import Graph
    return dict(torch=torch, models=models, part=partition, Graph=Graph)


def grads_of(model, keys):
    return {k: model.P.g(k).cpu().numpy().copy() for k in keys}


@pytest.mark.parametrize("P,overlap", [(2, True), (3, True), (2, False)])
def test_gcn_gat_partitioned(env, P, overlap):
    """overlap: GCN2's aggregations run NEXT-1's two phases (owned-neighbour edges from the rank's own rows, then
    the rest from the gathered table) -- the default when partitioned -- or one phase after the gather."""
    torch, models, part, Graph = env["torch"], env["models"], env["part"], env["Graph"]
    N, Fin = 3001, 120
    ip, ix = synth.powerlaw_sym(N, 30000, 0.5, 51)
    X = synth.uniform(1, (N, Fin))
    lab7, lab5 = synth.labels(2, N, 7), synth.labels(3, N, 5)
    pg = {"W1": synth.glorot(4, Fin, 16), "b1": synth.uniform(5, (16,), -.1, .1), "W2": synth.glorot(6, 16, 7),
          "b2": synth.uniform(7, (7,), -.1, .1)}
    heads, hid, C = 8, 8, 5
    pa = {"W1": synth.glorot(13, Fin, 64), "al1": synth.uniform(14, (heads, hid), -.5, .5),
          "ar1": synth.uniform(15, (heads, hid), -.5, .5), "b1": synth.uniform(16, (64,), -.1, .1),
          "W2": synth.glorot(17, 64, C), "al2": synth.uniform(18, (1, C), -.5, .5),
          "ar2": synth.uniform(19, (1, C), -.5, .5), "b2": synth.uniform(20, (C,), -.1, .1)}

    def build(r, comm):
        torch.cuda.set_device(0)
        rb, re = part.row_range(N, P, r)
        g = Graph(ip, ix, row_begin=rb, row_end=re)
        Xl = torch.from_numpy(X[rb:re]).cuda()
        mg = models.GCN2(g, Xl, torch.from_numpy(lab7[rb:re]).cuda(), pg, comm=comm,
                         n_pad_rows=part.gathered_rows(N, P), overlap=overlap)
        lg = mg.forward().item()
        mg.backward()
        ma = models.GAT2(g, Xl, torch.from_numpy(lab5[rb:re]).cuda(), pa, heads, hid, comm=comm,
                         n_pad_rows=part.gathered_rows(N, P))
        la = ma.forward().item()
        ma.backward()
        torch.cuda.synchronize()
        return lg, grads_of(mg, pg), la, grads_of(ma, pa)

    res = run_ranks(P, build)
    rl, rg = model_ref.gcn2(ip, ix, X, lab7, {k: v.astype(np.float64) for k, v in pg.items()})
    assert abs(sum(r[0] for r in res) - rl) <= TOL * abs(rl)
    for k in rg:
        assert rel_err(res[0][1][k], rg[k].reshape(res[0][1][k].shape)) <= TOL, ("gcn", k)
        assert all(np.array_equal(res[0][1][k], res[i][1][k]) for i in range(P))   # identical after all-reduce
    rl, rg = model_ref.gat2(ip, ix, X, lab5, {k: v.astype(np.float64) for k, v in pa.items()}, heads, hid)
    assert abs(sum(r[2] for r in res) - rl) <= TOL * abs(rl)
    for k in rg:
        assert rel_err(res[0][3][k], rg[k].reshape(res[0][3][k].shape)) <= TOL, ("gat", k)


def test_rgcn_partitioned(env):
    torch, models, part, Graph = env["torch"], env["models"], env["part"], env["Graph"]
    P, N, R, Fin, Hd, C = 2, 2001, 12, 16, 16, 11
    ip, ix, et = synth.powerlaw_directed_typed(N, 10000, 0.6, 0.6, R, 1.0, 52)
    X = synth.uniform(31, (N, Fin))
    lab = synth.labels(32, N, C)
    p = {"W1": synth.glorot(33, Fin, Hd, (R, Fin, Hd)), "b1": synth.uniform(34, (Hd,), -0.1, 0.1),
         "W2": synth.glorot(35, Hd, C, (R, Hd, C)), "b2": synth.uniform(36, (C,), -0.1, 0.1)}

    def build(r, comm):
        torch.cuda.set_device(0)
        rb, re = part.row_range(N, P, r)
        g = Graph(ip, ix, et, num_etypes=R, row_begin=rb, row_end=re, rgcn_norm=True)
        m = models.RGCN2(g, torch.from_numpy(X[rb:re]).cuda(), torch.from_numpy(lab[rb:re]).cuda(), p, comm=comm,
                         n_pad_rows=part.gathered_rows(N, P))
        l = m.forward().item()
        m.backward()
        torch.cuda.synchronize()
        return l, grads_of(m, p)

    res = run_ranks(P, build)
    rl, rg = model_ref.rgcn2(ip, ix, et, X, lab, {k: v.astype(np.float64) for k, v in p.items()})
    assert abs(sum(r[0] for r in res) - rl) <= TOL * abs(rl)
    for k in rg:
        assert rel_err(res[0][1][k], rg[k].reshape(res[0][1][k].shape)) <= TOL, k


@pytest.mark.parametrize("P", [2, 3])
def test_rgcnb_partitioned(env, P):
    """NEXT-2 model: V1 row-partitioned with the vertices (dV rows owned, never all-reduced), V1 all-gathered."""
    torch, models, part, Graph = env["torch"], env["models"], env["part"], env["Graph"]
    N, R, B1, B2, Hd, C = 2003, 14, 6, 4, 16, 3
    ip, ix, et = synth.powerlaw_directed_typed(N, 12000, 0.6, 0.6, R, 1.0, 53)
    lab = synth.labels(37, N, C)
    p = {"V1": synth.uniform(38, (N, B1, Hd), -0.5, 0.5), "a1": synth.uniform(39, (R, B1)),
         "b1": synth.uniform(40, (Hd,), -0.1, 0.1), "V2": synth.uniform(41, (B2, Hd, C), -0.5, 0.5),
         "a2": synth.uniform(42, (R, B2)), "b2": synth.uniform(43, (C,), -0.1, 0.1)}

    def build(r, comm):
        torch.cuda.set_device(0)
        rb, re = part.row_range(N, P, r)
        g = Graph(ip, ix, et, num_etypes=R, row_begin=rb, row_end=re, rgcn_norm=True)
        m = models.RGCNBasis2(g, torch.from_numpy(lab[rb:re]).cuda(), p, comm=comm,
                              n_pad_rows=part.gathered_rows(N, P))
        l = m.forward().item()
        m.backward()
        torch.cuda.synchronize()
        return l, {k: m.grad(k).cpu().numpy().copy() for k in p}, rb, re

    res = run_ranks(P, build)
    rl, rg = model_ref.rgcnb2(ip, ix, et, lab, {k: v.astype(np.float64) for k, v in p.items()})
    assert abs(sum(r[0] for r in res) - rl) <= TOL * abs(rl)
    for k in rg:
        if k == "V1":       # owned rows of each rank, concatenated
            got = np.concatenate([r[1]["V1"] for r in res], 0)
        else:
            got = res[0][1][k]
        assert rel_err(got, rg[k].reshape(got.shape)) <= TOL, k


@pytest.mark.parametrize("overlap,edge_p", [(True, 0.0), (False, 0.0), (True, 0.2)])
def test_appnp_partitioned(env, overlap, edge_p):
    """APPNP row-partitioned over P = 2 ranks: every propagation step's aggregation (forward and backward) in NEXT-1's
    two phases around its all-gather, or one phase; with and without edge dropout (masks keyed by user edge id)."""
    torch, models, part, Graph = env["torch"], env["models"], env["part"], env["Graph"]
    P, N, Fin, Hd, C, K = 2, 1601, 40, 16, 5, 4
    ip, ix = synth.powerlaw_sym(N, 12000, 0.5, 61)
    X, lab = synth.uniform(44, (N, Fin)), synth.labels(45, N, C)
    p = {"W1": synth.glorot(46, Fin, Hd), "b1": synth.uniform(47, (Hd,), -0.1, 0.1),
         "W2": synth.glorot(48, Hd, C), "b2": synth.uniform(49, (C,), -0.1, 0.1)}

    def build(r, comm):
        torch.cuda.set_device(0)
        rb, re = part.row_range(N, P, r)
        g = Graph(ip, ix, row_begin=rb, row_end=re)
        m = models.APPNPNet(g, torch.from_numpy(X[rb:re]).cuda(), torch.from_numpy(lab[rb:re]).cuda(), p, K=K,
                            alpha=0.1, comm=comm, n_pad_rows=part.gathered_rows(N, P), overlap=overlap,
                            edge_dropout=edge_p, seed=9)
        assert m.overlap == overlap
        l = m.forward().item()
        m.backward()
        torch.cuda.synchronize()
        return l, grads_of(m, p)

    res = run_ranks(P, build)
    drop = {"edge_p": edge_p, "seed": 9, "step": 0} if edge_p else None
    rl, rg = model_ref.appnp(ip, ix, X, lab, {k: v.astype(np.float64) for k, v in p.items()}, K, 0.1, drop=drop)
    assert abs(sum(r[0] for r in res) - rl) <= TOL * abs(rl)
    for k in rg:
        assert rel_err(res[0][1][k], rg[k].reshape(res[0][1][k].shape)) <= TOL, k
