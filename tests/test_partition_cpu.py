"""Multi-GPU sharding math on CPU: 2 processes, gloo, the product's Comm / partition modules, the
oracle standing in for each rank's kernels ("partition emulation").

Each rank owns a destination-row range, computes exactly what models.GCN2 / models.GAT2 compute for
its rows (same gathers, same per-rank normalisation, same gradient all-reduce, GAT der over owned rows
from the gathered forward tables -- no reduce-scatter), and rank 0 checks loss and every gradient
against the single-process oracle composition."""
import os
import socket
import sys

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

HERE = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, HERE)
sys.path.insert(0, os.path.dirname(HERE))


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _rel(a, b):
    den = np.abs(b).max() or 1.0
    return float(np.abs(a - b).max() / den)


def _gather(comm, loc, rows_all, n_pad):
    """Product Comm.all_gather on CPU fp64 tensors, padded chunks (as models._local_rows)."""
    buf = np.zeros((n_pad,) + loc.shape[1:])
    buf[:loc.shape[0]] = loc
    out = torch.zeros((rows_all,) + loc.shape[1:], dtype=torch.float64)
    return comm.all_gather(out, torch.from_numpy(buf)).numpy()


def _allreduce(comm, x):
    t = torch.from_numpy(np.ascontiguousarray(x, np.float64)).clone()
    comm.all_reduce(t)
    return t.numpy()


def _gcn_rank(comm, part, ip, ix, X, lab, p, N, P, rank):
    import oracle
    rb, re = part.row_range(N, P, rank)
    n_pad, rows_all = part.rows_per_rank(N, P), part.gathered_rows(N, P)
    own = np.arange(rb, re)
    in_n, out_n = oracle.degree_norms(ip, ix)
    T_loc = oracle.linear_fwd(X[rb:re], p["W1"]) * out_n[own, None]
    T_all = _gather(comm, T_loc, rows_all, n_pad)[:N]
    Z1 = oracle.gcn_aggregate(ip, ix, T_all, None, in_n, own) + p["b1"]
    H1 = oracle.act_fwd("relu", Z1)
    H1s_all = _gather(comm, H1 * out_n[own, None], rows_all, n_pad)[:N]
    P2 = oracle.gcn_aggregate(ip, ix, H1s_all, None, in_n, own)
    logits = oracle.linear_fwd(P2, p["W2"], p["b2"])
    loss_loc, dlog = oracle.softmax_xent(logits, lab[rb:re])
    loss_loc *= (re - rb) / N                    # seastar_softmax_xent normalises by the global N
    dlog *= (re - rb) / N
    dP2, dW2, db2 = oracle.linear_bwd(P2, p["W2"], dlog)
    dP2_all = _gather(comm, dP2 * in_n[own, None], rows_all, n_pad)[:N]
    dH1 = oracle.gcn_aggregate_T(ip, ix, dP2_all, out_n, None, own)
    dA1 = oracle.act_bwd("relu", Z1, dH1)
    dP1_all = _gather(comm, dA1 * in_n[own, None], rows_all, n_pad)[:N]
    dT1 = oracle.gcn_aggregate_T(ip, ix, dP1_all, out_n, None, own)
    _, dW1, _ = oracle.linear_bwd(X[rb:re], p["W1"], dT1, need_dX=False, need_db=False)
    grads = {"W1": dW1, "b1": dA1.sum(0), "W2": dW2, "b2": db2}
    return _allreduce(comm, np.array([loss_loc]))[0], {k: _allreduce(comm, v) for k, v in grads.items()}


def _gat_layer_rank(comm, part, ip, ix, Xin_loc, W, al, ar, b, act, H, F, N, P, rank, n_pad, rows_all):
    import oracle
    rb, re = part.row_range(N, P, rank)
    own = np.arange(rb, re)
    T_loc = oracle.linear_fwd(Xin_loc, W).reshape(-1, H, F)
    el_loc, er_loc = oracle.gat_attn_proj(T_loc, al, ar)
    T_all = _gather(comm, T_loc.reshape(-1, H * F), rows_all, n_pad)[:N].reshape(N, H, F)
    el_all = _gather(comm, el_loc, rows_all, n_pad)[:N]
    er_full = np.zeros((N, H))
    er_full[own] = er_loc                        # only owned destinations are evaluated in the forward
    A, _, _ = oracle.gat_fwd(ip, ix, T_all, el_all, er_full, 0.2, own)
    Z = A.reshape(-1, H * F) + b
    return dict(T_loc=T_loc, el_loc=el_loc, er_loc=er_loc, T_all=T_all, el_all=el_all, Z=Z,
                Y=oracle.act_fwd(act, Z), own=own)


def _gat_layer_bwd_rank(comm, part, ip, ix, Xin_loc, W, al, ar, act, H, F, st, dY, N, n_pad, rows_all, need_dX):
    import oracle
    own = st["own"]
    dZ = oracle.act_bwd(act, st["Z"], dY)
    db = dZ.sum(0)
    # the packed record D = [dA | er | lse | c] is all-gathered: dA and er of every destination
    dA_all = _gather(comm, dZ, rows_all, n_pad)[:N].reshape(N, H, F)
    er_all = _gather(comm, st["er_loc"], rows_all, n_pad)[:N]
    # src-major kernel over owned sources (rows=own): dT, del; the dst-major der kernel evaluates the
    # owned destinations from the gathered forward tables -> take der[own], no reduce-scatter
    dT, dl, dr_all = oracle.gat_bwd(ip, ix, st["T_all"], st["el_all"], er_all, dA_all, 0.2, own)
    dr = dr_all[own]
    dTp, dal, dar = oracle.gat_attn_proj_bwd(st["T_loc"], al, ar, dl, dr)
    dTt = (dT + dTp).reshape(-1, H * F)
    dX, dW, _ = oracle.linear_bwd(Xin_loc, W, dTt, need_dX=need_dX, need_db=False)
    return dX, dW, dal, dar, db


def _gat_rank(comm, part, ip, ix, X, lab, p, heads, hid, N, P, rank):
    import oracle
    rb, re = part.row_range(N, P, rank)
    n_pad, rows_all = part.rows_per_rank(N, P), part.gathered_rows(N, P)
    C = p["W2"].shape[1]
    s1 = _gat_layer_rank(comm, part, ip, ix, X[rb:re], p["W1"], p["al1"], p["ar1"], p["b1"], "elu", heads, hid, N,
                         P, rank, n_pad, rows_all)
    s2 = _gat_layer_rank(comm, part, ip, ix, s1["Y"], p["W2"], p["al2"], p["ar2"], p["b2"], "none", 1, C, N, P, rank,
                         n_pad, rows_all)
    loss_loc, dY2 = oracle.softmax_xent(s2["Y"], lab[rb:re])
    loss_loc *= (re - rb) / N
    dY2 *= (re - rb) / N
    dY1, dW2, dal2, dar2, db2 = _gat_layer_bwd_rank(comm, part, ip, ix, s1["Y"], p["W2"], p["al2"], p["ar2"], "none",
                                                    1, C, s2, dY2, N, n_pad, rows_all, True)
    _, dW1, dal1, dar1, db1 = _gat_layer_bwd_rank(comm, part, ip, ix, X[rb:re], p["W1"], p["al1"], p["ar1"], "elu",
                                                  heads, hid, s1, dY1, N, n_pad, rows_all, False)
    grads = {"W1": dW1, "al1": dal1, "ar1": dar1, "b1": db1, "W2": dW2, "al2": dal2, "ar2": dar2, "b2": db2}
    return _allreduce(comm, np.array([loss_loc]))[0], {k: _allreduce(comm, v) for k, v in grads.items()}


def _worker(rank, world, port, errfile):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        from oracle import model_ref
        import synth
        from paper_conf_eurosys_wumcjlzcy21_b200 import partition as part
        from paper_conf_eurosys_wumcjlzcy21_b200.models import Comm
        comm = Comm(world, rank)
        N = 501                                           # not divisible by the world size
        ip, ix = synth.powerlaw_sym(N, 4000, 0.6, 41)
        X = synth.uniform(1, (N, 40)).astype(np.float64)
        lab = synth.labels(2, N, 7)
        pg = {"W1": synth.glorot(3, 40, 16), "b1": synth.uniform(4, (16,), -.1, .1), "W2": synth.glorot(5, 16, 7),
              "b2": synth.uniform(6, (7,), -.1, .1)}
        pg = {k: v.astype(np.float64) for k, v in pg.items()}
        loss, grads = _gcn_rank(comm, part, ip, ix, X, lab, pg, N, world, rank)
        heads, hid, C = 4, 4, 5
        pa = {"W1": synth.glorot(13, 40, heads * hid), "al1": synth.uniform(14, (heads, hid), -.5, .5),
              "ar1": synth.uniform(15, (heads, hid), -.5, .5), "b1": synth.uniform(16, (heads * hid,), -.1, .1),
              "W2": synth.glorot(17, heads * hid, C), "al2": synth.uniform(18, (1, C), -.5, .5),
              "ar2": synth.uniform(19, (1, C), -.5, .5), "b2": synth.uniform(20, (C,), -.1, .1)}
        pa = {k: v.astype(np.float64) for k, v in pa.items()}
        lab5 = synth.labels(21, N, C)
        loss_a, grads_a = _gat_rank(comm, part, ip, ix, X, lab5, pa, heads, hid, N, world, rank)
        if rank == 0:
            rl, rg = model_ref.gcn2(ip, ix, X, lab, pg)
            assert abs(loss - rl) < 1e-12 * abs(rl), (loss, rl)
            for k in rg:
                assert _rel(grads[k], rg[k]) < 1e-12, ("gcn", k, _rel(grads[k], rg[k]))
            rl, rg = model_ref.gat2(ip, ix, X, lab5, pa, heads, hid)
            assert abs(loss_a - rl) < 1e-12 * abs(rl), (loss_a, rl)
            for k in rg:
                assert _rel(grads_a[k], rg[k]) < 1e-12, ("gat", k, _rel(grads_a[k], rg[k]))
    except BaseException as e:  # noqa: BLE001
        with open(errfile, "a") as f:
            f.write(f"rank {rank}: {type(e).__name__}: {e}\n")
        raise
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
def test_partitioned_training_step_matches_single_process(tmp_path, world):
    err = str(tmp_path / "err.txt")
    mp.spawn(_worker, args=(world, _free_port(), err), nprocs=world, join=True)
    assert not os.path.exists(err) or open(err).read() == ""


def test_row_ranges_cover_and_pad():
    from paper_conf_eurosys_wumcjlzcy21_b200 import partition as part
    for N, P in [(232965, 8), (10, 3), (7, 8), (16, 4)]:
        ranges = [part.row_range(N, P, r) for r in range(P)]
        assert ranges[0][0] == 0 and ranges[-1][1] == N
        assert all(a[1] == b[0] for a, b in zip(ranges, ranges[1:]))
        assert part.gathered_rows(N, P) >= N and part.gathered_rows(N, P) % P == 0
        assert all(r[1] - r[0] <= part.rows_per_rank(N, P) for r in ranges)
