"""a7 / a10 parity: fused R-GCN forward (type runs, W_r in shared memory), dX on the reverse CSR and
dW on the type-major view vs the fp64 oracle."""
import numpy as np
import pytest

import oracle
import synth
from conftest import rel_err
from helpers import padded, rnd

pytestmark = pytest.mark.gpu
TOL = 1e-5


@pytest.fixture(scope="module")
def env():
    import torch
    assert torch.cuda.is_available()
    from paper_conf_eurosys_wumcjlzcy21_b200 import _lib as L
    from paper_conf_eurosys_wumcjlzcy21_b200.graph import Graph
    N, R = 4000, 33
    ip, ix, et = synth.powerlaw_directed_typed(N, 30000, 0.6, 0.6, R, 1.0, 17)
    # add a typed hub (in-degree 1500 over a few types) so the warp-per-row bucket is exercised
    dst = np.repeat(np.arange(N), np.diff(ip))
    hub_src = (rnd(5, (1500,), 0, 1).astype(np.float64) * N).astype(np.int64).clip(0, N - 1)
    hub_t = (rnd(6, (1500,), 0, 1).astype(np.float64) * 4).astype(np.int64).clip(0, 3)
    ip, ix, et = synth.csr_from_edges(N + 7, np.concatenate([ix, hub_src]), np.concatenate([dst, np.full(1500, 11)]),
                                      np.concatenate([et, hub_t]))
    g = Graph(ip, ix, et, num_etypes=R, rgcn_norm=True)
    return dict(torch=torch, L=L, g=g, ip=ip, ix=ix, et=et, N=N + 7, R=R)


def dev(env, a):
    return env["torch"].from_numpy(np.ascontiguousarray(a)).cuda()


@pytest.mark.parametrize("Fin,Fout", [(16, 16), (16, 11), (4, 5), (8, 32), (32, 8)])
def test_rgcn_fwd(env, Fin, Fout):
    torch, L, g, N, R = env["torch"], env["L"], env["g"], env["N"], env["R"]
    ldx, ldy = (Fin + 3) // 4 * 4, (Fout + 3) // 4 * 4
    X, W, b = rnd(1, (N, Fin)), rnd(2, (R, Fin, Fout)), rnd(3, (Fout,))
    Y = torch.full((N, ldy), float("nan"), device="cuda")
    L.seastar_rgcn_fwd(g.handle, dev(env, padded(X, ldx)), Fin, ldx, dev(env, W), Fout, None, dev(env, b), "relu", Y,
                       ldy)
    ref = oracle.act_fwd("relu", oracle.rgcn_fwd(env["ip"], env["ix"], env["et"], X, W) + b)
    assert rel_err(Y.cpu().numpy()[:, :Fout], ref) <= TOL


def test_rgcn_fwd_user_norm(env):
    torch, L, g, N, R = env["torch"], env["L"], env["g"], env["N"], env["R"]
    X, W = rnd(7, (N, 16)), rnd(8, (R, 16, 16))
    nu = rnd(9, (len(env["ix"]),), 0.1, 1.0)
    Y = torch.empty((N, 16), device="cuda")
    L.seastar_rgcn_fwd(g.handle, dev(env, X), 16, 16, dev(env, W), 16, dev(env, nu), None, "none", Y, 16)
    ref = oracle.rgcn_fwd(env["ip"], env["ix"], env["et"], X, W, nu)
    assert rel_err(Y.cpu().numpy(), ref) <= TOL


@pytest.mark.parametrize("Fin,Fout", [(16, 16), (16, 11), (4, 5), (8, 32)])
def test_rgcn_bwd(env, Fin, Fout):
    torch, L, g, N, R = env["torch"], env["L"], env["g"], env["N"], env["R"]
    ldx, ldd = (Fin + 3) // 4 * 4, (Fout + 3) // 4 * 4
    X, W, dA = rnd(11, (N, Fin)), rnd(12, (R, Fin, Fout)), rnd(13, (N, Fout))
    dX = torch.full((N, ldx), float("nan"), device="cuda")
    dW = torch.empty((R, Fin, Fout), device="cuda")
    ws_b = L.seastar_rgcn_bwd_workspace(g.handle, Fin, Fout)
    ws = torch.empty(ws_b, dtype=torch.uint8, device="cuda")
    Z = rnd(14, (N, Fin)).astype(np.float64)           # fused activation backward on dX
    Yact = oracle.act_fwd("relu", Z).astype(np.float32)
    L.seastar_rgcn_bwd(g.handle, dev(env, padded(X, ldx)), Fin, ldx, dev(env, padded(dA, ldd)), Fout, ldd,
                       dev(env, W), None, dev(env, padded(Yact, ldx)), "relu", dX, dW, ws, ws_b)
    rdX, rdW = oracle.rgcn_bwd(env["ip"], env["ix"], env["et"], X, W, dA)
    assert rel_err(dX.cpu().numpy()[:, :Fin], oracle.act_bwd("relu", Z, rdX)) <= TOL
    assert rel_err(dW.cpu().numpy(), rdW) <= TOL
    # deterministic run to run (no atomics anywhere in the R-GCN backward)
    dW2 = torch.empty_like(dW)
    dX2 = torch.empty_like(dX)
    L.seastar_rgcn_bwd(g.handle, dev(env, padded(X, ldx)), Fin, ldx, dev(env, padded(dA, ldd)), Fout, ldd,
                       dev(env, W), None, None, "none", dX2, dW2, ws, ws_b)
    assert torch.equal(dW, dW2)
    assert rel_err(dX2.cpu().numpy()[:, :Fin], rdX) <= TOL


@pytest.fixture
def path(request, monkeypatch):
    """The R-GCN forward / dX formulation: "tile" (default: edge-balanced tiles with a CTA-local type grouping,
    rgcn_tile.cu, persistent CTAs with W resident in shared memory), "standalone" (SEASTAR_RGCN_TILE_STANDALONE=1:
    one tile per CTA, W through L1/L2), "rows" (SEASTAR_RGCN_ROWS=1: the one-pass row kernel, W_r in shared memory per type run) or
    "twophase" (SEASTAR_RGCN_TWOPHASE=1: lane-per-edge products in type-major order + per-row sums)."""
    monkeypatch.delenv("SEASTAR_RGCN_TWOPHASE", raising=False)
    monkeypatch.delenv("SEASTAR_RGCN_ROWS", raising=False)
    monkeypatch.delenv("SEASTAR_RGCN_TILE_STANDALONE", raising=False)
    if request.param == "standalone":
        monkeypatch.setenv("SEASTAR_RGCN_TILE_STANDALONE", "1")
    if request.param == "rows":
        monkeypatch.setenv("SEASTAR_RGCN_ROWS", "1")
    elif request.param == "twophase":
        monkeypatch.setenv("SEASTAR_RGCN_TWOPHASE", "1")
    return request.param


@pytest.mark.parametrize("path", ["tile", "standalone", "rows", "twophase"], indirect=True)
@pytest.mark.parametrize("Fin,Fout", [(16, 16), (16, 11), (3, 7)])
def test_rgcn_paths(env, path, Fin, Fout):
    """Every R-GCN formulation against the oracle, forward and dX, with a hub row of 1,500 typed in-edges (two tile
    borders inside it) and rows without in-edges."""
    torch, L, g, N, R = env["torch"], env["L"], env["g"], env["N"], env["R"]
    ws_f = L.seastar_rgcn_fwd_workspace(g.handle, Fin, Fout)
    assert (ws_f == 0) == (path == "rows")
    ldx, ldy = (Fin + 3) // 4 * 4, (Fout + 3) // 4 * 4
    X, W, b = rnd(21, (N, Fin)), rnd(22, (R, Fin, Fout)), rnd(23, (Fout,))
    Y = torch.full((N, ldy), float("nan"), device="cuda")
    L.seastar_rgcn_fwd(g.handle, dev(env, padded(X, ldx)), Fin, ldx, dev(env, W), Fout, None, dev(env, b), "elu", Y,
                       ldy)
    ref = oracle.act_fwd("elu", oracle.rgcn_fwd(env["ip"], env["ix"], env["et"], X, W) + b)
    assert rel_err(Y.cpu().numpy()[:, :Fout], ref) <= TOL
    dA = rnd(24, (N, Fout))
    dX = torch.full((N, ldx), float("nan"), device="cuda")
    ws_b = L.seastar_rgcn_bwd_workspace(g.handle, Fin, Fout)
    ws = torch.empty(ws_b, dtype=torch.uint8, device="cuda")
    L.seastar_rgcn_bwd(g.handle, dev(env, padded(X, ldx)), Fin, ldx, dev(env, padded(dA, ldy)), Fout, ldy,
                       dev(env, W), None, None, "none", dX, None, ws, ws_b)
    rdX, _ = oracle.rgcn_bwd(env["ip"], env["ix"], env["et"], X, W, dA, need_dW=False)
    assert rel_err(dX.cpu().numpy()[:, :Fin], rdX) <= TOL


@pytest.mark.parametrize("degs", [
    [1024, 1024, 512, 512, 256, 256, 256, 256],          # rows ending exactly on 1,024-edge borders
    [512, 512, 256, 256, 128, 128, 128, 128],             # ... on 512-edge borders (the default tile)
    [3000, 1025, 1023, 7, 1, 1, 1],                       # a row over three tiles, rows cut by every border
    [5000],                                               # one row, five tiles
    [1] * 2500,                                           # a row per edge: a whole tile of rows
    [40] * 300,                                           # rows cut by most borders, several tiles per CTA
])
def test_rgcn_tile_borders(degs):
    """Edge-balanced tiles (512 edges by default, RGCN_TILE_EDGES): rows cut by tile borders are summed over their tiles in tile order; rows
    without edges get the epilogue of 0.  Forward, dX (over the out-degrees) and dW against the oracle."""
    import torch
    from paper_conf_eurosys_wumcjlzcy21_b200 import _lib as L
    from paper_conf_eurosys_wumcjlzcy21_b200.graph import Graph
    R, Fin, Fout = 9, 16, 11
    N = max(len(degs) + 5, 64)
    rng = np.random.default_rng(sum(degs) + len(degs))
    dst = np.repeat(np.arange(len(degs)), degs)
    src = rng.integers(0, N, dst.size)
    et = rng.integers(0, R, dst.size)
    ip, ix, et = synth.csr_from_edges(N, src, dst, et)
    g = Graph(ip, ix, et, num_etypes=R, rgcn_norm=True)
    ldx, ldy = 16, 12
    X, W, b = rnd(41, (N, Fin)), rnd(42, (R, Fin, Fout)), rnd(43, (Fout,))
    Y = torch.full((N, ldy), float("nan"), device="cuda")
    L.seastar_rgcn_fwd(g.handle, torch.from_numpy(X).cuda(), Fin, ldx, torch.from_numpy(W).cuda(), Fout, None,
                       torch.from_numpy(b).cuda(), "relu", Y, ldy)
    ref = oracle.act_fwd("relu", oracle.rgcn_fwd(ip, ix, et, X, W) + b)
    assert rel_err(Y.cpu().numpy()[:, :Fout], ref) <= TOL
    dA = rnd(44, (N, Fout))
    dX = torch.full((N, ldx), float("nan"), device="cuda")
    dW = torch.empty((R, Fin, Fout), device="cuda")
    ws_b = L.seastar_rgcn_bwd_workspace(g.handle, Fin, Fout)
    ws = torch.empty(ws_b, dtype=torch.uint8, device="cuda")
    L.seastar_rgcn_bwd(g.handle, torch.from_numpy(X).cuda(), Fin, ldx, torch.from_numpy(padded(dA, ldy)).cuda(), Fout,
                       ldy, torch.from_numpy(W).cuda(), None, None, "none", dX, dW, ws, ws_b)
    rdX, rdW = oracle.rgcn_bwd(ip, ix, et, X, W, dA)
    assert rel_err(dX.cpu().numpy()[:, :Fin], rdX) <= TOL
    assert rel_err(dW.cpu().numpy(), rdW) <= TOL


def test_rgcn_fwd_workspace_required(env, monkeypatch):
    monkeypatch.setenv("SEASTAR_RGCN_TWOPHASE", "1")
    torch, L, g = env["torch"], env["L"], env["g"]
    need = L.seastar_rgcn_fwd_workspace(g.handle, 16, 16)
    assert need > 0
    X = torch.zeros((env["N"], 16), device="cuda")
    W = torch.zeros((env["R"], 16, 16), device="cuda")
    Y = torch.zeros((env["N"], 16), device="cuda")
    small = torch.empty(need - 256, dtype=torch.uint8, device="cuda")
    with pytest.raises(RuntimeError, match="workspace"):
        L.seastar_rgcn_fwd(g.handle, X, 16, 16, W, 16, None, None, "none", Y, 16, small, small.numel())


@pytest.mark.parametrize("R,Fin,Fout,ok", [(210, 32, 8, True), (240, 32, 8, False), (1200, 4, 4, True)])
def test_rgcn_shared_memory_limit(R, Fin, Fout, ok):
    """at R = 210 the padded W table (stride 272 floats) no longer fits but the dense one (256) does;
    R = 240 exceeds the shared memory of an SM (UNSUPPORTED); narrow layers with many relations (R = 1200, 4 x 4:
    76 KB padded, 77 KB) fit."""
    import torch
    from paper_conf_eurosys_wumcjlzcy21_b200 import _lib as L
    from paper_conf_eurosys_wumcjlzcy21_b200.graph import Graph
    N = 3000
    ip, ix, et = synth.powerlaw_directed_typed(N, 20000, 0.6, 0.6, R, 1.0, 23)
    g = Graph(ip, ix, et, num_etypes=R, rgcn_norm=True)
    X, W = rnd(31, (N, Fin)), rnd(32, (R, Fin, Fout))
    Y = torch.empty((N, Fout), device="cuda")
    if not ok:
        with pytest.raises(RuntimeError, match="does not fit"):
            L.seastar_rgcn_fwd(g.handle, torch.from_numpy(X).cuda(), Fin, Fin, torch.from_numpy(W).cuda(), Fout, None,
                               None, "none", Y, Fout)
        return
    L.seastar_rgcn_fwd(g.handle, torch.from_numpy(X).cuda(), Fin, Fin, torch.from_numpy(W).cuda(), Fout, None, None,
                       "none", Y, Fout)
    assert rel_err(Y.cpu().numpy(), oracle.rgcn_fwd(ip, ix, et, X, W)) <= TOL
