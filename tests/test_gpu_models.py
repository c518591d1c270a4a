"""End-to-end parity: one forward + backward of each model through the C ABI (models.py) vs the
oracle composition (model_ref.py): loss and every parameter gradient, then one Adam step."""
import numpy as np
import pytest

import oracle
import synth
from conftest import rel_err
from oracle import model_ref

pytestmark = pytest.mark.gpu
TOL = 1e-5


@pytest.fixture(scope="module")
def env():
    import torch
    assert torch.cuda.is_available()
    from paper_conf_eurosys_wumcjlzcy21_b200 import models
    from paper_conf_eurosys_wumcjlzcy21_b200.graph import Graph
    return dict(torch=torch, models=models, Graph=Graph)


def dev(env, a):
    return env["torch"].from_numpy(np.ascontiguousarray(a)).cuda()


def check(model, loss_ref, grads_ref):
    loss = model.forward()
    model.backward()
    assert abs(loss.item() - loss_ref) <= TOL * abs(loss_ref)
    grad = getattr(model, "grad", model.P.g)
    for k, ref in grads_ref.items():
        got = grad(k).cpu().numpy()
        assert rel_err(got, ref.reshape(got.shape)) <= TOL, k


def test_gcn2(env):
    ip, ix = synth.powerlaw_sym(2000, 16000, 0.6, 31)
    N, Fin, H, C = 2000, 300, 16, 7
    X, lab = synth.uniform(1, (N, Fin)), synth.labels(2, N, C)
    p = {"W1": synth.glorot(3, Fin, H), "b1": synth.uniform(4, (H,), -0.1, 0.1),
         "W2": synth.glorot(5, H, C), "b2": synth.uniform(6, (C,), -0.1, 0.1)}
    m = env["models"].GCN2(env["Graph"](ip, ix), dev(env, X), dev(env, lab), p)
    check(m, *model_ref.gcn2(ip, ix, X, lab, {k: v.astype(np.float64) for k, v in p.items()}))
    m.P.adam(0.01)                                            # one optimiser step runs and moves the weights
    assert not np.array_equal(m.P.p("W1").cpu().numpy(), p["W1"])


@pytest.mark.parametrize("save_B", [True, False])
def test_gat2(env, save_B):
    ip, ix = synth.powerlaw_sym(1500, 12000, 0.6, 32)
    N, Fin, heads, hid, C = 1500, 200, 8, 8, 41
    X, lab = synth.uniform(11, (N, Fin)), synth.labels(12, N, C)
    p = {"W1": synth.glorot(13, Fin, heads * hid), "al1": synth.uniform(14, (heads, hid), -0.5, 0.5),
         "ar1": synth.uniform(15, (heads, hid), -0.5, 0.5), "b1": synth.uniform(16, (heads * hid,), -0.1, 0.1),
         "W2": synth.glorot(17, heads * hid, C), "al2": synth.uniform(18, (1, C), -0.5, 0.5),
         "ar2": synth.uniform(19, (1, C), -0.5, 0.5), "b2": synth.uniform(20, (C,), -0.1, 0.1)}
    m = env["models"].GAT2(env["Graph"](ip, ix), dev(env, X), dev(env, lab), p, heads, hid, save_der_factors=save_B)
    check(m, *model_ref.gat2(ip, ix, X, lab, {k: v.astype(np.float64) for k, v in p.items()}, heads, hid))


def test_appnp(env):
    ip, ix = synth.powerlaw_sym(1800, 15000, 0.5, 33)
    N, Fin, Hd, C, K = 1800, 150, 64, 5, 10
    X, lab = synth.uniform(21, (N, Fin)), synth.labels(22, N, C)
    p = {"W1": synth.glorot(23, Fin, Hd), "b1": synth.uniform(24, (Hd,), -0.1, 0.1),
         "W2": synth.glorot(25, Hd, C), "b2": synth.uniform(26, (C,), -0.1, 0.1)}
    m = env["models"].APPNPNet(env["Graph"](ip, ix), dev(env, X), dev(env, lab), p, K=K, alpha=0.1)
    check(m, *model_ref.appnp(ip, ix, X, lab, {k: v.astype(np.float64) for k, v in p.items()}, K, 0.1))


def test_rgcn2(env):
    N, R, Fin, Hd, C = 3000, 20, 16, 16, 11
    ip, ix, et = synth.powerlaw_directed_typed(N, 12000, 0.6, 0.6, R, 1.0, 34)
    X, lab = synth.uniform(31, (N, Fin)), synth.labels(32, N, C)
    p = {"W1": synth.glorot(33, Fin, Hd, (R, Fin, Hd)), "b1": synth.uniform(34, (Hd,), -0.1, 0.1),
         "W2": synth.glorot(35, Hd, C, (R, Hd, C)), "b2": synth.uniform(36, (C,), -0.1, 0.1)}
    g = env["Graph"](ip, ix, et, num_etypes=R, rgcn_norm=True)
    m = env["models"].RGCN2(g, dev(env, X), dev(env, lab), p)
    check(m, *model_ref.rgcn2(ip, ix, et, X, lab, {k: v.astype(np.float64) for k, v in p.items()}))


def test_rgcnb2(env):
    """NEXT-2: featureless input layer with bases + dense basis output layer (aifb-like shape, B < R)."""
    N, R, B1, B2, Hd, C = 2500, 30, 12, 6, 16, 4
    ip, ix, et = synth.powerlaw_directed_typed(N, 18000, 0.6, 0.6, R, 1.0, 35)
    lab = synth.labels(36, N, C)
    p = {"V1": synth.uniform(37, (N, B1, Hd), -0.5, 0.5), "a1": synth.uniform(38, (R, B1)),
         "b1": synth.uniform(39, (Hd,), -0.1, 0.1), "V2": synth.uniform(40, (B2, Hd, C), -0.5, 0.5),
         "a2": synth.uniform(41, (R, B2)), "b2": synth.uniform(42, (C,), -0.1, 0.1)}
    g = env["Graph"](ip, ix, et, num_etypes=R, rgcn_norm=True)
    m = env["models"].RGCNBasis2(g, dev(env, lab), p)
    check(m, *model_ref.rgcnb2(ip, ix, et, lab, {k: v.astype(np.float64) for k, v in p.items()}))
    m.epoch()
    assert not np.array_equal(m.param("V1").cpu().numpy(), p["V1"])
