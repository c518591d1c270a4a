"""Parity at BASELINE.json's full sizes, in the launch configuration bench.py times.

Every config of BASELINE.json is built by ``synth.workload`` -- the same
seeded graph, features, labels and initial parameters the benchmark uses -- and one training step
of its model (forward, softmax cross-entropy, backward) runs through the C ABI exactly as
``bench.py`` (and ``bench.py --workload``) launches it: X padded to a 16-byte row stride for the
TMA-fed dense transform, the same model classes and options.  The oracle composition
(``model_ref``, fp64 edge loops) runs on the whole graph, so the comparison is element by element
over every output row, not a sample:

* a1-a2 on the Reddit shape (114.6 M edges): forward and reverse CSR bit-exact;
* loss, the hidden activations and every parameter gradient within 1e-5 (north_star tolerance,
  max-abs normalised per tensor).

These are the slowest GPU tests (the oracle needs ~1-2 CPU-minutes for the Reddit GAT step).
"""
import json
import os

import numpy as np
import pytest

import oracle
import synth
from conftest import rel_err
from oracle import model_ref
import kinks

pytestmark = pytest.mark.gpu
TOL = 1e-5


@pytest.fixture(scope="module")
def env():
    import torch
    assert torch.cuda.is_available()
    from paper_conf_eurosys_wumcjlzcy21_b200 import models
    from paper_conf_eurosys_wumcjlzcy21_b200.graph import Graph
    return dict(torch=torch, models=models, Graph=Graph)


_W = {}


def workload(name):
    if name not in _W:
        _W.clear()                     # keep at most one full-size input set in host memory
        _W[name] = synth.workload(name)
    return _W[name]


def device_X(env, X):
    """bench.py's layout: rows padded to a multiple of 4 floats (TMA row stride), unpadded view."""
    torch = env["torch"]
    N, F = X.shape
    Xp = torch.zeros((N, (F + 3) // 4 * 4), device="cuda")
    Xp[:, :F].copy_(torch.from_numpy(X))
    return Xp[:, :F]


def f64(p):
    return {k: np.asarray(v, np.float64) for k, v in p.items()}


def check_step(model, loss_ref, grads_ref, acts, envelope=None, n_ambiguous=0):
    """Every tensor's max-abs-normalised error is computed (and printed) before any assert, so a
    failure shows the whole error profile of the step.  ``envelope`` (tests/kinks.py) adds, per
    gradient element, the bound on what the ambiguous ReLU / LeakyReLU decisions can change."""
    envelope = envelope or {}
    loss = model.forward()
    model.backward()
    errs = {"loss": abs(loss.item() - loss_ref) / abs(loss_ref)}
    for name, (got, ref) in acts.items():
        errs[name] = rel_err(got().cpu().numpy(), ref)
    excess, width = {}, {}
    grad = getattr(model, "grad", model.P.g)
    for k, ref in grads_ref.items():
        got = grad(k).cpu().numpy().astype(np.float64)
        ref = ref.reshape(got.shape)
        errs["d" + k] = rel_err(got, ref)
        if k in envelope:
            den = np.abs(ref).max() or 1.0
            excess["d" + k] = float(np.maximum(np.abs(got - ref) - envelope[k].reshape(got.shape), 0).max() / den)
            width["d" + k] = float(envelope[k].max() / den)
    log = os.environ.get("SEASTAR_PARITY_LOG")
    if log:                     # committed under profiles/ from the GPU runs
        with open(log, "a") as f:
            f.write(json.dumps({"test": os.environ.get("PYTEST_CURRENT_TEST", "?").split(" ")[0], "tol": TOL,
                                "rel_err": errs, "ambiguous_kink_decisions": int(n_ambiguous),
                                "envelope_over_maxref": width, "error_beyond_envelope": excess}) + "\n")
    print("\nrel errors:", {k: f"{v:.2e}" for k, v in errs.items()}, "| ambiguous kink decisions:", n_ambiguous,
          "| envelope / max|ref|:", {k: f"{v:.2e}" for k, v in width.items()},
          "| error beyond the envelope:", {k: f"{v:.2e}" for k, v in excess.items()})
    bad = {k: v for k, v in errs.items() if not v <= TOL and not (k in excess and excess[k] <= TOL)}
    assert not bad, bad


def gat_envelope(ip, ix, acts, heads, hid, C):
    env, na = {}, 0
    for l, (H, F) in enumerate([(heads, hid), (1, C)], start=1):
        e, n = kinks.gat_layer(ip, ix, acts["layers"][l - 1], H, F)
        env.update({f"W{l}": e["W"], f"al{l}": e["al"], f"ar{l}": e["ar"]})
        na += n
    return env, na


# ---------------------------------------------------------------------------------------------
# configs[4]: Reddit-shaped (the bench workload)
# ---------------------------------------------------------------------------------------------
def test_reddit_preprocess_bitexact(env):
    w = workload("reddit")
    ip, ix = w["indptr"], w["indices"]
    g = env["Graph"](ip, ix)
    o = oracle.preprocess(ip, ix)
    f = {k: v.cpu().numpy() for k, v in g.export("fwd").items()}
    for k, ok in [("perm", "fwd_perm"), ("off", "fwd_off"), ("nbr", "fwd_src"), ("eid", "fwd_eid")]:
        assert np.array_equal(f[k], o[ok]), k
    del f
    r = {k: v.cpu().numpy() for k, v in g.export("rev").items()}
    for k, ok in [("perm", "rev_perm"), ("off", "rev_off"), ("nbr", "rev_dst"), ("eid", "rev_eid"),
                  ("pos", "rev_pos")]:
        assert np.array_equal(r[k], o[ok]), k
    info = g.info
    assert info["num_fwd_edges"] == info["num_rev_edges"] == w["cfg"].E


def test_reddit_gcn2_step(env):
    w = workload("reddit")
    ip, ix, X, lab = w["indptr"], w["indices"], w["X"], w["labels"]
    g = env["Graph"](ip, ix)
    m = env["models"].GCN2(g, device_X(env, X), env["torch"].from_numpy(lab).cuda(), w["gcn"])
    acts = {}
    loss, grads = model_ref.gcn2(ip, ix, X, lab, f64(w["gcn"]), acts)
    env, na = kinks.relu_gcn(ip, ix, X, acts["Z1"], acts["dH1"], {k: grads[k].shape for k in ("W1", "b1")})
    check_step(m, loss, grads, {"H1": (lambda: m.H1, acts["H1"]),
                                "logits": (lambda: m.logits[:, :m.C], acts["logits"])}, env, na)


def test_reddit_gat2_step(env):
    w = workload("reddit")
    ip, ix, X, lab = w["indptr"], w["indices"], w["X"], w["labels"]
    cfg = w["cfg"]
    heads, hid = cfg.heads, cfg.extra["gat_hidden"]
    g = env["Graph"](ip, ix)
    m = env["models"].GAT2(g, device_X(env, X), env["torch"].from_numpy(lab).cuda(), w["gat"], heads, hid)
    acts = {}
    loss, grads = model_ref.gat2(ip, ix, X, lab, f64(w["gat"]), heads, hid, acts)
    env, na = gat_envelope(ip, ix, acts, heads, hid, cfg.classes)
    check_step(m, loss, grads, {"Y1": (lambda: m.Y1[:, :heads * hid], acts["Y1"]),
                                "Y2": (lambda: m.Y2[:, :m.C], acts["Y2"])}, env, na)


# ---------------------------------------------------------------------------------------------
# configs[0..3]
# ---------------------------------------------------------------------------------------------
def test_cora_gcn2_step(env):
    w = workload("cora_gcn")
    ip, ix, X, lab = w["indptr"], w["indices"], w["X"], w["labels"]
    m = env["models"].GCN2(env["Graph"](ip, ix), device_X(env, X), env["torch"].from_numpy(lab).cuda(), w["gcn"])
    acts = {}
    loss, grads = model_ref.gcn2(ip, ix, X, lab, f64(w["gcn"]), acts)
    env, na = kinks.relu_gcn(ip, ix, X, acts["Z1"], acts["dH1"], {k: grads[k].shape for k in ("W1", "b1")})
    check_step(m, loss, grads, {"H1": (lambda: m.H1, acts["H1"])}, env, na)


def test_corafull_gat2_step(env):
    w = workload("corafull_gat")
    ip, ix, X, lab = w["indptr"], w["indices"], w["X"], w["labels"]
    cfg = w["cfg"]
    m = env["models"].GAT2(env["Graph"](ip, ix), device_X(env, X), env["torch"].from_numpy(lab).cuda(), w["gat"],
                           cfg.heads, cfg.hidden)
    acts = {}
    loss, grads = model_ref.gat2(ip, ix, X, lab, f64(w["gat"]), cfg.heads, cfg.hidden, acts)
    env, na = gat_envelope(ip, ix, acts, cfg.heads, cfg.hidden, cfg.classes)
    check_step(m, loss, grads, {"Y1": (lambda: m.Y1[:, :cfg.heads * cfg.hidden], acts["Y1"])}, env, na)


def test_physics_appnp_step(env):
    w = workload("physics_appnp")
    ip, ix, X, lab = w["indptr"], w["indices"], w["X"], w["labels"]
    cfg = w["cfg"]
    m = env["models"].APPNPNet(env["Graph"](ip, ix), device_X(env, X), env["torch"].from_numpy(lab).cuda(),
                               w["appnp"], K=cfg.K, alpha=cfg.alpha)
    acts = {}
    loss, grads = model_ref.appnp(ip, ix, X, lab, f64(w["appnp"]), cfg.K, cfg.alpha, acts)
    env, na = kinks.relu_mlp(X, acts["Z1"], acts["dH1"], {k: grads[k].shape for k in ("W1", "b1")})
    check_step(m, loss, grads, {"Z": (lambda: m.Z[cfg.K][:, :cfg.classes], acts["Z"])}, env, na)


def test_am_rgcn2_step(env):
    w = workload("am_rgcn")
    ip, ix, et, X, lab = w["indptr"], w["indices"], w["etypes"], w["X"], w["labels"]
    cfg = w["cfg"]
    g = env["Graph"](ip, ix, et, num_etypes=cfg.R, rgcn_norm=True)
    o = oracle.preprocess(ip, ix, et)
    f = {k: v.cpu().numpy() for k, v in g.export("fwd").items()}
    for k, ok in [("perm", "fwd_perm"), ("off", "fwd_off"), ("nbr", "fwd_src"), ("eid", "fwd_eid"),
                  ("type", "fwd_type")]:
        assert np.array_equal(f[k], o[ok]), k
    m = env["models"].RGCN2(g, device_X(env, X), env["torch"].from_numpy(lab).cuda(), w["rgcn"])
    acts = {}
    loss, grads = model_ref.rgcn2(ip, ix, et, X, lab, f64(w["rgcn"]), acts)
    env, na = kinks.relu_rgcn(ip, ix, et, cfg.R, X, acts["Z1"], acts["dH1"], {k: grads[k].shape for k in ("W1", "b1")})
    check_step(m, loss, grads, {"H1": (lambda: m.H1[:, :cfg.hidden], acts["H1"])}, env, na)


# ---------------------------------------------------------------------------------------------
# NEXT-2: R-GCN as the paper ran it (featureless input, bases), Table 2 shapes
# ---------------------------------------------------------------------------------------------
@pytest.mark.parametrize("name", ["aifb_rgcnb", "mutag_rgcnb", "bgs_rgcnb"])
def test_rgcnb2_step(env, name):
    w = workload(name)
    ip, ix, et, lab = w["indptr"], w["indices"], w["etypes"], w["labels"]
    cfg = w["cfg"]
    g = env["Graph"](ip, ix, et, num_etypes=cfg.R, rgcn_norm=True)
    m = env["models"].RGCNBasis2(g, env["torch"].from_numpy(lab).cuda(), w["rgcnb"])
    acts = {}
    p = f64(w["rgcnb"])
    loss, grads = model_ref.rgcnb2(ip, ix, et, lab, p, acts)
    envl, na = kinks.relu_rgcnb(ip, ix, et, cfg.R, p["V1"], p["a1"], acts["Z1"], acts["dH1"],
                                {k: grads[k].shape for k in ("V1", "a1", "b1")})
    check_step(m, loss, grads, {"H1": (lambda: m.H1[:, :cfg.hidden], acts["H1"])}, envl, na)
