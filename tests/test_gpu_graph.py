"""a1-a3 on the GPU: bit-exact against the oracle (and Fig. 7) through the C ABI."""
import json
import os

import numpy as np
import pytest

import oracle
import synth
from helpers import hub_graph

pytestmark = pytest.mark.gpu
GOLD = os.path.join(os.path.dirname(__file__), "golden")


@pytest.fixture(scope="module")
def G():
    import torch
    assert torch.cuda.is_available(), "GPU tests need a B200"
    from paper_conf_eurosys_wumcjlzcy21_b200.graph import Graph
    return Graph


def exported(g, which):
    return {k: v.cpu().numpy().astype(np.int64) for k, v in g.export(which).items()}


def compare(g, o, partitioned=False):
    f = exported(g, "fwd")
    r = exported(g, "rev")
    assert np.array_equal(f["perm"], o["fwd_perm"])
    assert np.array_equal(f["off"], o["fwd_off"])
    assert np.array_equal(f["nbr"], o["fwd_src"])
    assert np.array_equal(f["eid"], o["fwd_eid"])
    assert np.array_equal(r["perm"], o["rev_perm"])
    assert np.array_equal(r["off"], o["rev_off"])
    assert np.array_equal(r["nbr"], o["rev_dst"])
    assert np.array_equal(r["eid"], o["rev_eid"])
    assert np.array_equal(r["pos"], o["rev_pos"])
    if "type" in f:
        assert np.array_equal(f["type"], o["fwd_type"])
        assert np.array_equal(r["type"], o["rev_type"])
    if partitioned:
        s = exported(g, "lsf")
        assert np.array_equal(s["off"], o["lsf_off"])
        assert np.array_equal(s["eid"], o["lsf_eid"])


@pytest.mark.parametrize("fixture", ["fig7.json", "fig7_relabelled.json"])
def test_fig7(G, fixture):
    d = json.load(open(os.path.join(GOLD, fixture)))
    g = G(np.array(d["indptr"]), np.array(d["indices"]))
    f, r = exported(g, "fwd"), exported(g, "rev")
    for k, arr in [("fwd_perm", f["perm"]), ("fwd_off", f["off"]), ("fwd_src", f["nbr"]), ("fwd_eid", f["eid"]),
                   ("rev_perm", r["perm"]), ("rev_off", r["off"]), ("rev_dst", r["nbr"]), ("rev_eid", r["eid"]),
                   ("rev_pos", r["pos"])]:
        assert arr.tolist() == d[k], k


@pytest.mark.parametrize("seed,N,E,R", [(1, 1, 3, 0), (2, 7, 20, 0), (3, 30, 200, 0), (4, 50, 400, 5),
                                        (5, 64, 64, 3), (6, 17, 0, 0), (7, 300, 5000, 17)])
def test_random_graphs(G, seed, N, E, R):
    if E == 0:
        ip, ix, et = np.zeros(N + 1, np.int64), np.zeros(0, np.int64), None
    elif R:
        ip, ix, et = synth.random_graph(N, E, seed, R)
    else:
        (ip, ix), et = synth.random_graph(N, E, seed), None
    g = G(ip, ix, et, num_etypes=R)
    compare(g, oracle.preprocess(ip, ix, et))


def test_hub_graph_and_buckets(G):
    ip, ix = hub_graph()
    g = G(ip, ix)
    o = oracle.preprocess(ip, ix)
    compare(g, o)
    for key, off in (("fwd_bucket_rows", o["fwd_off"]), ("rev_bucket_rows", o["rev_off"])):
        deg = np.diff(off)
        want = [int((deg >= t).sum()) for t in (1024, 32, 1)] + [len(deg)]
        assert g.info[key] == want, key
    assert g.info["max_in_degree"] == np.diff(ip).max()


@pytest.mark.parametrize("P", [2, 3])
def test_partitions(G, P):
    ip, ix, et = synth.random_graph(400, 6000, 21, 6)
    N = 400
    for p in range(P):
        rb, re = N * p // P, N * (p + 1) // P
        g = G(ip, ix, et, num_etypes=6, row_begin=rb, row_end=re)
        compare(g, oracle.preprocess(ip, ix, et, rb, re), partitioned=True)


def test_typed_powerlaw_and_rgcn_norm(G):
    ip, ix, et = synth.powerlaw_directed_typed(5000, 40000, 0.6, 0.6, 33, 1.0, 8)
    g = G(ip, ix, et, num_etypes=33, rgcn_norm=True)
    o = oracle.preprocess(ip, ix, et)
    compare(g, o)
    nrm = oracle.rgcn_norm(ip, et, 33)
    f, r = g.export("fwd"), g.export("rev")
    np.testing.assert_allclose(f["norm"].cpu().numpy(), nrm[o["fwd_eid"]], rtol=1e-7)
    np.testing.assert_allclose(r["norm"].cpu().numpy(), nrm[o["rev_eid"]], rtol=1e-7)


def test_degree_norms(G):
    ip, ix = hub_graph(N=500, E_dir=4000, hub_deg=50)
    g = G(ip, ix)
    in_n, out_n = oracle.degree_norms(ip, ix)
    s, d = g.degree_norms("both")
    np.testing.assert_allclose(s.cpu().numpy(), out_n, rtol=1e-6)
    np.testing.assert_allclose(d.cpu().numpy(), in_n, rtol=1e-6)
    s, d = g.degree_norms("in")
    np.testing.assert_allclose(s.cpu().numpy(), in_n, rtol=1e-6)


def test_invalid_graphs_rejected(G):
    from paper_conf_eurosys_wumcjlzcy21_b200 import SeastarError
    with pytest.raises(SeastarError, match="INVALID_GRAPH"):
        G(np.array([0, 2, 1, 3]), np.array([0, 1, 2]))          # non-monotone indptr
    with pytest.raises(SeastarError, match="INVALID_GRAPH"):
        G(np.array([0, 1, 2]), np.array([0, 5]))                 # source out of range
    with pytest.raises(SeastarError, match="INVALID_ARGUMENT"):
        G(np.array([0, 1, 2]), np.array([0, 1]), row_begin=2, row_end=1)
