"""Pins for the oracle's graph representation (rows a1-a3).

* Fig. 7 of the paper, exact arrays, and a hand-relabelled copy.
* Brute force on small random graphs: Python ``sorted`` with the stated keys, and a naive
  O(E) transpose written independently here.
"""
import json
import os

import numpy as np
import pytest

import oracle
import synth

GOLD = os.path.join(os.path.dirname(__file__), "golden")
KEYS = ["fwd_perm", "fwd_off", "fwd_src", "fwd_eid", "rev_perm", "rev_off", "rev_dst", "rev_eid", "rev_pos"]


@pytest.mark.parametrize("fixture", ["fig7.json", "fig7_relabelled.json"])
def test_fig7_exact(fixture):
    g = json.load(open(os.path.join(GOLD, fixture)))
    o = oracle.preprocess(np.array(g["indptr"]), np.array(g["indices"]))
    for k in KEYS:
        assert o[k].tolist() == g[k], (fixture, k, o[k].tolist(), g[k])


def brute(indptr, indices, etypes=None, rb=0, re=None):
    """Independent brute force of L301 / L461-L463 / L475 with Python lists."""
    N = len(indptr) - 1
    re = N if re is None else re
    E = int(indptr[-1])
    dst = [v for v in range(N) for _ in range(indptr[v], indptr[v + 1])]
    src = [int(x) for x in indices]
    typ = [0] * E if etypes is None else [int(t) for t in etypes]
    indeg = [indptr[v + 1] - indptr[v] for v in range(N)]
    outdeg = [0] * N
    for s in src:
        outdeg[s] += 1
    owned = list(range(rb, re))
    fperm = sorted(owned, key=lambda v: (-indeg[v], v))
    f_eid = []
    f_off = [0]
    for v in fperm:
        row = sorted([e for e in range(E) if dst[e] == v], key=lambda e: (typ[e], e))
        f_eid += row
        f_off.append(len(f_eid))
    rperm = sorted(owned, key=lambda u: (-outdeg[u], u))
    r_eid = []
    r_off = [0]
    for u in rperm:
        row = sorted([e for e in range(E) if src[e] == u], key=lambda e: (typ[e], e))
        r_eid += row
        r_off.append(len(r_eid))
    if rb == 0 and re == N:
        pos = {e: i for i, e in enumerate(f_eid)}
    else:
        lsf = sorted([e for e in range(E) if rb <= src[e] < re], key=lambda e: (dst[e], typ[e], e))
        pos = {e: i for i, e in enumerate(lsf)}
    return {
        "fwd_perm": fperm, "fwd_off": f_off, "fwd_eid": f_eid, "fwd_src": [src[e] for e in f_eid],
        "fwd_type": [typ[e] for e in f_eid],
        "rev_perm": rperm, "rev_off": r_off, "rev_eid": r_eid, "rev_dst": [dst[e] for e in r_eid],
        "rev_type": [typ[e] for e in r_eid], "rev_pos": [pos[e] for e in r_eid],
    }


@pytest.mark.parametrize("seed,N,E,R", [(1, 1, 3, 0), (2, 7, 20, 0), (3, 30, 200, 0), (4, 50, 400, 5),
                                        (5, 64, 64, 3), (6, 17, 0, 0)])
def test_random_vs_brute(seed, N, E, R):
    if E == 0:
        indptr, indices = np.zeros(N + 1, np.int64), np.zeros(0, np.int64)
        et = None
    elif R:
        indptr, indices, et = synth.random_graph(N, E, seed, R)
    else:
        indptr, indices = synth.random_graph(N, E, seed)
        et = None
    o = oracle.preprocess(indptr, indices, et)
    b = brute(indptr.tolist(), indices.tolist(), None if et is None else et.tolist())
    for k in b:
        assert o[k].tolist() == b[k], k


@pytest.mark.parametrize("P", [2, 3])
def test_partial_ranges_vs_brute(P):
    N, E, R = 40, 300, 4
    indptr, indices, et = synth.random_graph(N, E, 11, R)
    bounds = [N * p // P for p in range(P + 1)]
    seen_fwd, seen_rev = [], []
    for p in range(P):
        rb, re = bounds[p], bounds[p + 1]
        o = oracle.preprocess(indptr, indices, et, rb, re)
        b = brute(indptr.tolist(), indices.tolist(), et.tolist(), rb, re)
        for k in b:
            assert o[k].tolist() == b[k], (p, k)
        # LSF index is consistent with rev_pos
        assert (o["lsf_eid"][o["rev_pos"]] == o["rev_eid"]).all()
        seen_fwd += o["fwd_eid"].tolist()
        seen_rev += o["rev_eid"].tolist()
    # every edge is owned exactly once on each side
    assert sorted(seen_fwd) == list(range(E)) and sorted(seen_rev) == list(range(E))


def test_typed_row_order_hand():
    # one destination (vertex 0) with in-edges of types [2,0,2,1] at eids 0..3 -> (type, eid) order [1,3,0,2]
    indptr = np.array([0, 4, 4])
    indices = np.array([1, 1, 0, 1])
    et = np.array([2, 0, 2, 1], np.int32)
    o = oracle.preprocess(indptr, indices, et)
    assert o["fwd_eid"][:4].tolist() == [1, 3, 0, 2]
    assert o["fwd_type"][:4].tolist() == [0, 1, 2, 2]
    # vertex 1 is the source of eids 0,1,3 (types 2,0,1) -> rev row order [1,3,0]
    k = o["rev_perm"].tolist().index(1)
    a, b = o["rev_off"][k], o["rev_off"][k + 1]
    assert o["rev_eid"][a:b].tolist() == [1, 3, 0]


def test_degree_norms_closed_form():
    indptr, indices = synth.random_graph(25, 90, 3)
    a, b = oracle.degree_norms(indptr, indices)
    indeg = np.diff(indptr)
    outdeg = np.bincount(indices, minlength=25)
    np.testing.assert_array_equal(a, 1.0 / np.sqrt(np.maximum(indeg, 1)))
    np.testing.assert_array_equal(b, 1.0 / np.sqrt(np.maximum(outdeg, 1)))
