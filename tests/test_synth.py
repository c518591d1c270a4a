"""The seeded input generator: deterministic, shaped as stated in DESIGN.md §4."""
import numpy as np

import synth


def test_deterministic_and_valid_csr():
    a = synth.powerlaw_sym(500, 4000, 0.5, 7)
    b = synth.powerlaw_sym(500, 4000, 0.5, 7)
    assert all(np.array_equal(x, y) for x, y in zip(a, b))
    indptr, indices = a
    assert indptr[0] == 0 and indptr[-1] == 4000 + 500 and (np.diff(indptr) >= 0).all()
    assert indices.min() >= 0 and indices.max() < 500
    # symmetric: the multiset of (src,dst) equals that of (dst,src)
    dst = np.repeat(np.arange(500), np.diff(indptr))
    fwd = np.sort(indices * 500 + dst)
    bwd = np.sort(dst * 500 + indices)
    assert np.array_equal(fwd, bwd)
    # one self loop per vertex, none elsewhere
    assert (indices == dst).sum() == 500


def test_typed_graph_shape():
    indptr, indices, et = synth.powerlaw_directed_typed(1000, 5000, 0.6, 0.6, 13, 1.0, 3)
    dst = np.repeat(np.arange(1000), np.diff(indptr))
    assert indptr[-1] == 5000 and (indices != dst).all()
    assert et.min() >= 0 and et.max() < 13
    cnt = np.bincount(et, minlength=13)
    assert cnt[0] > cnt[5] > cnt[12]          # Zipf-shaped relation frequencies


def test_power_law_skew():
    indptr, _ = synth.powerlaw_sym(20000, 200000, 0.5, 5)
    deg = np.diff(indptr)
    assert deg.max() > 20 * deg.mean()        # hubs exist


def test_dense_draws():
    x = synth.uniform(3, (1000,), -1, 1)
    assert x.dtype == np.float32 and -1 <= x.min() and x.max() < 1
    assert np.array_equal(x, synth.uniform(3, (1000,), -1, 1))
    w = synth.glorot(9, 30, 70)
    assert np.abs(w).max() <= np.sqrt(6 / 100)
    lab = synth.labels(4, 1000, 7)
    assert lab.min() == 0 and lab.max() == 6
