"""Shared test inputs (seeded, via synth) -- no method arithmetic here."""
import numpy as np

import synth


def hub_graph(N=3000, E_dir=30000, s=0.6, seed=5, hub_deg=1500, isolated=20, self_loops=True):
    """Power-law graph + one extra star hub (in-degree >= 1024 crosses the hub bucket) + isolated
    vertices (zero in- and out-degree) appended at the end: several tiles, ragged tails, all buckets."""
    ip, ix = synth.powerlaw_sym(N, E_dir, s, seed, self_loops)
    dst = np.repeat(np.arange(N), np.diff(ip))
    src = ix
    # star: hub_deg distinct leaves point at vertex 7
    leaves = (synth.uniform(seed + 99, (hub_deg,), 0, 1).astype(np.float64) * N).astype(np.int64).clip(0, N - 1)
    src = np.concatenate([src, leaves])
    dst = np.concatenate([dst, np.full(hub_deg, 7)])
    return synth.csr_from_edges(N + isolated, src, dst)


def rnd(seed, shape, lo=-1.0, hi=1.0):
    return synth.uniform(seed, shape, lo, hi)


def padded(a, ld):
    """[M,F] float32 -> [M,ld] float32 with the extra columns filled with NaN (must never be read
    into a result)."""
    M, F = a.shape
    out = np.full((M, ld), np.nan, np.float32)
    out[:, :F] = a
    return out
