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


BORDER_DEGREES = (0, 1, 31, 32, 33, 1023, 1024, 1025, 4096)


def border_graph(N=6000, E_bg=24000, seed=11):
    """Random background edges plus, for every d in BORDER_DEGREES, one destination with exactly d extra in-edges
    and one source with exactly d extra out-edges, at the bucket borders of a3 (1 / 32 / 1024).
    The border vertices take no background edges, so their degrees are exactly d (in) and d (out)."""
    nb = len(BORDER_DEGREES)
    dst_v = np.arange(nb)                    # vertices 0..nb-1: in-degree d_i
    src_v = np.arange(nb, 2 * nb)            # vertices nb..2nb-1: out-degree d_i
    lo = 2 * nb
    pick = lambda s, n: lo + (synth.uniform(s, (n,), 0, 1).astype(np.float64) * (N - lo)).astype(np.int64).clip(0, N - lo - 1)
    src = [pick(seed, E_bg)]
    dst = [pick(seed + 1, E_bg)]
    for i, d in enumerate(BORDER_DEGREES):
        src.append(pick(seed + 10 + i, d)); dst.append(np.full(d, dst_v[i]))       # in-degree d
        src.append(np.full(d, src_v[i])); dst.append(pick(seed + 30 + i, d))       # out-degree d
    return synth.csr_from_edges(N, np.concatenate(src), np.concatenate(dst))
