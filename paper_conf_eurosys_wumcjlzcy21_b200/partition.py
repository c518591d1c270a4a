"""Destination-row partitioning for P GPUs (the paper itself is single-GPU, L479).

Rank p owns the contiguous vertex range [p*n, min(N, (p+1)*n)) with n = ceil(N / P); every
per-layer all-gather is P*n rows high so that rank p's rows land at offset p*n = row_begin, i.e.
gathered tables are indexed by global vertex id.  Vertex ids are shuffled by the generator, so equal
ranges carry roughly equal edge counts (reported by edge_imbalance)."""
from __future__ import annotations

import numpy as np


def rows_per_rank(N: int, P: int) -> int:
    return (N + P - 1) // P


def row_range(N: int, P: int, rank: int) -> tuple[int, int]:
    n = rows_per_rank(N, P)
    return min(N, rank * n), min(N, (rank + 1) * n)


def gathered_rows(N: int, P: int) -> int:
    """Height of an all-gathered table (>= N; rows >= N are padding and never indexed)."""
    return rows_per_rank(N, P) * P


def edge_imbalance(indptr: np.ndarray, P: int) -> float:
    """max over ranks of owned in-edges / mean."""
    N = len(indptr) - 1
    counts = [int(indptr[row_range(N, P, p)[1]] - indptr[row_range(N, P, p)[0]]) for p in range(P)]
    return max(counts) / max(1e-9, sum(counts) / P)
