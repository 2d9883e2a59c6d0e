"""Oracle metrics.

ideal_bytes   compulsory SpMV traffic, PAPER.md:96 (§IV-B):
              (2*|N|*4B) + ((|N|+1+|NZ|+|NZ|)*4B); the build also reports it
              with the real row-offset width w_off (reading c2):
              2*N*4 + (N+1)*w_off + 2*NZ*4.
insularity    PAPER.md:132 (§V-A): intra-community edges / all edges (c12:
              distinct off-diagonal stored (i, j) of A, directed).
skew          PAPER.md:146 (§V-B): % of NZ in the top 10% most connected rows
              (c17: top ceil(0.1 N) rows by row length).
modularity    ref [34] PAPER.md:293: exact integer form
              Q' = sum_c (2m * in_c - tot_c^2),  Q = Q' / (2m)^2.
hub_footprint PAPER.md:205: distinct cache lines holding the hubs x line size.

TEST INFRASTRUCTURE ONLY (see oracle/__init__.py).
"""
from __future__ import annotations

import math

import numpy as np

from .rabbit import symmetrize


def ideal_bytes(n: int, nnz: int, w_off: int = 4) -> int:
    return 2 * n * 4 + (n + 1) * w_off + 2 * nnz * 4


def insularity(n, row_ptr, col, comm) -> float:
    row_ptr = np.asarray(row_ptr, np.int64)
    rows = np.repeat(np.arange(n, dtype=np.int64), np.diff(row_ptr))
    cols = np.asarray(col, np.int64)
    pairs = {(int(i), int(j)) for i, j in zip(rows.tolist(), cols.tolist()) if i != j}
    if not pairs:
        return 1.0
    comm = np.asarray(comm)
    intra = sum(1 for i, j in pairs if comm[i] == comm[j])
    return intra / len(pairs)


def skew(row_ptr) -> float:
    L = np.sort(np.diff(np.asarray(row_ptr, np.int64)))[::-1]
    n, nnz = len(L), int(np.asarray(row_ptr)[-1])
    if nnz == 0:
        return 0.0
    top = int(math.ceil(0.1 * n))
    return float(L[:top].sum()) / nnz


def modularity_int(n, row_ptr, col, comm) -> tuple[int, int]:
    """(Q', 2m) with Q' = sum_c (2m * in_c - tot_c^2) over S = Bp + Bp^T."""
    sp_ptr, sp_idx, sp_w = symmetrize(n, row_ptr, col)
    comm = np.asarray(comm)
    two_m = int(sp_w.sum())
    in_c, tot_c = {}, {}
    for v in range(n):
        c = int(comm[v])
        a, b = int(sp_ptr[v]), int(sp_ptr[v + 1])
        tot_c[c] = tot_c.get(c, 0) + int(sp_w[a:b].sum())
        for j, w in zip(sp_idx[a:b].tolist(), sp_w[a:b].tolist()):
            if comm[j] == c:
                in_c[c] = in_c.get(c, 0) + int(w)
    q = sum(two_m * in_c.get(c, 0) - t * t for c, t in tot_c.items())
    return q, two_m


def modularity(n, row_ptr, col, comm) -> float:
    q, two_m = modularity_int(n, row_ptr, col, comm)
    return q / (two_m * two_m) if two_m else 0.0


def hub_footprint(new_ids, line_bytes: int = 128, elem_bytes: int = 4) -> int:
    """Bytes of distinct cache lines holding x[new_ids]."""
    lines = {int(i) * elem_bytes // line_bytes for i in np.asarray(new_ids).tolist()}
    return len(lines) * line_bytes


def community_stats(comm) -> tuple[int, float]:
    """(#communities, largest community fraction)."""
    comm = np.asarray(comm)
    if len(comm) == 0:
        return 0, 0.0
    _, cnt = np.unique(comm, return_counts=True)
    return len(cnt), float(cnt.max()) / len(comm)
