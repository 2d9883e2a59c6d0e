"""Oracle of the plan's integer outputs: stream tiles, row classes, hub chunks,
hot prefix H, row-block partition bounds.

The paper runs cuSPARSE and never describes scheduling (Alg. 1
is a plain "parfor row"); these are build constants (reading c23), RE-DECLARED
here from DESIGN.md §Plan, not imported from the library:

  TILE_D      = 3072   stream tile "diagonal": row r (r < N) belongs to tile
                        k = floor((row_ptr[r] + r) / TILE_D); tiles
                        k = 0 .. K-1, K = ceil((NZ + N) / TILE_D);
                        bounds b_k = lower_bound_{r in [0,N]}(row_ptr[r] + r >= k*TILE_D)
  STREAM_MAX  = 1024   a stream tile computes its rows with L <= WARP_MAX,
                        except its LAST row when that row has L > STREAM_MAX
                        (the tile buffer holds < TILE_D + STREAM_MAX entries);
                        rows with L >= TILE_D are always last
  WARP_MAX    = 2048   last-in-tile rows with STREAM_MAX < L <= WARP_MAX: one
                        warp per row
  CTA_MAX     = 16384  WARP_MAX < L <= CTA_MAX (any position): one CTA per row
  SHORT_MAX   = 32     lane variant: L <= SHORT_MAX lane per row; the MID list
                        (SHORT_MAX < L <= WARP_MAX, any position) one warp per row
  HUB_CHUNK   = 16384  L > CTA_MAX: hub row cut into ceil(L / HUB_CHUNK)
                        chunks of HUB_CHUNK entries (merge-path split)

H: the length of the leading run of columns j of B with
colcnt_B[j] * N > NZ_B (the hot, hub-grouped prefix of x under RABBIT++).

Partition (SURVEY.md §8(e) "nnz-balanced" row blocks, refined by reading c29 of
DESIGN.md §2 to balance each rank's compulsory bytes of PAPER.md:96 -- 8 B per
entry (col, val) and w_off + 8 B per row (row_ptr, x, y), w_off = 8 when
NZ >= 2^31 else 4): with c(r) = 8 * row_ptr_B[r] + (w_off + 8) * r,
b_0 = 0, b_G = N, b_k = min{ r : c(r) >= ceil(k * c(N) / G) } for 0 < k < G.

TEST INFRASTRUCTURE ONLY (see oracle/__init__.py).
"""
from __future__ import annotations

import numpy as np

SHORT_MAX = 32
TILE_D = 3072
STREAM_MAX = 1024
WARP_MAX = 2048
CTA_MAX = 16384
HUB_CHUNK = 16384


def tile_bounds(row_ptr) -> np.ndarray:
    row_ptr = np.asarray(row_ptr, np.int64)
    n = len(row_ptr) - 1
    nnz = int(row_ptr[-1])
    if n == 0:
        return np.zeros(1, np.int64)
    K = -(-(nnz + n) // TILE_D)
    c = row_ptr + np.arange(n + 1, dtype=np.int64)       # strictly increasing
    b = np.empty(K + 1, np.int64)
    for k in range(K + 1):
        # lower_bound over r in [0, n]
        lo, hi = 0, n
        while lo < hi:
            mid = (lo + hi) // 2
            if c[mid] >= k * TILE_D:
                hi = mid
            else:
                lo = mid + 1
        b[k] = lo
    return b


def _last_in_tile(row_ptr, r):
    n = len(row_ptr) - 1
    if r + 1 >= n:
        return True
    return (int(row_ptr[r]) + r) // TILE_D != (int(row_ptr[r + 1]) + r + 1) // TILE_D


def row_classes(row_ptr):
    """(warp_rows, cta_rows, hub_rows, chunk_row, chunk_idx), all ascending."""
    row_ptr = np.asarray(row_ptr, np.int64)
    L = np.diff(row_ptr)
    warp = [r for r in range(len(L)) if STREAM_MAX < L[r] <= WARP_MAX and _last_in_tile(row_ptr, r)]
    cta = [r for r in range(len(L)) if WARP_MAX < L[r] <= CTA_MAX]
    hub = [r for r in range(len(L)) if L[r] > CTA_MAX]
    ch_r, ch_i = [], []
    for r in hub:
        for c in range(-(-int(L[r]) // HUB_CHUNK)):
            ch_r.append(r)
            ch_i.append(c)
    return (np.array(warp, np.int64), np.array(cta, np.int64), np.array(hub, np.int64),
            np.array(ch_r, np.int64), np.array(ch_i, np.int64))


def mid_rows(row_ptr) -> np.ndarray:
    """Rows computed warp-per-row by the lane variant: SHORT_MAX < L <= WARP_MAX
    (SHORT_MAX = 32), ascending, any position."""
    L = np.diff(np.asarray(row_ptr, np.int64))
    return np.nonzero((L > SHORT_MAX) & (L <= WARP_MAX))[0].astype(np.int64)


def stream_rows(row_ptr) -> np.ndarray:
    """Flag of rows computed inside their stream tile."""
    row_ptr = np.asarray(row_ptr, np.int64)
    L = np.diff(row_ptr)
    return np.array([L[r] <= WARP_MAX and not (L[r] > STREAM_MAX and _last_in_tile(row_ptr, r))
                     for r in range(len(L))], bool)


def hot_prefix(n, col_B) -> int:
    nnz = len(col_B)
    if n == 0:
        return 0
    colcnt = np.bincount(np.asarray(col_B, np.int64), minlength=n).astype(np.int64)
    hot = colcnt * np.int64(n) > nnz
    H = 0
    while H < n and hot[H]:
        H += 1
    return H


def partition(row_ptr, G: int) -> np.ndarray:
    row_ptr = np.asarray(row_ptr, np.int64)
    n = len(row_ptr) - 1
    nnz = int(row_ptr[-1])
    w_off = 8 if nnz >= 2**31 else 4
    cost = 8 * row_ptr + (w_off + 8) * np.arange(n + 1, dtype=np.int64)   # c(r), r = 0..N
    b = np.zeros(G + 1, np.int64)
    b[G] = n
    for k in range(1, G):
        target = -(-(k * int(cost[n])) // G)
        b[k] = int(np.searchsorted(cost, target, side="left"))
    return b
