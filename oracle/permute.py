"""Oracle symmetric permutation B = P A P^T and vector relabel.

PAPER.md:86 (§IV-A): reordering "assigns community members consecutive IDs";
PAPER.md:96 (§IV-B): A is a square |N| x |N| matrix.  Relabelling node i to
perm[i] on both rows and columns gives

    B[perm[i], perm[j]] = A[i, j]        (P x)[perm[i]] = x[i]

with perm[old] = new.  Each row of B is ordered by its new column index;
stored duplicates keep their order in A (stable), which fixes B uniquely
(reading c25).

TEST INFRASTRUCTURE ONLY (see oracle/__init__.py).
"""
from __future__ import annotations

import numpy as np


def is_bijection(perm, n: int) -> bool:
    perm = np.asarray(perm)
    if perm.shape != (n,):
        return False
    if n == 0:
        return True
    if perm.min() < 0 or perm.max() >= n:
        return False
    return np.bincount(perm, minlength=n).max() == 1


def inverse(perm) -> np.ndarray:
    """inv[perm[i]] = i."""
    perm = np.asarray(perm, np.int64)
    inv = np.empty_like(perm)
    inv[perm] = np.arange(len(perm))
    return inv


def permute_csr(n, row_ptr, col, val, perm):
    """B = P A P^T as CSR (row_ptr int64, col int32, val float32 bit-copied)."""
    row_ptr = np.asarray(row_ptr, np.int64)
    perm = np.asarray(perm, np.int64)
    nnz = int(row_ptr[-1])
    rows = np.repeat(np.arange(n, dtype=np.int64), np.diff(row_ptr))
    new_r = perm[rows]
    new_c = perm[np.asarray(col, np.int64)]
    # primary key new row, then new column, then position in A (stability)
    order = np.lexsort((np.arange(nnz), new_c, new_r))
    B_col = new_c[order].astype(np.int32)
    B_val = np.asarray(val, np.float32)[order]
    B_ptr = np.zeros(n + 1, np.int64)
    B_ptr[1:] = np.cumsum(np.bincount(new_r, minlength=n))
    return B_ptr, B_col, B_val


def permute_csr_scipy(n, row_ptr, col, val, perm):
    """B = P A P^T through scipy fancy indexing (B = A[inv][:, inv]) with
    sorted rows: a fast library route used only to prepare the input of the
    timed CPU baseline (duplicate order is not guaranteed stable)."""
    import scipy.sparse as sp
    inv = inverse(perm)
    M = sp.csr_matrix((np.asarray(val, np.float32), np.asarray(col), np.asarray(row_ptr)),
                      shape=(n, n))
    B = M[inv][:, inv]
    B.sort_indices()
    return B.indptr.astype(np.int64), B.indices.astype(np.int32), B.data.astype(np.float32)


def permute_rows(row_ptr, col, val, perm, inv, rows):
    """Rows `rows` of B = P A P^T only (large-size sampled parity):
    row r of B is row inv[r] of A relabelled by perm and stably sorted."""
    out = []
    for r in rows:
        i = int(inv[r])
        a, b = int(row_ptr[i]), int(row_ptr[i + 1])
        c = np.asarray(perm)[np.asarray(col[a:b], np.int64)]
        o = np.argsort(c, kind="stable")
        out.append((c[o].astype(np.int32), np.asarray(val[a:b], np.float32)[o]))
    return out


def permute_block(row_ptr, col, val, perm, inv, r0: int, r1: int):
    """Rows [r0, r1) of B = P A P^T as a CSR block (row_ptr rebased to 0):
    row r of B is row inv[r] of A with columns relabelled by perm, stably
    sorted by new column (the definition permute_csr follows), vectorised so
    that a bounded sample of a billion-entry matrix is cheap to build."""
    row_ptr = np.asarray(row_ptr, np.int64)
    src = np.asarray(inv, np.int64)[r0:r1]
    a, b = row_ptr[src], row_ptr[src + 1]
    L = b - a
    rp = np.concatenate([[0], np.cumsum(L)]).astype(np.int64)
    m = int(rp[-1])
    rowid = np.repeat(np.arange(r1 - r0, dtype=np.int64), L)
    k = np.arange(m, dtype=np.int64) - np.repeat(rp[:-1], L) + np.repeat(a, L)
    c = np.asarray(perm, np.int64)[np.asarray(col)[k].astype(np.int64)]
    o = np.lexsort((np.arange(m), c, rowid))          # by row, then new column, stable
    return rp, c[o].astype(np.int32), np.asarray(val, np.float32)[k][o]


def permute_vec(x, perm, inverse_: bool = False) -> np.ndarray:
    """out = P x  (out[perm[i]] = x[i]);  inverse: out = P^T x (out[i] = x[perm[i]])."""
    x = np.asarray(x)
    perm = np.asarray(perm, np.int64)
    if inverse_:
        return x[perm].copy()
    out = np.empty_like(x)
    out[perm] = x
    return out
