"""Oracle RABBIT and RABBIT++ orderings.

The paper describes RABBIT only as modularity-maximising, hierarchical
community detection followed by "assign[ing] community members consecutive
IDs" (§IV-A, §V-A; algorithm of ref [1] PAPER.md:259,
modularity of ref [34] PAPER.md:293).  The step-by-step reading below is
SURVEY.md §8(c) c5-c10, fixed deterministically so a library and this oracle
can agree bit for bit:

 1. S = Bp + Bp^T, Bp the 0/1 off-diagonal pattern of A (c5, c6): w_ij in
    {1, 2}; deg_i = sum_j w_ij; 2m = sum_i deg_i.
 2. Visit vertices in ascending (deg, id) (c7).
 3. root[v] = v, tot[v] = deg_v, children[v] = [] (merge order).
 4. For u in that order (u is a root when reached):
    a. aggregate u's S-row and the aggregated lists of the children merged
       into u so far; map every neighbour to its current root, sum weights
       per root, drop the root u itself (c9: lazy aggregation);
    b. dQ'(u, v) = 2m * w_uv - tot[u] * tot[v]   (= dQ * (2m)^2 / 2, exact int)
    c. v* = argmax dQ', ties -> smallest v (c8);
    d. if dQ'(u, v*) > 0: u becomes a child of v*, tot[v*] += tot[u];
       else u is appended to the top level.
 5. Pre-order DFS of the dendrogram from each top-level root in append order,
    children in merge order, hands out consecutive IDs (c10).  comm[v] is the
    top-level ancestor (c11).

RABBIT++ (§VI-A, Fig. 5): first group insular nodes
("nodes that are only connected to other nodes in their own
community"), then group hub nodes ("degree greater than the
average degree"; HUBGROUP keeps RABBIT's relative order).
Readings c13-c16: hub <=> colcount_A(v) * N > NZ; order
[non-insular hubs][non-insular non-hubs][insular], each RABBIT-ordered.

TEST INFRASTRUCTURE ONLY (see oracle/__init__.py).
"""
from __future__ import annotations

from dataclasses import dataclass, field

import numpy as np
import scipy.sparse as sp


def symmetrize(n, row_ptr, col):
    """S = Bp + Bp^T (c5): CSR (indptr, indices, data int64), sorted."""
    row_ptr = np.asarray(row_ptr, np.int64)
    rows = np.repeat(np.arange(n), np.diff(row_ptr))
    cols = np.asarray(col, np.int64)
    off = rows != cols                                  # c6: diagonal ignored
    Bp = sp.csr_matrix((np.ones(int(off.sum()), np.int64), (rows[off], cols[off])),
                       shape=(n, n))
    Bp.sum_duplicates()
    Bp.data[:] = 1                                      # 0/1 pattern
    S = (Bp + Bp.T).tocsr()
    S.sum_duplicates()
    S.sort_indices()
    return S.indptr.astype(np.int64), S.indices.astype(np.int64), S.data.astype(np.int64)


@dataclass
class RabbitResult:
    perm: np.ndarray                 # perm[old] = new
    comm: np.ndarray                 # top-level community (root id) per vertex
    toplevel: list
    children: list
    merges: list = field(default_factory=list)   # (u, v*, dQ') in merge order
    two_m: int = 0


def rabbit(n, row_ptr, col) -> RabbitResult:
    sp_ptr, sp_idx, sp_w = symmetrize(n, row_ptr, col)
    deg = [int(sp_w[sp_ptr[v]:sp_ptr[v + 1]].sum()) for v in range(n)]
    two_m = sum(deg)
    order = sorted(range(n), key=lambda v: (deg[v], v))          # c7

    parent = list(range(n))

    def find(v):
        r = v
        while parent[r] != r:
            r = parent[r]
        while parent[v] != r:                                       # path compression
            parent[v], v = r, parent[v]
        return r

    tot = list(deg)
    children = [[] for _ in range(n)]
    agg = [None] * n
    toplevel, merges = [], []
    for u in order:
        acc = {}
        lists = [zip(sp_idx[sp_ptr[u]:sp_ptr[u + 1]].tolist(),
                     sp_w[sp_ptr[u]:sp_ptr[u + 1]].tolist())]
        lists += [agg[c] for c in children[u]]                    # c9
        for lst in lists:
            for w, wt in lst:
                r = find(w)
                if r != u:
                    acc[r] = acc.get(r, 0) + wt
        for c in children[u]:
            agg[c] = None
        best_v, best_dq = -1, None
        for v in sorted(acc):
            dq = two_m * acc[v] - tot[u] * tot[v]                 # step 4b
            if best_dq is None or dq > best_dq:                    # ties -> smallest v
                best_v, best_dq = v, dq
        if best_dq is not None and best_dq > 0:                    # step 4d
            parent[u] = best_v
            tot[best_v] += tot[u]
            children[best_v].append(u)
            agg[u] = list(acc.items())
            merges.append((u, best_v, best_dq))
        else:
            toplevel.append(u)

    perm = np.full(n, -1, np.int64)
    nxt = 0
    for r in toplevel:                                             # step 5 / c10
        stack = [r]
        while stack:
            x = stack.pop()
            perm[x] = nxt
            nxt += 1
            stack.extend(reversed(children[x]))
    comm = np.array([find(v) for v in range(n)], np.int64)
    return RabbitResult(perm, comm, toplevel, children, merges, two_m)


# RABBIT++ variants (Table II design space)
RABBITPP, HUBSORT, INSULAR_ONLY, HUBGROUP_ONLY = "rabbitpp", "hubsort", "insular", "hubgroup"
HUBSORT_ONLY = "hubsort_only"


def insular_flags(n, row_ptr, col, comm) -> np.ndarray:
    """insular[v] <=> every S-neighbour j of v has comm[j] == comm[v]
    (c11 top-level community; isolated vertices vacuously)."""
    sp_ptr, sp_idx, _ = symmetrize(n, row_ptr, col)
    comm = np.asarray(comm)
    out = np.ones(n, bool)
    for v in range(n):
        nb = sp_idx[sp_ptr[v]:sp_ptr[v + 1]]
        out[v] = bool(np.all(comm[nb] == comm[v]))
    return out


def hub_flags(n, row_ptr, col) -> np.ndarray:
    """hub[v] <=> in-degree (column count of A) above the average NZ/N,
    compared exactly as colcnt * N > NZ (c13, c14)."""
    nnz = int(np.asarray(row_ptr)[-1])
    colcnt = np.bincount(np.asarray(col, np.int64), minlength=n)
    return colcnt.astype(np.int64) * np.int64(n) > nnz


def rabbitpp(n, row_ptr, col, rabbit_perm, comm, variant=RABBITPP) -> np.ndarray:
    """RABBIT++ = group insular nodes, then group hubs."""
    rabbit_perm = np.asarray(rabbit_perm, np.int64)
    ins = insular_flags(n, row_ptr, col, comm)
    hub = hub_flags(n, row_ptr, col)
    seq = np.empty(n, np.int64)
    seq[rabbit_perm] = np.arange(n)                 # vertices in RABBIT order
    colcnt = np.bincount(np.asarray(col, np.int64), minlength=n)
    if variant == RABBITPP:
        groups = [[v for v in seq if not ins[v] and hub[v]],
                  [v for v in seq if not ins[v] and not hub[v]],
                  [v for v in seq if ins[v]]]
    elif variant == HUBSORT:            # non-insular hubs by decreasing in-degree
        g0 = [v for v in seq if not ins[v] and hub[v]]
        pos = {v: i for i, v in enumerate(seq)}
        g0.sort(key=lambda v: (-int(colcnt[v]), pos[v]))
        groups = [g0, [v for v in seq if not ins[v] and not hub[v]],
                  [v for v in seq if ins[v]]]
    elif variant == INSULAR_ONLY:       # modification 1 only (Fig. 5)
        groups = [[v for v in seq if not ins[v]], [v for v in seq if ins[v]]]
    elif variant == HUBGROUP_ONLY:      # modification 2 only, no insular grouping
        groups = [[v for v in seq if hub[v]], [v for v in seq if not hub[v]]]
    elif variant == HUBSORT_ONLY:       # hubs by decreasing in-degree, no insular grouping
        g0 = [v for v in seq if hub[v]]  # (Table II, left half, RABBIT+HUBSORT)
        pos = {v: i for i, v in enumerate(seq)}
        g0.sort(key=lambda v: (-int(colcnt[v]), pos[v]))
        groups = [g0, [v for v in seq if not hub[v]]]
    else:
        raise ValueError(variant)
    perm = np.empty(n, np.int64)
    order = [v for g in groups for v in g]
    perm[np.array(order, np.int64)] = np.arange(n)
    return perm


def random_perm(n, seed) -> np.ndarray:
    """RANDOM (c19): Fisher-Yates driven by a splitmix64 counter stream.
    Step i (i = n-1 .. 1) swaps slot i with slot h1(seed, i) mod (i+1);
    result perm[old] = new is the shuffled identity."""
    M = (1 << 64) - 1
    G = 0x9E3779B97F4A7C15

    def mix(z):
        z = ((z ^ (z >> 30)) * 0xBF58476D1CE4E5B9) & M
        z = ((z ^ (z >> 27)) * 0x94D049BB133111EB) & M
        return z ^ (z >> 31)

    p = list(range(n))
    for i in range(n - 1, 0, -1):
        j = mix((seed + G * (i + 1)) & M) % (i + 1)
        p[i], p[j] = p[j], p[i]
    return np.array(p, np.int64)
