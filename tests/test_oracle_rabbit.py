"""Pins of the oracle RABBIT / RABBIT++ (readings
c5-c16) against closed forms, modularity identities and invariants."""
import json
import math
import os

import numpy as np
import pytest
import scipy.sparse as sp
from scipy.sparse.csgraph import connected_components

import synth
from oracle import metrics, permute, rabbit

GOLD = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "paper_pins.json")))
RC = GOLD["rabbit_closed_forms"]


def csr_from_edges(n, edges):
    rows = [[] for _ in range(n)]
    for i, j in edges:
        rows[i].append(j)
    rp = np.zeros(n + 1, np.int64)
    cols = []
    for i in range(n):
        rp[i + 1] = rp[i] + len(rows[i])
        cols += sorted(rows[i])
    return rp, np.array(cols, np.int32)


def order_of(perm):
    seq = np.empty(len(perm), np.int64)
    seq[perm] = np.arange(len(perm))
    return seq.tolist()


def star(k, both):
    e = [(j, k) for j in range(k)]
    if both:
        e += [(k, j) for j in range(k)]
    return csr_from_edges(k + 1, e)


@pytest.mark.parametrize("both,key", [(False, "star_one_direction_k5"), (True, "star_both_directions_k5")])
def test_star_closed_form(both, key):
    k = RC[key]["k"]
    rp, col = star(k, both)
    r = rabbit.rabbit(k + 1, rp, col)
    assert [m[2] for m in r.merges] == RC[key]["dq"]
    # general closed form: dQ'_j = c (k - j + 1), c = 1 (one direction) or 4 (both)
    c = 4 if both else 1
    assert [m[2] for m in r.merges] == [c * (k - j + 1) for j in range(1, k + 1)]
    assert order_of(r.perm) == RC[key]["order"]


def test_clique_closed_form():
    n = RC["clique_both_directions_n5"]["n"]
    e = [(i, j) for i in range(n) for j in range(n) if i != j]
    rp, col = csr_from_edges(n, e)
    r = rabbit.rabbit(n, rp, col)
    assert [m[2] for m in r.merges] == RC["clique_both_directions_n5"]["dq"]
    assert [m[2] for m in r.merges] == [4 * (k + 1) * (n - 1) for k in range(n - 1)]
    assert order_of(r.perm) == RC["clique_both_directions_n5"]["order"]


def k3k4():
    e = [(i, j) for i in range(3) for j in range(3) if i != j]
    e += [(i, j) for i in range(3, 7) for j in range(3, 7) if i != j]
    return csr_from_edges(7, e)


def test_k3_plus_k4():
    rp, col = k3k4()
    r = rabbit.rabbit(7, rp, col)
    g = RC["k3_plus_k4"]
    assert order_of(r.perm) == g["order"]
    assert r.comm.tolist() == g["comm"]
    q, two_m = metrics.modularity_int(7, rp, col, r.comm)
    assert (q, two_m) == (g["modularity_num"], g["two_m"])
    # textbook modularity of two disjoint cliques: sum_c e_c/m - (d_c/2m)^2
    m = 3 + 6
    text = (3 / m - (6 / (2 * m)) ** 2) + (6 / m - (12 / (2 * m)) ** 2)
    assert math.isclose(metrics.modularity(7, rp, col, r.comm), text, rel_tol=1e-12)
    assert math.isclose(text, g["Q"], rel_tol=1e-12)


def _rmat_small(scale=9, ef=8, seed=5):
    A = synth.rmat(scale, ef, seed, seed_v=1)
    return A.n, A.row_ptr, A.col


@pytest.mark.parametrize("seed", [1, 2, 3])
def test_rabbit_invariants(seed):
    n, rp, col = _rmat_small(9, 8, seed)
    r = rabbit.rabbit(n, rp, col)
    assert permute.is_bijection(r.perm, n)
    # (i) every merge strictly increases modularity
    assert all(m[2] > 0 for m in r.merges)
    # (ii) Q'_final - Q'_initial == 2 * sum dQ'   (exact integers)
    q_final, two_m = metrics.modularity_int(n, rp, col, r.comm)
    q_init, _ = metrics.modularity_int(n, rp, col, np.arange(n))
    assert q_final - q_init == 2 * sum(m[2] for m in r.merges)
    assert two_m == r.two_m
    # (iv) disconnected components never merge
    sp_ptr, sp_idx, sp_w = rabbit.symmetrize(n, rp, col)
    S = sp.csr_matrix((sp_w, sp_idx, sp_ptr), shape=(n, n))
    _, lab = connected_components(S, directed=False)
    for v in range(n):
        assert lab[v] == lab[r.comm[v]]
    # consecutive IDs: every community -- at every level of the
    # dendrogram -- occupies a contiguous ID range
    def subtree(v):
        out, st = [], [v]
        while st:
            x = st.pop()
            out.append(x)
            st.extend(r.children[x])
        return out
    for v in range(n):
        ids = sorted(r.perm[subtree(v)].tolist())
        assert ids == list(range(ids[0], ids[0] + len(ids)))
        assert r.perm[v] == ids[0]           # pre-order: root first


def test_rabbit_sbm_recovers_planted():
    # soft, paper-level quality check (not parity): RABBIT on a planted SBM
    # finds communities close to the planted insularity
    A = synth.sbm(8, 128, 8, 0.97, 11, True, 3, 0, 2)
    r = rabbit.rabbit(A.n, A.row_ptr, A.col)
    ins = metrics.insularity(A.n, A.row_ptr, A.col, r.comm)
    assert ins > 0.85
    ncomm, big = metrics.community_stats(r.comm)
    assert big < 0.5


def test_rabbitpp_block_diagonal_equals_rabbit():
    rp, col = k3k4()
    r = rabbit.rabbit(7, rp, col)
    assert rabbit.insular_flags(7, rp, col, r.comm).all()
    assert np.array_equal(rabbit.rabbitpp(7, rp, col, r.perm, r.comm), r.perm)


@pytest.mark.parametrize("seed", [1, 4])
def test_rabbitpp_groups(seed):
    n, rp, col = _rmat_small(9, 8, seed)
    r = rabbit.rabbit(n, rp, col)
    pp = rabbit.rabbitpp(n, rp, col, r.perm, r.comm)
    assert permute.is_bijection(pp, n)
    ins = rabbit.insular_flags(n, rp, col, r.comm)
    hub = rabbit.hub_flags(n, rp, col)
    grp = np.where(ins, 2, np.where(hub, 0, 1))
    seq = order_of(pp)
    # groups appear in order G0, G1, G2 and keep RABBIT's relative order
    assert all(grp[seq[i]] <= grp[seq[i + 1]] for i in range(n - 1))
    for g in range(3):
        members = [v for v in seq if grp[v] == g]
        assert all(r.perm[members[i]] < r.perm[members[i + 1]] for i in range(len(members) - 1))
    # independent recomputation of the flags
    sp_ptr, sp_idx, _ = rabbit.symmetrize(n, rp, col)
    for v in range(0, n, 7):
        nb = set(sp_idx[sp_ptr[v]:sp_ptr[v + 1]].tolist())
        assert ins[v] == all(r.comm[j] == r.comm[v] for j in nb)
        cnt = int(np.sum(col == v))
        assert hub[v] == (cnt > rp[-1] / n)


def test_rabbitpp_variants():
    n, rp, col = _rmat_small(8, 8, 2)
    r = rabbit.rabbit(n, rp, col)
    for v in (rabbit.HUBSORT, rabbit.INSULAR_ONLY, rabbit.HUBGROUP_ONLY):
        assert permute.is_bijection(rabbit.rabbitpp(n, rp, col, r.perm, r.comm, v), n)
    # HUBSORT: leading hubs in non-increasing in-degree
    hs = rabbit.rabbitpp(n, rp, col, r.perm, r.comm, rabbit.HUBSORT)
    hub = rabbit.hub_flags(n, rp, col)
    ins = rabbit.insular_flags(n, rp, col, r.comm)
    g0 = int(np.sum(hub & ~ins))
    seq = order_of(hs)
    cc = np.bincount(col, minlength=n)
    assert all(cc[seq[i]] >= cc[seq[i + 1]] for i in range(g0 - 1))
    # HUBSORT_ONLY: every hub first, in non-increasing in-degree, then the rest
    # in RABBIT order (no insular grouping)
    hso = rabbit.rabbitpp(n, rp, col, r.perm, r.comm, rabbit.HUBSORT_ONLY)
    assert permute.is_bijection(hso, n)
    s2 = order_of(hso)
    nh = int(hub.sum())
    assert all(hub[v] for v in s2[:nh]) and all(cc[s2[i]] >= cc[s2[i + 1]] for i in range(nh - 1))
    rest = [v for v in order_of(r.perm) if not hub[v]]
    assert list(s2[nh:]) == rest


def test_fig5_hub_arithmetic():
    f = GOLD["fig5_hubs"]
    # 9 rows, 28 NZ, column counts with two columns of degree >= 4
    counts = [5, 4, 3, 3, 3, 3, 3, 2, 2]
    assert sum(counts) == f["nnz"]
    col = np.concatenate([np.full(c, j, np.int32) for j, c in enumerate(counts)])
    rp = np.linspace(0, f["nnz"], f["n"] + 1).astype(np.int64)
    hub = rabbit.hub_flags(f["n"], rp, col)
    assert int(hub.sum()) == f["hub_count"]
    assert all((c >= f["hub_min_degree"]) == h for c, h in zip(counts, hub))


def test_random_perm():
    p = rabbit.random_perm(1000, 42)
    assert permute.is_bijection(p, 1000)
    assert np.array_equal(p, rabbit.random_perm(1000, 42))
    assert not np.array_equal(p, rabbit.random_perm(1000, 43))


# splitmix64 reference outputs for state 0 (Vigna's splitmix64.c; the same
# stream as java.util.SplittableRandom): output k = mix64(k * 0x9E3779B97F4A7C15).
# Reading c19 draws h1(seed, i) = output i+1 of the stream started at `seed`.
SPLITMIX64_SEED0 = [0xE220A8397B1DCDAF, 0x6E789E6AA1B965F4, 0x06C45D188009454F,
                    0xF88BB8A8724C81EC, 0x1B39896A51A8749B]


def test_random_perm_hand_worked_fisher_yates():
    """RANDOM (reading c19) pinned by hand from the published splitmix64 vector.

    n = 4, seed 0, p = [0, 1, 2, 3]:
      i = 3: j = out4 mod 4 = 0  -> swap p3, p0 -> [3, 1, 2, 0]
      i = 2: j = out3 mod 3 = 1  -> swap p2, p1 -> [3, 2, 1, 0]
      i = 1: j = out2 mod 2 = 0  -> swap p1, p0 -> [2, 3, 1, 0]
    n = 5 adds i = 4 first: j = out5 mod 5 = 2 -> [0, 1, 4, 3, 2], then the
      same three steps -> [3, 1, 4, 0, 2] -> [3, 4, 1, 0, 2] -> [4, 3, 1, 0, 2].
    A Sattolo slip (mod i instead of mod i+1) or an off-by-one counter gives
    other permutations."""
    o = SPLITMIX64_SEED0
    assert (o[1] % 2, o[2] % 3, o[3] % 4, o[4] % 5) == (0, 1, 0, 2)  # the j's above
    assert rabbit.random_perm(4, 0).tolist() == [2, 3, 1, 0]
    assert rabbit.random_perm(5, 0).tolist() == [4, 3, 1, 0, 2]
    assert rabbit.random_perm(1, 0).tolist() == [0]
    assert rabbit.random_perm(0, 0).tolist() == []
