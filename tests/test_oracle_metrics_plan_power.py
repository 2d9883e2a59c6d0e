"""Pins of the oracle metrics, plan rules (c23) and
power iteration (c22)."""
import json
import math
import os

import numpy as np
import pytest

import synth
from oracle import metrics, plan, power, spmv
from tests.test_oracle_rabbit import csr_from_edges

GOLD = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "paper_pins.json")))


def test_insularity_worked_number():
    g = GOLD["insularity_example"]
    # hand-built 9-node graph with communities {0..3}, {4..7}, {8}: 20 distinct
    # intra-community directed edges and 4 inter-community ones (the Fig. 1
    # graph itself is absent from PAPER.md, so only the formula is pinned)
    comm = np.array([0, 0, 0, 0, 1, 1, 1, 1, 2])
    intra = [(0, 1), (1, 0), (1, 2), (2, 1), (2, 3), (3, 2), (3, 0), (0, 3), (0, 2), (2, 0),
             (4, 5), (5, 4), (5, 6), (6, 5), (6, 7), (7, 6), (7, 4), (4, 7), (4, 6), (6, 4)]
    inter = [(3, 8), (8, 4), (1, 5), (7, 2)]
    assert len(set(intra)) == g["intra"] and len(set(intra + inter)) == g["total"]
    # diagonal entries and stored duplicates do not change it (c6, c12)
    edges = intra + inter + [(0, 0), (8, 8), (0, 1)]
    assert math.isclose(metrics.insularity(9, *csr_from_edges(9, edges), comm), g["value"])
    assert round(g["value"], 2) == 0.83


def test_skew_closed_form():
    # 20 rows: two rows of length 50, the rest length 5 -> top ceil(2) rows hold 100/190
    L = np.array([5] * 18 + [50, 50])
    rp = np.concatenate([[0], np.cumsum(L)])
    assert math.isclose(metrics.skew(rp), 100 / 190)


def test_community_stats_closed_form():
    """(#communities, largest fraction) ("largest community
    comprises 98% of the nodes", :144) on hand-counted labelings."""
    assert metrics.community_stats([]) == (0, 0.0)
    assert metrics.community_stats([7]) == (1, 1.0)
    # K3 + K4 under RABBIT (SURVEY 8(c) closed form): comm = {2,2,2,6,6,6,6}
    assert metrics.community_stats([2, 2, 2, 6, 6, 6, 6]) == (2, 4 / 7)
    # labels need not be contiguous or sorted; singletons count as communities
    n, big = metrics.community_stats([5, 0, 5, 9, 5, 0, 3])
    assert (n, big) == (4, 3 / 7)
    # n singletons: n communities of fraction 1/n
    assert metrics.community_stats(list(range(10))) == (10, 0.1)
    # the mawi case study shape: 98 of 100 nodes in one community
    assert metrics.community_stats([0] * 98 + [1, 2]) == (3, 0.98)


def test_hub_footprint_pin():
    g = GOLD["sx_stackoverflow_hub_footprint"]
    fp = metrics.hub_footprint(np.arange(g["hubs"]), g["line_bytes"], g["elem_bytes"])
    assert fp == g["contiguous_bytes"]
    assert round(fp / 2**20, 2) == g["mib"]
    # scattered hubs (one per line) occupy one line each
    assert metrics.hub_footprint(np.arange(100) * 32) == 100 * 128


def _tiles_bruteforce(rp):
    n = len(rp) - 1
    return [(int(rp[r]) + r) // plan.TILE_D for r in range(n)]


@pytest.mark.parametrize("case", ["rmat", "empty_tail", "long_rows", "empty"])
def test_tile_bounds(case):
    if case == "rmat":
        A = synth.rmat(12, 16, 3)
        rp = A.row_ptr
    elif case == "empty_tail":
        rp = np.concatenate([np.arange(0, 3000, 3), np.full(5000, 2997)]).astype(np.int64)
    elif case == "long_rows":
        L = np.array([1, 5000, 2, 2048, 2049, 0, 0, 40000, 3, 128, 129, 127, 0, 5, 1024, 1023,
                      1025, 0, 1, 512, 513, 511] + [7] * 500)
        rp = np.concatenate([[0], np.cumsum(L)]).astype(np.int64)
    else:
        rp = np.zeros(1, np.int64)
    b = plan.tile_bounds(rp)
    n = len(rp) - 1
    assert b[0] == 0 and b[-1] == n and np.all(np.diff(b) >= 0)
    tid = _tiles_bruteforce(rp)
    for k in range(len(b) - 1):
        for r in range(b[k], b[k + 1]):
            assert tid[r] == k
    L = np.diff(rp)
    inside = plan.stream_rows(rp)
    warp, cta, hub, _, _ = plan.row_classes(rp)
    assert sorted(np.nonzero(~inside)[0].tolist()) == sorted(warp.tolist() + cta.tolist() + hub.tolist())
    for k in range(len(b) - 1):
        rows = range(b[k], b[k + 1])
        huge = [r for r in rows if L[r] >= plan.TILE_D]
        assert not huge or huge == [b[k + 1] - 1]            # rows >= TILE_D are always last
        out = [r for r in rows if not inside[r] and L[r] <= plan.WARP_MAX]
        assert not out or out == [b[k + 1] - 1]              # short-enough rows leave only if last
        s = sum(L[r] for r in rows if inside[r])
        assert s < plan.TILE_D + plan.STREAM_MAX             # fits the tile buffer
        assert b[k + 1] - b[k] <= plan.TILE_D


def test_row_classes_and_partition():
    # a 1500-entry row followed by short rows of the same tile stays inside it
    rp2 = np.array([0, 1500, 1502, 1507])
    assert plan.stream_rows(rp2).all() and len(plan.row_classes(rp2)[0]) == 0
    L = np.array([1, 5000, 2, 2048, 2049, 0, 16384, 16385, 40000, 3, 1024, 1025])
    rp = np.concatenate([[0], np.cumsum(L)]).astype(np.int64)
    warp, cta, hub, cr, ci = plan.row_classes(rp)
    # c_r = row_ptr[r] + r = 0, 2, 5003, 5006, 7055, 9105, 9106, 25491, 41877, 81878,
    # 81882, 82907 -> tiles (// 3072) 0,0,1,1,2,2,2,8,13,26,26,26: rows 3 and 11
    # (1024 < L <= 2048) are last in their tile; row 10 is not; rows with
    # L > 2048 (1, 4, 6) never stay inside a tile
    assert plan.TILE_D == 3072
    assert warp.tolist() == [3, 11]
    assert plan.mid_rows(rp).tolist() == [3, 10, 11]
    assert cta.tolist() == [1, 4, 6]
    assert hub.tolist() == [7, 8]
    assert cr.tolist() == [7, 7] + [8, 8, 8]
    assert ci.tolist() == [0, 1, 0, 1, 2]
    for G in (1, 2, 3, 8):
        b = plan.partition(rp, G)
        assert b[0] == 0 and b[-1] == len(L) and np.all(np.diff(b) >= 0)
        c = 8 * rp + 12 * np.arange(len(rp))      # int32 offsets: 8 B / entry, 12 B / row
        for k in range(1, G):
            t = -(-(k * int(c[-1])) // G)
            assert c[b[k]] >= t and (b[k] == 0 or c[b[k] - 1] < t)


def test_partition_balances_compulsory_bytes():
    """Reading c29 by hand: L = [4, 0, 0, 0, 4], int32 offsets (w_off = 4).
    c(r) = 8 row_ptr[r] + 12 r = [0, 44, 56, 68, 80, 124]; G = 2: target
    ceil(124 / 2) = 62 -> b_1 = 3 (c = 68): rank 0 gets 4 entries + 3 rows
    (68 B of P:96 traffic), rank 1 4 entries + 2 rows (56 B).  The plain nnz
    split (lower_bound(row_ptr, 4) = 1) would give rank 1 all four empty rows."""
    rp = np.array([0, 4, 4, 4, 4, 8], np.int64)
    assert plan.partition(rp, 2).tolist() == [0, 3, 5]
    assert plan.partition(rp, 1).tolist() == [0, 5]
    # G larger than N: empty blocks, bounds still monotone and complete
    assert plan.partition(np.array([0, 2], np.int64), 3).tolist() == [0, 1, 1, 1]
    # int64 offsets (NZ >= 2^31) weigh a row 16 B: c(r) = 8 rp + 16 r
    rp64 = np.array([0, 2**31, 2**31, 2**31 + 2], np.int64)
    c = 8 * rp64 + 16 * np.arange(4)
    b = plan.partition(rp64, 2)
    t = -(-int(c[-1]) // 2)
    assert c[b[1]] >= t and c[b[1] - 1] < t


def test_hot_prefix():
    # columns 0,1 hot (count*N > NZ), column 2 cold, column 3 hot again -> H = 2
    col = np.array([0, 0, 0, 1, 1, 1, 3, 3, 3, 2], np.int32)
    assert plan.hot_prefix(5, col) == 2
    assert plan.hot_prefix(5, np.array([4, 4], np.int32)) == 0


def test_power_iteration_regular_fixed_point():
    # periodic 27-point stencil, unit values: 27-regular, x0 = 1/sqrt(N) is a
    # fixed point with lambda = 27
    A = synth.stencil27(4, periodic=True, relabel=True, seed_scr=3, valmode=2)
    x0 = np.full(A.n, np.float32(1 / math.sqrt(A.n)))
    x, lam = power.power_iteration(A.row_ptr, A.col, A.val, x0, 5)
    assert math.isclose(lam, 27.0, rel_tol=1e-6)
    assert np.allclose(x, x0, rtol=1e-6)


def test_power_iteration_perron_root():
    A = synth.rmat(7, 8, 2, valmode=synth.VAL_POS, seed_v=3)
    # make it strongly connected-ish: add the identity (shifts spectrum by +1)
    D = spmv.dense(A.n, A.row_ptr, A.col, A.val) + np.eye(A.n)
    ev = np.max(np.abs(np.linalg.eigvals(D)))
    rows = [np.nonzero(D[r])[0] for r in range(A.n)]
    rp = np.concatenate([[0], np.cumsum([len(c) for c in rows])]).astype(np.int64)
    col = np.concatenate(rows).astype(np.int32)
    val = np.concatenate([D[r, c] for r, c in enumerate(rows)]).astype(np.float32)
    x, lam = power.power_iteration(rp, col, val, np.ones(A.n, np.float32), 400)
    assert abs(lam - ev) / ev < 1e-3


def test_mid_rows():
    rng = np.random.default_rng(4)
    L = rng.integers(0, 40, 700)
    L[[3, 300, 650]] = [100, 2048, 5000]
    rp = np.concatenate([[0], np.cumsum(L)]).astype(np.int64)
    mid = plan.mid_rows(rp)
    assert set(mid.tolist()) == {r for r in range(len(L)) if 32 < L[r] <= 2048}
    assert np.all(np.diff(mid) > 0)
