"""Concurrent RABBIT merges (Rabbit Order's parallel
incremental aggregation, ref [1] PAPER.md:259) checked by invariants.

The concurrent detection (spmv_reorder | SPMV_REORDER_PARALLEL) is not
bit-exact with the sequential reading c5-c10 -- its merge order depends on
thread timing -- so it is pinned by what must hold for ANY run, each computed
independently by the oracle:

  * every merge has an exact integer gain dQ' = 2m w - tot tot > 0 (P:130:
    modularity-driven merging), so modularity strictly increases;
  * Q'_final - Q'_init = 2 * sum dQ' exactly (Q' from oracle.metrics on the
    final and the singleton communities) -- a merge recorded with a stale w or
    tot breaks this identity;
  * no merge joins two connected components (w = 0 there, dQ' < 0);
  * the merge log is a forest whose top-level ancestors are spmv_reorder's
    communities, and every community is a contiguous ID range (P:86
    "consecutive IDs"); the permutation is a bijection;
  * quality close to the sequential detection (soft: modularity and
    insularity within 5 %).
The sequential detection's own log obeys the first three as well."""
import os

import numpy as np
import pytest
import scipy.sparse as sp
import scipy.sparse.csgraph as csg

import synth
from oracle import metrics, permute, rabbit
from paper_conf_ispass_balajicjk23_b200 import spmv


def _graphs():
    yield "rmat12", synth.config(1, small=True).A
    yield "sbm16", synth.config(2, small=True).A
    yield "stencil24", synth.config(4, small=True).A
    yield "kron14", synth.config(5, small=True).A
    rp, col = _k3k4_and_isolated()
    yield "k3k4", synth.Csr(9, rp, col, np.ones(len(col), np.float32))


def _k3k4_and_isolated():
    e = [(i, j) for i in range(3) for j in range(3) if i != j]
    e += [(i, j) for i in range(3, 7) for j in range(3, 7) if i != j]
    rows = [[] for _ in range(9)]
    for i, j in e:
        rows[i].append(j)
    rp = np.zeros(10, np.int64)
    for i in range(9):
        rp[i + 1] = rp[i] + len(rows[i])
    return rp, np.array([c for r in rows for c in sorted(r)], np.int32)


def _components(A):
    rows = np.repeat(np.arange(A.n), np.diff(A.row_ptr))
    M = sp.csr_matrix((np.ones(A.nnz), (rows, A.col.astype(np.int64))), shape=(A.n, A.n))
    return csg.connected_components(M, directed=True, connection="weak")[1]


def _check_invariants(A, perm, comm, child, parent, dq):
    n = A.n
    assert permute.is_bijection(perm, n)
    assert np.all(dq > 0)
    q_final, two_m = metrics.modularity_int(n, A.row_ptr, A.col, comm)
    q_init, _ = metrics.modularity_int(n, A.row_ptr, A.col, np.arange(n))
    assert q_final - q_init == 2 * int(dq.astype(object).sum())
    cc = _components(A)
    assert np.all(cc[child] == cc[parent])
    # forest: every vertex merged at most once; the root of each chain is the community
    assert len(np.unique(child)) == len(child)
    up = np.arange(n)
    up[child] = parent
    top = np.arange(n)
    for _ in range(64):
        nxt = up[top]
        if np.array_equal(nxt, top):
            break
        top = nxt
    assert np.array_equal(top, comm)
    # each community a contiguous range of new IDs
    for c in np.unique(comm):
        ids = np.sort(perm[comm == c])
        assert ids[-1] - ids[0] + 1 == len(ids)


@pytest.mark.parametrize("name,A", list(_graphs()))
@pytest.mark.parametrize("parallel", [False, True])
def test_detection_invariants(name, A, parallel):
    perm, st = spmv.reorder(A.row_ptr, A.col, "rabbit", parallel=parallel, log=True)
    comm = spmv.reorder_last_comm(A.n)
    child, parent, dq = spmv.reorder_last_merges()
    assert st.parallel == int(parallel)
    assert st.n_merges == len(child)
    _check_invariants(A, perm, comm, child, parent, dq)
    if not parallel:  # the sequential detection is the oracle's, merge for merge
        r = rabbit.rabbit(A.n, A.row_ptr, A.col)
        assert [(int(u), int(v), int(g)) for u, v, g in zip(child, parent, dq)] == \
            [(int(u), int(v), int(g)) for u, v, g in r.merges]


@pytest.mark.parametrize("name,A", list(_graphs())[:4])
def test_parallel_quality_close_to_sequential(name, A):
    _, s_seq = spmv.reorder(A.row_ptr, A.col, "rabbit")
    _, s_par = spmv.reorder(A.row_ptr, A.col, "rabbit", parallel=True)
    assert s_par.modularity >= s_seq.modularity - 0.05 * abs(s_seq.modularity) - 1e-3
    assert s_par.insularity >= s_seq.insularity - 0.05


def test_parallel_rabbitpp_postpass_on_parallel_detection():
    """RABBIT++ on top of the concurrent detection: the post-pass (oracle
    rabbitpp) applied to the concurrent RABBIT order and its communities is
    exactly the library's RABBIT++ order from the same detection."""
    A = synth.config(1, small=True).A
    perm_r, _ = spmv.reorder(A.row_ptr, A.col, "rabbit", parallel=True)
    comm = spmv.reorder_last_comm(A.n)
    perm_pp, _ = spmv.reorder(A.row_ptr, A.col, "rabbitpp", parallel=True)  # cached detection
    ref = rabbit.rabbitpp(A.n, A.row_ptr, A.col, perm_r, comm)
    assert np.array_equal(perm_pp, ref)


@pytest.mark.skipif((os.cpu_count() or 1) < 2, reason="needs several threads")
def test_parallel_rmat16_full_size_invariants():
    """BASELINE configs[0] at full size with every host thread."""
    A = synth.config(1).A
    perm, st = spmv.reorder(A.row_ptr, A.col, "rabbit", parallel=True, log=True)
    comm = spmv.reorder_last_comm(A.n)
    child, parent, dq = spmv.reorder_last_merges()
    assert np.all(dq > 0)
    assert permute.is_bijection(perm, A.n)
    q_final, _ = metrics.modularity_int(A.n, A.row_ptr, A.col, comm)
    q_init, _ = metrics.modularity_int(A.n, A.row_ptr, A.col, np.arange(A.n))
    assert q_final - q_init == 2 * int(dq.astype(object).sum())
