"""C-ABI library: loads, exports every declared symbol, host-side calls.

spmv_reorder is host C++ (input preparation), so its bit-exact parity with
the oracle's RABBIT / RABBIT++ / RANDOM runs here without a GPU.
"""
import ctypes
import math

import numpy as np
import pytest

import synth
from oracle import metrics, rabbit
from paper_conf_ispass_balajicjk23_b200 import spmv


def test_library_exports_every_declared_symbol():
    L = spmv.lib()
    names = spmv.declared_symbols()
    assert len(names) == 34
    for nm in names:
        assert hasattr(L, nm), nm
    assert "sm_100a" in spmv.version()


def test_opts_default_and_errors_without_gpu():
    o = spmv._Opts()
    spmv.lib().spmv_opts_default(ctypes.byref(o))
    assert (o.l2_window, o.evict_first, o.rank, o.world, o.device) == (1, 1, 0, 1, -1)
    assert o.l2_hit_ratio == 1.0
    assert (o.nccl_comm, o.x_layout, o.exchange) == (None, spmv.XLAYOUT_GLOBAL, spmv.EXCHANGE_COLL)
    assert ctypes.sizeof(o) == 6 * 4 + 4 * 8 + 2 * 4 + 4 * 8   # layout of spmv_opts_t
    # collective backend / peers need a plan
    assert spmv.lib().spmv_set_coll(None, None) == 1
    assert spmv.lib().spmv_set_peers(None, None, 2) == 1
    h = ctypes.c_void_p()
    st = spmv.lib().spmv_plan(None, None, None, ctypes.byref(h))
    assert st == 1 and b"NULL" in spmv.lib().spmv_last_error()
    spmv.lib().spmv_destroy(None)  # safe on NULL


def _graphs():
    yield "rmat10", synth.rmat(10, 8, 3, seed_v=1)
    yield "sbm", synth.sbm(8, 64, 6, 0.9, 5, True, 2, 0, 1)
    yield "stencil", synth.stencil27(6, False, True, 4, 0, 1)


@pytest.mark.parametrize("name,A", list(_graphs()))
def test_reorder_rabbit_bitexact(name, A):
    r = rabbit.rabbit(A.n, A.row_ptr, A.col)
    perm, st = spmv.reorder(A.row_ptr, A.col, "rabbit")
    assert np.array_equal(perm, r.perm)
    comm = spmv.reorder_last_comm(A.n)
    assert np.array_equal(comm, r.comm)
    assert st.n_communities == len(r.toplevel)
    assert st.n_merges == len(r.merges)
    assert st.two_m == r.two_m
    q, two_m = metrics.modularity_int(A.n, A.row_ptr, A.col, r.comm)
    assert st.modularity_num == float(q)
    assert math.isclose(st.insularity, metrics.insularity(A.n, A.row_ptr, A.col, r.comm))
    assert math.isclose(st.skew, metrics.skew(A.row_ptr))
    _, big = metrics.community_stats(r.comm)
    assert math.isclose(st.largest_comm_frac, big)


@pytest.mark.parametrize("name,A", list(_graphs()))
@pytest.mark.parametrize("variant,method", [(rabbit.RABBITPP, "rabbitpp"),
                                            (rabbit.HUBSORT, "hubsort"),
                                            (rabbit.INSULAR_ONLY, "insular"),
                                            (rabbit.HUBGROUP_ONLY, "hubgroup"),
                                            (rabbit.HUBSORT_ONLY, "hubsort_only")])
def test_reorder_rabbitpp_bitexact(name, A, variant, method):
    r = rabbit.rabbit(A.n, A.row_ptr, A.col)
    ref = rabbit.rabbitpp(A.n, A.row_ptr, A.col, r.perm, r.comm, variant)
    perm, st = spmv.reorder(A.row_ptr, A.col, method)
    assert np.array_equal(perm, ref)
    assert st.n_hubs == int(rabbit.hub_flags(A.n, A.row_ptr, A.col).sum())
    ins = rabbit.insular_flags(A.n, A.row_ptr, A.col, r.comm)
    assert math.isclose(st.insular_frac, ins.mean())
    assert st.n_insular == int(ins.sum())


def test_reorder_rmat16_bitexact():
    # config-1-sized parity
    w = synth.config(1)
    r = rabbit.rabbit(w.A.n, w.A.row_ptr, w.A.col)
    perm, _ = spmv.reorder(w.A.row_ptr, w.A.col, "rabbit")
    assert np.array_equal(perm, r.perm)
    pp, _ = spmv.reorder(w.A.row_ptr, w.A.col, "rabbitpp")
    assert np.array_equal(pp, rabbit.rabbitpp(w.A.n, w.A.row_ptr, w.A.col, r.perm, r.comm))


def test_reorder_random_original_degsort():
    A = synth.rmat(9, 8, 2)
    p, _ = spmv.reorder(A.row_ptr, A.col, "random", seed=1234)
    assert np.array_equal(p, rabbit.random_perm(A.n, 1234))
    p, _ = spmv.reorder(A.row_ptr, A.col, "original")
    assert np.array_equal(p, np.arange(A.n))
    p, _ = spmv.reorder(A.row_ptr, A.col, "degsort")
    cc = np.bincount(A.col, minlength=A.n)
    seq = np.empty(A.n, np.int64)
    seq[p] = np.arange(A.n)
    assert all(cc[seq[i]] > cc[seq[i + 1]] or (cc[seq[i]] == cc[seq[i + 1]] and seq[i] < seq[i + 1])
               for i in range(A.n - 1))


def test_reorder_rejects_bad_input():
    with pytest.raises(spmv.SpmvError):
        spmv.reorder(np.array([0, 2, 1]), np.array([0, 1], np.int32), "rabbit")
    with pytest.raises(spmv.SpmvError):
        spmv.reorder(np.array([0, 1, 2]), np.array([0, 5], np.int32), "rabbit")
    with pytest.raises(spmv.SpmvError):
        spmv.reorder(np.array([0, 1, 2]), np.array([0, 1], np.int32), 99)


def test_reorder_empty_and_isolated():
    perm, st = spmv.reorder(np.zeros(4, np.int64), np.zeros(0, np.int32), "rabbitpp")
    assert sorted(perm.tolist()) == [0, 1, 2] and st.n_communities == 3
    perm, _ = spmv.reorder(np.zeros(1, np.int64), np.zeros(0, np.int32), "rabbit")
    assert perm.size == 0


def test_table4_entry_points_reject_null_plan_without_gpu():
    """spmv_exec_spmm4 / spmv_exec_coo / spmv_export_coo_rows validate their
    arguments before touching the device (EINVAL + message)."""
    L = spmv.lib()
    for fn, args in (("spmv_exec_spmm4", (None, None, None, None)),
                     ("spmv_exec_coo", (None, None, None, None)),
                     ("spmv_export_coo_rows", (None, None, None))):
        st = getattr(L, fn)(*args)
        assert st == 1, fn
        assert b"NULL" in L.spmv_last_error(), fn
