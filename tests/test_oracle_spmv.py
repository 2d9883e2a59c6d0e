"""Pins of the oracle SpMV (Alg. 1) and the compulsory-traffic
formula against things other than the oracle itself."""
import json
import os

import numpy as np
import pytest
import scipy.sparse as sp

from oracle import cref, metrics, permute, spmv

GOLD = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "paper_pins.json")))


def rand_csr(n, nnz_per_row, seed, dup=True, empty_frac=0.2):
    rng = np.random.default_rng(seed)
    L = rng.integers(0, 2 * nnz_per_row + 1, n)
    L[rng.random(n) < empty_frac] = 0
    rp = np.zeros(n + 1, np.int64)
    rp[1:] = np.cumsum(L)
    col = rng.integers(0, n, rp[-1]).astype(np.int32)
    if dup and rp[-1] > 3:
        col[1] = col[0] if L[0] >= 2 else col[1]
    val = rng.uniform(-1, 1, rp[-1]).astype(np.float32)
    x = rng.uniform(-1, 1, n).astype(np.float32)
    return rp, col, val, x


@pytest.mark.parametrize("seed", range(5))
def test_spmv_vs_dense_bruteforce(seed):
    n = 37
    rp, col, val, x = rand_csr(n, 4, seed)
    D = spmv.dense(n, rp, col, val)
    ref = D @ x.astype(np.float64)
    y = spmv.spmv_f64(rp, col, val, x)
    scale = spmv.abs_rowsum(rp, col, val, x)
    assert np.all(np.abs(y - ref) <= 1e-12 * scale + 1e-300)


@pytest.mark.parametrize("seed", range(3))
def test_spmv_vs_scipy(seed):
    n = 500
    rp, col, val, x = rand_csr(n, 8, seed)
    M = sp.csr_matrix((val.astype(np.float64), col, rp), shape=(n, n))
    ref = M @ x.astype(np.float64)
    y = spmv.spmv(rp, col, val, x)
    scale = spmv.abs_rowsum(rp, col, val, x)
    assert np.all(np.abs(y.astype(np.float64) - ref) <= 1e-7 * scale + 1e-30)


def test_spmv_exact_cancellation():
    # fp32 values 1e8, 1, -1e8 in one row: the exact sum is 1 (naive fp32 gives 0)
    rp = np.array([0, 3, 3])
    col = np.array([0, 1, 0], np.int32)
    val = np.array([1e8, 1.0, -1e8], np.float32)
    x = np.ones(2, np.float32)
    y = spmv.spmv(rp, col, val, x)
    assert y[0] == np.float32(1.0)
    assert y[1] == 0.0 and not np.signbit(y[1])     # empty row: Y initialised to 0 (c1)


def test_spmv_order_independent():
    rp, col, val, x = rand_csr(200, 10, 7)
    y = spmv.spmv(rp, col, val, x)
    rng = np.random.default_rng(1)
    col2, val2 = col.copy(), val.copy()
    for r in range(200):
        a, b = rp[r], rp[r + 1]
        o = rng.permutation(b - a) + a
        col2[a:b], val2[a:b] = col[o], val[o]
    assert np.array_equal(y.view(np.int32), spmv.spmv(rp, col2, val2, x).view(np.int32))


@pytest.mark.parametrize("seed", range(3))
def test_permutation_invariant_bitwise(seed):
    # P(A x) == (P A P^T)(P x) bitwise (exact row sums)
    n = 300
    rp, col, val, x = rand_csr(n, 6, seed)
    perm = np.random.default_rng(seed + 10).permutation(n)
    y = spmv.spmv(rp, col, val, x)
    Bp, Bc, Bv = permute.permute_csr(n, rp, col, val, perm)
    yB = spmv.spmv(Bp, Bc, Bv, permute.permute_vec(x, perm))
    assert np.array_equal(permute.permute_vec(y, perm).view(np.int32), yB.view(np.int32))


def test_spmv_rows_and_c_oracle():
    n = 2000
    rp, col, val, x = rand_csr(n, 12, 3)
    y = spmv.spmv_f64(rp, col, val, x)
    rows = [0, 5, 17, 1999]
    assert np.array_equal(spmv.spmv_rows(rp, col, val, x, rows), y[rows].astype(np.float32))
    yc = cref.spmv_f64(rp, col, val, x)
    yn, a = cref.spmv_neumaier(rp, col, val, x)
    scale = spmv.abs_rowsum(rp, col, val, x)
    assert np.allclose(a, scale, rtol=1e-12, atol=0)
    assert np.all(np.abs(yc - y) <= 1e-13 * scale + 1e-300)
    assert np.all(np.abs(yn - y) <= 1e-15 * scale + 1e-300)


def test_compulsory_traffic_pins():
    for c in GOLD["compulsory_traffic"]["cases"]:
        assert metrics.ideal_bytes(c["n"], c["nnz"], c["w_off"]) == c["bytes"]
    ai = GOLD["arithmetic_intensity_upper_bound"]
    assert ai["flops_per_nz"] / ai["bytes_per_nz"] == ai["ai"]


# ---- SpMM-CSR-4 (Table IV) -------------------------------
@pytest.mark.parametrize("seed", range(4))
def test_spmm_vs_dense_bruteforce_and_scipy(seed):
    n = 41
    rp, col, val, _ = rand_csr(n, 5, seed)
    X = np.random.default_rng(100 + seed).uniform(-1, 1, (n, 4)).astype(np.float32)
    Y = spmv.spmm(rp, col, val, X).astype(np.float64)
    D = spmv.dense(n, rp, col, val)
    scale = spmv.abs_rowsum_mat(rp, col, val, X)
    # dense brute force in fp64, then the one fp32 rounding: within 1 ulp-ish of fp32
    assert np.all(np.abs(Y - D @ X.astype(np.float64)) <= 2 ** -23 * scale + 1e-300)
    S = sp.csr_matrix((val.astype(np.float64), col, rp), shape=(n, n))
    assert np.all(np.abs(Y - S @ X.astype(np.float64)) <= 2 ** -23 * scale + 1e-300)


def test_spmm_exact_cancellation_and_empty_rows():
    # row 0: 1e8*1 + 1*1 - 1e8*1 = 1 exactly in column 0; column 1 uses x = 0
    rp = np.array([0, 3, 3, 4], np.int64)
    col = np.array([0, 1, 2, 0], np.int32)
    val = np.array([1e8, 1.0, -1e8, 2.0], np.float32)
    X = np.array([[1, 0, 0.5, -1], [1, 0, 0.5, -1], [1, 0, 0.5, -1]], np.float32)
    Y = spmv.spmm(rp, col, val, X)
    assert Y[0, 0] == 1.0 and Y[0, 1] == 0.0 and Y[0, 2] == 0.5 and Y[0, 3] == -1.0
    assert np.all(Y[1] == 0) and np.array_equal(Y[2], 2 * X[0])


def test_spmm_rows_sample_agrees():
    rp, col, val, _ = rand_csr(60, 6, 9)
    X = np.random.default_rng(3).uniform(-1, 1, (60, 4)).astype(np.float32)
    rows = [0, 7, 59, 31]
    assert np.array_equal(spmv.spmm_rows(rp, col, val, X, rows), spmv.spmm(rp, col, val, X)[rows])


# ---- SpMV-COO (Table IV) ---------------------------------
@pytest.mark.parametrize("seed", range(4))
def test_coo_rows_equal_scipy_and_spmv_coo_vs_dense(seed):
    n = 53
    rp, col, val, x = rand_csr(n, 4, seed)
    rows = spmv.coo_rows(rp)
    S = sp.csr_matrix((val, col, rp), shape=(n, n))
    assert np.array_equal(rows, S.tocoo().row)  # library routine, duplicates kept
    y = spmv.spmv_coo(n, rows, col, val, x).astype(np.float64)
    D = spmv.dense(n, rp, col, val)
    scale = spmv.abs_rowsum(rp, col, val, x)
    assert np.all(np.abs(y - D @ x.astype(np.float64)) <= 2 ** -23 * scale + 1e-300)
    # triplet order does not matter (exact sums)
    sh = np.random.default_rng(seed).permutation(len(rows))
    y2 = spmv.spmv_coo(n, rows[sh], col[sh], val[sh], x)
    assert np.array_equal(y2.view(np.int32), y.astype(np.float32).view(np.int32))


def test_coo_empty_rows_and_cancellation():
    rows = np.array([2, 2, 2], np.int64)
    col = np.array([0, 1, 2], np.int32)
    val = np.array([1e8, 1.0, -1e8], np.float32)
    y = spmv.spmv_coo(5, rows, col, val, np.ones(5, np.float32))
    assert list(y) == [0, 0, 1.0, 0, 0]
