"""Pins of the oracle permutation B = P A P^T against the dense
definition B[perm[i], perm[j]] = A[i, j] and vector identities."""
import numpy as np
import pytest

from oracle import permute, spmv
from tests.test_oracle_spmv import rand_csr


def test_bijection_check():
    assert permute.is_bijection(np.array([2, 0, 1]), 3)
    assert not permute.is_bijection(np.array([2, 0, 2]), 3)
    assert not permute.is_bijection(np.array([3, 0, 1]), 3)
    assert not permute.is_bijection(np.array([-1, 0, 1]), 3)
    assert permute.is_bijection(np.zeros(0, np.int64), 0)


@pytest.mark.parametrize("seed", range(4))
def test_dense_definition(seed):
    n = 23
    rp, col, val, x = rand_csr(n, 3, seed)
    perm = np.random.default_rng(seed).permutation(n)
    A = spmv.dense(n, rp, col, val)
    Bp, Bc, Bv = permute.permute_csr(n, rp, col, val, perm)
    B = spmv.dense(n, Bp, Bc, Bv)
    for i in range(n):
        for j in range(n):
            assert B[perm[i], perm[j]] == A[i, j]
    # rows sorted by new column
    for r in range(n):
        assert np.all(np.diff(Bc[Bp[r]:Bp[r + 1]]) >= 0)
    # multiset of values preserved bit for bit
    assert np.array_equal(np.sort(Bv.view(np.int32)), np.sort(val.view(np.int32)))


def test_stable_duplicates():
    # row 0 holds (0,1)=a, (0,2)=b, (0,1)=c; duplicates keep their order
    rp = np.array([0, 3, 3, 3])
    col = np.array([1, 2, 1], np.int32)
    val = np.array([1.5, 2.5, 3.5], np.float32)
    perm = np.array([2, 0, 1])            # 1 -> 0, 2 -> 1
    Bp, Bc, Bv = permute.permute_csr(3, rp, col, val, perm)
    assert list(Bp) == [0, 0, 0, 3]
    assert list(Bc) == [0, 0, 1] and list(Bv) == [1.5, 3.5, 2.5]


def test_vector_roundtrip_and_rows():
    n = 100
    rp, col, val, x = rand_csr(n, 5, 9)
    perm = np.random.default_rng(3).permutation(n)
    px = permute.permute_vec(x, perm)
    assert np.array_equal(permute.permute_vec(px, perm, inverse_=True), x)
    assert all(px[perm[i]] == x[i] for i in range(n))
    Bp, Bc, Bv = permute.permute_csr(n, rp, col, val, perm)
    inv = permute.inverse(perm)
    assert np.array_equal(inv[perm], np.arange(n))
    rows = [0, 7, 50, 99]
    for r, (c, v) in zip(rows, permute.permute_rows(rp, col, val, perm, inv, rows)):
        assert np.array_equal(c, Bc[Bp[r]:Bp[r + 1]])
        assert np.array_equal(v.view(np.int32), Bv[Bp[r]:Bp[r + 1]].view(np.int32))


def test_identity_perm_sorts_rows():
    rp = np.array([0, 3, 4])
    col = np.array([1, 0, 1], np.int32)
    val = np.array([1, 2, 3, 4], np.float32)[:3]
    rp = np.array([0, 3, 3])
    Bp, Bc, Bv = permute.permute_csr(2, rp, col, val, np.arange(2))
    assert list(Bc) == [0, 1, 1] and list(Bv) == [2, 1, 3]


def test_permute_block_equals_definition():
    """permute_block (the bounded-sample builder of bench.py's cpu_baseline)
    gives exactly the rows of permute_csr, which is pinned to the dense
    definition B[perm i, perm j] = A[i, j] above."""
    import synth
    from oracle import rabbit
    A = synth.rmat(10, 8, 5, seed_v=2)
    perm = rabbit.random_perm(A.n, 3)
    inv = permute.inverse(perm)
    Bp, Bc, Bv = permute.permute_csr(A.n, A.row_ptr, A.col, A.val, perm)
    for r0, r1 in ((0, A.n), (17, 400), (A.n - 5, A.n), (3, 3)):
        rp, c, v = permute.permute_block(A.row_ptr, A.col, A.val, perm, inv, r0, r1)
        assert np.array_equal(rp, Bp[r0:r1 + 1] - Bp[r0])
        assert np.array_equal(c, Bc[Bp[r0]:Bp[r1]])
        assert np.array_equal(v.view(np.int32), Bv[Bp[r0]:Bp[r1]].view(np.int32))
