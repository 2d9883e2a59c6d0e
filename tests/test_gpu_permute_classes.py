"""B = P A P^T on rows of every sort path of
spmv_permute, bit-exact against the oracle's permute_csr (the definition
B[perm i, perm j] = A[i, j], rows sorted by column, duplicates in A's order):

  * L <= 32: relabel + register sort (k_relabel_sort_short);
  * 32 < L <= 256: warp register bitonic, 4 keys per lane up to 128, 8 above
    (k_relabel_sort_mid);
  * 256 < L <= 4096: shared-memory bitonic sized to the row (k_sort_cta);
  * L > 4096: 4096-entry tiles sorted in shared memory, then merge-path passes
    of width 4096, 8192, ... (k_big_chunk_sort, k_big_split, k_big_merge_tile),
    including rows whose last run has no partner in a pass and rows that end
    exactly on a tile boundary.

Each special row gets runs of duplicate columns, so a sort that is not stable
(duplicates out of A's order) fails the value comparison."""
import numpy as np
import pytest

from oracle import permute, rabbit

from .test_gpu_parity import Mat, mk_plan

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

LENS = [1, 31, 32, 33, 64, 100, 127, 128, 129, 200, 255, 256, 257, 300, 1024, 1025, 4095, 4096,
        4097, 8191, 8192, 8193, 12288, 12289, 20000, 40961, 70000]


@pytest.fixture(scope="module")
def dev():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    return torch.device("cuda:0")


def _matrix(seed):
    rng = np.random.default_rng(seed)
    n = 90000
    L = rng.integers(0, 40, n)
    where = rng.choice(n, len(LENS), replace=False)
    L[where] = LENS
    rp = np.concatenate([[0], np.cumsum(L)]).astype(np.int64)
    col = rng.integers(0, n, rp[-1]).astype(np.int32)
    for r in where:
        a, e = rp[r], rp[r + 1]
        k = min(e - a, 50)
        col[a:a + k // 2] = col[a]            # a run of duplicates at the start
        col[e - k // 3:e] = n - 1             # and one on the largest column
    val = rng.uniform(-1, 1, rp[-1]).astype(np.float32)
    return Mat(n, rp, col, val)


@pytest.mark.parametrize("seed", [1, 2])
def test_permute_every_sort_path_bitexact(dev, seed):
    A = _matrix(seed)
    perm = rabbit.random_perm(A.n, 100 + seed)
    P = mk_plan(A, perm, dev)
    pm = np.asarray(perm, np.int64)
    Bp, Bc, Bv = permute.permute_csr(A.n, A.row_ptr, A.col, A.val, pm)
    rp, c, v = (t.cpu().numpy() for t in P.export_csr())
    assert np.array_equal(rp, Bp)
    assert np.array_equal(c, Bc)
    assert np.array_equal(v.view(np.int32), Bv.view(np.int32))
    P.close()
