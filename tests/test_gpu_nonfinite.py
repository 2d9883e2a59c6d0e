"""Non-finite matrix values stay in their own row (Alg. 1).

Under Alg. 1 a row's result depends only on that row's entries: an Inf or NaN
stored in row r makes y[r] non-finite and leaves every other row alone.  The
lane-per-row kernels (k_lane, k_lane4) read 8-entry chunks that can be shared
with neighbouring rows; a neighbour's slot must contribute exactly +0, never
Inf * 0 = NaN.  Every row class is covered: short rows sharing a chunk with the
poisoned row (k_lane / k_lane4), a MID row, a CTA row and a hub row (split into
chunks with the fp64 fixup), and the COO kernel on the same plan.

Expected values: rows whose own entries are all finite follow the oracle within
the north-star tolerance; a poisoned row holds exactly one non-finite value, so
its result class (+Inf, -Inf or NaN) does not depend on the summation order and
is compared with an fp64 evaluation of the same products.
"""
import numpy as np
import pytest

from oracle import spmv as ospmv
from tests.test_gpu_parity import Mat, long_rows_matrix, mk_plan

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu
TOL = 1e-5


@pytest.fixture(scope="module")
def dev():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_ispass_balajicjk23_b200 import spmv  # noqa: F401
    return torch.device("cuda:0")


def poisoned():
    A = long_rows_matrix(3)
    rp, col, val = A.row_ptr, A.col.copy(), A.val.copy()
    L = np.diff(rp)
    short = [r for r in range(10, 2000) if 2 <= L[r] <= 20 and 2 <= L[r - 1] <= 20
             and 2 <= L[r + 1] <= 20]
    bad = {}
    # short rows: the poisoned entry is the first / last of its row, so the
    # 8-entry chunk holding it is shared with the previous / next row
    for r, where, v in ((short[0], -1, np.inf), (short[5], 0, -np.inf), (short[10], -1, np.nan),
                        (short[15], 0, np.nan)):
        k = rp[r + 1] - 1 if where == -1 else rp[r]
        val[k] = v
        bad[r] = k
    for r, v in ((2500, np.inf), (1000, np.nan), (5, -np.inf), (29999, np.inf)):  # MID, CTA, hubs
        k = rp[r] + L[r] // 2
        val[k] = v
        bad[r] = k
    # a poisoned entry whose x is 0 gives Inf * 0 = NaN in that row only
    return Mat(A.n, rp, col, val), bad


def _check(y, A, x, bad):
    y = np.asarray(y, np.float64)
    n = A.n
    good = np.ones(n, bool)
    good[list(bad)] = False
    rows = np.flatnonzero(good)
    ref = ospmv.spmv_rows(A.row_ptr, A.col, A.val, x, rows).astype(np.float64)
    tol = TOL * ospmv.abs_rowsum(A.row_ptr, A.col, A.val, x, rows) + 1e-37
    err = np.abs(y[rows] - ref)
    assert np.all(np.isfinite(y[rows])), f"{int((~np.isfinite(y[rows])).sum())} finite rows poisoned"
    assert np.all(err <= tol)
    for r in bad:
        a, b = int(A.row_ptr[r]), int(A.row_ptr[r + 1])
        e = float(np.sum(A.val[a:b].astype(np.float64) * x[A.col[a:b]].astype(np.float64)))
        assert not np.isfinite(y[r]), r
        if np.isnan(e):
            assert np.isnan(y[r]), (r, y[r])
        else:
            assert y[r] == e, (r, y[r], e)


@pytest.mark.parametrize("zero_x", [False, True])
def test_nonfinite_values_stay_in_their_row(dev, zero_x):
    A, bad = poisoned()
    rng = np.random.default_rng(1)
    x = rng.uniform(-1, 1, A.n).astype(np.float32)
    if zero_x:  # x = 0 under a poisoned entry: Inf * 0 = NaN, still only that row
        for r, k in bad.items():
            x[A.col[k]] = 0.0
    P = mk_plan(A, None, dev)  # identity: B = A with rows sorted, neighbours kept
    xd = torch.from_numpy(x).to(dev)
    # B = A up to the order inside rows; the oracle sees the same rows
    Bp, Bc, Bv = (t.cpu().numpy() for t in P.export_csr())
    B = Mat(A.n, Bp, Bc, Bv)
    bad_B = {r: None for r in bad}
    _check(P.exec(xd).cpu().numpy(), B, x, bad_B)
    _check(P.exec_coo(xd).cpu().numpy(), B, x, bad_B)
    X = np.ascontiguousarray(np.stack([x, x[::-1], 0.5 * x, -x], 1).astype(np.float32))
    Y = P.exec_spmm4(torch.from_numpy(X).to(dev)).cpu().numpy()
    for k in range(4):
        # column k of Y is bitwise spmv_exec(X[:, k])
        yk = P.exec(torch.from_numpy(np.ascontiguousarray(X[:, k])).to(dev)).cpu().numpy()
        nan = np.isnan(yk)
        assert np.array_equal(np.isnan(Y[:, k]), nan)
        assert np.array_equal(Y[~nan, k].view(np.int32), yk[~nan].view(np.int32))
    P.close()
