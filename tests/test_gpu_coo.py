"""GPU parity of spmv_exec_coo (SpMV-COO, Table IV) against
the oracle's spmv_coo, through the C ABI.

Bars: COO row array bit-exact (integer output); y within 1e-5 * sum|a x| per
row; empty rows exactly 0; bitwise repeatable; rows crossing thread and tile
(2048-entry) boundaries, hub rows and empty leading / trailing rows covered."""
import numpy as np
import pytest

import synth
from oracle import permute, rabbit, spmv as ospmv

from .test_gpu_parity import CASES, Mat, mk_plan

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu
TOL = 1e-5


@pytest.fixture(scope="module")
def dev():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    return torch.device("cuda:0")


def _edge_matrices():
    rng = np.random.default_rng(4)
    # empty leading / trailing rows, one row spanning several 2048-tiles,
    # rows exactly 8 / 2048 long at thread / tile boundaries
    L = np.zeros(9000, np.int64)
    L[5:2053] = 1          # 2048 single-entry rows: one full tile of row starts
    L[3000] = 2048
    L[3001] = 7
    L[3002] = 9
    L[4000] = 10000        # crosses 5+ tiles
    L[4200:4264] = 512     # rows exactly one warp tile long
    L[4300:4310] = 16      # one lane each
    L[4400] = 513
    L[4001:4100] = rng.integers(0, 20, 99)
    L[8990] = 3
    rp = np.concatenate([[0], np.cumsum(L)])
    col = rng.integers(0, 9000, rp[-1]).astype(np.int32)
    val = rng.uniform(-1, 1, rp[-1]).astype(np.float32)
    yield "edges", Mat(9000, rp, col, val)
    yield "empty", Mat(100, np.zeros(101, np.int64), np.zeros(0, np.int32), np.zeros(0, np.float32))
    L = np.zeros(500, np.int64)
    L[-1] = 5000           # all entries in the last row
    rp = np.concatenate([[0], np.cumsum(L)])
    yield "lastrow", Mat(500, rp, rng.integers(0, 500, 5000).astype(np.int32),
                         rng.uniform(-1, 1, 5000).astype(np.float32))


ALL = CASES + [(nm, (lambda m=m: m)) for nm, m in _edge_matrices()]


@pytest.mark.parametrize("variant", ["1", "2", "2e8"])
@pytest.mark.parametrize("name,make", ALL)
def test_coo_matches_oracle(dev, name, make, variant, monkeypatch):
    """variant 1: CTA tiles of 2048 entries (k_coo); 2: warp tiles of 32 x 16
    entries (k_coo_w, the default); 2e8: warp tiles of 32 x 8 -- SPMV_COO_V /
    SPMV_COO_E dev knobs."""
    monkeypatch.setenv("SPMV_COO_V", variant[0])
    monkeypatch.setenv("SPMV_COO_E", "8" if variant == "2e8" else "16")
    A = make()
    perm = rabbit.random_perm(A.n, 21) if A.nnz and name not in ("edges", "lastrow") else None
    P = mk_plan(A, perm, dev)
    pm = np.arange(A.n) if perm is None else np.asarray(perm, np.int64)
    Bp, Bc, Bv = permute.permute_csr(A.n, A.row_ptr, A.col, A.val, pm)
    rows = P.export_coo_rows().cpu().numpy()
    assert np.array_equal(rows, ospmv.coo_rows(Bp))
    x = synth.vector(A.n, 7)
    xB = permute.permute_vec(x, pm)
    xd = torch.from_numpy(xB).to(dev)
    y = torch.full((A.n,), float("nan"), device=dev)
    P.exec_coo(xd, y)
    y = y.cpu().numpy()
    ref = ospmv.spmv_coo(A.n, ospmv.coo_rows(Bp), Bc, Bv, xB)
    scale = ospmv.abs_rowsum(Bp, Bc, Bv, xB)
    err = np.abs(y.astype(np.float64) - ref.astype(np.float64))
    bad = ~(err <= TOL * scale + 1e-37)  # NaN (unwritten y) counts as bad
    assert not bad.any(), f"{name}: {int(bad.sum())} rows bad, first {np.flatnonzero(bad)[:5]}"
    assert np.all(y[np.diff(Bp) == 0] == 0)
    y2 = P.exec_coo(xd).cpu().numpy()
    assert np.array_equal(y.view(np.int32), y2.view(np.int32))
    P.close()


def test_coo_full_size_rmat16_all_rows(dev):
    """BASELINE configs[0] (RMAT-16, 65K rows / 955K nnz), RABBIT++: every row."""
    from paper_conf_ispass_balajicjk23_b200 import spmv
    A = synth.config(1).A
    perm, _ = spmv.reorder(A.row_ptr, A.col, "rabbitpp")
    P = mk_plan(A, perm, dev)
    Bp, Bc, Bv = permute.permute_csr(A.n, A.row_ptr, A.col, A.val, perm.astype(np.int64))
    x = synth.vector(A.n, 3)
    xB = permute.permute_vec(x, perm)
    y = P.exec_coo(torch.from_numpy(xB).to(dev)).cpu().numpy()
    ref = ospmv.spmv(Bp, Bc, Bv, xB)
    scale = ospmv.abs_rowsum(Bp, Bc, Bv, xB)
    assert np.all(np.abs(y.astype(np.float64) - ref) <= TOL * scale + 1e-37)
    P.close()
