"""GPU parity of spmv_exec_spmm4 (SpMM-CSR-4, Table IV)
against the oracle's spmm, through the C ABI.

Bars: every Y[r, k] within 1e-5 * sum_j |a_rj X[j, k]| of the oracle's
correctly rounded sum; column k bitwise equal to spmv_exec on X[:, k] (same
row classes and canonical order, include/spmv.h); bitwise repeatable."""
import numpy as np
import pytest

import synth
from oracle import permute, rabbit, spmv as ospmv

from .test_gpu_parity import CASES, mk_plan

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu
TOL = 1e-5


@pytest.fixture(scope="module")
def dev():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    return torch.device("cuda:0")


def _X(n, seed):
    return np.stack([synth.vector(n, seed + k) for k in range(4)], 1).astype(np.float32)


@pytest.mark.parametrize("name,make", CASES)
def test_spmm4_matches_oracle_and_spmv_columns(dev, name, make):
    A = make()
    perm = rabbit.random_perm(A.n, 11)
    P = mk_plan(A, perm, dev)
    Bp, Bc, Bv = permute.permute_csr(A.n, A.row_ptr, A.col, A.val, perm)
    X = _X(A.n, 500)
    Xd = torch.from_numpy(X).to(dev).contiguous()
    Y = P.exec_spmm4(Xd).cpu().numpy()
    ref = ospmv.spmm(Bp, Bc, Bv, X)
    scale = ospmv.abs_rowsum_mat(Bp, Bc, Bv, X)
    err = np.abs(Y.astype(np.float64) - ref.astype(np.float64))
    bad = err > TOL * scale + 1e-37
    assert not bad.any(), f"{name}: {int(bad.sum())} entries out of tolerance"
    for k in range(4):
        yk = P.exec(Xd[:, k].contiguous()).cpu().numpy()
        assert np.array_equal(yk.view(np.int32), Y[:, k].copy().view(np.int32)), f"{name} col {k}"
    Y2 = P.exec_spmm4(Xd).cpu().numpy()
    assert np.array_equal(Y.view(np.int32), Y2.view(np.int32))
    assert np.all(Y[np.diff(Bp) == 0] == 0)
    P.close()


def test_spmm4_rejects_misaligned(dev):
    from paper_conf_ispass_balajicjk23_b200 import spmv
    A = synth.config(1, small=True).A
    P = mk_plan(A, None, dev)
    buf = torch.zeros(4 * A.n + 1, dtype=torch.float32, device=dev)
    with pytest.raises(spmv.SpmvError):
        P.exec_spmm4(buf[1:].view(A.n, 4))
    P.close()


def test_spmm4_full_size_sbm_sampled(dev):
    """BASELINE configs[1] at full size (4M rows / 64M nnz), RABBIT++ order:
    sampled rows against the oracle, columns against spmv_exec bitwise."""
    from paper_conf_ispass_balajicjk23_b200 import spmv
    w = synth.config(2)
    A = w.A
    perm, _ = spmv.reorder(A.row_ptr, A.col, "rabbitpp")
    P = mk_plan(A, perm, dev, rp_dtype=torch.int32)
    Bp, Bc, Bv = permute.permute_csr_scipy(A.n, A.row_ptr, A.col, A.val, perm.astype(np.int64))
    X = _X(A.n, 900)
    Xd = torch.from_numpy(X).to(dev)
    Y = P.exec_spmm4(Xd).cpu().numpy()
    rows = np.random.default_rng(1).choice(A.n, 2000, replace=False)
    rows = np.concatenate([rows, [0, A.n - 1]])
    ref = ospmv.spmm_rows(Bp, Bc, Bv, X, rows)
    for t, r in enumerate(rows):
        a, b = Bp[r], Bp[r + 1]
        scale = np.abs(Bv[a:b].astype(np.float64)[:, None] * X[Bc[a:b]].astype(np.float64)).sum(0)
        assert np.all(np.abs(Y[r].astype(np.float64) - ref[t]) <= TOL * scale + 1e-37), r
    y0 = P.exec(Xd[:, 2].contiguous()).cpu().numpy()
    assert np.array_equal(y0.view(np.int32), Y[:, 2].copy().view(np.int32))
    P.close()
