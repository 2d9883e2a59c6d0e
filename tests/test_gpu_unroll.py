"""Stream-load modes of the warp-per-row, CTA-per-row and hub-chunk kernels
(SPMV_MID_STREAM dev knob: ld.cs; no L1 allocation; no L1 allocation + L2
evict_first policy).  They change where col / val are cached, never the
values or the association (each lane sums its strided entries j, j + W, ...
in that order, four in flight, a guarded slot past the row adding +0), so y
is bitwise the same for every mode (include/spmv.h canonical order) and
within 1e-5 * sum|a x| of the oracle.  Row lengths sit on both sides of every
32*4 and 256*4 boundary and of the class bounds (32 / 2048 / 16384, hub
chunking above)."""
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


def _boundaries():
    rng = np.random.default_rng(48)
    lens = [33, 127, 128, 129, 255, 256, 257, 383, 511, 512, 1000, 1023, 1024, 1025, 2047,
            2048, 2049, 3000, 4095, 4096, 4097, 8191, 8192, 16383, 16384, 16385, 40000, 50001]
    n = 20000
    L = rng.integers(0, 20, n)
    where = rng.choice(n, len(lens), replace=False)
    L[where] = lens
    rp = np.concatenate([[0], np.cumsum(L)])
    col = rng.integers(0, n, rp[-1]).astype(np.int32)
    val = rng.uniform(-1, 1, rp[-1]).astype(np.float32)
    return Mat(n, rp, col, val)


ALL = CASES + [("boundaries", _boundaries)]


@pytest.mark.parametrize("name,make", ALL)
def test_stream_modes_bitwise_and_oracle(dev, name, make, monkeypatch):
    A = make()
    perm = rabbit.random_perm(A.n, 5) if A.nnz and name != "boundaries" else None
    P = mk_plan(A, perm, dev)
    pm = np.arange(A.n) if perm is None else np.asarray(perm, np.int64)
    Bp, Bc, Bv = permute.permute_csr(A.n, A.row_ptr, A.col, A.val, pm)
    xB = permute.permute_vec(synth.vector(A.n, 3), pm)
    xd = torch.from_numpy(xB).to(dev)
    ref = ospmv.spmv(Bp, Bc, Bv, xB)
    scale = ospmv.abs_rowsum(Bp, Bc, Bv, xB)
    ys = []
    for mode in ("0", "1", "2"):
        monkeypatch.setenv("SPMV_MID_STREAM", mode)
        monkeypatch.setenv("SPMV_SMALL", "0")        # the per-class kernels, not k_small
        y = P.exec(xd).cpu().numpy()
        err = np.abs(y.astype(np.float64) - ref.astype(np.float64))
        bad = ~(err <= TOL * scale + 1e-37)
        assert not bad.any(), f"{name} mode {mode}: {int(bad.sum())} rows bad"
        ys.append(y.view(np.int32).copy())
    for y in ys[1:]:
        assert np.array_equal(ys[0], y)
    P.close()
