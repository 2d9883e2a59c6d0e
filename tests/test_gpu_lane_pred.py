"""Gather policy of the short-row kernel (plan decision `lane_pred_gather`,
SPMV_LANE_PRED dev knob to force it): with it, k_lane gathers x only for a
row's own slots of each 8-entry chunk; without it every slot is gathered and
the foreign ones are zeroed.  Either way a row's sum is the same sequence of
fp32 operations (include/spmv.h canonical order, L <= 32 sequential), so y is
bitwise identical, in the per-class kernels and in k_small, and within
1e-5 * sum|a x| of the fsum oracle (north_star tolerance, reading c3).

The plan's choice: the 27-point stencil (every row a short row, 27 entries
straddling 4-5 chunks) takes the predicated gathers; the planted-community
SBM (16-entry rows, chunk-aligned) does not."""
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


@pytest.mark.parametrize("name,make", CASES)
def test_lane_gather_policy_bitwise_and_oracle(dev, name, make, monkeypatch):
    A = make()
    perm = rabbit.random_perm(A.n, 13)
    P = mk_plan(A, perm, dev)
    pm = np.asarray(perm, np.int64)
    Bp, Bc, Bv = permute.permute_csr(A.n, A.row_ptr, A.col, A.val, pm)
    xB = permute.permute_vec(synth.vector(A.n, 4), pm)
    xd = torch.from_numpy(xB).to(dev)
    ref = ospmv.spmv(Bp, Bc, Bv, xB)
    scale = ospmv.abs_rowsum(Bp, Bc, Bv, xB)
    ys = []
    for small in ("0", "1"):
        for pred in ("0", "1"):
            monkeypatch.setenv("SPMV_SMALL", small)
            monkeypatch.setenv("SPMV_LANE_PRED", pred)
            y = P.exec(xd).cpu().numpy()
            err = np.abs(y.astype(np.float64) - ref.astype(np.float64))
            bad = ~(err <= TOL * scale + 1e-37)
            assert not bad.any(), f"{name} small={small} pred={pred}: {int(bad.sum())} rows bad"
            ys.append(y.view(np.int32).copy())
    for y in ys[1:]:
        assert np.array_equal(ys[0], y)
    P.close()


def test_plan_chooses_lane_gather_policy(dev):
    st = synth.config(4, small=True).A                 # stencil 24^3: 27-entry rows
    P = mk_plan(st, rabbit.random_perm(st.n, 1), dev)
    i = P.info()
    assert i["lane_nnz"] == st.nnz                      # every row is a short row
    assert 5 * i["lane_waste_slots"] >= i["lane_nnz"]
    assert i["lane_pred_gather"] == 1
    P.close()
    sb = synth.config(2, small=True).A                 # SBM: 16 entries per row
    P = mk_plan(sb, None, dev)
    i = P.info()
    assert i["lane_waste_slots"] == 0                   # row_ptr = 16 r: chunk-aligned
    assert i["lane_pred_gather"] == 0
    P.close()
