"""The power-iteration norm of spmv_exec_scaled (reading c22): sumsq_out =
sum over the rank's rows of (double) y^2, summed from y itself in fixed
16384-row segments, then the segment sums in order (include/spmv.h).

Pins: (1) it equals the exactly rounded sum math.fsum(y^2) of the y the call
returned to within the error bound of a recursive fp64 sum (depth < 64
additions over non-negative terms: <= 64 * 2^-53 relative); (2) since the
association depends only on the row count, it is bitwise the same for every
kernel schedule that produces the same y -- the single-launch k_small and the
per-class kernels, the short-row kernel variants 0 (lane) and 1 (panel) --
and for repeated calls."""
import math

import numpy as np
import pytest

import synth
from oracle import rabbit

from .test_gpu_parity import CASES, mk_plan

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def dev():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    return torch.device("cuda:0")


@pytest.mark.parametrize("name,make", CASES)
def test_norm_from_y_exact_and_schedule_independent(dev, name, make, monkeypatch):
    A = make()
    perm = rabbit.random_perm(A.n, 31)
    x = torch.from_numpy(synth.vector(A.n, 8)).to(dev)
    seen = []
    for variant in (0, 1):
        P = mk_plan(A, perm, dev, variant=variant)
        for small in ("0", "1"):
            monkeypatch.setenv("SPMV_SMALL", small)
            y = torch.empty(A.n, dtype=torch.float32, device=dev)
            ss = torch.zeros(1, dtype=torch.float64, device=dev)
            P.exec_scaled(x, y, None, ss)
            yh = y.cpu().numpy().astype(np.float64)
            s = float(ss.item())
            exact = math.fsum((yh * yh).tolist())
            assert abs(s - exact) <= 64 * 2.0**-53 * exact + 1e-300, (name, variant, small)
            P.exec_scaled(x, y, None, ss)
            assert float(ss.item()) == s                      # repeatable, bitwise
            seen.append((s, y.cpu().numpy().view(np.int32).copy()))
        P.close()
    for s, yb in seen[1:]:
        assert np.array_equal(yb, seen[0][1])                  # the same y ...
        assert s == seen[0][0]                                 # ... the same norm, bitwise
