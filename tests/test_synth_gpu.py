"""The GPU RMAT / Kronecker generator (synth/csrc/synth_gpu.cu) produces the
same CSR as the host generator (synth/csrc/synth.cpp), bit for bit: row
pointer, columns and value bits.  Input generation only -- this module is
shared by the oracle and the CUDA path and holds none of the method."""
import numpy as np
import pytest

import synth

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu


def _same(h, d):
    g = d.to_host()
    assert g.n == h.n and g.nnz == h.nnz
    assert np.array_equal(g.row_ptr, h.row_ptr)
    assert np.array_equal(g.col, h.col)
    assert np.array_equal(g.val.view(np.int32), h.val.view(np.int32))


@pytest.mark.parametrize("scale,ef,scr,vm", [(1, 1, False, 0), (5, 4, True, 1), (10, 8, False, 0),
                                             (12, 16, True, 1), (13, 3, True, 2), (9, 0, False, 0)])
def test_rmat_gpu_equals_host(scale, ef, scr, vm):
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    kw = dict(seed=77 + scale, scramble=scr, seed_scr=5, valmode=vm, seed_v=9)
    _same(synth.rmat(scale, ef, **kw), synth.rmat_gpu(scale, ef, **kw))


@pytest.mark.parametrize("k,small", [(1, False), (5, True), (3, False)])
def test_config_gpu_equals_host(k, small):
    """BASELINE configs[0] (RMAT-16) and configs[2] (RMAT-26, 1.06 G nnz) at
    full size, Kronecker-14 (the small C5)."""
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    w = synth.config(k, small=small)
    name, A, x = synth.config_gpu(k, small=small)
    assert name == w.name
    assert np.array_equal(x.view(np.int32), w.x.view(np.int32))
    _same(w.A, A)
