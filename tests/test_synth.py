"""The seeded generators: fast C++ == plain reference loops, and shape facts."""
import numpy as np
import pytest

import synth
from synth import gen


def _same(ref, m):
    rp, c, v = ref
    assert np.array_equal(rp, m.row_ptr)
    assert np.array_equal(c, m.col)
    assert np.array_equal(v.view(np.int32), m.val.view(np.int32))


def test_hash_matches():
    for s, a, b in [(0, 0, 0), (20230423, 5, 7), (2**63 + 11, 2**40, 3)]:
        assert synth.lib().synth_h1(s, a) == gen.h1(s, a)
        assert synth.lib().synth_h2(s, a, b) == gen.h2(s, a, b)


@pytest.mark.parametrize("scr,valmode", [(False, 0), (True, 1), (False, 2)])
def test_rmat_equal(scr, valmode):
    _same(gen.rmat(7, 4, 11, scramble=scr, seed_scr=9, valmode=valmode, seed_v=5),
          synth.rmat(7, 4, 11, scramble=scr, seed_scr=9, valmode=valmode, seed_v=5))


def test_sbm_equal_and_shape():
    ref = gen.sbm(6, 37, 5, 0.8, 3, True, 7, 0, 2)
    m = synth.sbm(6, 37, 5, 0.8, 3, True, 7, 0, 2)
    _same(ref, m)
    assert np.all(np.diff(m.row_ptr) == 5)
    for r in range(m.n):
        cs = m.col[m.row_ptr[r]:m.row_ptr[r + 1]]
        assert len(set(cs.tolist())) == 5 and np.all(np.diff(cs) > 0)


@pytest.mark.parametrize("periodic", [False, True])
def test_stencil_equal_and_shape(periodic):
    _same(gen.stencil27(5, periodic, True, 3, 0, 4), synth.stencil27(5, periodic, True, 3, 0, 4))
    m = synth.stencil27(6, periodic, False, 0, 2, 0)
    L = np.diff(m.row_ptr)
    if periodic:
        assert np.all(L == 27)
    else:
        assert L.max() == 27 and L.min() == 8 and m.nnz == (3 * 6 - 2) ** 3


def test_vector_and_scramble():
    assert np.array_equal(gen.vector(257, 7), synth.vector(257, 7))
    assert np.array_equal(gen.vector(64, 7, 1), synth.vector(64, 7, 1))
    t = synth.scramble_table(1000, 99)
    assert np.array_equal(np.sort(t), np.arange(1000))
    assert np.array_equal(gen.scramble_table(1000, 99), t)


def test_value_grids_exact_fp32():
    # sym values are k*2^-23 - 1 and pos values (k+1)*2^-24: exact in fp32
    h = np.array([gen.h1(1, i) for i in range(1000)], dtype=object)
    for hh in h[:50]:
        v = gen.sym_f32(int(hh))
        assert float(v) == (int(hh) >> 40) * 2.0**-23 - 1.0
        p = gen.pos_f32(int(hh))
        assert 0.0 < float(p) <= 1.0


def test_config_small_shapes():
    w = synth.config(1, small=True)
    assert w.A.n == 4096 and 0 < w.A.nnz <= 16 * 4096
    w2 = synth.config(2, small=True)
    assert w2.A.nnz == 16 * w2.A.n
    # planted order is the inverse of the label scramble
    assert np.array_equal(np.sort(w2.planted), np.arange(w2.A.n))
