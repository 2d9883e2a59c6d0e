"""Plain numpy reference of the synthetic generators (small sizes only).

Same definitions as ``synth/csrc/synth.cpp`` (see its header); the fast C++
library is checked bit-for-bit against these loops in tests/test_synth.py.
Holds none of the method's arithmetic.
"""
from __future__ import annotations

import numpy as np

_M = (1 << 64) - 1
GOLDEN = 0x9E3779B97F4A7C15


def mix64(z: int) -> int:
    z &= _M
    z = ((z ^ (z >> 30)) * 0xBF58476D1CE4E5B9) & _M
    z = ((z ^ (z >> 27)) * 0x94D049BB133111EB) & _M
    return z ^ (z >> 31)


def h1(s: int, a: int) -> int:
    return mix64((s + GOLDEN * (a + 1)) & _M)


def h2(s: int, a: int, b: int) -> int:
    return h1(h1(s, a), b)


def sym_f32(h: int) -> np.float32:
    return np.float32((h >> 40) * (1.0 / 8388608.0) - 1.0)


def pos_f32(h: int) -> np.float32:
    return np.float32(((h >> 40) + 1) * (1.0 / 16777216.0))


def val_of(mode: int, h: int) -> np.float32:
    return sym_f32(h) if mode == 0 else pos_f32(h) if mode == 1 else np.float32(1.0)


def thr53(p: float) -> int:
    return int(p * 9007199254740992.0)


class Bij:
    """Bijection on [0, 2^k): 4 rounds of odd-multiply+add and xor-shift."""

    def __init__(self, k: int, seed: int):
        self.k = k
        self.mask = (1 << k) - 1
        self.shift = max(1, (k + 1) // 2)
        self.mul = [(h1(seed, 2 * r) | 1) & self.mask for r in range(4)]
        self.add = [h1(seed, 2 * r + 1) & self.mask for r in range(4)]

    def __call__(self, v: int) -> int:
        if self.k == 0:
            return 0
        for r in range(4):
            v = (v * self.mul[r] + self.add[r]) & self.mask
            v ^= v >> self.shift
        return v


class Scramble:
    """Cycle-walking bijection on [0, n)."""

    def __init__(self, n: int, seed: int):
        k = 0
        while (1 << k) < n:
            k += 1
        self.n = n
        self.b = Bij(k, seed)

    def __call__(self, v: int) -> int:
        u = self.b(v)
        while u >= self.n:
            u = self.b(u)
        return u


def _csr_from_rows(n, rows, valmode, seed_v):
    row_ptr = np.zeros(n + 1, np.int64)
    cols, vals = [], []
    for i in range(n):
        cs = sorted(set(rows[i]))
        row_ptr[i + 1] = row_ptr[i] + len(cs)
        for c in cs:
            cols.append(c)
            vals.append(val_of(valmode, h2(seed_v, i, c)))
    return row_ptr, np.array(cols, np.int32), np.array(vals, np.float32)


def rmat(scale, edge_factor, seed, a=0.57, b=0.19, c=0.19, scramble=False,
         seed_scr=0, valmode=0, seed_v=0):
    n = 1 << scale
    t1, t2, t3 = thr53(a), thr53(a + b), thr53(a + b + c)
    scr = Scramble(n, seed_scr)
    rows = [[] for _ in range(n)]
    for e in range(edge_factor << scale):
        he = h1(seed, e)
        r = cc = 0
        for lv in range(scale):
            u = h1(he, lv) >> 11
            rb = 1 if u >= t2 else 0
            cb = 1 if ((t1 <= u < t2) or u >= t3) else 0
            r |= rb << (scale - 1 - lv)
            cc |= cb << (scale - 1 - lv)
        if scramble:
            r, cc = scr(r), scr(cc)
        rows[r].append(cc)
    return _csr_from_rows(n, rows, valmode, seed_v)


def sbm(n_comm, comm_size, deg, p_in, seed, scramble=True, seed_scr=0,
        valmode=0, seed_v=0):
    n = n_comm * comm_size
    scr = Scramble(n, seed_scr)
    tin = thr53(p_in)
    rows = [[] for _ in range(n)]
    for p in range(n):
        cb = (p // comm_size) * comm_size
        got = []
        k = 0
        while len(got) < deg:
            hA, hB = h2(seed, p, 2 * k), h2(seed, p, 2 * k + 1)
            q = cb + hB % comm_size if (hA >> 11) < tin else hB % n
            if q not in got:
                got.append(q)
            k += 1
        row = scr(p) if scramble else p
        rows[row] = [scr(q) if scramble else q for q in got]
    return _csr_from_rows(n, rows, valmode, seed_v)


def stencil27(nx, periodic=False, relabel=True, seed_scr=0, valmode=0, seed_v=0):
    n = nx ** 3
    scr = Scramble(n, seed_scr)
    lab = [scr(g) if relabel else g for g in range(n)]
    rows = [[] for _ in range(n)]
    for g in range(n):
        x, y, z = g % nx, (g // nx) % nx, g // (nx * nx)
        for dz in (-1, 0, 1):
            for dy in (-1, 0, 1):
                for dx in (-1, 0, 1):
                    X, Y, Z = x + dx, y + dy, z + dz
                    if periodic:
                        X, Y, Z = X % nx, Y % nx, Z % nx
                    elif not (0 <= X < nx and 0 <= Y < nx and 0 <= Z < nx):
                        continue
                    rows[lab[g]].append(lab[(Z * nx + Y) * nx + X])
    return _csr_from_rows(n, rows, valmode, seed_v)


def vector(n, seed_x, mode=0):
    return np.array([val_of(mode, h1(seed_x, i)) for i in range(n)], np.float32)


def scramble_table(n, seed_scr):
    s = Scramble(n, seed_scr)
    return np.array([s(i) for i in range(n)], np.int64)
