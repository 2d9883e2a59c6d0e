"""Oracle power iteration (reading c22; north_star "iterated SpMV (power
iteration)"; PAPER.md:221 iterations amortise reordering).

    y_t = B x_{t-1}                       (Alg. 1, exact row sums, fp64)
    s_t = ||y_t||_2                        (fp64)
    x_t = fp32(y_t / s_t)
    lambda = s_iters

TEST INFRASTRUCTURE ONLY (see oracle/__init__.py).
"""
from __future__ import annotations

import math

import numpy as np

from .spmv import spmv_f64


def power_iteration(row_ptr, col, val, x0, iters: int):
    x = np.asarray(x0, np.float32).copy()
    s = 0.0
    for _ in range(iters):
        y = spmv_f64(row_ptr, col, val, x)
        s = math.sqrt(math.fsum((y * y).tolist()))
        x = (y / s).astype(np.float32) if s > 0 else np.zeros_like(x)
    return x, s


def power_step(row_ptr, col, val, x):
    """One step from a given x (step-wise parity): (y_t fp32, s_t)."""
    y = spmv_f64(row_ptr, col, val, x)
    return y.astype(np.float32), math.sqrt(math.fsum((y * y).tolist()))
