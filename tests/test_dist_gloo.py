"""Multi-rank host logic of the row-block power iteration on
CPU: world_size 2 over gloo, driving paper_conf_ispass_balajicjk23_b200.dist
exactly as the NCCL run does, with the oracle standing in for the local
kernel (the CUDA kernels themselves are covered by tests/test_gpu_parity.py,
including partitioned == single bitwise)."""
import math
import os
import socket

import numpy as np
import pytest

import synth
from oracle import permute, plan as oplan, power, rabbit, spmv as ospmv

torch = pytest.importorskip("torch")


class OracleLocal:
    """CPU stand-in with the Plan interface used by dist.iterate: rows
    [b_r, b_{r+1}) of B, padded x layout x[k*M + i - b_k]."""

    def __init__(self, Bp, Bc, Bv, world, rank):
        n = len(Bp) - 1
        self.world, self.rank = world, rank
        self.bounds = oplan.partition(Bp, world)
        M = int(max(np.diff(self.bounds).max(), 1))
        M = (M + 31) // 32 * 32
        self.x_stride, self.y_offset = M, rank * M
        b0, b1 = self.bounds[rank], self.bounds[rank + 1]
        self.nrows = int(b1 - b0)
        owner = np.searchsorted(self.bounds, np.arange(n), side="right") - 1
        self.pad_index = owner * M + (np.arange(n) - self.bounds[owner])
        lo, hi = Bp[b0], Bp[b1]
        self.rp = Bp[b0:b1 + 1] - lo
        self.col = self.pad_index[Bc[lo:hi]].astype(np.int32)
        self.val = Bv[lo:hi]

    def exec_scaled(self, x, y, ss_in, ss_out):
        alpha = 1.0 if ss_in is None else np.float32(1.0 / math.sqrt(float(ss_in.item())))
        yy = ospmv.spmv(self.rp, self.col, self.val, x.numpy()) * np.float32(alpha)
        y.copy_(torch.from_numpy(yy.astype(np.float32)))
        ss_out.fill_(float(np.sum(yy.astype(np.float64) ** 2)))

    def scale(self, u, x, ss):
        x.copy_(u * np.float32(1.0 / math.sqrt(float(ss.item()))))


def _worker(rank, world, port, out_dir):
    import torch.distributed as dist
    from paper_conf_ispass_balajicjk23_b200 import dist as pdist
    dist.init_process_group("gloo", init_method=f"tcp://127.0.0.1:{port}", rank=rank,
                            world_size=world)
    w = synth.config(5, small=True)
    A = w.A
    perm = rabbit.random_perm(A.n, 3)
    Bp, Bc, Bv = permute.permute_csr(A.n, A.row_ptr, A.col, A.val, perm)
    loc = OracleLocal(Bp, Bc, Bv, world, rank)
    xB = permute.permute_vec(w.x, perm)
    xpad = np.zeros(world * loc.x_stride, np.float32)
    xpad[loc.pad_index] = xB
    x, lam = pdist.iterate(loc, torch.from_numpy(xpad), 6)
    np.save(os.path.join(out_dir, f"x{rank}.npy"), x.numpy()[loc.pad_index])
    np.save(os.path.join(out_dir, f"lam{rank}.npy"), np.array([lam]))
    dist.destroy_process_group()


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


@pytest.mark.parametrize("world", [2])
def test_gloo_power_iteration_matches_oracle(tmp_path, world):
    import torch.multiprocessing as mp
    mp.spawn(_worker, args=(world, _free_port(), str(tmp_path)), nprocs=world, join=True)
    w = synth.config(5, small=True)
    A = w.A
    perm = rabbit.random_perm(A.n, 3)
    Bp, Bc, Bv = permute.permute_csr(A.n, A.row_ptr, A.col, A.val, perm)
    xr, lr = power.power_iteration(Bp, Bc, Bv, permute.permute_vec(w.x, perm), 6)
    xs = [np.load(tmp_path / f"x{r}.npy") for r in range(world)]
    lams = [float(np.load(tmp_path / f"lam{r}.npy")[0]) for r in range(world)]
    for r in range(world):
        assert np.array_equal(xs[r], xs[0])          # every replica identical
        assert abs(lams[r] - lr) <= 1e-5 * lr
        assert np.max(np.abs(xs[r] - xr)) <= 1e-5 * np.max(np.abs(xr))


def test_single_rank_path_matches_oracle():
    # world == 1 through the same driver (no collectives)
    from paper_conf_ispass_balajicjk23_b200 import dist as pdist
    A = synth.rmat(9, 8, 4, valmode=synth.VAL_POS, seed_v=2)
    Bp, Bc, Bv = A.row_ptr, A.col, A.val
    loc = OracleLocal(Bp, Bc, Bv, 1, 0)
    x0 = np.ones(A.n, np.float32) / np.float32(math.sqrt(A.n))
    xpad = np.zeros(loc.x_stride, np.float32)
    xpad[loc.pad_index] = x0
    x, lam = pdist.iterate(loc, torch.from_numpy(xpad), 4)
    xr, lr = power.power_iteration(Bp, Bc, Bv, x0, 4)
    assert abs(lam - lr) <= 1e-6 * lr
    assert np.allclose(x.numpy()[loc.pad_index], xr, rtol=1e-5, atol=1e-7)
