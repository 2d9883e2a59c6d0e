"""spmv_iterate across ranks (reading c22) against the
oracle power iteration, with two ranks sharing cuda:0.

Each rank runs the library's own loop (spmv_iterate, world 2): the scaled SpMV
of its row block, the all-reduce of sum y^2 and the exchange, through a
host-staged gloo backend (dist.HostColl, installed with spmv_set_coll) -- the
same calls the NCCL backend makes.  Both exchanges are covered: COLL (y slices
written locally, then an all-gatherv of the uneven slices) and PEER (the SpMV
stores its rows into both ranks' next x through CUDA IPC mappings).

Parity is step-wise, from the GPU's own previous iterate (running T steps and
T - 1 steps from the same x_0; the loop is deterministic, so the shorter run
is a prefix): one exact step of the oracle (Alg. 1 row sums in fp64, s = its
2-norm) gives x_ref = y / s.  Per-row bound, positive values (Kronecker, values
in (0, 1], x > 0, so sum_j |a_rj x_j| = y_r):
  the SpMV row error is <= 1e-5 * y_r (north star), hence the
  norm's relative error is <= 1e-5; the GPU applies 1/s in fp32 and stores fp32
  u and x: four roundings of 2^-24 each.  So
  |x_gpu[r] - x_ref[r]| <= 2e-5 * x_ref[r] + 2^-22 * x_ref[r].
The eigenvalue estimate lambda = s_T gets the norm's bound plus the roundings,
(1e-5 + 2^-22) relative.
"""
import math
import os
import socket

import numpy as np
import pytest

import synth
from oracle import permute, power, spmv as ospmv

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu
T = 5


def _port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _inputs():
    from paper_conf_ispass_balajicjk23_b200 import spmv
    w = synth.config(5, small=True)
    A = w.A
    perm, _ = spmv.reorder(A.row_ptr, A.col, "rabbitpp")
    return A, perm, w.x


def _worker(rank, world, port, exchange, out_dir):
    import torch.distributed as dist
    from paper_conf_ispass_balajicjk23_b200 import dist as pdist, spmv
    dist.init_process_group("gloo", init_method=f"tcp://127.0.0.1:{port}", rank=rank,
                            world_size=world)
    dev = torch.device("cuda:0")
    torch.cuda.set_device(dev)
    A, perm, x0 = _inputs()
    P = spmv.Plan(torch.from_numpy(A.row_ptr).to(dev), torch.from_numpy(A.col).to(dev),
                  torch.from_numpy(A.val).to(dev), torch.from_numpy(perm).to(dev),
                  world=world, rank=rank,
                  exchange=spmv.EXCHANGE_PEER if exchange == "peer" else spmv.EXCHANGE_COLL)
    hc = pdist.HostColl(device=dev)
    P.set_coll(hc.coll)
    pb = pdist.PeerBuffers(P, dev) if exchange == "peer" else None
    info = P.info()
    xB = P.permute_vec(torch.from_numpy(x0).to(dev))
    out = {"x_len": info["x_len"], "row_begin": info["row_begin"], "row_end": info["row_end"]}
    for t in (T - 1, T):
        x = xB.clone()
        lam = pdist.iterate(P, x, t)
        out[f"x{t}"] = x.cpu().numpy()
        out[f"lam{t}"] = lam
    out["calls"] = [hc.calls["allreduce"], hc.calls["allgatherv"]]
    np.savez(os.path.join(out_dir, f"{exchange}{rank}.npz"), **out)
    if pb is not None:
        pb.close()
    P.close()
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("exchange", ["coll", "peer"])
def test_iterate_world2_matches_oracle_stepwise(tmp_path, exchange):
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import torch.multiprocessing as mp
    world = 2
    mp.start_processes(_worker, args=(world, _port(), exchange, str(tmp_path)), nprocs=world,
                       join=True, start_method="spawn")
    A, perm, x0 = _inputs()
    Bp, Bc, Bv = permute.permute_csr(A.n, A.row_ptr, A.col, A.val, perm.astype(np.int64))
    d = [np.load(tmp_path / f"{exchange}{r}.npz") for r in range(world)]
    assert d[0]["row_begin"] == 0 and d[1]["row_end"] == A.n
    assert d[0]["row_end"] == d[1]["row_begin"]
    for r in range(world):
        assert int(d[r]["x_len"]) == A.n                     # global layout, no padding
        assert np.array_equal(d[r]["x5"], d[0]["x5"])        # replicas identical
        assert d[r]["lam5"] == d[0]["lam5"]
        ar, ag = d[r]["calls"].tolist()
        assert ar == 2 * T - 1                               # one all-reduce per step
        assert ag == (2 * T - 1 if exchange == "coll" else 0)
    xp = d[0][f"x{T - 1}"]
    _, s = power.power_step(Bp, Bc, Bv, xp)
    xref = ospmv.spmv_f64(Bp, Bc, Bv, xp) / s
    xg = d[0][f"x{T}"].astype(np.float64)
    tol = (2e-5 + 2.0 ** -22) * np.abs(xref) + 1e-37
    assert np.all(np.abs(xg - xref) <= tol), float(np.max(np.abs(xg - xref) / tol))
    assert abs(float(d[0][f"lam{T}"]) - s) <= (1e-5 + 2.0 ** -22) * s
    assert math.isfinite(s) and s > 0
