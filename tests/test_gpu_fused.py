"""Multi-rank spmv_iterate against the single-GPU
power iteration: the PEER exchange (spmv_exec_scaled_bcast + CUDA IPC, the
fused NVLink path) and the COLL exchange in the padded x layout.

Two processes share cuda:0 (CUDA IPC maps the peer's buffers exactly as it
would across NVLink-connected GPUs; only the link differs), gloo carries the
8-byte all-reduce (dist.HostColl) and the handle exchange.  The iteration must
give the single-GPU spmv_iterate result: y rows bitwise (same kernels, same
association; the partition never changes y), the fp64 norm up
to its summation order across ranks (the per-rank partial sums are all-reduced:
another association of the same fp64 terms), so x = fp32(u / s) by at most one
ulp and lambda within 1e-12 relative."""
import os
import socket

import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu


def _port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, cfg, iters, mode, out_dir):
    import torch.distributed as dist

    import synth
    from paper_conf_ispass_balajicjk23_b200 import dist as pdist, spmv
    dist.init_process_group("gloo", init_method=f"tcp://127.0.0.1:{port}", rank=rank,
                            world_size=world)
    dev = torch.device("cuda:0")
    torch.cuda.set_device(dev)
    A = synth.config(cfg, small=True).A
    perm, _ = spmv.reorder(A.row_ptr, A.col, "rabbitpp")
    peer = mode == "peer"
    P = spmv.Plan(torch.from_numpy(A.row_ptr).to(dev), torch.from_numpy(A.col).to(dev),
                  torch.from_numpy(A.val).to(dev), torch.from_numpy(perm).to(dev),
                  world=world, rank=rank,
                  exchange=spmv.EXCHANGE_PEER if peer else spmv.EXCHANGE_COLL,
                  x_layout=spmv.XLAYOUT_PADDED if mode == "padded" else spmv.XLAYOUT_GLOBAL)
    hc = pdist.HostColl(device=dev)
    P.set_coll(hc.coll)
    pb = pdist.PeerBuffers(P, dev) if peer else None
    x0 = torch.ones(A.n, dtype=torch.float32, device=dev) / float(np.sqrt(A.n))
    xp = P.pad_vec(x0, to_padded=True)
    lam = pdist.iterate(P, xp, iters)
    xfull = P.pad_vec(xp, to_padded=False).cpu().numpy()
    np.savez(os.path.join(out_dir, f"r{rank}.npz"), x=xfull, lam=lam)
    if pb is not None:
        pb.close()
    P.close()
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("cfg", [1, 5])
@pytest.mark.parametrize("mode", ["peer", "padded"])
def test_multirank_iterate_equals_single_gpu(tmp_path, cfg, mode):
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import torch.multiprocessing as mp

    import synth
    from paper_conf_ispass_balajicjk23_b200 import spmv
    iters, world = 6, 2
    mp.start_processes(_worker, args=(world, _port(), cfg, iters, mode, str(tmp_path)),
                       nprocs=world, join=True, start_method="spawn")
    dev = torch.device("cuda:0")
    A = synth.config(cfg, small=True).A
    perm, _ = spmv.reorder(A.row_ptr, A.col, "rabbitpp")
    P = spmv.Plan(torch.from_numpy(A.row_ptr).to(dev), torch.from_numpy(A.col).to(dev),
                  torch.from_numpy(A.val).to(dev), torch.from_numpy(perm).to(dev))
    x = torch.ones(A.n, dtype=torch.float32, device=dev) / float(np.sqrt(A.n))
    lam = P.iterate(x, iters)
    ref = x.cpu().numpy()
    for r in range(world):
        d = np.load(tmp_path / f"r{r}.npz")
        err = np.abs(d["x"].astype(np.float64) - ref.astype(np.float64))
        assert np.all(err <= 2.0 ** -23 * np.abs(ref.astype(np.float64))), f"rank {r}"
        assert abs(float(d["lam"]) - lam) <= 1e-12 * lam
    P.close()


def test_bcast_argument_errors():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import synth
    from paper_conf_ispass_balajicjk23_b200 import spmv
    dev = torch.device("cuda:0")
    A = synth.config(1, small=True).A
    P = spmv.Plan(torch.from_numpy(A.row_ptr).to(dev), torch.from_numpy(A.col).to(dev),
                  torch.from_numpy(A.val).to(dev), None, world=2, rank=0)
    x = torch.zeros(P.info()["x_len"], device=dev)
    ss = torch.zeros(1, dtype=torch.float64, device=dev)
    with pytest.raises(spmv.SpmvError):  # more destinations than ranks
        P.exec_scaled_bcast(x, [x.data_ptr()] * 3, None, ss)
    with pytest.raises(spmv.SpmvError):  # sumsq_out is required
        P.exec_scaled_bcast(x, [x.data_ptr()], None, None)
    with pytest.raises(spmv.SpmvError):  # world > 1 without a collective backend
        P.iterate(x, 2)
    with pytest.raises(spmv.SpmvError):  # peer list of the wrong size
        P.set_peers([x.data_ptr()] * 2)
    P.close()
