"""Multi-rank plumbing of spmv_iterate (reading c22).

One process per GPU.  Rank k owns rows [b_k, b_{k+1}) of B (partition by
spmv_plan, reading c29) and a full replica of x.  The power-iteration loop --
scaled SpMV, all-reduce of sum y^2, exchange of the y slices, final
normalisation and lambda -- runs inside libspmv (spmv_iterate).  This module
only connects it to torch.distributed:

  nccl_comm_ptr   the ncclComm_t of a ProcessGroupNCCL (opts.nccl_comm), so
                  libspmv issues ncclAllReduce / grouped ncclBroadcast itself;
  HostColl        an spmv_coll_t over any torch.distributed group with host
                  staging (gloo): the test / CPU-box backend;
  PeerBuffers     the ping-pong next-x buffers of the PEER exchange: allocated
                  with spmv_dev_alloc, IPC handles swapped with
                  all_gather_object, peers' buffers mapped (NVLink/NVSwitch)
                  and registered with spmv_set_peers;
  iterate         plan.iterate (the C loop) with the above in place.

No arithmetic of the method is done here.
"""
from __future__ import annotations

import ctypes

import numpy as np


def nccl_comm_ptr(group=None, device=None) -> int:
    """ncclComm_t (as an int) of the NCCL backend of `group` on `device`.
    The communicator is created eagerly (init_process_group(device_id=...)),
    or by the first collective; a barrier forces it."""
    import torch
    import torch.distributed as dist
    g = group if group is not None else dist.distributed_c10d._get_default_group()
    dev = device if device is not None else torch.device("cuda", torch.cuda.current_device())
    be = g._get_backend(dev)
    ptr = be._comm_ptr()
    if not ptr:
        dist.barrier(group=g, device_ids=[dev.index])
        ptr = be._comm_ptr()
    if not ptr:
        raise RuntimeError("no NCCL communicator on this process group")
    return int(ptr)


class _DevView:
    """torch view of a raw fp32 / fp64 device range (__cuda_array_interface__)."""

    def __init__(self, ptr: int, n: int, typestr: str):
        self.__cuda_array_interface__ = {"shape": (int(n),), "typestr": typestr,
                                         "data": (int(ptr), False), "version": 3}


class HostColl:
    """spmv_coll_t over a torch.distributed group, staged through host memory
    (gloo).  device=None: the buffers are host memory (CPU tests);
    otherwise device buffers on `device`, whose stream is synchronised before
    the host copy (the callbacks run on the thread that called spmv_iterate)."""

    def __init__(self, group=None, device=None):
        from . import spmv
        self.group, self.device = group, device
        self._ar = spmv.ALLREDUCE_FN(self._allreduce)
        self._ag = spmv.ALLGATHERV_FN(self._allgatherv)
        self.coll = spmv._Coll(None, self._ar, self._ag)
        self.calls = {"allreduce": 0, "allgatherv": 0}

    def _view(self, ptr, n, dtype):
        import torch
        if self.device is None:
            ct = ctypes.c_double if dtype == np.float64 else ctypes.c_float
            return torch.from_numpy(np.ctypeslib.as_array((ct * int(n)).from_address(int(ptr))))
        ts = "<f8" if dtype == np.float64 else "<f4"
        return torch.as_tensor(_DevView(ptr, n, ts), device=self.device)

    def _sync(self, stream):
        import torch
        if self.device is not None:
            torch.cuda.ExternalStream(int(stream or 0), device=self.device).synchronize() \
                if stream else torch.cuda.synchronize(self.device)

    def _allreduce(self, ctx, buf, count, stream):
        import torch.distributed as dist
        try:
            self._sync(stream)
            t = self._view(buf, count, np.float64)
            h = t.cpu()
            dist.all_reduce(h, op=dist.ReduceOp.SUM, group=self.group)
            t.copy_(h)
            self._sync(stream)
            self.calls["allreduce"] += 1
            return 0
        except Exception:  # reported as SPMV_ENCCL by the library
            return 1

    def _allgatherv(self, ctx, x, bounds, world, stream):
        import torch.distributed as dist
        try:
            self._sync(stream)
            b = [int(bounds[k]) for k in range(world + 1)]
            t = self._view(x + 4 * b[0], b[world] - b[0], np.float32)
            h = t.cpu()
            for k in range(world):  # all-gatherv = one broadcast per root
                if b[k + 1] > b[k]:
                    sl = h[b[k] - b[0]:b[k + 1] - b[0]].clone()
                    dist.broadcast(sl, src=k, group=self.group)
                    h[b[k] - b[0]:b[k + 1] - b[0]] = sl
            t.copy_(h)
            self._sync(stream)
            self.calls["allgatherv"] += 1
            return 0
        except Exception:
            return 1


class PeerBuffers:
    """Ping-pong next-x buffers of every rank for the PEER exchange (SURVEY
    §8(f1)): two spmv_dev_alloc buffers per rank, the other ranks' mapped
    through CUDA IPC (peer access over NVLink / NVSwitch) and registered with
    spmv_set_peers.  close() unmaps after a barrier (no peer may still store)."""

    def __init__(self, plan, device, group=None):
        import torch.distributed as dist
        from . import spmv
        self._spmv, self.plan, self.group = spmv, plan, group
        i = plan.info()
        self.world, self.rank, xlen = i["world"], i["rank"], i["x_len"]
        idx = device.index if device.index is not None else 0
        self.bufs = [spmv.DeviceBuffer(xlen, idx) for _ in range(2)]
        self.opened = []
        mine = [b.handle() for b in self.bufs]
        allh = [None] * self.world
        dist.all_gather_object(allh, mine, group=group)
        ptrs = []
        for j in range(2):
            for k in range(self.world):
                if k == self.rank:
                    ptrs.append(self.bufs[j].ptr)
                else:
                    q = spmv.ipc_open(allh[k][j])
                    self.opened.append(q)
                    ptrs.append(q)
        plan.set_peers(ptrs)

    def close(self):
        import torch
        import torch.distributed as dist
        if self.bufs is None:
            return
        torch.cuda.synchronize()
        dist.barrier(group=self.group)
        for q in self.opened:
            self._spmv.ipc_close(q)
        for b in self.bufs:
            b.close()
        self.bufs = None


def iterate(plan, x, iters: int, stream=None) -> float:
    """spmv_iterate on this rank: x (full length, plan's x layout, the same on
    every rank) is overwritten with x_iters; returns lambda = s_iters.  The
    plan carries its collective backend (nccl_comm at creation, or
    plan.set_coll(HostColl(...).coll)) and, for the PEER exchange, its
    PeerBuffers."""
    return plan.iterate(x, iters, stream)
