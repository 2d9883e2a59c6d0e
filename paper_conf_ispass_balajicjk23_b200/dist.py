"""Row-block power iteration across ranks (reading c22).

One process per GPU.  Rank k owns rows [b_k, b_{k+1}) of B (nnz-balanced
partition computed by spmv_plan), a full replica of x in the padded layout
x[k*M + (i - b_k)] (M = plan x_stride), and writes its y slice straight into
its own segment of the next x buffer.  Per iteration:

    exec_scaled   y_k = (B_k u_{t-1}) / s_{t-1},  partial sum y_k^2   (libspmv)
    all_reduce    s_t^2 = sum_k partial                               (NCCL, 8 B)
    all_gather    in place, equal-size segments of M floats           (NCCL over NVLink)

The padded layout turns NCCL's missing all-gatherv into an in-place
equal-count all-gather with zero copies.  The
collectives go through torch.distributed (plumbing); all arithmetic runs in
libspmv.  ``local`` may be any object with the Plan interface below, which is
how the gloo/CPU tests drive this exact code with a stand-in local SpMV.
"""
from __future__ import annotations

import math


def iterate(local, x, iters: int, group=None):
    """Run `iters` normalised steps from x (padded layout, every rank the same).

    local: object with attributes world, rank, x_stride, y_offset, nrows and
    methods exec_scaled(x, y, ss_in, ss_out) and scale(u, x, ss).
    Returns (x_iters normalised, padded layout; lambda = s_iters).
    """
    import torch
    import torch.distributed as dist

    if iters < 1:
        raise ValueError("iters must be >= 1")
    M, off, nr = local.x_stride, local.y_offset, local.nrows
    xa, xb = x, torch.empty_like(x)
    ss = torch.zeros(2, dtype=torch.float64, device=x.device)
    ss_in = None
    for t in range(iters):
        ss_out = ss[t & 1:(t & 1) + 1]
        local.exec_scaled(xa, xb[off:off + nr], ss_in, ss_out)
        if local.world > 1:
            dist.all_reduce(ss_out, op=dist.ReduceOp.SUM, group=group)
            dist.all_gather_into_tensor(xb, xb[off:off + M].clone() if not xb.is_cuda
                                        else xb[off:off + M], group=group)
        ss_in = ss_out
        xa, xb = xb, xa
    local.scale(xa, xa, ss_in)
    return xa, math.sqrt(float(ss_in.item()))


def _all_reduce_sum(t, group, host_staged):
    import torch.distributed as dist
    if host_staged:  # gloo: stage through the host (this also syncs the stream)
        h = t.cpu()
        dist.all_reduce(h, op=dist.ReduceOp.SUM, group=group)
        t.copy_(h)
    else:
        dist.all_reduce(t, op=dist.ReduceOp.SUM, group=group)


class FusedExchange:
    """Peer-mapped ping-pong x buffers for the fused exec + exchange (SURVEY
    §8(f1)): every rank maps every other rank's two next-x buffers (CUDA IPC
    over NVLink / NVSwitch), and spmv_exec_scaled_bcast stores each y row
    straight into all of them -- no all-gather.  One collective remains per
    step, the 8-byte all-reduce of sum y^2, which also orders the data: a rank
    passes step t's all-reduce only after every rank's step-t kernels have
    completed, so the next read sees all peers' stores and no peer overwrites a
    buffer that is still being read."""

    def __init__(self, plan, device, group=None, host_staged: bool = False):
        import torch.distributed as dist
        from . import spmv
        self._spmv, self.plan, self.group, self.host_staged = spmv, plan, group, host_staged
        i = plan.info()
        self.world, self.rank, xlen = i["world"], i["rank"], i["x_len"]
        idx = device.index if device.index is not None else 0
        self.bufs = [spmv.DeviceBuffer(xlen, idx) for _ in range(2)]
        self.opened = []
        mine = [b.handle() for b in self.bufs]
        allh = [None] * self.world
        dist.all_gather_object(allh, mine, group=group)
        self.dst = [[0] * self.world for _ in range(2)]
        for k in range(self.world):
            for j in range(2):
                if k == self.rank:
                    self.dst[j][k] = self.bufs[j].ptr
                else:
                    self.dst[j][k] = spmv.ipc_open(allh[k][j])
                    self.opened.append(self.dst[j][k])
        self.cur = 0

    @property
    def x(self):
        """The current x (padded layout) -- the buffer the next step reads."""
        return self.bufs[self.cur].tensor

    def step(self, ss_in, ss_out):
        """x <- B x / s (fused store into every rank's next buffer), then the
        all-reduce of ss_out; flips the ping-pong."""
        self.plan.exec_scaled_bcast(self.x, self.dst[1 - self.cur], ss_in, ss_out)
        _all_reduce_sum(ss_out, self.group, self.host_staged)
        self.cur = 1 - self.cur

    def close(self):
        import torch
        import torch.distributed as dist
        if self.bufs is None:
            return
        torch.cuda.synchronize()
        dist.barrier(group=self.group)  # nobody unmaps while a peer may still store
        for q in self.opened:
            self._spmv.ipc_close(q)
        for b in self.bufs:
            b.close()
        self.bufs = None


def iterate_fused(plan, x, iters: int, group=None, host_staged: bool = False):
    """iterate() with the exchange fused into the SpMV (FusedExchange).
    Returns (x_iters normalised, padded layout; lambda = s_iters)."""
    import torch

    if iters < 1:
        raise ValueError("iters must be >= 1")
    fx = FusedExchange(plan, x.device, group, host_staged)
    try:
        fx.x.copy_(x)
        ss = torch.zeros(2, dtype=torch.float64, device=x.device)
        ss_in = None
        for t in range(iters):
            ss_out = ss[t & 1:(t & 1) + 1]
            fx.step(ss_in, ss_out)
            ss_in = ss_out
        out = torch.empty_like(x)
        fx._spmv.scale_vec(fx.x, out, ss_in)
        lam = math.sqrt(float(ss_in.item()))
    finally:
        fx.close()
    return out, lam


class PlanLocal:
    """Adapter: a libspmv Plan as the `local` of iterate()."""

    def __init__(self, plan):
        from . import spmv
        self._spmv = spmv
        self.plan = plan
        i = plan.info()
        self.world, self.rank = i["world"], i["rank"]
        self.x_stride, self.y_offset = i["x_stride"], i["y_offset"]
        self.nrows = i["row_end"] - i["row_begin"]

    def exec_scaled(self, x, y, ss_in, ss_out):
        self.plan.exec_scaled(x, y, ss_in, ss_out)

    def scale(self, u, x, ss):
        self._spmv.scale_vec(u, x, ss)
