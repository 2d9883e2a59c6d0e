"""Fig. 6 of the paper on B200: DRAM
traffic of SpMV on the INSULAR sub-matrix, normalised to its compulsory
traffic.

PAPER.md:179: "the DRAM traffic for SpMV on just the insular sub-matrix
(evaluated by masking all non-zeros that do not connect to insular nodes) is
very close to compulsory traffic (Figure 6)", after the insular nodes were
grouped (modification 1, RABBIT++ / INSULAR order).  Reading c30: the insular
sub-matrix is B restricted to rows AND columns of insular nodes -- under
RABBIT++ the trailing block B[N-I:, N-I:] (I = #insular), renumbered
0..I-1; its compulsory traffic is P:96 over that I x I matrix.

Under gpurun:  python scripts/fig6.py --config 2 [--ncu]   (with --ncu run
inside `ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum ...`; the
script prints the block's ideal bytes and the kernel launch it makes).
The sub-matrix is cut from B on the device (torch index ops: input
preparation of a measurement, not the hot path) and run through a plan of
its own (identity permutation), cold (512 MiB read + persisting-L2 reset).
"""
import argparse
import json
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import synth  # noqa: E402
from paper_conf_ispass_balajicjk23_b200 import spmv  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--config", type=int, default=2)
ap.add_argument("--ordering", default="rabbitpp")
ap.add_argument("--execs", type=int, default=5)
a = ap.parse_args()
dev = torch.device("cuda:0")
torch.cuda.set_device(dev)
st = torch.cuda.Stream()
torch.cuda.set_stream(st)
if a.config in (1, 3, 5):
    name, A, x = synth.config_gpu(a.config)
    rp_h, col_h = A.row_ptr.cpu().numpy(), A.col.cpu().numpy()
    rp_d, col_d, val_d = A.row_ptr, A.col, A.val
else:
    w = synth.config(a.config)
    name, x = w.name, w.x
    rp_h, col_h = w.A.row_ptr, w.A.col
    rp_d, col_d, val_d = (torch.from_numpy(t).to(dev) for t in (w.A.row_ptr, w.A.col, w.A.val))
n, nnz = len(rp_h) - 1, int(rp_h[-1])
perm, rs = spmv.reorder(rp_h, col_h, a.ordering, parallel=True)
I = int(rs.n_insular)
if nnz < 2**31:
    rp_d = rp_d.to(torch.int32)
P = spmv.Plan(rp_d, col_d, val_d, torch.from_numpy(perm).to(dev))
Bp, Bc, Bv = P.export_csr()
P.close()
lo = n - I
# rows [lo, n), entries with column >= lo, renumbered
r0, r1 = int(Bp[lo]), int(Bp[n])
c = Bc[r0:r1].to(torch.int64)
keep = c >= lo
rows = torch.repeat_interleave(torch.arange(I, device=dev), (Bp[lo + 1:] - Bp[lo:-1]))
cnt = torch.bincount(rows[keep], minlength=I)
rp_s = torch.zeros(I + 1, dtype=torch.int64, device=dev)
rp_s[1:] = torch.cumsum(cnt, 0)
col_s = (c[keep] - lo).to(torch.int32).contiguous()
val_s = Bv[r0:r1][keep].contiguous()
nz_s = int(rp_s[-1])
masked = (r1 - r0) - nz_s
del Bp, Bc, Bv, c, keep, rows
if nz_s < 2**31:
    rp_s = rp_s.to(torch.int32)
S = spmv.Plan(rp_s, col_s, val_s, None)
xs = torch.from_numpy(np.ascontiguousarray(x[:I], np.float32)).to(dev)
ys = torch.empty(I, dtype=torch.float32, device=dev)
flush = torch.zeros(512 * 2**20 // 4, device=dev)
sink = torch.zeros((), device=dev)
ideal = 8 * I + (I + 1) * (8 if nz_s >= 2**31 else 4) + 8 * nz_s
ts = []
for i in range(a.execs):
    torch.sum(flush, dim=0, out=sink)
    spmv.lib().spmv_reset_persisting_l2(None)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    S.exec(xs, ys)
    e1.record()
    torch.cuda.synchronize()
    ts.append(e0.elapsed_time(e1))
hbm = json.load(open("MEASURED_PEAKS.json"))["hbm_gbs"] if os.path.exists("MEASURED_PEAKS.json") else 6548.8
print(json.dumps({"workload": name, "ordering": a.ordering, "n": n, "nnz": nnz, "insular": I,
                  "insular_frac": I / n, "sub_nnz": nz_s, "masked_in_block_rows": masked,
                  "sub_ideal_bytes": ideal, "ms": round(float(np.median(ts)), 5),
                  "runtime_over_ideal": round(float(np.median(ts)) * 1e-3 * hbm * 1e9 / ideal, 4),
                  "exec_launches": S.info()["exec_launches"]}), flush=True)
S.close()
