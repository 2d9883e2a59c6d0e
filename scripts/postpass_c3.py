"""dev (GPU): RABBIT++ post-pass on the GPU vs the host at full size (C3)."""
import json
import sys
import time

import numpy as np
import torch

sys.path.insert(0, ".")
import synth  # noqa: E402
from paper_conf_ispass_balajicjk23_b200 import spmv  # noqa: E402

cfg = int(sys.argv[1]) if len(sys.argv) > 1 else 3
A = synth.config(cfg).A
dev = torch.device("cuda:0")
t = time.perf_counter()
pr, st = spmv.reorder(A.row_ptr, A.col, "rabbit")
t_rabbit = time.perf_counter() - t
comm = spmv.reorder_last_comm(A.n)
t = time.perf_counter()
ppp, st2 = spmv.reorder(A.row_ptr, A.col, "rabbitpp")  # detection reused from the cache
t_host_total = time.perf_counter() - t
rp = torch.from_numpy(A.row_ptr).to(dev)
if A.nnz < 2**31:
    rp = rp.to(torch.int32)
col = torch.from_numpy(A.col).to(dev)
prd, cd = torch.from_numpy(pr).to(dev), torch.from_numpy(comm).to(dev)
spmv.rabbitpp_gpu(rp, col, prd, cd)
torch.cuda.synchronize()
t = time.perf_counter()
out = spmv.rabbitpp_gpu(rp, col, prd, cd)
torch.cuda.synchronize()
t_gpu = time.perf_counter() - t
print(json.dumps({"workload": cfg, "n": A.n, "nnz": A.nnz, "rabbit_s": round(t_rabbit, 2),
                  "host_rabbitpp_call_s (detection cached)": round(t_host_total, 3),
                  "gpu_postpass_s": round(t_gpu, 4),
                  "bitexact": bool(np.array_equal(out.cpu().numpy(), ppp))}))
