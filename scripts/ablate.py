"""Dev: stream-pattern ablation on the C2 workload (see ablate.cu)."""
import ctypes
import json
import os
import sys

import numpy as np
import torch

sys.path.insert(0, ".")
import synth  # noqa: E402
from paper_conf_ispass_balajicjk23_b200 import spmv  # noqa: E402

lib = ctypes.CDLL(os.path.abspath("scripts/ablate.so"))
lib.ablate.argtypes = [ctypes.c_int, ctypes.c_void_p, ctypes.c_int] + [ctypes.c_void_p] * 4 + \
    [ctypes.c_int, ctypes.c_long, ctypes.c_int, ctypes.c_void_p]
dev = torch.device("cuda:0")
st = torch.cuda.Stream()
torch.cuda.set_stream(st)
w = synth.config(int(os.environ.get("CFG", "2")))
A = w.A
rp64 = A.nnz >= 2**31
rp = torch.from_numpy(A.row_ptr).to(dev)
if not rp64:
    rp = rp.to(torch.int32)
col = torch.from_numpy(A.col).to(dev)
val = torch.from_numpy(A.val).to(dev)
o = os.environ.get("ORD", "rabbit")
f = f"/tmp/permcache/{w.name}_{o}_20230423.npz"
if o == "planted":
    perm = w.planted.astype(np.int32)
else:
    perm = np.load(f, allow_pickle=True)["perm"] if os.path.exists(f) else spmv.reorder(A.row_ptr, A.col, o)[0]
P = spmv.Plan(rp, col, val, torch.from_numpy(perm).to(dev))
Brp, Bcol, Bval = P.export_csr()
Brp = Brp if rp64 else Brp.to(torch.int32)
del rp, col, val
Bcol = torch.cat([Bcol, torch.zeros(16, dtype=Bcol.dtype, device=dev)])
Bval = torch.cat([Bval, torch.zeros(16, dtype=Bval.dtype, device=dev)])
xB = P.permute_vec(torch.from_numpy(w.x).to(dev))
y = torch.empty(max(A.n, 148 * 64 * 256), device=dev)
buf = torch.zeros(512 * 2**20 // 4, device=dev)
sink = torch.zeros((), device=dev)
ideal = 8 * A.n + (A.n + 1) * (8 if rp64 else 4) + 8 * A.nnz


def ev():
    return torch.cuda.Event(enable_timing=True)


def timeit(fn, cold, K=20):
    for _ in range(3):
        fn()
    torch.cuda.synchronize()
    torch.cuda._sleep(int(1e8))
    es = []
    for _ in range(K):
        if cold:
            torch.sum(buf, dim=0, out=sink)
        a, b = ev(), ev()
        a.record()
        fn()
        b.record()
        es.append((a, b))
    torch.cuda.synchronize()
    return round(float(np.median([a.elapsed_time(b) * 1e3 for a, b in es])), 2)


out = {"ideal_us": round(ideal / 6538.6e9 * 1e6, 2), "ord": o}
VAR = [(20, "ef_nogather"), (10, "canon"), (12, "canon_ef"), (13, "canon_ef_panel")]
for which, name in VAR:
    for per_sm in (4, 32):
        g = 148 * per_sm
        fn = (lambda wh=which, g=g: lib.ablate(wh, Brp.data_ptr(), int(rp64), Bcol.data_ptr(), Bval.data_ptr(),
                                               xB.data_ptr(), y.data_ptr(), A.n, A.nnz, g,
                                               st.cuda_stream))
        out[f"{name}/g{per_sm}"] = (timeit(fn, True), timeit(fn, False))
out["k_lane"] = (timeit(lambda: P.exec(xB, y[:A.n]), True), timeit(lambda: P.exec(xB, y[:A.n]), False))
print(json.dumps(out))
