"""Dev microbenchmark: one plan, several exec variants and flush styles."""
import json
import os
import sys

import numpy as np
import torch

sys.path.insert(0, ".")
import synth  # noqa: E402
from paper_conf_ispass_balajicjk23_b200 import spmv  # noqa: E402

cfg = int(os.environ.get("CFG", "2"))
ords = os.environ.get("ORDS", "rabbit").split(",")
dev = torch.device("cuda:0")
torch.cuda.set_device(dev)
st = torch.cuda.Stream()
torch.cuda.set_stream(st)
w = synth.config(cfg)
A = w.A
rp = torch.from_numpy(A.row_ptr).to(dev)
if A.nnz < 2**31:
    rp = rp.to(torch.int32)
col = torch.from_numpy(A.col).to(dev)
val = torch.from_numpy(A.val).to(dev)
buf = torch.zeros(512 * 2**20 // 4, device=dev)
sink = torch.zeros((), device=dev)
ideal = 8 * A.n + (A.n + 1) * (8 if A.nnz >= 2**31 else 4) + 8 * A.nnz
res = {}
for o in ords:
    f = f"/tmp/permcache/{w.name}_{o}_20230423.npz"
    if os.path.exists(f):
        perm = np.load(f, allow_pickle=True)["perm"]
    else:
        perm, _ = spmv.reorder(A.row_ptr, A.col, o)
    pd = torch.from_numpy(perm).to(dev)
    for variant, ctas in [(1, None), (0, 4), (0, 8)]:
        os.environ.pop("SPMV_LANE_CTAS", None)
        if ctas:
            os.environ["SPMV_LANE_CTAS"] = str(ctas)
        P = spmv.Plan(rp, col, val, pd, variant=variant)
        xB = P.permute_vec(torch.from_numpy(w.x).to(dev))
        y = torch.empty(A.n, device=dev)
        for fl in ("read", "write", "none"):
            K = 30
            ts = []
            for i in range(K + 3):
                if fl == "read":
                    torch.sum(buf, dim=0, out=sink)
                elif fl == "write":
                    buf.zero_()
                a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                a.record()
                P.exec(xB, y)
                b.record()
                ts.append((a, b))
            torch.cuda.synchronize()
            ms = [a.elapsed_time(b) for a, b in ts[3:]]
            res[f"{o}/v{variant}c{ctas}/{fl}"] = round(float(np.median(ms)), 4)
        # graph of K execs (launch overhead removed), warm
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g, stream=st):
            for _ in range(10):
                P.exec(xB, y)
        g.replay()
        torch.cuda.synchronize()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        g.replay()
        b.record()
        torch.cuda.synchronize()
        res[f"{o}/v{variant}c{ctas}/graph_warm"] = round(a.elapsed_time(b) / 10, 4)
        P.close()
        print(json.dumps({k: v for k, v in res.items() if k.startswith(f"{o}/v{variant}c{ctas}")}),
              flush=True)
print("ideal_us", ideal / 6545.9e9 * 1e6)
