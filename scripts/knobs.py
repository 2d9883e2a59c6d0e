"""Dev sweep of exec knobs that need a fresh plan (SPMV_L2_FETCH, SPMV_WIN_COLS,
SPMV_LANE_EF, SPMV_CONCURRENT ...): one plan per combination, cold (512 MiB
read flush) and warm per-exec times, y checked bitwise against the first combo.
    CFG=3 ORDS=rabbitpp COMBOS='[{}, {"SPMV_L2_FETCH": "32"}]' python scripts/knobs.py"""
import json
import os
import sys

import numpy as np
import torch

sys.path.insert(0, ".")
import synth  # noqa: E402
from paper_conf_ispass_balajicjk23_b200 import spmv  # noqa: E402

cfg = int(os.environ.get("CFG", "3"))
ords = os.environ.get("ORDS", "rabbitpp").split(",")
combos = json.loads(os.environ.get("COMBOS", "[{}]"))
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
print(json.dumps({"workload": w.name, "ideal_us": round(ideal / 6539.2e9 * 1e6, 2)}), flush=True)


def ev():
    return torch.cuda.Event(enable_timing=True)


def timeit(fn, flush, K=int(os.environ.get("K", "15"))):
    for _ in range(3):
        flush()
        fn()
    torch.cuda.synchronize()
    es = []
    for _ in range(K):
        flush()
        a, b = ev(), ev()
        a.record()
        fn()
        b.record()
        es.append((a, b))
    torch.cuda.synchronize()
    return round(float(np.median([a.elapsed_time(b) * 1e3 for a, b in es])), 1)


for o in ords:
    f = f"/tmp/permcache/{w.name}_{o}_20230423.npz"
    if o == "planted":
        perm = w.planted.astype(np.int32)
    elif o == "original":
        perm = np.arange(A.n, dtype=np.int32)
    elif os.path.exists(f):
        perm = np.load(f, allow_pickle=True)["perm"]
    else:
        perm, stt = spmv.reorder(A.row_ptr, A.col, o)
        os.makedirs("/tmp/permcache", exist_ok=True)
        np.savez(f, perm=perm, stats=np.array(stt.__dict__, dtype=object))
    perm_d = torch.from_numpy(perm).to(dev)
    xB = None
    ref = None
    kind = os.environ.get("KIND", "exec")  # exec | spmm4 | coo
    for c in combos:
        saved = {k: os.environ.get(k) for k in c}
        os.environ.update({k: str(v) for k, v in c.items()})
        P = spmv.Plan(rp, col, val, perm_d)
        if xB is None:
            xB = P.permute_vec(torch.from_numpy(w.x).to(dev))
            y = torch.empty(A.n, device=dev)
            X4 = xB[:, None].repeat(1, 4).contiguous() if kind == "spmm4" else None
            Y4 = torch.empty_like(X4) if kind == "spmm4" else None
        run = {"exec": lambda: P.exec(xB, y), "coo": lambda: P.exec_coo(xB, y),
               "spmm4": lambda: P.exec_spmm4(X4, Y4)}[kind]
        run()
        torch.cuda.synchronize()
        out = Y4 if kind == "spmm4" else y
        if ref is None:
            ref = out.clone()
        same = bool(torch.equal(ref, out))
        cold = timeit(run, lambda: torch.sum(buf, dim=0, out=sink))
        warm = timeit(run, lambda: None)
        info = P.info()
        print(json.dumps({"ord": o, "kind": kind, **c, "cold_us": cold, "warm_us": warm,
                          "x_ideal": round(cold / (ideal / 6539.2e9 * 1e6), 3),
                          "win_bytes": info["l2_window_bytes"], "bitwise_same": same}), flush=True)
        P.close()
        for k, v in saved.items():
            if v is None:
                os.environ.pop(k, None)
            else:
                os.environ[k] = v
