"""Dev tool (under gpurun): one plan of config K in ordering O, timed execs.

    python scripts/kprof.py --config 5 --ordering rabbitpp [--steps 10] [--iterate]
                            [--ncu 1] [--env SPMV_MID_STREAM=1 ...]

Generation on the GPU for RMAT / Kronecker configs, the reorder memoised in
/tmp/permcache (survives within one gpurun call), cold execs (512 MiB read +
persisting-L2 reset before each) and warm back-to-back execs, y's bits hashed
so knob variants can be compared.  --ncu N runs N bare execs after one warm-up
and nothing else (for `ncu -k regex:... -c ...` captures).
"""
import argparse
import hashlib
import json
import os
import resource
import sys
import time

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import synth  # noqa: E402
from paper_conf_ispass_balajicjk23_b200 import spmv  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--config", type=int, default=5)
ap.add_argument("--ordering", default="rabbitpp")
ap.add_argument("--steps", type=int, default=10)
ap.add_argument("--iterate", action="store_true", help="time spmv_iterate steps instead of execs")
ap.add_argument("--ncu", type=int, default=0)
ap.add_argument("--ncu-scaled", action="store_true", help="--ncu N: N execs, then N exec_scaled (fixed x)")
ap.add_argument("--env", nargs="*", default=[])
ap.add_argument("--sequential-reorder", action="store_true")
ap.add_argument("--no-reset", action="store_true", help="flush without the persisting-L2 reset")
ap.add_argument("--so", default=None, help="load this libspmv build instead of the in-tree one (A/B)")
a = ap.parse_args()
if a.so:
    spmv.SO_PATH = os.path.abspath(a.so)
for kv in a.env:
    k, v = kv.split("=", 1)
    os.environ[k] = v
dev = torch.device("cuda:0")
torch.cuda.set_device(dev)
st = torch.cuda.Stream()
torch.cuda.set_stream(st)
t0 = time.time()
if a.config in (1, 3, 5):
    name, A, x = synth.config_gpu(a.config)
    rp_d, col_d, val_d = A.row_ptr, A.col, A.val
    n, nnz = A.n, A.nnz
    host_rp = host_col = None
else:
    w = synth.config(a.config)
    name, x = w.name, w.x
    n, nnz = w.A.n, w.A.nnz
    rp_d, col_d, val_d = (torch.from_numpy(t).to(dev) for t in (w.A.row_ptr, w.A.col, w.A.val))
    host_rp, host_col = w.A.row_ptr, w.A.col
gen_s = time.time() - t0
if nnz < 2**31:
    rp_d = rp_d.to(torch.int32)
os.makedirs("/tmp/permcache", exist_ok=True)
f = f"/tmp/permcache/{name}_{a.ordering}{'_seq' if a.sequential_reorder else ''}.npy"
t0 = time.time()
if a.ordering == "original":
    perm = np.arange(n, dtype=np.int32)
elif a.ordering == "planted":
    perm = np.ascontiguousarray(w.planted, np.int32)
elif os.path.exists(f):
    perm = np.load(f)
else:
    if host_rp is None:
        host_rp, host_col = A.row_ptr.cpu().numpy(), A.col.cpu().numpy()
    perm, _ = spmv.reorder(host_rp, host_col, a.ordering, parallel=not a.sequential_reorder)
    np.save(f, perm)
reorder_s = time.time() - t0
perm_d = torch.from_numpy(perm).to(dev)
torch.cuda.synchronize()
t0 = time.time()
P = spmv.Plan(rp_d, col_d, val_d, perm_d, permute=False)
torch.cuda.synchronize()
plan_s = time.time() - t0
t0 = time.time()
P.permute()
torch.cuda.synchronize()
permute_s = time.time() - t0
info = P.info()
xB = P.permute_vec(torch.from_numpy(np.ascontiguousarray(x, np.float32)).to(dev))
y = torch.empty(n, dtype=torch.float32, device=dev)
ideal = 8 * n + (n + 1) * (8 if nnz >= 2**31 else 4) + 8 * nnz
flush = torch.zeros(512 * 2**20 // 4, device=dev)
sink = torch.zeros((), device=dev)


def fl():
    torch.sum(flush, dim=0, out=sink)
    if not a.no_reset:
        spmv.lib().spmv_reset_persisting_l2(None)


P.exec(xB, y)
torch.cuda.synchronize()
if a.ncu:
    for _ in range(a.ncu):
        fl()
        P.exec(xB, y)
    if a.ncu_scaled:
        ss = torch.zeros(2, dtype=torch.float64, device=dev)
        P.exec_scaled(xB, y, None, ss[:1])
        for _ in range(a.ncu):
            fl()
            P.exec_scaled(xB, y, ss[:1], ss[1:])
    torch.cuda.synchronize()
    print(json.dumps({"ncu_execs": a.ncu, "workload": name, "ordering": a.ordering}))
    sys.exit(0)


def ev():
    return torch.cuda.Event(enable_timing=True)


cold = []
for _ in range(a.steps):
    fl()
    e0, e1 = ev(), ev()
    e0.record()
    P.exec(xB, y)
    e1.record()
    cold.append((e0, e1))
torch.cuda.synchronize()
cold_ms = float(np.median([e0.elapsed_time(e1) for e0, e1 in cold]))
e0, e1 = ev(), ev()
e0.record()
for _ in range(a.steps):
    P.exec(xB, y)
e1.record()
torch.cuda.synchronize()
warm_ms = e0.elapsed_time(e1) / a.steps
it_ms = None
sc_ms = None
if a.iterate:  # exec_scaled back to back with FIXED x / y (the norm's cost without alternation)
    ss = torch.zeros(2, dtype=torch.float64, device=dev)
    P.exec_scaled(xB, y, None, ss[:1])
    e0, e1 = ev(), ev()
    e0.record()
    for _ in range(a.steps):
        P.exec_scaled(xB, y, ss[:1], ss[1:])
    e1.record()
    torch.cuda.synchronize()
    sc_ms = e0.elapsed_time(e1) / a.steps
if a.iterate:
    xs = xB.clone()
    P.iterate(xs, 3)
    e0, e1 = ev(), ev()
    e0.record()
    P.iterate(xs, a.steps)
    e1.record()
    torch.cuda.synchronize()
    it_ms = e0.elapsed_time(e1) / a.steps
h = hashlib.sha1(y.cpu().numpy().tobytes()).hexdigest()[:16]
hbm = json.load(open("MEASURED_PEAKS.json"))["hbm_gbs"] if os.path.exists("MEASURED_PEAKS.json") else 6548.8
print(json.dumps({"workload": name, "ordering": a.ordering, "env": a.env + (["no-reset"] if a.no_reset else []),
                  "so": a.so,
                  "n": n, "nnz": nnz,
                  "cold_ms": round(cold_ms, 4), "warm_ms": round(warm_ms, 4), "iterate_ms": it_ms, "scaled_fixed_ms": sc_ms,
                  "x_ideal_cold": round(cold_ms * 1e-3 * hbm * 1e9 / ideal, 3),
                  "gen_s": round(gen_s, 2), "reorder_s": round(reorder_s, 1),
                  "plan_s": round(plan_s, 3), "permute_ms": round(permute_s * 1e3, 1),
                  "mid_rows": info["n_mid_rows"], "cta_rows": info["n_cta_rows"],
                  "hub_rows": info["n_hub_rows"], "H": info["hot_prefix"],
                  "win": P.info()["l2_window_bytes"], "ef": info["stream_evict_first"],
                  "lane_pred": info.get("lane_pred_gather"), "lane_waste": info.get("lane_waste_slots"), "lane_nnz": info.get("lane_nnz"),
                  "y_sha": h,
                  "peak_rss_gb": round(resource.getrusage(resource.RUSAGE_SELF).ru_maxrss / 2**20, 1)}),
      flush=True)
P.close()
