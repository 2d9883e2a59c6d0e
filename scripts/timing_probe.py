"""Dev probe: why does the bench's cold step time exceed ncu's kernel time?

Times one plan's spmv_exec on the C2 workload under several protocols.
"""
import json
import os
import sys
import time

import numpy as np
import torch

sys.path.insert(0, ".")
import synth  # noqa: E402
from paper_conf_ispass_balajicjk23_b200 import spmv  # noqa: E402

cfg = int(os.environ.get("CFG", "2"))
o = os.environ.get("ORD", "rabbitpp")
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
f = f"/tmp/permcache/{w.name}_{o}_20230423.npz"
if os.path.exists(f):
    perm = np.load(f, allow_pickle=True)["perm"]
else:
    perm, _ = spmv.reorder(A.row_ptr, A.col, o)
P = spmv.Plan(rp, col, val, torch.from_numpy(perm).to(dev))
xB = P.permute_vec(torch.from_numpy(w.x).to(dev))
y = torch.empty(A.n, device=dev)
res = {"ideal_us": ideal / 6538.6e9 * 1e6}


def ev():
    return torch.cuda.Event(enable_timing=True)


def run(name, flush, sleep_ahead, K=40):
    for _ in range(3):
        flush()
        P.exec(xB, y)
    torch.cuda.synchronize()
    if sleep_ahead:
        torch.cuda._sleep(int(2e8))
    es = []
    for _ in range(K):
        flush()
        a, b = ev(), ev()
        a.record()
        P.exec(xB, y)
        b.record()
        es.append((a, b))
    torch.cuda.synchronize()
    t = [a.elapsed_time(b) * 1e3 for a, b in es]
    res[name] = {"mean": round(float(np.mean(t)), 2), "median": round(float(np.median(t)), 2),
                 "min": round(float(np.min(t)), 2)}


def fl_read():
    torch.sum(buf, dim=0, out=sink)


def fl_write():
    buf.fill_(1.0)


def fl_none():
    pass


run("read", fl_read, False)
run("read_sleep", fl_read, True)
run("write_sleep", fl_write, True)
run("none_sleep", fl_none, True)
# host cost of one exec call
torch.cuda.synchronize()
torch.cuda._sleep(int(5e8))
t0 = time.perf_counter()
for _ in range(200):
    P.exec(xB, y)
res["host_us_per_exec_call"] = round((time.perf_counter() - t0) / 200 * 1e6, 2)
torch.cuda.synchronize()
t0 = time.perf_counter()
for _ in range(200):
    fl_read()
res["host_us_per_flush_call"] = round((time.perf_counter() - t0) / 200 * 1e6, 2)
torch.cuda.synchronize()
# graph: flush+exec pairs, minus flush-only graph
for nm, body in (("g_pair", lambda: (fl_read(), P.exec(xB, y))), ("g_flush", lambda: fl_read())):
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=st):
        for _ in range(20):
            body()
    g.replay()
    torch.cuda.synchronize()
    a, b = ev(), ev()
    a.record()
    g.replay()
    b.record()
    torch.cuda.synchronize()
    res[nm] = round(a.elapsed_time(b) * 1e3 / 20, 2)
res["g_pair_minus_flush"] = round(res["g_pair"] - res["g_flush"], 2)
print(json.dumps(res), flush=True)

# --- probe 2: is the cold penalty a property of the kernel or of the system?
if os.environ.get("PROBE2"):
    big = torch.zeros(2 * 2**30 // 4, device=dev)
    r2 = {}
    mat = torch.empty(ideal // 4, device=dev)

    def t_of(fn, flush, K=20):
        for _ in range(3):
            flush()
            fn()
        torch.cuda.synchronize()
        torch.cuda._sleep(int(2e8))
        es = []
        for _ in range(K):
            flush()
            a, b = ev(), ev()
            a.record()
            fn()
            b.record()
            es.append((a, b))
        torch.cuda.synchronize()
        return round(float(np.median([a.elapsed_time(b) * 1e3 for a, b in es])), 2)

    for mb in (128, 256, 512, 1024, 2048):
        sub = big[: mb * 2**20 // 4]
        fl = (lambda s=sub: torch.sum(s, dim=0, out=sink))
        r2[f"exec_flush{mb}"] = t_of(lambda: P.exec(xB, y), fl)
        r2[f"stream_sum_flush{mb}"] = t_of(lambda: torch.sum(mat, dim=0, out=sink), fl)
    r2["exec_noflush"] = t_of(lambda: P.exec(xB, y), fl_none)
    r2["stream_sum_noflush"] = t_of(lambda: torch.sum(mat, dim=0, out=sink), fl_none)
    # flush that touches only x's lines (evict x, keep TLB): read x-sized other buffer? no:
    # re-read the matrix arrays themselves (same pages as the kernel) as the flush
    fl_same = (lambda: (torch.sum(col.view(torch.float32)[:128 * 2**20 // 4], dim=0, out=sink),
                        torch.sum(val[-(128 * 2**20 // 4):], dim=0, out=sink)))
    r2["exec_flush_samepages"] = t_of(lambda: P.exec(xB, y), fl_same)
    print(json.dumps(r2), flush=True)
