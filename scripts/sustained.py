"""Dev: sustained exec loop (~2 s) with nvidia-smi sampling: SM clock/power under load."""
import os
import subprocess
import sys
import threading
import time

import numpy as np
import torch

sys.path.insert(0, ".")
import synth  # noqa: E402
from paper_conf_ispass_balajicjk23_b200 import spmv  # noqa: E402

dev = torch.device("cuda:0")
st = torch.cuda.Stream()
torch.cuda.set_stream(st)
w = synth.config(2)
A = w.A
rp = torch.from_numpy(A.row_ptr).to(dev).to(torch.int32)
col = torch.from_numpy(A.col).to(dev)
val = torch.from_numpy(A.val).to(dev)
o = os.environ.get("ORD", "rabbit")
f = f"/tmp/permcache/{w.name}_{o}_20230423.npz"
perm = np.load(f, allow_pickle=True)["perm"] if os.path.exists(f) else spmv.reorder(A.row_ptr, A.col, o)[0]
pd = torch.from_numpy(perm).to(dev)
for variant in (1, 0):
    P = spmv.Plan(rp, col, val, pd, variant=variant)
    xB = P.permute_vec(torch.from_numpy(w.x).to(dev))
    y = torch.empty(A.n, device=dev)
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=st):
        for _ in range(100):
            P.exec(xB, y)
    g.replay()
    torch.cuda.synchronize()
    samples = []
    proc = subprocess.Popen(["nvidia-smi", "--query-gpu=clocks.sm,clocks.mem,power.draw,clocks_event_reasons.active",
                             "--format=csv,noheader,nounits", "-lms", "50"], stdout=subprocess.PIPE, text=True)
    th = threading.Thread(target=lambda: [samples.append(l.strip()) for l in proc.stdout], daemon=True)
    th.start()
    time.sleep(0.3)
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    for _ in range(30):
        g.replay()
    b.record()
    torch.cuda.synchronize()
    proc.terminate()
    ms = a.elapsed_time(b) / 3000
    print(f"variant {variant}: {ms*1000:.1f} us/exec over {a.elapsed_time(b):.0f} ms", flush=True)
    for s in samples[::4]:
        print("   ", s)
    P.close()
