"""spmv_iterate's built-in NCCL backend on a one-GPU box: a world-1 NCCL
process group (the communicator torch's ProcessGroupNCCL created, handed to
the library as opts.nccl_comm) and SPMV_FORCE_COLL=1, so the loop issues
ncclAllReduce and the grouped ncclBroadcast all-gatherv (dlsym'd from the
process's libnccl) exactly as with eight ranks.  Over one rank both are the
identity, so x and lambda must equal the collective-free iteration bitwise."""
import os
import subprocess
import sys

import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

WORKER = r'''
import os, socket, sys
sys.path.insert(0, os.environ["ROOT"])
import numpy as np, torch, torch.distributed as dist
import synth
from paper_conf_ispass_balajicjk23_b200 import dist as pdist, spmv
s = socket.socket(); s.bind(("127.0.0.1", 0)); port = s.getsockname()[1]; s.close()
dev = torch.device("cuda:0"); torch.cuda.set_device(dev)
dist.init_process_group("nccl", init_method=f"tcp://127.0.0.1:{port}", rank=0, world_size=1,
                        device_id=dev)
comm = pdist.nccl_comm_ptr(device=dev)
assert comm
A = synth.config(5, small=True).A
perm, _ = spmv.reorder(A.row_ptr, A.col, "rabbitpp")
mk = lambda **kw: spmv.Plan(torch.from_numpy(A.row_ptr).to(dev), torch.from_numpy(A.col).to(dev),
                            torch.from_numpy(A.val).to(dev), torch.from_numpy(perm).to(dev), **kw)
P0, P1 = mk(), mk(nccl_comm=comm)
x0 = P0.permute_vec(torch.ones(A.n, device=dev) / float(np.sqrt(A.n)))
xa, xb = x0.clone(), x0.clone()
la = P0.iterate(xa, 7)
os.environ["SPMV_FORCE_COLL"] = "1"
lb = P1.iterate(xb, 7)
assert torch.equal(xa.view(torch.int32), xb.view(torch.int32)) and la == lb, (la, lb)
print("NCCL_OK", la)
dist.destroy_process_group()
'''


def test_builtin_nccl_backend_world1():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    r = subprocess.run([sys.executable, "-c", WORKER], capture_output=True, text=True, timeout=600,
                       env={**os.environ, "ROOT": ROOT})
    assert r.returncode == 0, r.stderr[-3000:]
    assert "NCCL_OK" in r.stdout
