"""bench.py's N > 1 path (row-block power iteration through spmv_iterate)
end to end on one GPU: two ranks share cuda:0 (--single-device) over gloo
(dist.HostColl as the collective backend), with the all-gatherv exchange and
with the SpMV's own peer stores.  The small Kronecker (config 5 shape, scale
14 via --small) keeps it quick.  Checks the contract fields of the JSON line
rank 0 prints."""
import json
import os
import subprocess
import sys

import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.mark.parametrize("exchange", ["coll", "peer"])
def test_bench_two_ranks_single_device(exchange):
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import socket
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node=2",
           "--master-addr=127.0.0.1", f"--master-port={port}", os.path.join(ROOT, "bench.py"),
           "--gpus", "2", "--steps", "4", "--warmup", "3", "--config", "5", "--small",
           "--orderings", "original,rabbitpp", "--backend", "gloo", "--single-device",
           "--exchange", exchange]
    r = subprocess.run(cmd, capture_output=True, text=True, timeout=600, cwd=ROOT)
    assert r.returncode == 0, r.stderr[-3000:]
    lines = [ln for ln in r.stdout.splitlines() if ln.startswith("{")]
    assert len(lines) == 1, r.stdout[-2000:]
    d = json.loads(lines[0])
    assert d["n_gpus"] == 2 and d["steps"] == 4 and d["value"] > 0
    assert d["e2e"]["value"] > 0 and d["gpu_launches"] > 0
    assert ("peer-store" in d["config"]["step"]) == (exchange == "peer")
    assert d["config"]["ordering"] == "rabbitpp" and d["orderings"]["rabbitpp"]["partition_rows"]
    assert sum(d["orderings"]["rabbitpp"]["partition_rows"]) == d["config"]["n"]
