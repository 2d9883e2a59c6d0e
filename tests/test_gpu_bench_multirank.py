"""bench.py's N > 1 path (row-block power iteration) end to end on one GPU:
two ranks share cuda:0 (--single-device) over gloo, with the NCCL-style
all-gather exchange and with the fused exec + peer-store exchange.  Checks the
contract fields of the JSON line rank 0 prints."""
import json
import os
import subprocess
import sys

import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.mark.parametrize("exchange", ["nccl", "fused"])
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
           "--gpus", "2", "--steps", "4", "--warmup", "3", "--config", "1",
           "--orderings", "rabbitpp", "--backend", "gloo", "--single-device",
           "--exchange", exchange]
    r = subprocess.run(cmd, capture_output=True, text=True, timeout=600, cwd=ROOT)
    assert r.returncode == 0, r.stderr[-3000:]
    lines = [ln for ln in r.stdout.splitlines() if ln.startswith("{")]
    assert len(lines) == 1, r.stdout[-2000:]
    d = json.loads(lines[0])
    assert d["n_gpus"] == 2 and d["steps"] == 4 and d["value"] > 0
    assert d["e2e"]["value"] > 0 and d["gpu_launches"] > 0
    assert ("fused" in d["config"]["step"]) == (exchange == "fused")
