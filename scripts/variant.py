"""Dev (A/B): build libspmv from the csrc/ of a git revision into another .so.

    python scripts/variant.py --rev HEAD --out variants/head.so
    python scripts/variant.py --rev WORKTREE -D SOME_KNOB=1 --out variants/knob.so
    python scripts/kprof.py --so variants/head.so ...      (on the GPU box)

The in-tree libspmv.so is untouched; built .so files travel to the GPU box
with the gpurun snapshot (git-ignored, not gpurun-ignored).
"""
import argparse
import os
import subprocess
import sys
import tempfile

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from paper_conf_ispass_balajicjk23_b200 import build as B  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--rev", required=True)
ap.add_argument("--out", required=True)
ap.add_argument("-D", action="append", default=[], help="extra -D macro (A/B builds)")
a = ap.parse_args()
top = tempfile.mkdtemp(prefix="spmv_variant_")
tmp = os.path.join(top, "pkg", "csrc")  # common.cuh includes ../../include/spmv.h
os.makedirs(tmp)
rel = os.path.relpath(B.CSRC, ROOT)
for f in B.SOURCES + B.HEADERS:
    if a.rev == "WORKTREE":
        src = open(os.path.join(B.CSRC, f)).read()
    else:
        src = subprocess.run(["git", "-C", ROOT, "show", f"{a.rev}:{rel}/{f}"], capture_output=True, text=True,
                             check=True).stdout
    open(os.path.join(tmp, f), "w").write(src)
if a.rev == "WORKTREE":
    hdr = open(os.path.join(ROOT, "include", "spmv.h")).read()
else:
    hdr = subprocess.run(["git", "-C", ROOT, "show", f"{a.rev}:include/spmv.h"], capture_output=True, text=True,
                         check=True).stdout
os.makedirs(os.path.join(top, "include"), exist_ok=True)
open(os.path.join(top, "include", "spmv.h"), "w").write(hdr)
common = ["-std=c++17", "-O3", "-Xcompiler", "-fPIC,-fopenmp", f"-I{os.path.join(top, 'include')}"] + [f"-D{d}" for d in a.D]
gpu = ["-gencode", "arch=compute_100a,code=sm_100a", "-lineinfo", "-Xptxas", "-O3"]
objs = []
for src in B.SOURCES:
    obj = os.path.join(tmp, src + ".o")
    cmd = [B.nvcc(), "-c", os.path.join(tmp, src), "-o", obj] + common + (gpu if src.endswith(".cu") else ["-x", "c++"])
    subprocess.run(cmd, check=True)
    objs.append(obj)
os.makedirs(os.path.dirname(os.path.abspath(a.out)), exist_ok=True)
subprocess.run([B.nvcc(), "-shared", "-o", a.out] + objs + ["-Xcompiler", "-fopenmp", "-lgomp", "-lcudart", "-ldl"],
               check=True)
print(a.out)
