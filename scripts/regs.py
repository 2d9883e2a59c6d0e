"""Dev: per-kernel register counts from `nvcc -Xptxas -v` output (stdin), demangled."""
import re
import subprocess
import sys

cur = None
for line in sys.stdin:
    m = re.search(r"Compiling entry function '(\S+)'", line)
    if m:
        cur = m.group(1)
        continue
    m = re.search(r"Used (\d+) registers", line)
    if m and cur:
        name = subprocess.run(["c++filt", cur], capture_output=True, text=True).stdout.strip()
        name = re.sub(r"\(.*", "", name.replace("spmv::(anonymous namespace)::", ""))
        pat = sys.argv[1] if len(sys.argv) > 1 else ""
        if pat in name:
            print(f"{m.group(1):>4} {name}")
        cur = None
