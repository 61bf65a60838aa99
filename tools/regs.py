"""Registers / stack per kernel instantiation of a built object: python tools/regs.py build/k3_ids.o [filter]"""
import re
import subprocess
import sys

out = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "-res-usage", sys.argv[1]], capture_output=True, text=True).stdout
flt = sys.argv[2] if len(sys.argv) > 2 else ""
lines = out.splitlines()
for i, l in enumerate(lines):
    m = re.search(r"Function (\S+):", l)
    if not m or i + 1 >= len(lines):
        continue
    name = subprocess.run(["c++filt", m.group(1)], capture_output=True, text=True).stdout.strip()
    name = re.sub(r"\(.*", "", name)
    r = re.search(r"REG:(\d+) STACK:(\d+)", lines[i + 1])
    if flt in name and r:
        print(f"REG {r.group(1):>3} STACK {r.group(2):>3}  {name}")
