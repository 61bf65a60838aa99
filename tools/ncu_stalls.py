"""Per-CUDA-line stall shares (all samples) + top SASS lines: python tools/ncu_stalls.py rep [top]"""
import csv
import io
import subprocess
import sys


def f(x):
    try:
        return float(x)
    except ValueError:
        return 0.0


rep = sys.argv[1]
top = int(sys.argv[2]) if len(sys.argv) > 2 else 25
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
for i, r in enumerate(rows[:6]):
    if "Instructions Executed" in r:
        hdr, start = r, i + 1
ia, ist = hdr.index("Instructions Executed"), hdr.index("Warp Stall Sampling (All Samples)")
isrc2 = 3
cuda, sass, cur = [], [], None
for r in rows[start:]:
    if r[0].strip():
        cur = f"L{r[0]}: {r[1].strip()[:80]}"
        if len(r) > ist:
            cuda.append((f(r[ist]), f(r[ia]), cur))
    elif len(r) > ist and r[isrc2].strip():
        sass.append((f(r[ist]), f(r[ia]), r[2], r[isrc2].strip()[:60], cur))
ts = sum(x[0] for x in cuda) or 1
ti = sum(x[1] for x in cuda) or 1
print("--- CUDA lines by stall share")
for s, i, c in sorted(cuda, reverse=True)[:top]:
    print(f"stall {s / ts * 100:5.1f}% instr {i / ti * 100:5.1f}%  {c}")
ts2 = sum(x[0] for x in sass) or 1
print("--- SASS by stall share")
for s, i, a, src, c in sorted(sass, reverse=True)[:top]:
    print(f"stall {s / ts2 * 100:5.1f}%  {a} {src:60s} <- {c[:50]}")
