"""Per-CUDA-line instruction and stall shares from an ncu report: python tools/ncu_lines.py rep.ncu-rep [top]."""
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
top = int(sys.argv[2]) if len(sys.argv) > 2 else 30
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
for i, r in enumerate(rows[:6]):
    if "Instructions Executed" in r:
        hdr, start = r, i + 1
ia, ist = hdr.index("Instructions Executed"), hdr.index("Warp Stall Sampling (All Samples)")
cur, agg, st = None, {}, {}
for r in rows[start:]:
    if r[0].strip():
        cur = (r[0], r[1].strip()[:100])
    if len(r) > ia:
        agg[cur] = agg.get(cur, 0) + f(r[ia])
        st[cur] = st.get(cur, 0) + f(r[ist])
tot, ts = sum(agg.values()) or 1, sum(st.values()) or 1
print(f"total warp-instructions {tot:.0f}")
for k, v in sorted(agg.items(), key=lambda x: -x[1])[:top]:
    print(f"{v / tot * 100:5.1f}% instr {st[k] / ts * 100:5.1f}% stall  L{k[0]}: {k[1]}")
