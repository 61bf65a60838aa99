"""Summarise a round's ncu artefacts into profiles/: python tools/summarize_profiles.py r01
Writes profiles/<tag>_summary.md (profiles/ncu_traffic.json is written by tools/ncu_traffic.py)."""
import csv
import io
import json
import os
import re
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import bench  # noqa: E402
from paper_conf_ppopp_ashkianidmo16_b200 import model  # noqa: E402

tag = sys.argv[1]
src = os.environ.get("PROF_SRC", os.path.join(ROOT, "gpurun_out"))
out = []


def short(name):
    m = re.match(r"(?:void )?(?:ms::)?([A-Za-z0-9_]+)", name)
    return m.group(1) if m else name[:40]


# (1) launch list
lp = os.path.join(src, f"prof_{tag}_launches.csv")
if os.path.exists(lp):
    lines = [l for l in open(lp) if l.startswith('"')]
    rows = list(csv.DictReader(io.StringIO("".join(lines))))
    agg = {}
    for r in rows:
        if r["Metric Name"] != "gpu__time_duration.sum":
            continue
        k = short(r["Kernel Name"])
        v = float(r["Metric Value"].replace(",", "")) * {"nsecond": 1e-3, "ns": 1e-3, "usecond": 1.0, "us": 1.0, "msecond": 1e3}.get(r["Metric Unit"], 1.0)  # -> us
        a = agg.setdefault(k, [0, 0.0])
        a[0] += 1
        a[1] += v
    ours = {k: v for k, v in agg.items() if re.match(r"k[0-9_]", k)}
    tot = sum(v[1] for v in ours.values())
    out.append(f"## Launch list (`ncu --metrics gpu__time_duration.sum --clock-control none`, "
               f"`python bench.py --steps 3 --warmup 3 --no-extra --no-cpu`, config {bench.DEFAULT})\n")
    out.append("Cold-cache, serialised per-launch times: compare shares, not absolutes.\n")
    out.append("| kernel | launches | total us | avg us | share of our kernels |\n|---|---|---|---|---|")
    for k, (c, t) in sorted(agg.items(), key=lambda x: -x[1][1]):
        share = f"{t / tot * 100:.1f} %" if k in ours else "(torch: data gen / L2 flush)"
        out.append(f"| {k} | {c} | {t:.1f} | {t / c:.2f} | {share} |")
    out.append("")

# (2) full captures
PROF_OUT = os.environ.get("PROF_OUT", os.path.join(ROOT, "profiles"))
keys = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "dram__throughput.avg.pct_of_peak_sustained_elapsed", "smsp__issue_active.avg.pct_of_peak_sustained_active",
        "sm__warps_active.avg.pct_of_peak_sustained_active", "l1tex__data_pipe_lsu_wavefronts.avg.pct_of_peak_sustained_elapsed",
        "launch__registers_per_thread", "launch__grid_size", "smsp__inst_executed.sum",
        "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum"]
units = {"gpu__time_duration.sum": 1.0}
for f in sorted(os.listdir(src)):
    m = re.match(rf"prof_{tag}_(\w+?)_(k1_prescan|k1r_prescan|k1s_prescan|k1a_prescan|k2_scan|k2r_scan|k3v_postscan|k3p_postscan|k3_postscan)\.ncu-rep$", f)
    if not m:
        continue
    cfg, kern = m.group(1), m.group(2)
    raw = subprocess.run(["ncu", "-i", os.path.join(src, f), "--page", "raw", "--csv"], capture_output=True,
                         text=True).stdout
    r = list(csv.reader(io.StringIO(raw)))
    h, u, d = r[0], r[1], r[2]
    get = lambda k: (float(d[h.index(k)]), u[h.index(k)]) if k in h else (None, "")  # noqa: E731

    def to_bytes(v, unit):
        return v * {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "KB": 1e3, "MB": 1e6, "GB": 1e9}.get(unit, 1)

    t, tu = get("gpu__time_duration.sum")
    t_us = t * {"nsecond": 1e-3, "ns": 1e-3, "usecond": 1, "us": 1, "msecond": 1e3, "ms": 1e3}.get(tu, 1)
    rd, rdu = get("dram__bytes_read.sum")
    wr, wru = get("dram__bytes_write.sum")
    dram = to_bytes(rd, rdu) + to_bytes(wr, wru)
    c = bench.CONFIGS[cfg]
    pre, post = model.pass_bytes_per_key(c["kv"], 1 if c["kind"] == "ids" else 0)
    alg = (post if kern.startswith("k3") else pre if kern.startswith("k1") else 0) * c["n"]
    # the library's own variant choice (ms_plan_geometry): ONE runs K1 + K3 in one cooperative
    # k3v_postscan launch -> all of the step's bytes
    from paper_conf_ppopp_ashkianidmo16_b200 import Plan
    one = kern == "k3v_postscan" and Plan(bench.spec_of(c), c["n"], with_values=c["kv"]).geometry(c["n"])[2] == 2
    if one:
        alg = (pre + post) * c["n"]
    stalls = [(hh.replace("smsp__average_warps_issue_stalled_", "").replace("_per_issue_active.ratio", ""),
               float(d[i] or 0)) for i, hh in enumerate(h)
              if hh.startswith("smsp__average_warps_issue_stalled_") and hh.endswith("_per_issue_active.ratio")]
    stalls.sort(key=lambda x: -x[1])
    out.append(f"## {kern}{' (ONE: K1 + K3 in one launch)' if one else ''} on {cfg} ({c['desc']})\n")
    out.append(f"- duration {t_us:.1f} us (under ncu, clocks not locked); dram read+write {dram / 1e9:.4f} GB"
               + (f" vs algorithmic {alg / 1e9:.4f} GB (ratio {dram / alg:.3f})" if alg else ""))
    for k in keys[3:]:
        v, un = get(k)
        if v is not None:
            out.append(f"- {k}: {v:g} {un}")
    out.append("- top stalls (cycles per issued instruction): " + ", ".join(f"{a} {b:.2f}" for a, b in stalls[:6]))
    out.append("")
os.makedirs(PROF_OUT, exist_ok=True)
with open(os.path.join(PROF_OUT, f"{tag}_summary.md"), "w") as fh:
    fh.write(f"# ncu summary, round tag {tag}\n\nGenerated by tools/summarize_profiles.py from "
             f"tools/profile_round.sh output (1 B200, clocks not locked).\n\n" + "\n".join(out) + "\n")
print("\n".join(out))
