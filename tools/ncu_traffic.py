"""DRAM traffic per launch of every libms kernel, per bench workload, measured with ncu
(dram__bytes_read.sum + dram__bytes_write.sum, gpu__time_duration.sum; one capture of the
second of two runs, L2 flushed before each) -> profiles/ncu_traffic.json, which bench.py
reports as roofline.traffic.  Run on the GPU box:  python tools/ncu_traffic.py NAME[,NAME...]"""
import csv
import io
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
NCU = "/usr/local/cuda/bin/ncu"
METRICS = "dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum"


def capture(name):
    cmd = [NCU, "--metrics", METRICS, "--clock-control", "none", "--kernel-name", "regex:^k",
           "--csv", "--page", "raw", "--print-units", "base", sys.executable, os.path.join(ROOT, "tools", "run_one.py"),
           name, "2"]
    r = subprocess.run(cmd, capture_output=True, text=True, timeout=1800)
    lines = [ln for ln in r.stdout.splitlines() if ln.startswith('"')]
    rows = list(csv.DictReader(io.StringIO("\n".join(lines))))
    def base_name(s):
        s = s.strip()
        if s.startswith("void "):
            s = s[5:]
        return s.split("<")[0].split("(")[0].strip()
    rows = [x for x in rows if base_name(x.get("Kernel Name", "")).startswith("k")]
    if not rows:
        sys.stderr.write(r.stdout[-2000:] + r.stderr[-2000:])
        return None
    half = len(rows) // 2  # two runs: keep the second
    out = []
    for x in rows[half:]:
        def num(k):
            return float(str(x[k]).replace(",", ""))
        rd, wr = num("dram__bytes_read.sum"), num("dram__bytes_write.sum")
        out.append({"kernel": base_name(x["Kernel Name"]), "instance": x["Kernel Name"].split("(")[0].strip(),
                    "dram_read": rd, "dram_write": wr, "dram_bytes": rd + wr,
                    "time_ns": num("gpu__time_duration.sum")})
    return out


def main():
    import bench
    names = sys.argv[1].split(",")
    path = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    db = {"how": "ncu --metrics " + METRICS + " --clock-control none, second of two runs (L2 flushed before "
                 "each), tools/ncu_traffic.py; bytes per launch", "configs": {}}
    if os.path.exists(path):
        try:
            old = json.load(open(path))
            if "configs" in old:
                db["configs"].update(old["configs"])
        except Exception:
            pass
    from paper_conf_ppopp_ashkianidmo16_b200 import model
    for nm in names:
        cfg = bench.CONFIGS[nm]
        ks = capture(nm)
        if ks is None:
            print(f"{nm}: capture failed", flush=True)
            continue
        idb = cfg.get("id_bytes", 1) if cfg["kind"] == "ids" else 0
        alg = model.algorithmic_bytes_per_key(cfg["kv"], idb) * cfg["n"]
        db["configs"][nm] = {"kernels": ks, "algorithmic_bytes_step": alg,
                             "dram_bytes_step": sum(k["dram_bytes"] for k in ks)}
        print(nm, json.dumps(db["configs"][nm]), flush=True)
    out = os.path.join(ROOT, "gpurun_out", "ncu_traffic.json")
    os.makedirs(os.path.dirname(out), exist_ok=True)
    json.dump(db, open(out, "w"), indent=1)
    print("wrote", out)


if __name__ == "__main__":
    main()
