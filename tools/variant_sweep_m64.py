"""Key-only 33..64 buckets, ONE (8192-key tiles, blocked counting) vs tile (ballot K3), by size:
python tools/variant_sweep_m64.py > profiles/r02_variants_m64.md  (the rule: ONE for every size)"""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import bench
steps = 15
print("| workload | n | one | tile | default |\n|---|---|---|---|---|")
for base in ("sweep_m64_ko", "wide_m4096_ko"):
    for e in (18, 20, 22, 24, 26, 28):
        cfg = dict(bench.CONFIGS[base], n=1 << e)
        row = []
        for v in (("one", "3k", None) if base.startswith("sweep") else (None,)):
            r = bench.bench_config(base, dict(cfg, variant=v), steps, 3, torch.device("cuda"), 1, 0, with_e2e=False)
            row.append(f"{r['value']:.1f}")
        print(f"| {base} | 2^{e} | " + " | ".join(row) + " |", flush=True)
cfg = dict(bench.CONFIGS["sweep_m64_ko"], m=33, delta=(1 << 32) // 33 + 1)
for e in (20, 24, 28):
    row = []
    for v in ("one", "3k", None):
        r = bench.bench_config("m33", dict(cfg, n=1 << e, variant=v), steps, 3, torch.device("cuda"), 1, 0, with_e2e=False)
        row.append(f"{r['value']:.1f}")
    print(f"| m33 delta | 2^{e} | " + " | ".join(row) + " |", flush=True)
