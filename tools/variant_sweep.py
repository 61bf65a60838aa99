"""Which variant wins where (the measured rule of ms_api.cu choose_variant):
G keys/s of ONE / ranged / tile for a set of workloads at several n.
usage: python tools/variant_sweep.py [steps] [base,base,...] > profiles/r02_variants.md"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import bench  # noqa: E402

steps = int(sys.argv[1]) if len(sys.argv) > 1 else 10
print("| workload | n | one | ranged | tile | default (variant) |")
print("|---|---|---|---|---|---|")
BASES = ("C3", "C3bin", "sweep_m2_kv", "sweep_m8_kv", "sweep_m16_kv", "sweep_m32_kv", "IDSkv", "sweep_m32_ko",
         "sweep_m8_ko", "sweep_m64_kv", "sweep_m64_ko")
for base in (sys.argv[2].split(",") if len(sys.argv) > 2 else BASES):
    for e in (23, 25, 26, 27):
        cfg = dict(bench.CONFIGS[base], n=1 << e)
        row = []
        for v in ("one", "ranged", "3k", None):
            r = bench.bench_config(base, dict(cfg, variant=v), steps, 3, torch.device("cuda"), 1, 0, with_e2e=False)
            row.append(f"{r['value']:.1f}" + (f" ({r['variant']})" if v is None else ""))
        print(f"| {base} | 2^{e} | " + " | ".join(row) + " |", flush=True)
