"""Key-only variant sweep (ONE / ranged / tile): python tools/variant_sweep_ko.py > profiles/r02_variants_ko.md"""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import bench
steps = 15
print("| workload | n | one | ranged | tile | default |")
for base in ("sweep_m2_ko", "sweep_m4_ko", "sweep_m8_ko", "sweep_m16_ko", "C2", "C2far", "IDSko", "sweep_m32_ko"):
    for e in (23, 25, 27, 28):
        cfg = dict(bench.CONFIGS[base], n=1 << e)
        row = []
        for v in ("one", "ranged", "3k", None):
            r = bench.bench_config(base, dict(cfg, variant=v), steps, 3, torch.device("cuda"), 1, 0, with_e2e=False)
            row.append(f"{r['value']:.1f}")
        print(f"| {base} | 2^{e} | " + " | ".join(row) + " |", flush=True)
