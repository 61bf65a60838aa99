"""Compact multi-config timing: python tools/quick_bench.py NSko,C2,C3 [steps]  (one line per config)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import bench  # noqa: E402

names = sys.argv[1].split(",") if len(sys.argv) > 1 else ["NSko", "NSkv", "C2", "C3", "C4ko", "IDSko"]
steps = int(sys.argv[2]) if len(sys.argv) > 2 else 20
tag = os.environ.get("TAG", "")
for nm in names:
    r = bench.bench_config(nm, bench.CONFIGS[nm], steps, 3, torch.device("cuda"), 1, 0, with_e2e=False)
    st = r["stages_ms"]
    print(f"{tag} {nm:8s} {r['value']:8.2f} Gk/s  median {r['ms_stats']['median']:.4f} ms  whole {r['whole_step_frac']:.3f}  "
          f"K1 {st['k1_prescan']:.4f} K2 {st['k2_scan']:.4f} K3 {st['k3_postscan']:.4f} ({r['roofline']['frac']:.3f})  "
          f"{r['variant']} x{r['launches_per_step']}", flush=True)
