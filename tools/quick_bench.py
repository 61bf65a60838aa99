"""Compact multi-config timing: python tools/quick_bench.py C2,NSko,NSkv [steps]  (one line per config)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import bench  # noqa: E402

names = sys.argv[1].split(",") if len(sys.argv) > 1 else ["C2", "NSko", "NSkv", "C4ko", "C3"]
steps = int(sys.argv[2]) if len(sys.argv) > 2 else 10
tag = os.environ.get("TAG", "")
for nm in names:
    r = bench.bench_config(nm, bench.CONFIGS[nm], steps, 3, torch.device("cuda"), 1, 0, with_e2e=False)
    st = r["stages_ms"]
    print(f"{tag} {nm:6s} {r['value']:8.2f} Gk/s  step {r['ms_per_step']:.4f} ms  whole {r['whole_step_frac']:.3f}  "
          f"K1 {st['k1_prescan']:.4f} ({r['roofline']['k1_prescan_frac'] or 0:.3f})  K2 {st['k2_scan']:.4f}  "
          f"K3 {st['k3_postscan']:.4f} ({r['roofline']['frac']:.3f})  nopdl {st['sum_without_pdl']:.4f}  "
          f"T={r['tile']} v={r['variant']} launches={r['gpu_launches'] // steps}", flush=True)
