"""Run one bench config a few times (for ncu captures): python tools/run_case.py C2 [reps] [variant]."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import bench  # noqa: E402
import paper_conf_ppopp_ashkianidmo16_b200 as P  # noqa: E402

name = sys.argv[1] if len(sys.argv) > 1 else "C2"
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 3
variant = sys.argv[3] if len(sys.argv) > 3 else None
cfg = bench.CONFIGS[name]
keys, vals = bench.inputs_torch(cfg, cfg["n"], 0, "cuda")
plan = P.Plan(bench.spec_of(cfg), cfg["n"], with_values=cfg["kv"], variant=variant)
ko = torch.empty_like(keys)
vo = torch.empty_like(vals) if vals is not None else None
flush = bench.L2Flush("cuda")
for _ in range(reps):
    flush()
    plan.run(keys, vals, keys_out=ko, vals_out=vo)
torch.cuda.synchronize()
print("ok", name, plan.geometry(cfg["n"]))
