"""One bench workload's multisplit, run `reps` times on resident inputs (for ncu / sanitizer captures).

usage: python tools/run_one.py NAME [reps]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import bench  # noqa: E402
import paper_conf_ppopp_ashkianidmo16_b200 as P  # noqa: E402

name = sys.argv[1]
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 2
cfg = bench.CONFIGS[name]
dev = torch.device("cuda", 0)
n = cfg["n"]
keys, vals, ids = bench.inputs_torch(cfg, n, 0, dev)
plan = P.Plan(bench.spec_of(cfg), n, with_values=cfg["kv"], variant=cfg.get("variant"))
ko = torch.empty_like(keys)
vo = torch.empty_like(vals) if vals is not None else None
flush = bench.L2Flush(dev)
for _ in range(reps):
    flush()
    plan.run(keys, vals, ids, keys_out=ko, vals_out=vo)
torch.cuda.synchronize()
print(f"{name}: {reps} runs, {plan.last_launches()} launches per run, variant {plan.geometry(n)[2]}", flush=True)
