"""Design-space ablation (the paper's Table 4 question on B200): does the local
reorder pay?  For m in {2,4,8,16,32}, key-only and key-value, DELTA buckets that equally divide the
32-bit domain (one shift), n = 2^25 and 2^28, time (G keys/s, L2 flushed, CUDA events):
  reorder  -- the default path (ONE launch for key-only, ranged/tile otherwise)
  tile     -- the 3-kernel tile variant with the local reorder (plan flag MS_VARIANT_3K)
  direct   -- the 3-kernel tile variant WITHOUT the local reorder: every key stored from registers
              straight to its global position (MS_ABLATION_DIRECT; the paper's "Direct" method)
Writes a markdown table to stdout.  usage: python tools/ablation.py [steps]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import bench  # noqa: E402
import workloads as W  # noqa: E402

steps = int(sys.argv[1]) if len(sys.argv) > 1 else 10
modes = {"reorder": None, "tile": "3k", "direct": "direct"}
print("| n | mode | m | KO G keys/s | KO K3 ms | KV G keys/s | KV K3 ms |")
print("|---|---|---|---|---|---|---|")
for e in (25, 28):
    for m in (2, 4, 8, 16, 32):
        for mode, variant in modes.items():
            row = []
            for kv in (False, True):
                cfg = dict(desc=f"delta m={m}", kind="delta", m=m, delta=(1 << 32) // m, n=1 << e, kv=kv,
                           dist="uniform", seed=W.SEEDS["C4"], variant=variant)
                r = bench.bench_config(f"abl_{m}", cfg, steps, 3, torch.device("cuda"), 1, 0, with_e2e=False)
                row += [f"{r['value']:.1f}", f"{r['stages_ms']['k3_postscan']:.4f}"]
            print(f"| 2^{e} | {mode} | {m} | " + " | ".join(row) + " |", flush=True)
