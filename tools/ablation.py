"""Design-space ablation on B200 (the paper's Table 4 / Table 6 / §6.1 questions).

Table 4 analogue: per-stage time (pre-scan / scan / post-scan, ms) and G keys/s of
every post-scan method for m in {2, 8, 32}, key-only and key-value, n = 2^25, DELTA buckets that
equally divide the 32-bit domain (one shift), L2 flushed, CUDA events:
  direct  -- tile variant WITHOUT the local reorder: every key stored from registers straight to
             its global position (MS_ABLATION_DIRECT; the paper's "Direct" method)
  warp    -- the paper's Warp-level MS: Alg. 3 ballot ranks, every warp reorders and
             stores its own 512-key segment (MS_ABLATION_WARP, tile variant)
  ballot  -- the same ballot post-scan with the block-level reorder of the 4096-key tile
             (MS_ABLATION_BALLOT; the paper's Block-level MS with Alg. 3)
  nw2     -- blocked-count reorder over 2 warps (1024-key tiles; MS_ABLATION_NW2, ranged variant)
  nw4     -- reorder over 4 warps (2048-key tiles; MS_ABLATION_NW4, ranged)
  tile    -- blocked-count block-level reorder over 8 warps (4096-key tiles), K1 -> K2 -> K3
             (MS_VARIANT_3K; the library's K3 v2)
  ranged  -- the same over CTA ranges, K1r -> K3 (MS_VARIANT_RANGED)
  one     -- the same in one cooperative launch (MS_VARIANT_ONE)
nw2 / nw4 / ranged together are the NW (warps per CTA) sweep of §6.1.
Per-stage times come from the per-stage trace (no PDL between kernels); G keys/s from the
whole-run trace.  usage: python tools/ablation.py [steps] [log2 n] > profiles/r02_ablation.md"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import bench  # noqa: E402
import workloads as W  # noqa: E402

steps = int(sys.argv[1]) if len(sys.argv) > 1 else 10
e = int(sys.argv[2]) if len(sys.argv) > 2 else 25
modes = ["direct", "warp", "ballot", "nw2", "nw4", "tile", "ranged", "one"]
variant = {"direct": "direct", "warp": "warp", "ballot": "ballot", "nw2": "nw2", "nw4": "nw4", "tile": "3k",
           "ranged": "ranged", "one": "one"}
print(f"| m | mode | method | launches | pre-scan ms | scan ms | post-scan ms | total ms (traced) | G keys/s |")
print("|---|---|---|---|---|---|---|---|---|")
for m in (2, 8, 32):
    for kv in (False, True):
        for mode in modes:
            cfg = dict(desc=f"delta m={m}", kind="delta", m=m, delta=(1 << 32) // m, n=1 << e, kv=kv,
                       dist="uniform", seed=W.SEEDS["C4"], variant=variant[mode])
            r = bench.bench_config(f"abl_{m}", cfg, steps, 3, torch.device("cuda"), 1, 0, with_e2e=False)
            st = r["stages_ms"]
            print(f"| {m} | {'KV' if kv else 'KO'} | {mode} | {r['launches_per_step']} | {st['k1_prescan']:.4f} | "
                  f"{st['k2_scan']:.4f} | {st['k3_postscan']:.4f} | {st['sum_without_pdl']:.4f} | "
                  f"{r['value']:.1f} |", flush=True)
