"""Delta-stepping SSSP on seeded synthetic graphs: multisplit re-bucketing vs sort-based
re-bucketing (the paper's motivating comparison, P:100-153 and footnote 1,
P:192-205).  Both loops compute identical distances (checked) with identical iteration counts;
reported: whole-loop wall time (synchronised), the summed device time of the re-bucketing
steps (CUDA events) and the keys re-bucketed.  Each loop runs twice; the second (warm) run is
reported.  usage: python tools/sssp_bench.py > profiles/r02_sssp.md"""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_ppopp_ashkianidmo16_b200.sssp import delta_stepping, synthetic_graph  # noqa: E402

print("| graph V, E, wmax | delta | m | iterations | keys re-bucketed | re-bucketing | device ms | "
      "G keys/s | loop ms (wall) |")
print("|---|---|---|---|---|---|---|---|---|")
for V, E, wmax, delta, m in [(1 << 20, 4 << 20, 1000, 1000, 8), (1 << 22, 16 << 20, 1000, 2000, 8),
                             (1 << 22, 16 << 20, 100000, 50000, 32), (1 << 23, 32 << 20, 1000, 4000, 16)]:
    g = synthetic_graph(V, E, wmax, seed=V + delta, device="cuda")
    ref = None
    for rb in ("multisplit", "sort"):
        for rep in range(2):
            torch.cuda.synchronize()
            t0 = time.perf_counter()
            dist, st = delta_stepping(g, 0, delta, m, rebucket=rb, time_rebucket=True)
            torch.cuda.synchronize()
            wall = (time.perf_counter() - t0) * 1e3
            if ref is None:
                ref = dist
            assert torch.equal(dist, ref), "re-bucketing methods disagree"
        print(f"| {V}, {E}, {wmax} | {delta} | {m} | {st['iterations']} | {st['multisplit_keys']} | {rb} | "
              f"{st['rebucket_ms']:.2f} | {st['multisplit_keys'] / (st['rebucket_ms'] * 1e-3) / 1e9:.2f} | "
              f"{wall:.1f} |", flush=True)
    del g
    torch.cuda.empty_cache()
