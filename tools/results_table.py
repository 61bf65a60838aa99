"""DESIGN.md §8 results table from one bench line: python tools/results_table.py profiles/r02f_bench_line.json

One row per workload (the headline first): G keys/s, variant (launches), whole-step fraction of the
measured copy rate and of 8 TB/s nominal, and the reduced-bit sort comparator (torch.sort of the
bucket ids + gather, bit-identity checked in the run) with our speed-up over it."""
import json
import sys

d = json.loads(open(sys.argv[1]).read().strip().splitlines()[-1])
rows = [(d["config"]["workload"], d)] + list(d.get("extra", {}).items())
print("| workload | G keys/s | variant (launches) | whole step / copy | / 8 TB/s | reduced-bit sort G keys/s (x ours) |")
print("|---|---|---|---|---|---|")
for name, r in rows:
    c = r.get("comparators", {}).get("torch_sort_on_bucket_id", {})
    cmp_ = f"{c['value']:.1f} ({r['value'] / c['value']:.1f}x)" if c.get("value") else ""
    if c and c.get("bit_identical_to_multisplit") is False:
        cmp_ += " NOT bit-identical"
    print(f"| {name} | {r['value']:.1f} | {r.get('variant', '')} ({r.get('launches_per_step', '')}) | "
          f"{r.get('whole_step_frac', 0):.3f} | {r.get('whole_step_frac_nominal_8tbs', 0):.3f} | {cmp_} |")
