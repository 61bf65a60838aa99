"""Small multisplit cases for compute-sanitizer (memcheck / racecheck / synccheck / initcheck):
every kernel family once -- ONE (KO, KV, IDS), CTA-range K1r -> K3, tile K1 -> K2 -> K3 for m <= 32
and m = 256, the Direct / NW / ballot / warp-level ablations, and the fused sharded scatter over virtual ranks -- each checked
against the CPU oracle so a run under the sanitizer is also a parity run.

usage: compute-sanitizer --tool racecheck python tools/sanitize_cases.py [n]"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))

import numpy as np  # noqa: E402
import torch  # noqa: E402

import oracle  # noqa: E402
import workloads as W  # noqa: E402
from msutil import from_dev, make_case, to_dev  # noqa: E402
import paper_conf_ppopp_ashkianidmo16_b200 as P  # noqa: E402
from paper_conf_ppopp_ashkianidmo16_b200.dist import scatter_multisplit_virtual  # noqa: E402

n = int(sys.argv[1]) if len(sys.argv) > 1 else 3 * 4096 * 148 + 77  # > 1 tile per resident CTA, ragged
cases = [("delta", 8, False, "one"), ("delta", 8, True, "one"), ("splitters", 32, False, "one"),
         ("ids", 32, True, "one"), ("lowbits", 16, True, "ranged"), ("splitters", 32, True, "ranged"),
         ("delta", 32, False, "3k"), ("ids", 5, True, "3k"), ("delta", 256, False, "3k"),
         ("splitters", 200, True, "3k"), ("ids", 100, False, "3k"), ("delta", 256, True, None),
         ("splitters", 100, False, None), ("delta", 8, False, "nw2"), ("delta", 32, True, "nw4"),
         ("delta", 32, True, "warp"), ("delta", 256, False, "warp"), ("delta", 8, False, "ballot")]
fails = 0
for kind, m, kv, variant in cases:
    # even seeds for the NW ablations: make_case then picks delta = 2^32 / m (the one-shift kind they need)
    case = make_case(kind, m, n, seed=2 * m if variant in ("nw2", "nw4", "warp", "ballot") else m + 3, kv=kv, dist="binomial")
    plan = P.Plan(P.BucketSpec(**case["spec_kw"]), n, with_values=kv, variant=variant)
    ko, vo, off = plan.run(to_dev(case["keys"]), to_dev(case["vals"]), to_dev(case["ids"]))
    torch.cuda.synchronize()
    eko, evo, eoff = oracle.multisplit(case["ospec"], case["keys"], case["vals"], ids=case["ids"])
    ok = np.array_equal(from_dev(ko), eko) and (evo is None or np.array_equal(from_dev(vo), evo)) and \
        np.array_equal(from_dev(off).astype(np.uint64), eoff)
    fails += not ok
    print(f"{kind:9s} m={m:3d} kv={kv:d} variant={variant}: launches={plan.last_launches()} "
          f"{'ok' if ok else 'MISMATCH'}", flush=True)
for kv in (False, True):  # the Direct ablation
    case = make_case("delta", 8, n, seed=8, kv=kv)
    plan = P.Plan(P.BucketSpec(**case["spec_kw"]), n, with_values=kv, variant="direct")
    ko, vo, _ = plan.run(to_dev(case["keys"]), to_dev(case["vals"]))
    eko, evo, _ = oracle.multisplit(case["ospec"], case["keys"], case["vals"])
    ok = np.array_equal(from_dev(ko), eko) and (evo is None or np.array_equal(from_dev(vo), evo))
    fails += not ok
    print(f"direct    m=  8 kv={kv:d}: {'ok' if ok else 'MISMATCH'}", flush=True)
for kv in (False, True):  # fused sharded scatter, 3 virtual ranks
    case = make_case("splitters", 32, n, seed=11, kv=kv, dist="hot")
    cuts = [0, n // 3, n // 3 + 4097, n]
    ks = [to_dev(case["keys"][cuts[r]:cuts[r + 1]]) for r in range(3)]
    vs = [to_dev(case["vals"][cuts[r]:cuts[r + 1]]) for r in range(3)] if kv else None
    k2, v2 = scatter_multisplit_virtual(ks, vs, P.BucketSpec(**case["spec_kw"]))
    eko, evo, _ = oracle.multisplit(case["ospec"], case["keys"], case["vals"])
    ok = np.array_equal(from_dev(k2), eko) and (evo is None or np.array_equal(from_dev(v2), evo))
    fails += not ok
    print(f"fused scatter P=3 kv={kv:d}: {'ok' if ok else 'MISMATCH'}", flush=True)
for kind, m, kw, kv in (("delta", 1000, dict(delta=4000037), True), ("ids", 4096, dict(id_bytes=4), False)):
    # m > 256: two passes + the offsets kernel
    ospec = oracle.Spec(kind, m, delta=kw.get("delta", 1), id_bytes=kw.get("id_bytes", 1))
    keys = W.keys_np(n, 5)
    ids = W.bucket_draw_np(n, 5, "binomial", m).astype(np.uint32) if kind == "ids" else None
    vals = W.values_np(n, 5, "index") if kv else None
    plan = P.Plan(P.BucketSpec(kind, m, **kw), n, with_values=kv)
    ko, vo, off = plan.run(to_dev(keys), to_dev(vals), to_dev(ids))
    eko, evo, eoff = oracle.multisplit(ospec, keys, vals, ids=ids)
    ok = np.array_equal(from_dev(ko), eko) and (evo is None or np.array_equal(from_dev(vo), evo)) and \
        np.array_equal(from_dev(off).astype(np.uint64), eoff)
    fails += not ok
    print(f"wide {kind} m={m} kv={kv:d}: launches={plan.last_launches()} {'ok' if ok else 'MISMATCH'}", flush=True)
print("SANITIZE_CASES", "FAIL" if fails else "OK", flush=True)
sys.exit(1 if fails else 0)
