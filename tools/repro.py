"""Run one parity case (for compute-sanitizer): python tools/repro.py kind m n kv [dist] [variant]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "tests"))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import oracle  # noqa: E402
import paper_conf_ppopp_ashkianidmo16_b200 as P  # noqa: E402
from msutil import from_dev, make_case, to_dev  # noqa: E402

kind, m, n, kv = sys.argv[1], int(sys.argv[2]), int(sys.argv[3]), sys.argv[4] == "1"
dist = sys.argv[5] if len(sys.argv) > 5 else "uniform"
variant = sys.argv[6] if len(sys.argv) > 6 else None
case = make_case(kind, m, n, seed=1000 * m + 1, dist=dist, kv=kv)
plan = P.Plan(P.BucketSpec(**case["spec_kw"]), max(n, 1), with_values=kv, variant=variant)
ko, vo, off = plan.run(to_dev(case["keys"]), to_dev(case["vals"]), to_dev(case["ids"]))
torch.cuda.synchronize()
eko, evo, eoff = oracle.multisplit(case["ospec"], case["keys"], case["vals"], ids=case["ids"])
ok = np.array_equal(from_dev(ko), eko) and (evo is None or np.array_equal(from_dev(vo), evo))
print("match" if ok else "MISMATCH", kind, m, n, kv, plan.geometry(n))
