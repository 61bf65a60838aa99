"""Debug: which CTA ranges / tiles the ONE-launch path gets wrong (L tiles of 4096 keys)."""
import os, sys
sys.path.insert(0, os.path.join(os.path.dirname(os.path.abspath(__file__)), "..", "tests"))
sys.path.insert(0, os.path.join(os.path.dirname(os.path.abspath(__file__)), ".."))
import numpy as np, torch
import oracle
from msutil import make_case, to_dev, from_dev
import paper_conf_ppopp_ashkianidmo16_b200 as P
L = int(sys.argv[1]) if len(sys.argv) > 1 else 889
kind, m = (sys.argv[2], int(sys.argv[3])) if len(sys.argv) > 3 else ("delta", 8)
T = 4096
n = L * T
KV = os.environ.get("KV", "0") == "1"
case = make_case(kind, m, n, seed=int(os.environ.get("SEED", "81")), kv=True)
spec = P.BucketSpec(**case["spec_kw"])
plan = P.Plan(spec, n, with_values=KV, variant="ranged")
kd = to_dev(case["keys"]); vd = to_dev(case["vals"]) if KV else None
eko0 = oracle.multisplit(case["ospec"], case["keys"], case["vals"])[0]
fails = 0
ws = plan.workspace(n)
C = min(L, 444)
ids_np = np.asarray(oracle.bucket_ids(case["ospec"], case["keys"]) if hasattr(oracle, "bucket_ids") else None)
for rep in range(int(os.environ.get("REPS", "1"))):
    ko = torch.empty_like(kd)
    vo = torch.empty_like(vd) if vd is not None else None
    plan.run(kd, vd, keys_out=ko, vals_out=vo, workspace=ws)
    torch.cuda.synchronize()
    if not np.array_equal(from_dev(ko), eko0):
        fails += 1
        if fails == 1 and ids_np is not None and ids_np.ndim:
            HC = ws[256:256 + C * m * 4].view(torch.int32).cpu().numpy().view(np.uint32).reshape(C, m)
            bnd = [c * L // C * T for c in range(C + 1)]
            exp = np.stack([np.bincount(ids_np[bnd[c]:bnd[c + 1]], minlength=m) for c in range(C)])
            badc = np.flatnonzero((HC != exp).any(axis=1))
            print("bad ranges", badc[:10], "count", len(badc))
            for c in badc[:3]:
                print(c, "got", HC[c], "exp", exp[c], "tiles", bnd[c] // T, bnd[c + 1] // T)
print("rep failures", fails)
ko = from_dev(ko)
eko, evo, eoff = oracle.multisplit(case["ospec"], case["keys"], case["vals"])
if not KV:  # recover input indices of the keys by a stable match (keys may repeat: use oracle order)
    vo = np.full(n, -1, np.int64); evo = evo.astype(np.int64)
    same = ko == eko
    vo[same] = evo[same]
else:
    vo = from_dev(vo)
off = torch.empty(m + 1, dtype=torch.int32, device="cuda")
plan.run(kd, vd, offsets=off)
print("offsets ok", np.array_equal(from_dev(off).astype(np.uint64), eoff))
bad = np.flatnonzero(vo != evo)
print("bad", len(bad), "of", n)
if len(bad):
    idx = vo[bad].astype(np.int64)  # vals = input index
    tiles = np.unique(idx // T)
    C = min(L, 444)
    rng = [int(np.searchsorted([c * L // C for c in range(C + 1)], t, side="right") - 1) for t in tiles[:20]]
    print("tiles", tiles[:20], "ranges", rng)
    b = bad[0]
    print("first bad pos", b, "got idx", vo[b], "exp idx", evo[b])
