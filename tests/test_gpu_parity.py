"""GPU parity: the CUDA path through the C ABI vs the CPU oracle, bit for bit.

Every comparison is element-wise and exact (integer work; the stable result
is unique).  Inputs come from the seeded generators (workloads/); expected
values only from oracle/ (or, for the bucket functors, the closed form).
"""
import numpy as np
import pytest

import oracle
import workloads as W
from msutil import from_dev, make_case, to_dev

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")


def _pkg():
    import paper_conf_ppopp_ashkianidmo16_b200 as P
    return P


FORCED = {"3k": 0, "tile": 0, "direct": 0, "ranged": 1, "one": 2, "nw2": 1, "nw4": 1, "ballot": 0, "warp": 0}


def _run_case(case, variant=None, want_offsets=True, expect_variant=None):
    """Runs the case through ms_run and checks that the kernels which ran are the ones the
    variant names: ms_plan_last_launches must equal the launch count of the variant the plan
    reports (or was forced to), so a silent re-routing to another path fails the test."""
    P = _pkg()
    from paper_conf_ppopp_ashkianidmo16_b200 import _abi
    spec = P.BucketSpec(**case["spec_kw"])
    n = len(case["keys"])
    kv = case["vals"] is not None
    plan = P.Plan(spec, max(n, 1), with_values=kv, variant=variant)
    ko, vo, off = plan.run(to_dev(case["keys"]), to_dev(case["vals"]), to_dev(case["ids"]),
                           want_offsets=want_offsets)
    torch.cuda.synchronize()
    v = plan.geometry(n)[2]
    if variant is not None:
        assert v == FORCED[variant], f"geometry reports variant {v} for forced {variant}"
    if expect_variant is not None:
        assert v == expect_variant, f"variant {v}, expected {expect_variant}"
    if v == _abi.VARIANT_WIDE:  # m > 256: two passes (each 1..3 launches) + the offsets pass
        assert (2 <= plan.last_launches() <= 2 * 3 * (2 if spec.kind == "ids" else 1) + 2) if n else \
            plan.last_launches() == 0
    else:
        assert plan.last_launches() == (_abi.LAUNCHES[v] if n else 0), \
            f"{plan.last_launches()} launches for variant {v} (n={n})"
    return from_dev(ko), from_dev(vo), (None if off is None else from_dev(off)), plan


def _expect(case):
    return oracle.multisplit(case["ospec"], case["keys"], case["vals"], ids=case["ids"])


def _assert_equal(case, got, exp, what=""):
    ko, vo, off, _ = got
    eko, evo, eoff = exp
    assert np.array_equal(ko, eko), f"keys differ {what}: first at {np.flatnonzero(ko != eko)[:5]}"
    if evo is not None:
        assert np.array_equal(vo, evo), f"vals differ {what}: first at {np.flatnonzero(vo != evo)[:5]}"
    if off is not None:
        assert np.array_equal(off.astype(np.uint64), eoff), f"offsets differ {what}"


NS = [0, 1, 31, 2047, 2048, 2049, 4095, 4097, 8191, 8193, 100003]
MS = [1, 2, 3, 5, 8, 31, 32, 33, 64, 127, 255, 256]


# Low-bit buckets need a power-of-two m (reading #10); m > 32 always uses the tile variant, so the
# forced CTA-range and ONE variants are only generated for m <= 32.
MATRIX = [(kind, m, variant) for variant in (None, "3k", "ranged", "one")
          for kind in ("lowbits", "delta", "splitters", "ids")
          for m in MS if not (kind == "lowbits" and m & (m - 1)) and not (variant in ("ranged", "one") and m > 32)]


@pytest.mark.parametrize("kind,m,variant", MATRIX)
def test_parity_matrix(kind, m, variant):
    """kind x m x n (empty, ragged, tile edges) x KO/KV, uniform keys; the default variant
    (ONE for m <= 32 at these sizes, tile above) and every forced variant, each run asserting
    the number of kernels it launched."""
    for i, n in enumerate(NS):
        for kv in (False, True):
            case = make_case(kind, m, n, seed=1000 * m + i, kv=kv, id_bytes=1 if i % 2 else 4)
            _assert_equal(case, _run_case(case, variant), _expect(case), f"{kind} m={m} n={n} kv={kv} {variant}")


@pytest.mark.parametrize("variant", ["ranged", "one"])
@pytest.mark.parametrize("kind,m,kv", [("delta", 8, False), ("splitters", 32, True), ("ids", 5, True),
                                       ("lowbits", 2, False), ("delta", 32, True), ("delta", 16, True),
                                       ("ids", 32, False)])
def test_ranged_range_edges(kind, m, kv, variant):
    """CTA-range (K1r -> K3, 2 launches) and ONE (1 launch) variants around C = resident K3 CTAs:
    L < C, L = C +- 1, L = 3C + r (ranges of 1..4 tiles, the ragged last tile at the end of the
    last range); every run asserts its launch count."""
    T = 4096
    sms = torch.cuda.get_device_properties(0).multi_processor_count
    for i, L in enumerate([sms - 1, 2 * sms, 4 * sms + 1, 6 * sms - 1, 6 * sms, 6 * sms + 1, 13 * sms + 7]):
        for n in (L * T, L * T - T + 3):
            case = make_case(kind, m, n, seed=77 + i, kv=kv)
            _assert_equal(case, _run_case(case, variant), _expect(case), f"{kind} m={m} L={L} n={n} {variant}")


@pytest.mark.parametrize("kind,m", [("delta", 32), ("delta", 17), ("splitters", 32), ("lowbits", 32), ("delta", 24),
                                    ("delta", 9), ("lowbits", 16), ("splitters", 12), ("ids", 32), ("ids", 9),
                                    ("delta", 64), ("lowbits", 64), ("splitters", 40), ("ids", 64), ("delta", 33),
                                    ("delta", 2), ("lowbits", 8), ("splitters", 5), ("ids", 3)])
def test_one_k32_edges(kind, m):
    """Key-only ONE with 2..64 buckets runs tiles of 8192 keys (32 per thread, 2 CTAs/SM; computed
    ids: phase 1 double-buffered through the reorder buffer; u8 ids: 32 prefetched per thread): L = ceil(n / 8192) around C = 2 x SMs ranges --
    L < C, L = C +- 1, 2C + 1, 3C + r, 5C + 3 (ranges of 1..6 full tiles, odd and even counts),
    the ragged last tile -- and inputs of one tile or less, 1 launch each."""
    T = 8192
    C = 2 * torch.cuda.get_device_properties(0).multi_processor_count
    sizes = [1, 4095, 4097, 8191, 8192, 8193, 3 * T + 5]
    for L in (C - 1, C, C + 1, 2 * C + 1, 3 * C + 7, 5 * C + 3):
        sizes += [L * T, L * T - T + 3]
    for i, n in enumerate(sizes):
        case = make_case(kind, m, n, seed=4100 + i, kv=False)
        _assert_equal(case, _run_case(case, "one"), _expect(case), f"{kind} m={m} n={n} one-k32")


@pytest.mark.parametrize("kind,m", [("delta", 2), ("lowbits", 8), ("splitters", 5), ("ids", 4), ("delta", 3)])
def test_parity_default_large_ko_small_m(kind, m):
    """Key-only m <= 8 takes the 8192-key ONE tiles: the library's default at n = 2^26 + 5 (ranges of
    ~27 tiles), bit-exact, 1 launch."""
    n = (1 << 26) + 5
    case = make_case(kind, m, n, seed=900 + m, kv=False)
    _assert_equal(case, _run_case(case, expect_variant=2), _expect(case), f"{kind} m={m} n={n}")


@pytest.mark.parametrize("n", [(1 << 26) + 5, 1 << 28])
@pytest.mark.parametrize("kind,m", [("delta", 2), ("delta", 8), ("lowbits", 16), ("splitters", 16), ("ids", 8),
                                    ("delta", 32), ("ids", 32)])
def test_parity_default_large_kv(kind, m, n):
    """The library's DEFAULT key-value path at n = 2^26 + 5 and 2^28 (K1r -> K3, 2 launches), full
    compare."""
    case = make_case(kind, m, n, seed=900 + m, kv=True, vals_kind="random")
    want = _abi_mod().VARIANT_RANGED
    _assert_equal(case, _run_case(case, expect_variant=want), _expect(case), f"default KV {kind} m={m} n={n}")


def _abi_mod():
    from paper_conf_ppopp_ashkianidmo16_b200 import _abi
    return _abi


@pytest.mark.parametrize("kv", [False, True])
def test_parity_2p28_m32(kv):
    """Headline size n = 2^28, m = 32 (DELTA 2^27, the NS configs), full element-wise compare."""
    n = 1 << 28
    keys = W.keys_np(n, W.SEEDS["C4"])
    vals = W.values_np(n, W.SEEDS["C4"], "random") if kv else None
    case = dict(spec_kw=dict(kind="delta", m=32, delta=1 << 27), ospec=oracle.Spec("delta", 32, delta=1 << 27),
                keys=keys, vals=vals, ids=None)
    _assert_equal(case, _run_case(case), _expect(case), "2^28 m=32")


@pytest.mark.parametrize("dist", ["buckets", "binomial", "hot", "one"])
@pytest.mark.parametrize("kind,m", [("lowbits", 2), ("delta", 8), ("splitters", 32), ("ids", 32),
                                    ("delta", 256), ("splitters", 255)])
def test_parity_distributions(kind, m, dist):
    """Skewed workloads (§6.5): binomial, 75 % hot bucket, all in one bucket."""
    for n in (4097, (1 << 20) + 7):
        case = make_case(kind, m, n, seed=7 + m, dist=dist, kv=True)
        for variant in ([None, "3k", "ranged", "one"] if m <= 32 else [None, "3k"]):
            _assert_equal(case, _run_case(case, variant), _expect(case), f"{kind} m={m} {dist} n={n} {variant}")


@pytest.mark.parametrize("dist", ["uniform", "binomial", "hot", "one"])
@pytest.mark.parametrize("kind,m", [("delta", 64), ("splitters", 48), ("ids", 40), ("lowbits", 64)])
def test_parity_ko_33_64(kind, m, dist):
    """Key-only 33..64 buckets: ONE with 8192-key tiles (the default) and the forced tile variant
    (ballot K3), uniform and skewed, ragged sizes up to 3 * 2^22 + 5 keys."""
    for n in (4097, (1 << 20) + 7, 3 * (1 << 22) + 5):
        case = make_case(kind, m, n, seed=11 + m, dist=dist, kv=False)
        for variant in (None, "3k", "one"):
            _assert_equal(case, _run_case(case, variant, expect_variant=0 if variant == "3k" else 2),
                          _expect(case), f"{kind} m={m} {dist} n={n} {variant}")


@pytest.mark.parametrize("variant", [None, "3k", "ranged", "one"])
@pytest.mark.parametrize("kind,m,kv", [("delta", 8, False), ("splitters", 32, True), ("lowbits", 32, True),
                                       ("lowbits", 2, True), ("ids", 32, False), ("ids", 16, True)])
def test_parity_2p25(kind, m, kv, variant):
    """BJ configs C2 / C3 size (n = 2^25), full element-wise compare, every variant."""
    case = make_case(kind, m, 1 << 25, seed=W.SEEDS["C3"], kv=kv, vals_kind="random")
    _assert_equal(case, _run_case(case, variant), _expect(case), f"2^25 {kind} m={m} {variant}")


@pytest.mark.parametrize("kv", [False, True])
def test_parity_2p28_m256(kv):
    """BJ config C4 (n = 2^28, m = 256, DELTA = 2^24), full element-wise compare."""
    n = 1 << 28
    keys = W.keys_np(n, W.SEEDS["C4"])
    vals = W.values_np(n, W.SEEDS["C4"], "random") if kv else None
    case = dict(spec_kw=dict(kind="delta", m=256, delta=1 << 24), ospec=oracle.Spec("delta", 256, delta=1 << 24),
                keys=keys, vals=vals, ids=None)
    _assert_equal(case, _run_case(case), _expect(case), "2^28 m=256")


def test_intermediates_H_G_offsets():
    """K1 / K2 intermediates vs the CPU Eq. (2) evaluation with the GPU's tile size T."""
    P = _pkg()
    for kind, m, n in [("delta", 8, 100003), ("splitters", 32, (1 << 20) + 7), ("lowbits", 256, 3 * 8192 + 5),
                       ("ids", 17, 50000), ("lowbits", 256, 297 * 4096 + 1), ("delta", 100, 299 * 4096 + 77),
                       ("splitters", 200, 298 * 4096), ("ids", 64, 300 * 4096 + 5),
                       ("delta", 256, 299 * 8192 + 4097), ("lowbits", 128, 297 * 8192)]:
        case = make_case(kind, m, n, seed=m + n, kv=False)
        plan = P.Plan(P.BucketSpec(**case["spec_kw"]), n)
        T, L, _ = plan.geometry(n)
        kd, idd = to_dev(case["keys"]), to_dev(case["ids"])
        H = plan.prescan(kd, idd)
        Hh = from_dev(H).reshape(m, L).copy()
        ids = oracle.bucket_ids(case["ospec"], case["keys"], ids=case["ids"])
        eH, eG = oracle.tile_matrices(ids, m, T)
        assert np.array_equal(Hh, eH), f"H differs {kind} m={m}"
        off = torch.empty(m + 1, dtype=torch.int32, device="cuda")
        plan.scan(H, n, off)
        assert np.array_equal(from_dev(H).reshape(m, L), eG), f"G differs {kind} m={m}"
        _, _, eoff = oracle.multisplit(case["ospec"], case["keys"], ids=case["ids"])
        assert np.array_equal(from_dev(off).astype(np.uint64), eoff)
        ko, _ = plan.postscan(kd, H, ids=idd)
        assert np.array_equal(from_dev(ko), oracle.multisplit(case["ospec"], case["keys"], ids=case["ids"])[0])


# m > 32: 2048-key subproblems below 296 x 4096 keys, 4096-key up to 296 x 8192, and on key-only plans
# 8192-key ones above (reordered as two 4096-key windows per CTA with a running G): sizes around both
# boundaries, ragged last subproblems (one full window + a partial one, a partial first window only)
K1B_N = [296 * 4096, 296 * 4096 + 1, 297 * 4096 + 4095, 299 * 4096 + 77,
         296 * 8192, 296 * 8192 + 1, 297 * 8192 + 4095, 299 * 8192 + 4097, 300 * 8192 + 77]


@pytest.mark.parametrize("n", K1B_N)
@pytest.mark.parametrize("kind,m,seed", [("lowbits", 64, 3), ("lowbits", 256, 0), ("delta", 33, 2),
                                         ("delta", 100, 1), ("delta", 256, 4), ("splitters", 255, 5),
                                         ("splitters", 128, 7)])
def test_parity_m_gt32_4096_tiles(kind, m, seed, n):
    case = make_case(kind, m, n, seed=seed, kv=seed % 2 == 1)
    got = _run_case(case)
    assert got[3].geometry(n)[0] == (8192 if n >= 296 * 8192 and seed % 2 == 0 else 4096)  # key-value: 4096
    _assert_equal(case, got, _expect(case), f"{kind} m={m} n={n}")


def test_scan_many_chunks():
    """K2 look-back across many chunks (m*L >> 4096) against numpy's exclusive cumsum of H."""
    P = _pkg()
    n = 1 << 24
    plan = P.Plan(P.BucketSpec.delta_range(256, 1 << 24), n)
    T, L, _ = plan.geometry(n)
    rng = np.random.default_rng(0)
    H = rng.integers(0, 60, size=256 * L).astype(np.uint32)
    exp = np.concatenate([[0], np.cumsum(H.astype(np.uint64))[:-1]]).astype(np.uint32)
    d = to_dev(H)
    plan.scan(d, n)
    assert np.array_equal(from_dev(d), exp)


def test_torch_stable_sort_cross_check():
    """Independent GPU cross-check: torch.sort(ids, stable=True) + gather (the RBS analogue, §3.4)."""
    P = _pkg()
    n, m, delta = (1 << 22) + 3, 8, 400000000
    keys = W.keys_torch(n, 5, "cuda")
    vals = W.values_torch(n, 5, "cuda", "random")
    ko, vo, off = P.multisplit(keys, vals, P.BucketSpec.delta_range(m, delta))
    k64 = keys.to(torch.int64) & 0xFFFFFFFF
    ids = torch.clamp(k64 // delta, max=m - 1)
    _, idx = torch.sort(ids, stable=True)
    assert torch.equal(ko, keys[idx]) and torch.equal(vo, vals[idx])


@pytest.mark.parametrize("delta", [1, 3, 7, 400000000, 1 << 24, 0xFFFFFFFF, 0x80000001, 65535])
def test_delta_functor_exhaustive(delta):
    """Device DELTA functor == min(k // delta, m-1) for EVERY 32-bit key (exact magic division)."""
    P = _pkg()
    m = 256
    plan = P.Plan(P.BucketSpec.delta_range(m, delta), 1 << 30)
    chunk = 1 << 30
    for c in range(4):
        k64 = torch.arange(c * chunk, (c + 1) * chunk, dtype=torch.int64, device="cuda")
        keys = (k64 - ((k64 >> 31) << 32)).to(torch.int32)
        got = plan.bucket_ids(keys)
        exp = torch.clamp(k64 // delta, max=m - 1).to(torch.int32)
        assert torch.equal(got, exp), f"delta={delta} chunk {c}"
        del k64, keys, got, exp


def test_splitter_functor_dense():
    """Device splitter search == #{j: s_j < k} on keys at and around every splitter (incl. duplicates)."""
    P = _pkg()
    for m in (2, 3, 32, 200, 256):
        spl = sorted(W.gen_splitters(m, m).tolist())
        if m > 3:
            spl[1] = spl[2]
        keys = sorted({0, 1, 0xFFFFFFFF} | {s + d for s in spl for d in (-1, 0, 1) if 0 <= s + d <= 0xFFFFFFFF})
        kn = np.array(keys, dtype=np.uint32)
        plan = P.Plan(P.BucketSpec.from_splitters(spl), len(kn))
        got = from_dev(plan.bucket_ids(to_dev(kn)))
        exp = np.searchsorted(np.array(spl, dtype=np.uint64), kn.astype(np.uint64), side="left")
        assert np.array_equal(got, exp.astype(np.uint32))


def _clustered_splitter_sets():
    """Splitter sets that stress the top-byte table: crowded 2^24 windows (fallback
    search), splitters exactly on window boundaries, at 0 / 2^32-1, and duplicates."""
    rng = np.random.default_rng(11)
    sets = []
    for m in (2, 5, 32, 33, 200, 256):
        sets.append(sorted(int(x) for x in rng.integers(0x37000000, 0x37001000, m - 1)))   # one window
        sets.append(sorted(int(t) << 24 for t in rng.integers(0, 256, m - 1)))             # boundaries
        half = (m - 1) // 2
        mix = [int(x) for x in rng.integers(0, 1 << 32, half)] + [0xA0FFFFFF] * ((m - 1) - half)
        sets.append(sorted(mix))
    # the 1024-bin table of K1/K3 (bins of 2^22 keys, ms_device.cuh id_spl_table):
    # many splitters in one bin, splitters on bin starts, on the last and the
    # second-to-last key of a bin, and runs of duplicates inside one bin
    for m in (3, 32, 256):
        sets.append(sorted(int(x) for x in rng.integers(0x12C00000, 0x12C00000 + (1 << 22), m - 1)))
        sets.append(sorted(int(t) << 22 for t in rng.integers(0, 1024, m - 1)))
        sets.append(sorted((int(t) << 22) + (1 << 22) - 1 - int(t % 2) for t in rng.integers(0, 1024, m - 1)))
        sets.append(sorted([0x40000005] * ((m - 1) // 2) + [int(x) for x in rng.integers(0, 1 << 32, m - 1 - (m - 1) // 2)]))
    sets.append([0])
    sets.append([0xFFFFFFFF])
    sets.append([0, 0xFFFFFFFF, 0xFFFFFFFF])
    return sets


def test_splitter_functor_clustered():
    P = _pkg()
    for spl in _clustered_splitter_sets():
        near = {s + d for s in spl for d in (-1, 0, 1) if 0 <= s + d <= 0xFFFFFFFF}
        near |= {(t << 22) + d for t in range(1024) for d in (-2, -1, 0, 1) if 0 <= (t << 22) + d <= 0xFFFFFFFF}
        kn = np.array(sorted(near | {0xFFFFFFFF}), dtype=np.uint32)
        plan = P.Plan(P.BucketSpec.from_splitters(spl), len(kn))
        got = from_dev(plan.bucket_ids(to_dev(kn)))
        exp = np.searchsorted(np.array(spl, dtype=np.uint64), kn.astype(np.uint64), side="left")
        assert np.array_equal(got, exp.astype(np.uint32)), f"m={len(spl) + 1}"


def test_parity_clustered_splitters():
    """Full K1/K2/K3 pipeline with clustered splitters, keys drawn near the splitters."""
    for i, spl in enumerate(_clustered_splitter_sets()):
        m = len(spl) + 1
        rng = np.random.default_rng(100 + i)
        n = 70001
        base = np.array(spl, dtype=np.int64)[rng.integers(0, len(spl), n)]
        keys = np.clip(base + rng.integers(-3000, 3000, n), 0, 0xFFFFFFFF).astype(np.uint32)
        keys[::7] = W.keys_np(n, i)[::7]
        for kv in (False, True):
            vals = W.values_np(n, i, "index") if kv else None
            case = dict(spec_kw=dict(kind="splitters", m=m, splitters=spl), keys=keys, vals=vals, ids=None,
                        ospec=oracle.Spec("splitters", m, splitters=spl))
            _assert_equal(case, _run_case(case), _expect(case), f"clustered set {i} m={m} kv={kv}")


def test_validate_flags_out_of_range_ids():
    P = _pkg()
    n, m = 10000, 16
    ids = W.bucket_draw_np(n, 1, "buckets", m)
    keys = W.keys_np(n, 1)
    plan = P.Plan(P.BucketSpec.precomputed(m, 1), n, validate=True)
    plan.run(to_dev(keys), ids=to_dev(ids))
    assert plan.check() == 0
    bad = ids.copy()
    bad[777] = 200
    plan.run(to_dev(keys), ids=to_dev(bad))
    assert plan.check() == -8
    plan.run(to_dev(keys), ids=to_dev(ids))
    assert plan.check() == 0


def test_run_host_matches_oracle():
    """ms_run_host (host buffers, copies inside the call) == oracle."""
    P = _pkg()
    case = make_case("splitters", 32, (1 << 20) + 9, seed=3, kv=True, vals_kind="random")
    plan = P.Plan(P.BucketSpec(**case["spec_kw"]), len(case["keys"]), with_values=True)
    kh = torch.from_numpy(case["keys"].view(np.int32).copy()).pin_memory()
    vh = torch.from_numpy(case["vals"].view(np.int32).copy()).pin_memory()
    ko, vo, off = plan.run_host(kh, vh)
    eko, evo, eoff = _expect(case)
    assert np.array_equal(ko.numpy().view(np.uint32), eko)
    assert np.array_equal(vo.numpy().view(np.uint32), evo)
    assert np.array_equal(off.numpy().view(np.uint32).astype(np.uint64), eoff)


def test_repeated_runs_same_workspace():
    """Look-back status is re-zeroed each run: repeated runs on one workspace stay exact."""
    P = _pkg()
    case = make_case("delta", 256, (1 << 21) + 1, seed=9, kv=True)
    plan = P.Plan(P.BucketSpec(**case["spec_kw"]), len(case["keys"]), with_values=True)
    kd, vd = to_dev(case["keys"]), to_dev(case["vals"])
    exp = _expect(case)
    for _ in range(3):
        ko, vo, off = plan.run(kd, vd)
        assert np.array_equal(from_dev(ko), exp[0]) and np.array_equal(from_dev(vo), exp[1])


@pytest.mark.parametrize("kind,m,kv,dist", [("delta", 32, False, "uniform"), ("delta", 64, False, "binomial"),
                                          ("lowbits", 8, False, "hot"), ("ids", 32, False, "uniform"),
                                          ("splitters", 32, True, "binomial"), ("delta", 16, True, "uniform"),
                                          ("delta", 256, False, "uniform")])
def test_repeat_stress(kind, m, kv, dist):
    """Race canary (compute-sanitizer was closed on the pool for the round's last kernel changes):
    1000 back-to-back runs of the default path on one workspace -- the mbarrier / TMA stage reuse,
    the double-buffered phase 1, the grid barrier and the bulk-store drain all cycle many times per
    run at this size (~7 tiles per persistent CTA, an odd partial last tile) -- every output compared
    element-wise on the device with the oracle's."""
    P = _pkg()
    n = 296 * 8192 * 3 + 4097 if not kv else 296 * 4096 * 7 + 4097
    case = make_case(kind, m, n, seed=31 + m, kv=kv, dist=dist)
    plan = P.Plan(P.BucketSpec(**case["spec_kw"]), n, with_values=kv)
    kd, vd, idd = to_dev(case["keys"]), to_dev(case["vals"]), to_dev(case["ids"])
    eko, evo, eoff = _expect(case)
    ek, ev = to_dev(eko), to_dev(evo)
    eo = torch.as_tensor(eoff.astype(np.int64), device="cuda")
    bad = 0
    for _ in range(1000):
        ko, vo, off = plan.run(kd, vd, idd)
        bad += int(not torch.equal(ko, ek)) + int(kv and not torch.equal(vo, ev)) + \
            int(not torch.equal(off.to(torch.int64) & 0xFFFFFFFF, eo))
    torch.cuda.synchronize()
    assert bad == 0, f"{bad} mismatching outputs in 1000 runs"


@pytest.mark.parametrize("P", [1, 2, 3, 4, 8])
@pytest.mark.parametrize("kind,m", [("lowbits", 2), ("delta", 8), ("splitters", 32), ("delta", 5), ("lowbits", 1)])
def test_fused_scatter_virtual_ranks(P, kind, m):
    """Fused sharded scatter (ms_postscan_scatter) with P virtual ranks on one GPU:
    each shard's K3 writes its runs straight into all P windows; the windows concatenated must equal
    the oracle's stable multisplit of the concatenated shards.  Ragged shards (empty, < 1 tile,
    several tiles + tail), skewed buckets so window boundaries cut runs, KO and KV."""
    from paper_conf_ppopp_ashkianidmo16_b200.dist import scatter_multisplit_virtual
    rng = np.random.default_rng(1000 * P + m)
    for trial, dist in enumerate(["uniform", "hot", "binomial"]):
        sizes = [int(x) for x in rng.integers(0, 3 * 4096 + 77, size=P)]
        if trial == 1 and P > 1:
            sizes[0] = 0
        if trial == 2:
            sizes[-1] = 4097
        for kv in (False, True):
            case = make_case(kind, m, sum(sizes), seed=50 + trial + 10 * P, dist=dist if m > 1 else "uniform", kv=kv)
            P_ = _pkg()
            spec = P_.BucketSpec(**case["spec_kw"])
            cuts = np.concatenate([[0], np.cumsum(sizes)])
            ks = [to_dev(case["keys"][cuts[r]:cuts[r + 1]]) for r in range(P)]
            vs = [to_dev(case["vals"][cuts[r]:cuts[r + 1]]) for r in range(P)] if kv else None
            ko, vo = scatter_multisplit_virtual(ks, vs, spec)
            eko, evo, _ = _expect(case)
            what = f"P={P} {kind} m={m} {dist} sizes={sizes} kv={kv}"
            assert np.array_equal(from_dev(ko), eko), what
            if kv:
                assert np.array_equal(from_dev(vo), evo), what


@pytest.mark.parametrize("kv", [False, True])
def test_fused_scatter_virtual_large(kv):
    """C5-shaped (splitters m = 32, uniform) at 2^26 keys over 4 virtual ranks, full compare."""
    from paper_conf_ppopp_ashkianidmo16_b200.dist import scatter_multisplit_virtual
    n, P = 1 << 26, 4
    case = make_case("splitters", 32, n, seed=W.SEEDS["C3"], kv=kv, vals_kind="random")
    spec = _pkg().BucketSpec(**case["spec_kw"])
    q = n // P
    ks = [to_dev(case["keys"][r * q:(r + 1) * q]) for r in range(P)]
    vs = [to_dev(case["vals"][r * q:(r + 1) * q]) for r in range(P)] if kv else None
    ko, vo = scatter_multisplit_virtual(ks, vs, spec)
    eko, evo, _ = _expect(case)
    assert np.array_equal(from_dev(ko), eko)
    if kv:
        assert np.array_equal(from_dev(vo), evo)


def test_fused_scatter_rejects_unsupported():
    """m > 32 or precomputed ids: the fused scatter is K3 v2 only (MS_ERR_UNSUPPORTED)."""
    from paper_conf_ppopp_ashkianidmo16_b200 import _abi
    from paper_conf_ppopp_ashkianidmo16_b200.dist import scatter_target
    P_ = _pkg()
    keys = torch.zeros(4096, dtype=torch.int32, device="cuda")
    out = torch.empty_like(keys)
    for spec in (P_.BucketSpec.delta_range(64, 1 << 26), P_.BucketSpec.precomputed(8, 1)):
        plan = P_.Plan(spec, 4096, variant="3k")
        t = scatter_target([out.data_ptr()], None, [0, 4096], [0] * 32)
        G = torch.zeros(spec.m, dtype=torch.int32, device="cuda")
        with pytest.raises(_abi.MultisplitError) as e:
            plan.postscan_scatter(keys, G, t)
        assert e.value.status == _abi.MS_ERR_UNSUPPORTED


@pytest.mark.parametrize("m", [2, 8, 32])
def test_parity_direct_ablation(m):
    """The Direct (no local reorder) K3 ablation, MS_ABLATION_DIRECT (SHIFT bucket kind: DELTA with
    m * delta = 2^32), bit-exact on ragged sizes, KO and KV (3 launches: K1, K2, Direct K3)."""
    for i, n in enumerate([1, 4095, 4097, 100003, (1 << 21) + 3]):
        for kv in (False, True):
            case = make_case("delta", m, n, seed=2 * (400 + i), kv=kv)  # even seed: delta = 2^32 / m
            assert case["spec_kw"]["delta"] == (1 << 32) // m
            _assert_equal(case, _run_case(case, "direct"), _expect(case), f"direct m={m} n={n} kv={kv}")


@pytest.mark.parametrize("variant", ["ballot", "warp"])
@pytest.mark.parametrize("m", [2, 8, 16, 32, 64, 128, 256])
def test_parity_ballot_warp_ablations(variant, m):
    """The ballot post-scan (Alg. 3 ranks) at any m with block-level (MS_ABLATION_BALLOT) or the
    paper's warp-level reorder (MS_ABLATION_WARP, §5.2.1: every warp reorders and stores its own
    512-key segment), bit-exact on ragged sizes (2048- and 4096-key tiles, partial last tiles,
    partly filled warp segments), uniform and skewed buckets, KO and KV (3 launches)."""
    for i, n in enumerate([1, 31, 513, 4095, 4097, 100003, 297 * 4096 + 1, (1 << 22) + 3]):
        for kv in (False, True):
            dist = ("uniform", "binomial", "hot")[i % 3]
            case = make_case("delta", m, n, seed=2 * (700 + i), kv=kv, dist=dist)
            assert case["spec_kw"]["delta"] == (1 << 32) // m  # even seed: the SHIFT kind
            _assert_equal(case, _run_case(case, variant), _expect(case), f"{variant} m={m} n={n} kv={kv}")


# ---------------------------------------------------------------- m > 256
WIDE = [("lowbits", 512, dict(shift=0)), ("lowbits", 65536, dict(shift=7)), ("lowbits", 1024, dict(shift=22)),
        ("delta", 300, dict(delta=1 << 20)),        # power of two, m * delta < 2^32: clamped (SHIFTC_LO + B)
        ("delta", 1000, dict(delta=1 << 22)),
        ("delta", 4096, dict(delta=1 << 20)),       # m * delta = 2^32: a bit field (LOWBITS passes)
        ("delta", 65536, dict(delta=1 << 16)),
        ("delta", 777, dict(delta=5000003)),        # magic division (DELTA_LO + DELTA)
        ("delta", 3000, dict(delta=123457)),        # far pile holds most keys
        ("delta", 65535, dict(delta=3)),
        ("delta", 400, dict(delta=400000000)),      # high digit always 0: one pass + offsets
        ("ids", 257, dict(id_bytes=4)), ("ids", 5000, dict(id_bytes=4)), ("ids", 65536, dict(id_bytes=4))]


def _wide_case(kind, m, kw, n, seed, kv, dist="uniform"):
    ospec = oracle.Spec(kind, m, shift=kw.get("shift", 0), delta=kw.get("delta", 1), id_bytes=kw.get("id_bytes", 1))
    ids = None
    if kind == "ids":
        keys = W.keys_np(n, seed)
        ids = W.bucket_draw_np(n, seed, "buckets" if dist == "uniform" else dist, m).astype(np.uint32)
    elif kind == "delta" and dist != "uniform":
        keys = W.keys_np(n, seed, dist, m, W.ranges_delta(m, kw["delta"]))
    else:
        keys = W.keys_np(n, seed)
    vals = W.values_np(n, seed, "index") if kv else None
    return dict(spec_kw=dict(kind=kind, m=m, **kw), ospec=ospec, keys=keys, vals=vals, ids=ids)


@pytest.mark.parametrize("kind,m,kw", WIDE)
def test_parity_wide(kind, m, kw):
    """m in (256, 65536]: two stable passes (low digit, high digit) + offsets from the sorted output,
    bit-exact vs the oracle on ragged sizes, KO and KV, uniform and skewed."""
    for i, n in enumerate([0, 1, 31, 4095, 100003, (1 << 20) + 7]):
        for kv in (False, True):
            for dist in (["uniform", "binomial", "hot"] if (kind != "lowbits" and n > 4095) else ["uniform"]):
                case = _wide_case(kind, m, kw, n, seed=31 * m + i, kv=kv, dist=dist)
                got = _run_case(case)
                _assert_equal(case, got, _expect(case), f"wide {kind} m={m} {kw} n={n} kv={kv} {dist}")
                assert got[3].geometry(max(n, 1))[2] == 3


@pytest.mark.parametrize("kind,m,kw,n,kv", [("delta", 65536, dict(delta=1 << 16), 1 << 28, False),
                                            ("delta", 4096, dict(delta=1 << 20), (1 << 26) + 3, True),
                                            ("delta", 1000, dict(delta=4000037), 1 << 26, False),
                                            ("ids", 4096, dict(id_bytes=4), (1 << 25) + 1, True)])
def test_parity_wide_large(kind, m, kw, n, kv):
    """m > 256 at up to 2^28 keys, full compare (the Fig. 4-style sweep's sizes)."""
    case = _wide_case(kind, m, kw, n, seed=4242, kv=kv)
    _assert_equal(case, _run_case(case), _expect(case), f"wide {kind} m={m} n={n}")


def test_wide_validate_flags_out_of_range_ids():
    P = _pkg()
    n, m = 100000, 1000
    ids = W.bucket_draw_np(n, 3, "buckets", m).astype(np.uint32)
    keys = W.keys_np(n, 3)
    plan = P.Plan(P.BucketSpec.precomputed(m, 4), n, validate=True)
    plan.run(to_dev(keys), ids=to_dev(ids))
    assert plan.check() == 0
    bad = ids.copy()
    bad[12345] = 1000
    plan.run(to_dev(keys), ids=to_dev(bad))
    assert plan.check() == -8
@pytest.mark.parametrize("variant", ["nw2", "nw4"])
@pytest.mark.parametrize("m", [2, 4, 8, 16, 32])
def test_parity_nw_ablation(variant, m):
    """The NW sweep ablation (MS_ABLATION_NW2 / NW4: 2 or 4 warps per post-scan CTA, T = 1024 / 2048,
    the local reorder spanning fewer warps; ranged variant, 2 launches), bit-exact on ragged sizes
    around the range boundaries, KO and KV."""
    sms = torch.cuda.get_device_properties(0).multi_processor_count
    T = 1024 if variant == "nw2" else 2048
    for i, n in enumerate([1, T - 1, T + 1, 100003, 37 * sms * T + 11, (1 << 22) + 3]):
        for kv in (False, True):
            case = make_case("delta", m, n, seed=2 * (600 + i), kv=kv, dist="binomial" if i % 2 else "uniform")
            assert case["spec_kw"]["delta"] == (1 << 32) // m  # even seed: the SHIFT kind
            got = _run_case(case, variant)
            assert got[3].geometry(n)[0] == T
            _assert_equal(case, got, _expect(case), f"{variant} m={m} n={n} kv={kv}")


# ---------------------------------------------------------------- the largest sizes (n up to 2^32 - 5)
def _torch_ids(keys_i32, kind, m, spl=None, delta=None):
    k = keys_i32.to(torch.int64) & 0xFFFFFFFF
    if kind == "delta":
        return torch.clamp(k // delta, max=m - 1)
    return torch.searchsorted(torch.as_tensor(spl.astype(np.int64), device=keys_i32.device), k, side="left")


def test_max_size_kv_vs_definition():
    """n = 2^31 + 7 key-value pairs (C5's total on one GPU, m = 32 splitters), the whole output
    element for element against the definition evaluated independently with torch on the GPU:
    bucket j of the output must be exactly the input's elements with id j, in input order
    (Eq. (1)) -- built chunk by chunk with boolean selection (torch's sort stops at
    2^31 elements) -- and the offsets the exclusive scan of the id histogram."""
    P = _pkg()
    n, m = (1 << 31) + 7, 32
    spl = W.gen_splitters(m, W.SEEDS["C5"])
    keys = W.keys_torch(n, W.SEEDS["C5"], "cuda")
    vals = W.values_torch(n, W.SEEDS["C5"], "cuda", "random")
    plan = P.Plan(P.BucketSpec.from_splitters(spl.tolist()), n, with_values=True)
    ko, vo, off = plan.run(keys, vals)
    torch.cuda.synchronize()
    assert plan.last_launches() == 3 - (plan.geometry(n)[2])  # ranged (2) at this size
    ids = _torch_ids(keys, "splitters", m, spl=spl).to(torch.uint8)
    hist = torch.bincount(ids, minlength=m).to(torch.int64)
    exp_off = torch.cat([torch.zeros(1, dtype=torch.int64, device="cuda"), torch.cumsum(hist, 0)])
    assert torch.equal(off.to(torch.int64) & 0xFFFFFFFF, exp_off)
    cursor = exp_off[:-1].clone()
    C = 1 << 28
    for c in range(0, n, C):
        idc, kc, vc = ids[c:c + C], keys[c:c + C], vals[c:c + C]
        for j in range(m):
            sel = idc == j
            ek, ev = kc[sel], vc[sel]
            a = int(cursor[j])
            assert torch.equal(ko[a:a + ek.numel()], ek), f"keys of bucket {j}, input chunk {c}"
            assert torch.equal(vo[a:a + ev.numel()], ev), f"values of bucket {j}, input chunk {c}"
            cursor[j] += ek.numel()
    assert torch.equal(cursor, exp_off[1:])


@pytest.mark.parametrize("m", [8, 32])
def test_max_size_ko_properties(m):
    """n = 2^32 - 5 keys (the largest n the ABI takes), key-only, m = 8 / 32 delta (one ONE launch,
    tiles of 4096 / 8192 keys; either way > 1024 tiles per CTA, so ONE's counter folding runs): the
    output is the same multiset as the input (order-insensitive 64-bit hashes), its bucket ids never
    decrease, and the offsets are exactly the id boundaries (for key-only output, equal keys are
    interchangeable, so these properties determine the result)."""
    P = _pkg()
    n, delta = (1 << 32) - 5, (1 << 32) // m
    keys = W.keys_torch(n, 424242, "cuda")
    plan = P.Plan(P.BucketSpec.delta_range(m, delta), n)
    ko, _, off = plan.run(keys)
    torch.cuda.synchronize()
    assert plan.last_launches() == 1

    def mh(t):  # order-insensitive multiset hash of u32 values: sum of a mixing function, mod 2^64
        h = 0
        for c in range(0, t.numel(), 1 << 28):
            x = t[c:c + (1 << 28)].to(torch.int64) & 0xFFFFFFFF
            x = (x ^ (x >> 16)) * 0x45D9F3B
            x = (x ^ (x >> 13)) * 0x2C1B3C6D
            h = (h + int(x.sum())) & ((1 << 64) - 1)
        return h
    assert mh(ko) == mh(keys)
    offh = (off.to(torch.int64) & 0xFFFFFFFF).tolist()
    assert offh[0] == 0 and offh[m] == n and all(a <= b for a, b in zip(offh, offh[1:]))
    for j in range(m):  # every position in [off[j], off[j+1]) has id j (checked chunk-wise)
        for c in range(offh[j], offh[j + 1], 1 << 28):
            seg = ko[c:min(c + (1 << 28), offh[j + 1])]
            ids = _torch_ids(seg, "delta", m, delta=delta)
            assert bool((ids == j).all()), f"bucket {j} chunk at {c}"


@pytest.mark.parametrize("kind,m,kv,n", [("lowbits", 2, False, 1 << 20), ("splitters", 32, True, 100003),
                                         ("delta", 256, False, 50000), ("delta", 1000, True, 70001)])
def test_cuda_graph_capture(kind, m, kv, n):
    """ms_run is stream-ordered with no host synchronisation, so it can be captured in a CUDA graph
    (ONE's cooperative launch, the 3-kernel path and the two-pass plan alike) and replayed: the
    replayed output equals the oracle's."""
    P = _pkg()
    if m > 256:
        case = _wide_case(kind, m, dict(delta=4000037), n, seed=5, kv=kv)
    else:
        case = make_case(kind, m, n, seed=5, kv=kv)
    plan = P.Plan(P.BucketSpec(**case["spec_kw"]), n, with_values=kv)
    kd, vd = to_dev(case["keys"]), to_dev(case["vals"])
    ko, vo = torch.empty_like(kd), (torch.empty_like(vd) if kv else None)
    off = torch.empty(m + 1, dtype=torch.int32, device="cuda")
    ws = plan.workspace(n)
    s = torch.cuda.Stream()
    s.wait_stream(torch.cuda.current_stream())
    with torch.cuda.stream(s):
        plan.run(kd, vd, keys_out=ko, vals_out=vo, offsets=off, workspace=ws)
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=s):
        plan.run(kd, vd, keys_out=ko, vals_out=vo, offsets=off, workspace=ws)
    ko.fill_(0)
    g.replay()
    torch.cuda.synchronize()
    _assert_equal(case, (from_dev(ko), from_dev(vo), from_dev(off), plan), _expect(case), f"graph {kind} m={m}")
