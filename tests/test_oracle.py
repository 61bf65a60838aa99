"""Pins for the CPU oracle (runs on CPU; no GPU).

Each test checks the oracle against something other than itself: the paper's
printed worked example (Fig. 1), brute force over every id sequence, a
different algorithm (Python's stable sort / numpy's stable argsort), closed
forms, invariants and special cases that reduce to sort / partition.
PAPER.md line citations are "P:<line>".
"""
import bisect
import collections
import itertools
import os
import random

import numpy as np
import pytest

import oracle
from oracle import warp_sim

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def _golden(name):
    d = {}
    with open(os.path.join(GOLD, name)) as f:
        for line in f:
            line = line.strip()
            if not line or line.startswith("#"):
                continue
            k, v = line.split(":", 1)
            d[k.strip()] = v.split()
    return d


def _is_prime(k):
    return k > 1 and all(k % d for d in range(2, int(k ** 0.5) + 1))


# ---------------------------------------------------------------- Fig. 1
def test_fig1_row1_prime_composite():
    """Fig. 1(1): stable multisplit, B0 = prime, B1 = composite."""
    g = _golden("fig1.txt")
    keys = np.array([int(x) for x in g["input"]], dtype=np.uint32)
    ids = np.array([0 if _is_prime(int(k)) else 1 for k in keys], dtype=np.uint8)
    ko, _, off = oracle.multisplit(oracle.Spec("ids", 2, id_bytes=1), keys, ids=ids)
    assert ko.tolist() == [int(x) for x in g["row1"]]
    assert off.tolist() == [0, 4, 8]


def test_fig1_row2_range_buckets():
    """Fig. 1(2): three range buckets {i<=20}, {20<i<=48}, {i>48} (reading #9 tie rule)."""
    g = _golden("fig1.txt")
    keys = np.array([int(x) for x in g["input"]], dtype=np.uint32)
    spl = [int(x) for x in g["row2_splitters"]]
    ko, _, off = oracle.multisplit(oracle.Spec("splitters", 3, splitters=spl), keys)
    for b in range(3):
        got = sorted(ko[off[b]:off[b + 1]].tolist())
        assert got == sorted(int(x) for x in g[f"row2_bucket{b}"])
    # a key equal to a splitter belongs to the lower bucket (B0 = {i <= 20})
    ko2, _, off2 = oracle.multisplit(oracle.Spec("splitters", 3, splitters=spl),
                                     np.array([20, 21, 48, 49], dtype=np.uint32))
    assert off2.tolist() == [0, 1, 3, 4]


def test_fig1_row3_sort_based():
    """Fig. 1(3): with one bucket per distinct key (ordered buckets) multisplit is a sort."""
    g = _golden("fig1.txt")
    keys = np.array([int(x) for x in g["input"]], dtype=np.uint32)
    spl = sorted(keys.tolist())[:-1]
    ko, _, _ = oracle.multisplit(oracle.Spec("splitters", len(keys), splitters=spl), keys)
    assert ko.tolist() == [int(x) for x in g["row3"]]


# ---------------------------------------------------------------- brute force
def _brute(keys, vals, ids, m):
    """Different algorithm: Python's (stable) sorted() of indices by id."""
    idx = sorted(range(len(ids)), key=lambda i: ids[i])
    cnt = collections.Counter(ids)
    off = [0]
    for b in range(m):
        off.append(off[-1] + cnt.get(b, 0))
    return [keys[i] for i in idx], [vals[i] for i in idx], off


@pytest.mark.parametrize("m", [1, 2, 3])
def test_bruteforce_all_id_sequences(m):
    """Every id sequence with n <= 7 (m <= 3): oracle == stable sort by id (A12, Eq. 1)."""
    spec = oracle.Spec("ids", m, id_bytes=1)
    for n in range(0, 8):
        keys = np.arange(100, 100 + n, dtype=np.uint32)
        vals = np.arange(n, dtype=np.uint32)
        for seq in itertools.product(range(m), repeat=n):
            ids = np.array(seq, dtype=np.uint8)
            ko, vo, off = oracle.multisplit(spec, keys, vals, ids=ids)
            bk, bv, boff = _brute(keys.tolist(), vals.tolist(), list(seq), m)
            assert ko.tolist() == bk and vo.tolist() == bv and off.tolist() == boff


def _py_ids(kind, m, keys, shift=0, delta=1, spl=None):
    """Bucket ids from the plain formulas, in Python integers (independent of oracle.c)."""
    if kind == "lowbits":
        return [(k >> shift) & (m - 1) for k in keys]
    if kind == "delta":
        return [min(k // delta, m - 1) for k in keys]
    if kind == "splitters":
        return [sum(1 for s in spl if s < k) for k in keys]
    raise ValueError(kind)


@pytest.mark.parametrize("kind", ["lowbits", "delta", "splitters", "ids"])
def test_random_vs_stable_argsort(kind):
    rng = random.Random(1234 + len(kind))
    for trial in range(60):
        m = rng.choice([1, 2, 3, 5, 8, 31, 32, 33, 64, 127, 255, 256])
        if kind == "lowbits":
            m = 1 << rng.randrange(0, 9)
        n = rng.choice([0, 1, 31, 32, 33, 1000, 4096, 4097])
        keys = np.array([rng.getrandbits(32) for _ in range(n)], dtype=np.uint32)
        vals = np.arange(n, dtype=np.uint32)
        ids = None
        if kind == "lowbits":
            shift = rng.randrange(0, 33 - max(1, (m - 1).bit_length()))
            spec = oracle.Spec(kind, m, shift=shift)
            pid = _py_ids(kind, m, keys.tolist(), shift=shift)
        elif kind == "delta":
            delta = rng.choice([1, 3, 7, 1 << 24, 400000000, rng.getrandbits(32) or 1, 0xFFFFFFFF])
            spec = oracle.Spec(kind, m, delta=delta)
            pid = _py_ids(kind, m, keys.tolist(), delta=delta)
        elif kind == "splitters":
            spl = sorted(rng.getrandbits(32) for _ in range(m - 1))
            if m > 3 and trial % 3 == 0:   # duplicates -> empty buckets
                spl[1] = spl[2]
                spl = sorted(spl)
            spec = oracle.Spec(kind, m, splitters=spl)
            pid = [bisect.bisect_left(spl, k) for k in keys.tolist()]
        else:
            ib = 1 if m <= 256 and trial % 2 == 0 else 4
            spec = oracle.Spec(kind, m, id_bytes=ib)
            pid = [rng.randrange(m) for _ in range(n)]
            ids = np.array(pid, dtype=np.uint8 if ib == 1 else np.uint32)
        ko, vo, off = oracle.multisplit(spec, keys, vals, ids=ids)
        order = np.argsort(np.array(pid, dtype=np.int64), kind="stable")
        assert np.array_equal(vo, order.astype(np.uint32))
        assert np.array_equal(ko, keys[order])
        cnt = np.bincount(np.array(pid, dtype=np.int64), minlength=m)
        assert off.tolist() == [0] + np.cumsum(cnt).tolist()


def test_splitters_linear_count():
    """Splitter kind vs the plain linear count #{j : s_j < k}, incl. duplicates and edges."""
    rng = random.Random(7)
    for m in [2, 3, 17, 32, 256]:
        spl = sorted(rng.getrandbits(32) for _ in range(m - 1))
        if m > 2:
            spl[0] = spl[1]
        keys = [0, 1, 0xFFFFFFFF, 0xFFFFFFFE] + spl + [s + 1 for s in spl if s < 0xFFFFFFFF] + \
               [rng.getrandbits(32) for _ in range(500)]
        got = oracle.bucket_ids(oracle.Spec("splitters", m, splitters=spl), np.array(keys, dtype=np.uint32))
        assert got.tolist() == _py_ids("splitters", m, keys, spl=spl)


@pytest.mark.parametrize("delta", [1, 3, 7, 400000000, 1 << 24, 0xFFFFFFFF])
def test_delta_closed_form_edges(delta):
    """DELTA kind vs floor division at bucket edges (reading #8: clamp to m-1)."""
    for m in [1, 2, 8, 256]:
        keys = {0, 1, 0xFFFFFFFF, 0xFFFFFFFE}
        for b in range(0, 300):
            for d in (-1, 0, 1):
                v = b * delta + d
                if 0 <= v <= 0xFFFFFFFF:
                    keys.add(v)
        keys = sorted(keys)
        got = oracle.bucket_ids(oracle.Spec("delta", m, delta=delta), np.array(keys, dtype=np.uint32))
        assert got.tolist() == [min(k // delta, m - 1) for k in keys]


def test_out_of_range_id_rejected():
    with pytest.raises(ValueError):
        oracle.multisplit(oracle.Spec("ids", 4, id_bytes=1), np.zeros(3, np.uint32),
                          ids=np.array([0, 4, 1], np.uint8))


# ---------------------------------------------------------------- invariants
@pytest.mark.parametrize("kind,m", [("delta", 8), ("splitters", 32), ("lowbits", 256), ("delta", 256),
                                    ("delta", 1000), ("lowbits", 4096), ("splitters", 700)])
def test_invariants_large(kind, m):
    """Permutation, id order, stability, offsets (BJ north_star invariants) at n = 2^16 + 5."""
    import workloads
    n = (1 << 16) + 5
    keys = workloads.keys_np(n, 99)
    vals = np.arange(n, dtype=np.uint32)
    spl = workloads.gen_splitters(m, 5) if kind == "splitters" else None
    spec = oracle.Spec(kind, m, shift=3, delta=(1 << 32) // m, splitters=spl)
    ko, vo, off = oracle.multisplit(spec, keys, vals)
    assert np.array_equal(np.sort(vo), vals)                  # bijection
    assert np.array_equal(ko, keys[vo])                       # keys travel with values
    ido = oracle.bucket_ids(spec, ko)
    assert np.all(np.diff(ido.astype(np.int64)) >= 0)         # ascending bucket ids
    for b in range(m):                                        # stable: input order kept in-bucket
        seg = vo[off[b]:off[b + 1]].astype(np.int64)
        assert np.all(np.diff(seg) > 0)
        assert np.all(ido[off[b]:off[b + 1]] == b)
    hist = np.bincount(oracle.bucket_ids(spec, keys), minlength=m)
    assert off.tolist() == [0] + np.cumsum(hist).tolist()     # offsets = exclusive scan of histogram


# ---------------------------------------------------------------- reductions
def test_identity_buckets_is_stable_sort():
    """Identity buckets B_i = {i}: multisplit == stable sort of keys in [0, m)."""
    rng = np.random.default_rng(3)
    for m in [2, 7, 32, 256, 257, 4096, 65536]:   # m > 256: SURVEY NEXT-3
        keys = rng.integers(0, m, size=5000).astype(np.uint32)
        vals = np.arange(5000, dtype=np.uint32)
        ko, vo, _ = oracle.multisplit(oracle.Spec("delta", m, delta=1), keys, vals)
        assert np.array_equal(ko, np.sort(keys))
        assert np.array_equal(vo, np.argsort(keys, kind="stable").astype(np.uint32))


def test_two_lowbit_buckets_is_stable_partition():
    """m = 2 low-bit buckets == the split / stable partition."""
    rng = random.Random(11)
    keys = [rng.getrandbits(32) for _ in range(3001)]
    ko, _, off = oracle.multisplit(oracle.Spec("lowbits", 2), np.array(keys, np.uint32))
    evens = [k for k in keys if k % 2 == 0]
    odds = [k for k in keys if k % 2 == 1]
    assert ko.tolist() == evens + odds and off.tolist() == [0, len(evens), len(keys)]


def test_range_buckets_match_sorted_segments():
    """Ordered range buckets: each bucket's multiset == the matching segment of sorted(keys)."""
    import workloads
    keys = workloads.keys_np(20000, 17)
    spl = workloads.gen_splitters(32, 17)
    ko, _, off = oracle.multisplit(oracle.Spec("splitters", 32, splitters=spl), keys)
    srt = np.sort(keys)
    for b in range(32):
        assert np.array_equal(np.sort(ko[off[b]:off[b + 1]]), srt[off[b]:off[b + 1]])


# ---------------------------------------------------------------- Eq. (2)
@pytest.mark.parametrize("T", [1, 32, 100, 4096])
def test_eq2_matrices_and_positions(T):
    """H and G of Eq. (2): G == exclusive scan of row-vectorised H, G[:,0] == offsets,
    and G[j][l] + local offset reproduces every output position of Eq. (1)."""
    rng = np.random.default_rng(T)
    m, n = 13, 5000 + T
    ids = rng.integers(0, m, size=n).astype(np.uint32)
    H, G = oracle.tile_matrices(ids, m, T)
    L = H.shape[1]
    assert L == (n + T - 1) // T
    hrow = H.reshape(-1).astype(np.int64)
    assert np.array_equal(G.reshape(-1).astype(np.int64), np.concatenate([[0], np.cumsum(hrow)[:-1]]))
    _, vo, off = oracle.multisplit(oracle.Spec("ids", m, id_bytes=4), np.zeros(n, np.uint32),
                                   np.arange(n, dtype=np.uint32), ids=ids)
    assert np.array_equal(G[:, 0].astype(np.uint64), off[:-1])
    pos = np.empty(n, dtype=np.int64)
    pos[vo.astype(np.int64)] = np.arange(n)
    seen = collections.Counter()
    for i in range(n):                                           # term 3: local offset in subproblem
        l, j = i // T, int(ids[i])
        assert pos[i] == int(G[j, l]) + seen[(j, l)]
        seen[(j, l)] += 1


# ---------------------------------------------------------------- Alg. 2 / Alg. 3
def test_warp_histogram_alg2():
    """Alg. 2: histo[i] = count of bucket i for lanes i < m (reading #5 for m not 2^k)."""
    rng = random.Random(5)
    for _ in range(400):
        m = rng.randint(1, 32)
        ids = [rng.randrange(m) for _ in range(32)]
        h = warp_sim.warp_histogram(ids, m)
        c = collections.Counter(ids)
        assert [h[i] for i in range(m)] == [c.get(i, 0) for i in range(m)]


def test_warp_offsets_alg3_reading4():
    """Alg. 3: the printed mask yields exclusive+1; the corrected mask the exclusive rank."""
    rng = random.Random(6)
    for _ in range(400):
        m = rng.randint(1, 32)
        ids = [rng.randrange(m) for _ in range(32)]
        excl = [sum(1 for r in range(i) if ids[r] == ids[i]) for i in range(32)]
        assert warp_sim.warp_offsets_exclusive(ids, m) == excl
        assert warp_sim.warp_offsets_printed(ids, m) == [e + 1 for e in excl]


# ---------------------------------------------------------------- speed of light
def test_speed_of_light_byte_model():
    """§6.2.2: 3 / 5 four-byte accesses per key give 24 / 14.4 G keys/s at 288 GB/s;
    the bench's byte model must reproduce the paper's arithmetic."""
    from paper_conf_ppopp_ashkianidmo16_b200 import model
    g = _golden("speed_of_light.txt")
    bw = float(g["bandwidth_GBps"][0])
    assert model.algorithmic_bytes_per_key(False) == 4 * int(g["accesses_key_only"][0])
    assert model.algorithmic_bytes_per_key(True) == 4 * int(g["accesses_key_value"][0])
    assert bw / model.algorithmic_bytes_per_key(False) == pytest.approx(float(g["sol_key_only_Gkeys"][0]))
    assert bw / model.algorithmic_bytes_per_key(True) == pytest.approx(float(g["sol_key_value_Gkeys"][0]))
