"""Seeded synthetic inputs for the multisplit tests and bench.

This module is shared scaffolding: both the oracle side (tests) and the CUDA
side (tests, bench) draw their inputs from here, and it holds none of the
method's arithmetic (it never maps a key to a bucket id, counts, scans or
permutes).  Where a distribution is defined over buckets, it draws the bucket
b first and then a key inside a key range the *caller* states for b (the
inverse direction of the bucket function), which is the input recipe of
SURVEY.md §8(d) / DESIGN.md "Input recipe".

Generator: counter-based splitmix64 finaliser, so every value depends only on
(seed, stream, i) and the numpy (host) and torch (device) twins produce
identical arrays:

    r64(seed, stream, i) = fmix(seed ^ (stream << 56) ^ ((i + 1) * PHI))
    fmix(z): z = (z ^ z>>30) * C1; z = (z ^ z>>27) * C2; return z ^ z>>31

Distributions of the paper's workloads (§6.1 P:1366-1369 uniform keys
over equal-width buckets; §6.5 P:2147-2170 binomial B(m-1, 1/2) and
"25 % uniform, the rest in one bucket"):

* ``uniform``   keys uniform over uint32 (hi 32 bits of stream 0).
* ``buckets``   b uniform over [0, m), then key uniform in range(b).
* ``binomial``  b = popcount of (m-1) random bits (exactly B(m-1, 1/2)).
* ``hot``       with prob 3/4 b = m // 2, else b uniform; key uniform in range(b).
* ``one``       every key in bucket m // 2 (degenerate case: one non-empty bucket).
"""
from __future__ import annotations

import numpy as np

PHI = 0x9E3779B97F4A7C15
C1 = 0xBF58476D1CE4E5B9
C2 = 0x94D049BB133111EB
M64 = (1 << 64) - 1

# stream ids
S_KEY, S_VAL, S_BUCKET, S_POS, S_BINOM = 0, 1, 2, 3, 8

SEEDS = {  # SURVEY.md §8(d) per-config seeds
    "C1": 0x4D530001, "C2": 0x4D530002, "C3": 0x4D530003,
    "C4": 0x4D530004, "C5": 0x4D530005,
}


# ----------------------------------------------------------------- numpy twin
def r64_np(seed: int, stream: int, start: int, n: int) -> np.ndarray:
    """uint64 random words for indices start..start+n-1 (numpy, host)."""
    with np.errstate(over="ignore"):
        i = np.arange(start + 1, start + n + 1, dtype=np.uint64)
        z = i * np.uint64(PHI)
        z ^= np.uint64(((seed & M64) ^ ((stream & 0xFF) << 56)) & M64)
        z = (z ^ (z >> np.uint64(30))) * np.uint64(C1)
        z = (z ^ (z >> np.uint64(27))) * np.uint64(C2)
        z ^= z >> np.uint64(31)
    return z


def u32_np(seed: int, stream: int, start: int, n: int) -> np.ndarray:
    return (r64_np(seed, stream, start, n) >> np.uint64(32)).astype(np.uint32)


def uniform_in_np(r32: np.ndarray, lo: np.ndarray, hi: np.ndarray) -> np.ndarray:
    """lo + floor(r32 * (hi - lo + 1) / 2^32): a value in [lo, hi] (inclusive)."""
    width = hi.astype(np.uint64) - lo.astype(np.uint64) + np.uint64(1)
    return (lo.astype(np.uint64) + ((r32.astype(np.uint64) * width) >> np.uint64(32))).astype(np.uint32)


def draw_buckets_np(dist: str, m: int, seed: int, start: int, n: int) -> np.ndarray:
    """Bucket indices (uint32) drawn from a bucket-level distribution."""
    if dist == "buckets":
        r = u32_np(seed, S_BUCKET, start, n).astype(np.uint64)
        return ((r * np.uint64(m)) >> np.uint64(32)).astype(np.uint32)
    if dist == "binomial":
        b = np.zeros(n, dtype=np.uint32)
        bits_left, word = m - 1, 0
        while bits_left > 0:
            take = min(64, bits_left)
            r = r64_np(seed, S_BINOM + word, start, n)
            if take < 64:
                r &= np.uint64((1 << take) - 1)
            b += np.bitwise_count(r).astype(np.uint32)
            bits_left -= take
            word += 1
        return b
    if dist == "hot":
        r = r64_np(seed, S_BUCKET, start, n)
        hot = (r & np.uint64(3)) != 0
        u = ((((r >> np.uint64(32)) * np.uint64(m)) >> np.uint64(32))).astype(np.uint32)
        return np.where(hot, np.uint32(m // 2), u).astype(np.uint32)
    if dist == "one":
        return np.full(n, m // 2, dtype=np.uint32)
    raise ValueError(dist)


# ----------------------------------------------------------------- torch twin
def _i64(x: int) -> int:
    x &= M64
    return x - (1 << 64) if x >= (1 << 63) else x


def _srl(t, k: int):
    import torch
    return torch.bitwise_and(torch.bitwise_right_shift(t, k), _i64((1 << (64 - k)) - 1))


def r64_torch(seed: int, stream: int, start: int, n: int, device):
    """Same words as r64_np, as int64 tensor (two's complement) on `device`."""
    import torch
    i = torch.arange(start + 1, start + n + 1, dtype=torch.int64, device=device)
    z = i * _i64(PHI)
    z ^= _i64((seed & M64) ^ ((stream & 0xFF) << 56))
    z = (z ^ _srl(z, 30)) * _i64(C1)
    z = (z ^ _srl(z, 27)) * _i64(C2)
    z = z ^ _srl(z, 31)
    return z


def u32_torch(seed, stream, start, n, device):
    """uint32 values as int64 tensor in [0, 2^32)."""
    return _srl(r64_torch(seed, stream, start, n, device), 32)


def _popcount64_torch(x):
    import torch
    # SWAR popcount on int64 with logical shifts
    x = x - torch.bitwise_and(_srl(x, 1), _i64(0x5555555555555555))
    x = torch.bitwise_and(x, _i64(0x3333333333333333)) + torch.bitwise_and(_srl(x, 2), _i64(0x3333333333333333))
    x = torch.bitwise_and(x + _srl(x, 4), _i64(0x0F0F0F0F0F0F0F0F))
    return _srl(x * _i64(0x0101010101010101), 56)


def draw_buckets_torch(dist, m, seed, start, n, device):
    import torch
    if dist == "buckets":
        return (u32_torch(seed, S_BUCKET, start, n, device) * m) >> 32
    if dist == "binomial":
        b = torch.zeros(n, dtype=torch.int64, device=device)
        bits_left, word = m - 1, 0
        while bits_left > 0:
            take = min(64, bits_left)
            r = r64_torch(seed, S_BINOM + word, start, n, device)
            if take < 64:
                r = torch.bitwise_and(r, (1 << take) - 1)
            b += _popcount64_torch(r)
            bits_left -= take
            word += 1
        return b
    if dist == "hot":
        r = r64_torch(seed, S_BUCKET, start, n, device)
        hot = torch.bitwise_and(r, 3) != 0
        u = (_srl(r, 32) * m) >> 32
        return torch.where(hot, torch.full_like(u, m // 2), u)
    if dist == "one":
        return torch.full((n,), m // 2, dtype=torch.int64, device=device)
    raise ValueError(dist)


def _as_u32_tensor(t64):
    """int64 tensor holding values in [0, 2^32) -> int32 tensor with the same bits."""
    import torch
    return (t64 - ((t64 >> 31) << 32)).to(torch.int32) if t64.numel() else t64.to(torch.int32)


# ------------------------------------------------------------ key recipes
class KeyRanges:
    """Per-bucket key ranges [lo[b], hi[b]] for bucket-targeted draws (numpy uint32)."""

    def __init__(self, lo, hi):
        self.lo = np.asarray(lo, dtype=np.uint32)
        self.hi = np.asarray(hi, dtype=np.uint32)


def ranges_delta(m: int, delta: int) -> KeyRanges:
    lo = [min(b * delta, 0xFFFFFFFF) for b in range(m)]
    hi = [min((b + 1) * delta - 1, 0xFFFFFFFF) for b in range(m - 1)] + [0xFFFFFFFF]
    return KeyRanges(lo, hi)


def ranges_splitters(splitters) -> KeyRanges:
    """Buckets {k <= s_0}, {s_0 < k <= s_1}, ..., {k > s_{m-2}}; splitters strictly increasing."""
    s = [int(x) for x in splitters]
    lo = [0] + [x + 1 for x in s]
    hi = s + [0xFFFFFFFF]
    return KeyRanges(lo, hi)


def ranges_equal(m: int) -> KeyRanges:
    """The paper's equal division of the 32-bit domain."""
    lo = [(b << 32) // m for b in range(m)]
    hi = [((b + 1) << 32) // m - 1 for b in range(m)]
    return KeyRanges(lo, hi)


def gen_splitters(m: int, seed: int) -> np.ndarray:
    """m-1 distinct sorted splitters in [1, 2^32-2] (irregular widths)."""
    out, start = set(), 0
    while len(out) < m - 1:
        r = u32_np(seed, 0x40, start, 4 * m)
        start += 4 * m
        for x in r.tolist():
            if 1 <= x <= 0xFFFFFFFE:
                out.add(x)
            if len(out) == m - 1:
                break
    return np.array(sorted(out), dtype=np.uint32)


def keys_np(n: int, seed: int, dist: str = "uniform", m: int = 0, ranges: KeyRanges | None = None,
            start: int = 0, lowbits_shift: int | None = None) -> np.ndarray:
    """Keys (uint32) on the host.

    dist == 'uniform': uniform over uint32.  Otherwise a bucket b is drawn from
    `dist` over m buckets and the key is drawn uniformly from ranges[b]; for
    low-bit buckets pass `lowbits_shift` instead of ranges (key bits
    [shift, shift+log2 m) are set to b, the rest uniform).
    """
    if dist == "uniform":
        return u32_np(seed, S_KEY, start, n)
    b = draw_buckets_np(dist, m, seed, start, n)
    r = u32_np(seed, S_POS, start, n)
    if lowbits_shift is not None:
        mask = np.uint32(((m - 1) << lowbits_shift) & 0xFFFFFFFF)
        return ((r & ~mask) | (b.astype(np.uint32) << np.uint32(lowbits_shift))).astype(np.uint32)
    return uniform_in_np(r, ranges.lo[b], ranges.hi[b])


def keys_torch(n: int, seed: int, device, dist: str = "uniform", m: int = 0,
               ranges: KeyRanges | None = None, start: int = 0, lowbits_shift: int | None = None):
    """Same keys as keys_np, as an int32 tensor (uint32 bit pattern) on `device`."""
    import torch
    if dist == "uniform":
        return _as_u32_tensor(u32_torch(seed, S_KEY, start, n, device))
    b = draw_buckets_torch(dist, m, seed, start, n, device)
    r = u32_torch(seed, S_POS, start, n, device)
    if lowbits_shift is not None:
        mask = ((m - 1) << lowbits_shift) & 0xFFFFFFFF
        k = torch.bitwise_or(torch.bitwise_and(r, 0xFFFFFFFF ^ mask), b << lowbits_shift)
        return _as_u32_tensor(k)
    lo = torch.as_tensor(ranges.lo.astype(np.int64), device=device)[b]
    hi = torch.as_tensor(ranges.hi.astype(np.int64), device=device)[b]
    k = lo + ((r * (hi - lo + 1)) >> 32)
    return _as_u32_tensor(k)


def bucket_draw_np(n: int, seed: int, dist: str, m: int, start: int = 0) -> np.ndarray:
    """Precomputed-id workloads (MS_IDS): the ids themselves, uint8 when m <= 256."""
    if dist == "uniform":
        dist = "buckets"
    return draw_buckets_np(dist, m, seed, start, n).astype(np.uint8 if m <= 256 else np.uint32)


def bucket_draw_torch(n, seed, dist, m, device, start: int = 0):
    import torch
    if dist == "uniform":
        dist = "buckets"
    return draw_buckets_torch(dist, m, seed, start, n, device).to(torch.uint8)


def values_np(n: int, seed: int, kind: str = "index", start: int = 0) -> np.ndarray:
    """'index' -> vals[i] = i (parity runs: makes stability visible); 'random' -> stream 1."""
    if kind == "index":
        return np.arange(start, start + n, dtype=np.uint64).astype(np.uint32)
    return u32_np(seed, S_VAL, start, n)


def values_torch(n, seed, device, kind="index", start: int = 0):
    import torch
    if kind == "index":
        return _as_u32_tensor(torch.arange(start, start + n, dtype=torch.int64, device=device) & 0xFFFFFFFF)
    return _as_u32_tensor(u32_torch(seed, S_VAL, start, n, device))
