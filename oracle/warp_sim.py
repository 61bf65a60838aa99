"""Bit-level simulator of the paper's warp procedures -- TEST INFRASTRUCTURE ONLY.

A 32-lane model of ``ballot`` / ``popc`` running Algorithm 2 (warp
histogram, §5.1) and Algorithm 3 (warp local offsets,
P:1128-1162) exactly as printed, plus the corrected local offset of reading
#4 in DESIGN.md (the printed mask ``0xFFFFFFFF >> (31-i)`` keeps lanes 0..i,
so it returns the inclusive rank; the text, "number of preceding
elements", asks for the exclusive one).  Pure Python; small inputs only.
"""
from __future__ import annotations

import math

FULL = 0xFFFFFFFF


def ballot(preds):
    """ballot(): bit i set iff lane i's predicate is true."""
    r = 0
    for lane, p in enumerate(preds):
        if p:
            r |= 1 << lane
    return r


def popc(x: int) -> int:
    return bin(x & FULL).count("1")


def rounds(m: int) -> int:
    """ceil(log2(m)) ballot rounds (Alg. 2 line 4); 0 for m = 1."""
    return 0 if m <= 1 else math.ceil(math.log2(m))


def warp_histogram(bucket_id, m):
    """Algorithm 2 as printed: returns histo[i] for every lane i (0..31)."""
    ids = list(bucket_id)
    bmp = [FULL] * 32
    for k in range(rounds(m)):
        t = ballot([b & 1 for b in ids])                       # line 5
        for i in range(32):
            if (i >> k) & 1:                                    # line 6
                bmp[i] &= t                                     # line 7
            else:
                bmp[i] &= FULL ^ t                              # line 9
        ids = [b >> 1 for b in ids]                             # line 11
    return [popc(bmp[i]) for i in range(32)]                    # line 13


def warp_offsets_printed(bucket_id, m):
    """Algorithm 3 as printed (line 13 mask 0xFFFFFFFF >> (31 - i))."""
    ids = list(bucket_id)
    bmp = [FULL] * 32
    for _ in range(rounds(m)):
        t = ballot([b & 1 for b in ids])                       # line 5
        for i in range(32):
            if ids[i] & 1:                                      # line 6
                bmp[i] &= t
            else:
                bmp[i] &= FULL ^ t
        ids = [b >> 1 for b in ids]
    return [popc(bmp[i] & (FULL >> (31 - i))) for i in range(32)]


def warp_offsets_exclusive(bucket_id, m):
    """Alg. 3 with reading #4: popc(bmp & lanemask_lt) = number of PRECEDING same-bucket lanes."""
    ids = list(bucket_id)
    bmp = [FULL] * 32
    for _ in range(rounds(m)):
        t = ballot([b & 1 for b in ids])
        for i in range(32):
            bmp[i] &= t if (ids[i] & 1) else (FULL ^ t)
        ids = [b >> 1 for b in ids]
    return [popc(bmp[i] & ((1 << i) - 1)) for i in range(32)]
