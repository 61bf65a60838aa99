"""Test helpers: build matching (product spec, oracle spec, inputs) from the seeded generators."""
from __future__ import annotations

import numpy as np

import oracle
import workloads as W


def power_of_two(m):
    return m & (m - 1) == 0


def make_case(kind: str, m: int, n: int, seed: int, dist: str = "uniform", kv: bool = True,
              id_bytes: int = 1, vals_kind: str = "index"):
    """Returns dict(spec_kw, ospec, keys, vals, ids) with numpy inputs."""
    spec_kw = dict(kind=kind, m=m)
    ranges, shift = None, None
    if kind == "lowbits":
        lb = (m - 1).bit_length()
        spec_kw["shift"] = shift = (seed % (33 - lb)) if lb < 32 else 0
        if m == 1:
            spec_kw["shift"] = shift = 0
    elif kind == "delta":
        delta = min(0xFFFFFFFF, max(1, (1 << 32) // m)) if seed % 2 == 0 else 400000000
        spec_kw["delta"] = delta
        ranges = W.ranges_delta(m, delta)
    elif kind == "splitters":
        spl = W.gen_splitters(m, seed) if m > 1 else np.zeros(0, np.uint32)
        spec_kw["splitters"] = spl.tolist()
        ranges = W.ranges_splitters(spl)
    elif kind == "ids":
        spec_kw["id_bytes"] = id_bytes
    ids = None
    if kind == "ids":
        keys = W.keys_np(n, seed)
        ids = W.bucket_draw_np(n, seed, dist, m).astype(np.uint8 if id_bytes == 1 else np.uint32)
    elif dist == "uniform" or m == 1:
        keys = W.keys_np(n, seed)
    else:
        keys = W.keys_np(n, seed, dist, m, ranges, lowbits_shift=shift if kind == "lowbits" else None)
    vals = W.values_np(n, seed, vals_kind) if kv else None
    ospec = oracle.Spec(kind, m, shift=spec_kw.get("shift", 0), delta=spec_kw.get("delta", 1),
                        splitters=spec_kw.get("splitters"), id_bytes=id_bytes)
    return dict(spec_kw=spec_kw, ospec=ospec, keys=keys, vals=vals, ids=ids)


def to_dev(a):
    import torch
    if a is None:
        return None
    if a.dtype == np.uint8:
        return torch.from_numpy(a.copy()).cuda()
    return torch.from_numpy(a.view(np.int32).copy()).cuda()


def from_dev(t):
    if t is None:
        return None
    return t.cpu().numpy().view(np.uint32)
