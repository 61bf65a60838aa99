"""Delta-stepping bucketing with the multisplit (§1).

The paper's motivating use: delta-stepping SSSP keeps the pending vertices in buckets of width
Delta by tentative distance, processes the lowest non-empty bucket, and re-buckets what the
relaxations changed; Davidson et al. do the re-bucketing with a sort, the paper with a multisplit
("delta-range" buckets floor(d / Delta) with a far pile).  Here every re-bucketing step
is ONE stable multisplit (libms, the same kernels as the benchmark) of the pending set:

    keys = tentative distance - base (u32),   vals = vertex id,
    spec = delta_range(m, Delta)   ->  bucket 0 = [base, base + Delta), ..., bucket m-1 = far pile

and the offsets give the lowest bucket's extent without any other pass.  Graph generation and the
edge relaxation (gather / scatter-min over the CSR) are plain torch ops -- plumbing around the
method, not part of it; the bucketing is the multisplit.  Synthetic seeded graphs only (the paper's
road networks are not available).
"""
from __future__ import annotations

from dataclasses import dataclass


from .api import BucketSpec, Plan

INF = 0xFFFFFFFF


@dataclass
class Graph:
    V: int
    row_ptr: "torch.Tensor"  # int64 [V+1]
    col: "torch.Tensor"      # int64 [E]
    w: "torch.Tensor"        # int64 [E], weights >= 1


def synthetic_graph(V: int, E: int, wmax: int, seed: int, device) -> Graph:
    """Seeded random directed graph: E edges with endpoints uniform over V vertices plus a ring
    (so every vertex is reachable from 0), integer weights uniform in [1, wmax]."""
    import torch
    import workloads as W
    r = W.u32_torch(seed, 20, 0, 3 * E, device)
    src = torch.cat([r[:E] % V, torch.arange(V, device=device)])
    dst = torch.cat([r[E:2 * E] % V, (torch.arange(V, device=device) + 1) % V])
    w = torch.cat([1 + r[2 * E:] % wmax, 1 + (torch.arange(V, device=device) * 7919) % wmax])
    order = torch.argsort(src, stable=True)
    src, dst, w = src[order], dst[order], w[order]
    row_ptr = torch.zeros(V + 1, dtype=torch.int64, device=device)
    row_ptr[1:] = torch.cumsum(torch.bincount(src, minlength=V), 0)
    return Graph(V, row_ptr, dst.to(torch.int64), w.to(torch.int64))


def delta_stepping(g: Graph, source: int, delta: int, m: int = 8, max_iters: int = 1 << 20):
    """Single-source shortest paths by delta-stepping with multisplit re-bucketing.
    Returns (dist int64 [V] with INF for unreachable, stats dict)."""
    import torch
    dev = g.row_ptr.device
    dist = torch.full((g.V,), INF, dtype=torch.int64, device=dev)
    dist[source] = 0
    pending = torch.tensor([source], dtype=torch.int64, device=dev)
    spec = BucketSpec.delta_range(m, delta)
    plans = {}
    stats = {"iterations": 0, "multisplits": 0, "relaxed_edges": 0, "multisplit_keys": 0}
    while pending.numel() and stats["iterations"] < max_iters:
        stats["iterations"] += 1
        d = dist[pending]
        base = int(d.min())
        n = pending.numel()
        cap = 1 << max(10, (n - 1).bit_length())  # one plan per power-of-two size class
        plan = plans.get(cap)
        if plan is None:
            plan = plans[cap] = Plan(spec, cap, with_values=True)
        keys = (d - base).to(torch.int32)  # u32 bit pattern (< 2^31 here)
        vals = pending.to(torch.int32)
        ko, vo, off = plan.run(keys, vals)  # the re-bucketing step: one stable multisplit
        stats["multisplits"] += 1
        stats["multisplit_keys"] += n
        n0 = int(off[1])                     # bucket 0 = [base, base + delta)
        frontier = vo[:n0].to(torch.int64)
        rest = vo[n0:].to(torch.int64)
        # relax every out-edge of the frontier (gather / scatter-min: plumbing)
        beg, end = g.row_ptr[frontier], g.row_ptr[frontier + 1]
        deg = end - beg
        tot = int(deg.sum())
        changed = torch.empty(0, dtype=torch.int64, device=dev)
        if tot:
            owner = torch.repeat_interleave(torch.arange(frontier.numel(), device=dev), deg)
            first = torch.cumsum(deg, 0) - deg
            eidx = beg[owner] + (torch.arange(tot, device=dev) - first[owner])
            tgt = g.col[eidx]
            nd = dist[frontier][owner] + g.w[eidx]
            old = dist.clone()
            dist.scatter_reduce_(0, tgt, nd, reduce="amin")
            changed = torch.nonzero(dist < old).flatten()
            stats["relaxed_edges"] += tot
        pending = torch.unique(torch.cat([rest, changed]))
    return dist, stats
