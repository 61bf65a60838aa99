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


def delta_stepping(g: Graph, source: int, delta: int, m: int = 8, max_iters: int = 1 << 20,
                   rebucket: str = "multisplit", time_rebucket: bool = False):
    """Single-source shortest paths by delta-stepping.  Every iteration re-buckets the pending
    vertices by tentative distance -- rebucket="multisplit": ONE stable libms multisplit (the
    paper's proposal); rebucket="sort": the sort-based re-bucketing it replaces (Davidson et al.,
    P:192-205): a stable torch.sort of the bucket ids + gathers, bit-identical output.  The
    pending set carries no duplicates (a per-vertex queue flag; no torch.unique), and an
    iteration synchronises with the host twice (the lowest bucket's size with its edge count,
    then the number of improved vertices).  time_rebucket: CUDA events around every re-bucketing
    step (stats["rebucket_ms"]).  Returns (dist int64 [V] with INF for unreachable, stats)."""
    import torch
    dev = g.row_ptr.device
    dist = torch.full((g.V,), INF, dtype=torch.int64, device=dev)
    dist[source] = 0
    inq = torch.zeros(g.V, dtype=torch.bool, device=dev)
    inq[source] = True
    pending = torch.tensor([source], dtype=torch.int64, device=dev)
    spec = BucketSpec.delta_range(m, delta)
    plans = {}
    stats = {"iterations": 0, "multisplits": 0, "relaxed_edges": 0, "multisplit_keys": 0, "rebucket_ms": 0.0}
    events = []
    while pending.numel() and stats["iterations"] < max_iters:
        stats["iterations"] += 1
        d = dist[pending]
        n = pending.numel()
        keys = (d - d.min()).to(torch.int32)  # u32 bit pattern (< 2^31 here), base = the lowest distance
        vals = pending.to(torch.int32)
        if time_rebucket:
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
        if rebucket == "multisplit":
            cap = 1 << max(10, (n - 1).bit_length())  # one plan per power-of-two size class
            plan = plans.get(cap)
            if plan is None:
                plan = plans[cap] = Plan(spec, cap, with_values=True)
            ko, vo, off = plan.run(keys, vals)  # the re-bucketing step: one stable multisplit
            n0_dev = off[1]                      # bucket 0 = [base, base + delta)
        else:
            ids = torch.clamp((keys.to(torch.int64) & 0xFFFFFFFF) // delta, max=m - 1).to(torch.uint8)
            _, idx = torch.sort(ids, stable=True)
            vo = vals[idx]
            n0_dev = (ids == 0).sum()
        if time_rebucket:
            e1.record()
            events.append((e0, e1))
        stats["multisplits"] += 1
        stats["multisplit_keys"] += n
        # the lowest bucket's vertices and their out-degree total, fetched together (sync 1)
        vo64 = vo.to(torch.int64)
        in0 = torch.arange(n, device=dev) < n0_dev
        deg_all = torch.where(in0, g.row_ptr[vo64 + 1] - g.row_ptr[vo64], 0)
        n0, tot = (int(x) for x in torch.stack([n0_dev.to(torch.int64), deg_all.sum()]).tolist())
        frontier = vo64[:n0]
        rest = vo64[n0:]
        inq[frontier] = False
        newc = torch.empty(0, dtype=torch.int64, device=dev)
        if tot:
            # relax every out-edge of the frontier (gather / scatter-min: plumbing)
            deg = deg_all[:n0]
            beg = g.row_ptr[frontier]
            owner = torch.repeat_interleave(torch.arange(n0, device=dev), deg, output_size=tot)
            first = torch.cumsum(deg, 0) - deg
            eidx = beg[owner] + (torch.arange(tot, device=dev) - first[owner])
            tgt = g.col[eidx]
            nd = dist[frontier][owner] + g.w[eidx]
            old = dist.clone()
            dist.scatter_reduce_(0, tgt, nd, reduce="amin")
            changed = torch.nonzero(dist < old).flatten()  # sync 2 (data-dependent size)
            newc = changed[~inq[changed]]                   # improved vertices not yet pending
            inq[newc] = True
            stats["relaxed_edges"] += tot
        pending = torch.cat([rest, newc])
    if time_rebucket:
        torch.cuda.synchronize()
        stats["rebucket_ms"] = sum(a.elapsed_time(b) for a, b in events)
    return dist, stats
