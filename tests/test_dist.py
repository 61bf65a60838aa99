"""Sharded multisplit: host planning + the exchange, on CPU with gloo (world size 2..4).

The local per-rank step here is the CPU oracle (test infrastructure) so the
whole N>1 orchestration -- count all-gather, ms_dist_pieces planning (native,
libms.so), grouped point-to-point exchange -- runs without a GPU; the product
path uses ms_run on the GPU for the local step.  Expected: the concatenation of
the rank windows equals the single-GPU stable multisplit of the concatenated
shards."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import oracle
import workloads as W
from paper_conf_ppopp_ashkianidmo16_b200.dist import dist_multisplit, dist_pieces, dist_targets
from paper_conf_ppopp_ashkianidmo16_b200.api import BucketSpec


# ------------------------------------------------------------ planning alone
@pytest.mark.parametrize("P,m", [(1, 1), (2, 3), (3, 32), (4, 8), (8, 32), (8, 256), (5, 1)])
def test_pieces_cover_and_match(P, m):
    rng = np.random.default_rng(P * 100 + m)
    for trial in range(20):
        counts = rng.integers(0, 50, size=(P, m)).astype(np.uint64)
        if trial % 4 == 0:
            counts[:, m // 2] *= 20            # skew: one heavy bucket
        if trial % 5 == 0:
            counts[rng.integers(P)] = 0         # an empty shard
        N = int(counts.sum())
        plans = [dist_pieces(P, r, m, counts) for r in range(P)]
        B = np.concatenate([[0], np.cumsum(counts.sum(axis=0))]).astype(np.uint64)
        for r in range(P):
            assert np.array_equal(plans[r][2], B)                    # global bucket starts
        wins = [(p[3], p[4]) for p in plans]
        assert wins[0][0] == 0 and sum(w[1] for w in wins) == N
        assert max(w[1] for w in wins) - min(w[1] for w in wins) <= 1  # balanced windows
        for r in range(P - 1):
            assert wins[r][0] + wins[r][1] == wins[r + 1][0]
        cover = np.zeros(N, dtype=np.int64)
        for g in range(P):
            send = plans[g][0]
            assert len(send) <= m + P - 1                            # monotone output: <= m+P-1 pieces
            assert sum(p[1] for p in send) == int(counts[g].sum())   # every local element leaves once
            for s_off, ln, peer, d_off in send:
                cover[wins[peer][0] + d_off: wins[peer][0] + d_off + ln] += 1
                # the matching receive exists at the peer with the same geometry
                assert (s_off, ln, g, d_off) in plans[peer][1]
        assert np.all(cover == 1)
        for r in range(P):                                           # receives tile the window exactly
            assert sum(p[1] for p in plans[r][1]) == wins[r][1]


@pytest.mark.parametrize("P,m", [(1, 1), (2, 3), (3, 32), (4, 8), (8, 32), (5, 2)])
def test_targets_match_pieces(P, m):
    """ms_dist_targets (fused scatter planning) agrees with ms_dist_pieces: same windows, and every
    piece rank g sends sits at global position local position + delta[bucket of that position]."""
    rng = np.random.default_rng(7 * P + m)
    for trial in range(20):
        counts = rng.integers(0, 40, size=(P, m)).astype(np.uint64)
        if trial % 3 == 0:
            counts[:, 0] *= 25
        if trial % 4 == 0:
            counts[rng.integers(P)] = 0
        for g in range(P):
            delta, wst = dist_targets(P, g, m, counts)
            send, _, _, ws, wl = dist_pieces(P, g, m, counts)
            assert wst[g] == ws and wst[g + 1] - wst[g] == wl
            assert wst[0] == 0 and wst[P] == counts.sum()
            off = np.concatenate([[0], np.cumsum(counts[g])]).astype(np.uint64)
            for s_off, ln, peer, d_off in send:
                b = int(np.searchsorted(off, s_off, side="right") - 1)
                while counts[g][b] == 0:
                    b += 1
                assert int(wst[peer]) + d_off == s_off + int(delta[b])


def test_targets_reject_bad_sizes():
    from paper_conf_ppopp_ashkianidmo16_b200._abi import MultisplitError
    with pytest.raises(MultisplitError):
        dist_targets(9, 0, 4, np.zeros((9, 4), np.uint64))   # more than MS_MAX_PEERS ranks


def test_pieces_follow_eq2():
    """Global position of local element i of bucket b on rank g = B[b] + sum_{g'<g} h[g'][b] + (i - off_g[b])."""
    P, m = 3, 4
    counts = np.array([[2, 0, 3, 1], [1, 1, 0, 4], [0, 2, 2, 0]], dtype=np.uint64)
    B = np.concatenate([[0], np.cumsum(counts.sum(axis=0))])
    for g in range(P):
        send, _, _, _, _ = dist_pieces(P, g, m, counts)
        off = np.concatenate([[0], np.cumsum(counts[g])])
        gpos = {}
        plans = [dist_pieces(P, r, m, counts) for r in range(P)]
        for s_off, ln, peer, d_off in send:
            for k in range(ln):
                gpos[s_off + k] = plans[peer][3] + d_off + k
        for b in range(m):
            for i in range(int(off[b]), int(off[b + 1])):
                assert gpos[i] == B[b] + counts[:g, b].sum() + (i - off[b])


# ------------------------------------------------------------ full exchange with gloo
def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _shard_sizes(P, n, mode):
    if mode == "equal":
        return [n // P + (1 if r < n % P else 0) for r in range(P)]
    sizes = [(n * (r + 1)) // (P * (P + 1) // 2) for r in range(P)]   # unequal, rank-increasing
    sizes[-1] += n - sum(sizes)
    if mode == "empty":
        sizes[0], sizes[-1] = 0, sizes[-1] + sizes[0]
    return sizes


def _case(kind, m):
    if kind == "splitters":
        spl = W.gen_splitters(m, 3)
        return BucketSpec.from_splitters(spl.tolist()), oracle.Spec("splitters", m, splitters=spl), W.ranges_splitters(spl)
    delta = max(1, (1 << 32) // m)
    return BucketSpec.delta_range(m, delta), oracle.Spec("delta", m, delta=delta), W.ranges_delta(m, delta)


def _worker(rank, P, port, n, kind, m, dist_name, mode, kv):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=P)
    try:
        spec, ospec, ranges = _case(kind, m)
        sizes = _shard_sizes(P, n, mode)
        start = sum(sizes[:rank])
        keys = W.keys_np(sizes[rank], 11, dist_name, m, ranges, start=start) if dist_name != "uniform" else \
            W.keys_np(sizes[rank], 11, start=start)
        vals = W.values_np(sizes[rank], 11, "index", start=start) if kv else None

        def local(k, v):  # CPU oracle as the local step (test infrastructure)
            ko, vo, off = oracle.multisplit(ospec, k.numpy().view(np.uint32),
                                            None if v is None else v.numpy().view(np.uint32))
            t = lambda a: torch.from_numpy(a.view(np.int32).copy())  # noqa: E731
            return t(ko), (t(vo) if vo is not None else None), torch.from_numpy(off.astype(np.int64))

        kt = torch.from_numpy(keys.view(np.int32).copy())
        vt = torch.from_numpy(vals.view(np.int32).copy()) if kv else None
        wk, wv, offg, ws = dist_multisplit(kt, vt, spec, local=local)
        # expected: oracle of the concatenated input, sliced to my window
        allk = W.keys_np(n, 11, dist_name, m, ranges) if dist_name != "uniform" else W.keys_np(n, 11)
        allv = W.values_np(n, 11, "index") if kv else None
        eko, evo, eoff = oracle.multisplit(ospec, allk, allv)
        assert np.array_equal(offg, eoff)
        assert np.array_equal(wk.numpy().view(np.uint32), eko[ws:ws + wk.numel()])
        if kv:
            assert np.array_equal(wv.numpy().view(np.uint32), evo[ws:ws + wv.numel()])
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("P,kind,m,dist_name,mode,kv", [
    (2, "delta", 8, "uniform", "equal", True),
    (3, "splitters", 32, "hot", "unequal", True),
    (4, "delta", 256, "binomial", "empty", False),
    (4, "splitters", 5, "one", "equal", True),
])
def test_dist_multisplit_gloo(P, kind, m, dist_name, mode, kv):
    n = 20011
    mp.spawn(_worker, args=(P, _free_port(), n, kind, m, dist_name, mode, kv), nprocs=P, join=True)


# ------------------------------------------------------------ the CUDA local step (GPU box)
def _worker_cuda(rank, P, port, n, kind, m, dist_name, mode, kv):
    """Like _worker, but every rank's local step is the product path: ms_run on cuda:0 (all ranks
    share the one GPU of the test box), the exchange over gloo on host copies of its output."""
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=P)
    try:
        from paper_conf_ppopp_ashkianidmo16_b200.api import Plan
        torch.cuda.set_device(0)
        spec, ospec, ranges = _case(kind, m)
        sizes = _shard_sizes(P, n, mode)
        start = sum(sizes[:rank])
        keys = W.keys_np(sizes[rank], 11, dist_name, m, ranges, start=start) if dist_name != "uniform" else \
            W.keys_np(sizes[rank], 11, start=start)
        vals = W.values_np(sizes[rank], 11, "index", start=start) if kv else None
        plan = Plan(spec, max(1, sizes[rank]), with_values=kv)

        def local(k, v):  # the CUDA multisplit of this rank's shard; outputs staged to the host for gloo
            ko, vo, off = plan.run(k.cuda(), None if v is None else v.cuda())
            torch.cuda.synchronize()
            assert plan.last_launches() == (1 if k.numel() else 0)  # ONE at these sizes (m <= 32)
            return ko.cpu(), (vo.cpu() if vo is not None else None), off.cpu().to(torch.int64) & 0xFFFFFFFF

        kt = torch.from_numpy(keys.view(np.int32).copy())
        vt = torch.from_numpy(vals.view(np.int32).copy()) if kv else None
        wk, wv, offg, ws = dist_multisplit(kt, vt, spec, local=local)
        allk = W.keys_np(n, 11, dist_name, m, ranges) if dist_name != "uniform" else W.keys_np(n, 11)
        allv = W.values_np(n, 11, "index") if kv else None
        eko, evo, eoff = oracle.multisplit(ospec, allk, allv)
        assert np.array_equal(offg, eoff)
        assert np.array_equal(wk.numpy().view(np.uint32), eko[ws:ws + wk.numel()])
        if kv:
            assert np.array_equal(wv.numpy().view(np.uint32), evo[ws:ws + wv.numel()])
    finally:
        dist.destroy_process_group()


@pytest.mark.gpu
@pytest.mark.parametrize("P,kind,m,dist_name,mode,kv", [
    (2, "delta", 8, "uniform", "equal", True),
    (3, "splitters", 32, "hot", "empty", False),
])
def test_dist_multisplit_gloo_cuda_local(P, kind, m, dist_name, mode, kv):
    """World size 2-3 on gloo with the REAL local step (libms ms_run on cuda:0) on every rank."""
    n = 3 * 4096 * 148 + 1234  # several tiles per resident CTA, ragged
    ctx = mp.get_context("spawn")
    port = _free_port()
    procs = [ctx.Process(target=_worker_cuda, args=(r, P, port, n, kind, m, dist_name, mode, kv)) for r in range(P)]
    for p in procs:
        p.start()
    for p in procs:
        p.join(600)
    assert all(p.exitcode == 0 for p in procs), [p.exitcode for p in procs]


@pytest.mark.gpu
@pytest.mark.parametrize("kind,m,kv", [("delta", 8, False), ("splitters", 32, True), ("delta", 256, True)])
def test_dist_run_nccl_single_rank(kind, m, kv):
    """ms_dist_run (the native collective: local ms_run, NCCL count all-gather, piece planning, NCCL
    group send/recv) on a one-rank NCCL communicator: the window is the whole output and must equal
    the oracle; offsets_global equal the oracle's offsets.  (A one-GPU box cannot host P > 1 NCCL
    ranks -- NCCL rejects two ranks on one device; the P > 1 piece planning is pinned by the CPU
    tests above and the exchange by the gloo runs.)"""
    from paper_conf_ppopp_ashkianidmo16_b200.dist import DistPlan, NcclComm
    torch.cuda.set_device(0)
    spec, ospec, ranges = _case(kind, m)
    n = (1 << 22) + 333
    keys = W.keys_np(n, 5, "binomial", m, ranges)
    vals = W.values_np(n, 5, "index") if kv else None
    comm = NcclComm.single(0)
    dp = DistPlan(spec, comm, n, n, with_values=kv)
    kd = torch.from_numpy(keys.view(np.int32).copy()).cuda()
    vd = torch.from_numpy(vals.view(np.int32).copy()).cuda() if kv else None
    eko, evo, eoff = oracle.multisplit(ospec, keys, vals)
    for _ in range(2):  # repeated runs on one workspace
        wk, wv, offg, ws = dp.run(kd, vd)
        torch.cuda.synchronize()
        assert ws == 0 and wk.numel() == n
        assert np.array_equal(offg, eoff)
        assert np.array_equal(wk.cpu().numpy().view(np.uint32), eko)
        if kv:
            assert np.array_equal(wv.cpu().numpy().view(np.uint32), evo)
    comm.close()


@pytest.mark.gpu
@pytest.mark.parametrize("kind,m,kv", [("delta", 8, False), ("splitters", 32, True), ("delta", 5, True)])
def test_dist_run_fused_single_rank(kind, m, kv):
    """ms_dist_run_fused (local K1 + K2, NCCL count all-gather, targets, the scatter post-scan into
    the window, NCCL barrier) on a one-rank communicator with an explicit window: bit-exact vs the
    oracle, offsets_global included, repeated runs."""
    from paper_conf_ppopp_ashkianidmo16_b200.dist import FusedDistPlan, NcclComm
    torch.cuda.set_device(0)
    spec, ospec, ranges = _case(kind, m)
    n = (1 << 22) + 333
    keys = W.keys_np(n, 6, "hot", m, ranges)
    vals = W.values_np(n, 6, "index") if kv else None
    comm = NcclComm.single(0)
    wk = torch.empty(n + 1, dtype=torch.int32, device="cuda")
    wv = torch.empty(n + 1, dtype=torch.int32, device="cuda") if kv else None
    fp = FusedDistPlan(spec, comm, n, n, with_values=kv,
                       peer_windows=([wk.data_ptr()], [wv.data_ptr()] if kv else None))
    kd = torch.from_numpy(keys.view(np.int32).copy()).cuda()
    vd = torch.from_numpy(vals.view(np.int32).copy()).cuda() if kv else None
    eko, evo, eoff = oracle.multisplit(ospec, keys, vals)
    for _ in range(2):
        wk.fill_(-1)
        _, _, offg, ws = fp.run(kd, vd)
        torch.cuda.synchronize()
        assert ws == 0 and np.array_equal(offg, eoff)
        assert np.array_equal(wk[:n].cpu().numpy().view(np.uint32), eko)
        if kv:
            assert np.array_equal(wv[:n].cpu().numpy().view(np.uint32), evo)
    comm.close()
