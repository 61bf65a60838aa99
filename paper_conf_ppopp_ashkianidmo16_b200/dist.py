"""Sharded stable multisplit over P ranks (include/ms.h `ms_dist_pieces`).

Eq. (2) with the ranks as the outermost subproblems:

1. every rank multisplits its shard locally (``ms_run``; its local output is
   bucket-major and stable);
2. one all-gather of the m per-rank bucket counts;
3. ``ms_dist_pieces`` (native host planning in libms.so) gives the global
   bucket starts, this rank's balanced output window and the <= m+P-1
   contiguous pieces it sends / receives;
4. one grouped point-to-point exchange (NCCL send/recv over NVLink/NVSwitch on
   a GPU box) lands every piece directly at its final offset in the owner's
   window -- no receive-side permutation.

The concatenation of the windows over ranks is the single-GPU stable
multisplit of the concatenated shards (rank order), so the same oracle checks it.
torch.distributed is plumbing here (process group, collectives); all per-key
work is the local multisplit's kernels.
"""
from __future__ import annotations

import ctypes

import numpy as np

from . import _abi
from ._abi import check


class ms_piece(ctypes.Structure):
    _fields_ = [("src_off", ctypes.c_uint64), ("len", ctypes.c_uint64), ("peer", ctypes.c_int32),
                ("pad_", ctypes.c_int32), ("dst_off", ctypes.c_uint64)]


def dist_pieces(nranks: int, rank: int, m: int, counts):
    """Host planning: counts (P x m, uint64) -> (send, recv, offsets_global[m+1], win_start, win_len).

    send/recv are lists of (src_off, len, peer, dst_off)."""
    L = _abi.lib()
    counts = np.ascontiguousarray(counts, dtype=np.uint64)
    assert counts.shape == (nranks, m)
    scap, rcap = m + nranks, m * nranks + 1
    send = (ms_piece * scap)()
    recv = (ms_piece * rcap)()
    ns, nr = ctypes.c_int32(), ctypes.c_int32()
    offg = np.zeros(m + 1, dtype=np.uint64)
    ws, wl = ctypes.c_uint64(), ctypes.c_uint64()
    check(L.ms_dist_pieces(nranks, rank, m, counts.ctypes.data_as(ctypes.c_void_p), send, scap, ctypes.byref(ns),
                           recv, rcap, ctypes.byref(nr), offg.ctypes.data_as(ctypes.c_void_p), ctypes.byref(ws),
                           ctypes.byref(wl)), "ms_dist_pieces")
    conv = lambda p: (int(p.src_off), int(p.len), int(p.peer), int(p.dst_off))  # noqa: E731
    return [conv(send[i]) for i in range(ns.value)], [conv(recv[i]) for i in range(nr.value)], offg, ws.value, wl.value


def _gpu_local(spec, with_values):
    from .api import Plan
    plans = {}

    def run(keys, vals):
        n = keys.numel()
        key = (max(n, 1), with_values)
        if key not in plans:
            plans[key] = Plan(spec, max(n, 1), with_values=with_values)
        return plans[key].run(keys, vals)
    return run


def dist_multisplit(keys, vals=None, spec=None, group=None, local=None):
    """Collective: every rank passes its shard (keys[, vals]); returns
    (keys_window, vals_window, offsets_global[m+1] as numpy uint64, window_start).

    `local(keys, vals) -> (keys_out, vals_out, offsets[m+1])` is the local stable
    multisplit; the default is libms's ms_run on the tensors' CUDA device."""
    import torch
    import torch.distributed as dist
    P = dist.get_world_size(group)
    g = dist.get_rank(group)
    m = spec.m
    if local is None:
        local = _gpu_local(spec, vals is not None)
    ko, vo, off = local(keys, vals)
    off64 = off.to(torch.int64) & 0xFFFFFFFF
    counts = (off64[1:] - off64[:-1]).contiguous()
    gathered = torch.empty(P * m, dtype=torch.int64, device=counts.device)
    dist.all_gather_into_tensor(gathered, counts, group=group)
    counts_host = gathered.cpu().numpy().astype(np.uint64).reshape(P, m)
    send, recv, offg, ws, wl = dist_pieces(P, g, m, counts_host)
    out_k = torch.empty(wl, dtype=ko.dtype, device=ko.device)
    out_v = torch.empty(wl, dtype=vo.dtype, device=vo.device) if vals is not None else None
    ops = []
    arrays = [(ko, out_k)] + ([(vo, out_v)] if vals is not None else [])
    for src_arr, dst_arr in arrays:
        for s_off, ln, peer, d_off in send:
            if peer == g:
                # local piece: straight device copy into my own window
                dst_arr[d_off:d_off + ln].copy_(src_arr[s_off:s_off + ln])
            else:
                ops.append(dist.P2POp(dist.isend, src_arr[s_off:s_off + ln], peer, group))
        for s_off, ln, peer, d_off in recv:
            if peer != g:
                ops.append(dist.P2POp(dist.irecv, dst_arr[d_off:d_off + ln], peer, group))
    if ops:
        for req in dist.batch_isend_irecv(ops):
            req.wait()
    return out_k, out_v, offg, ws


# ---------------------------------------------------------------------------
# Fused sharded scatter (include/ms.h ms_postscan_scatter):
# K1 + K2 locally, the count all-gather, then ONE post-scan kernel that stores
# every bucket run straight into the owners' windows (peer memory over
# NVLink/NVSwitch) -- no local output, no staging copy, no send/recv.
def dist_targets(nranks: int, rank: int, m: int, counts):
    """Host planning (ms_dist_targets): counts (P x m) -> (delta u64[m], win_start u64[P+1])."""
    counts = np.ascontiguousarray(counts, dtype=np.uint64)
    assert counts.shape == (nranks, m)
    delta = np.zeros(m, dtype=np.uint64)
    wst = np.zeros(nranks + 1, dtype=np.uint64)
    check(_abi.lib().ms_dist_targets(nranks, rank, m, counts.ctypes.data_as(ctypes.c_void_p),
                                     delta.ctypes.data_as(ctypes.c_void_p), wst.ctypes.data_as(ctypes.c_void_p)),
          "ms_dist_targets")
    return delta, wst


def scatter_target(keys_ptrs, vals_ptrs, win_start, delta):
    """ms_scatter_target from per-rank window base pointers (device addresses valid on this GPU)."""
    P = len(keys_ptrs)
    if not 1 <= P <= _abi.MS_MAX_PEERS:
        raise ValueError(f"fused scatter supports 1..{_abi.MS_MAX_PEERS} ranks, got {P}")
    t = _abi.ms_scatter_target()
    t.nranks = P
    for r in range(P):
        t.keys_dst[r] = int(keys_ptrs[r]) or None
        t.vals_dst[r] = (int(vals_ptrs[r]) or None) if vals_ptrs is not None else None
    for r in range(P + 1):
        t.win_start[r] = int(win_start[r])
    for b, d in enumerate(delta):
        t.delta[b] = int(d)
    return t


def _local_scan(plan, keys, ws):
    """K1 + K2 on this rank's shard: (G = m*L u32 matrix, counts u64[m] on the host)."""
    import torch
    n = keys.numel()
    off = torch.empty(plan.spec.m + 1, dtype=torch.int32, device=keys.device)
    G = plan.prescan(keys, workspace=ws)
    plan.scan(G, n, offsets=off, workspace=ws)
    o = off.cpu().numpy().view(np.uint32).astype(np.uint64)
    return G, o[1:] - o[:-1]


def _fused_plan(spec, n, with_values):
    from .api import Plan
    if spec.m > 32 or spec.kind == "ids":
        raise NotImplementedError("the fused sharded scatter runs on K3 v2 (m <= 32, computed bucket ids)")
    return Plan(spec, max(n, 1), with_values=with_values, variant="3k")


def scatter_multisplit_virtual(shards_keys, shards_vals=None, spec=None):
    """P VIRTUAL ranks on one GPU, same kernels and arithmetic as dist_multisplit_fused: each
    shard's K1+K2, then each shard's scatter-K3 writing into all P windows (here plain local
    allocations standing in for peer mappings).  Returns (keys, vals) = the windows concatenated,
    which equal the single-GPU stable multisplit of the concatenated shards."""
    import torch
    P = len(shards_keys)
    m = spec.m
    kv = shards_vals is not None
    plans, scans = [], []
    for r in range(P):
        plan = _fused_plan(spec, shards_keys[r].numel(), kv)
        ws = plan.workspace(shards_keys[r].numel())
        G, cnt = _local_scan(plan, shards_keys[r], ws)
        plans.append((plan, ws))
        scans.append((G, cnt))
    counts = np.stack([c for _, c in scans])
    dev = shards_keys[0].device
    _, wst = dist_targets(P, 0, m, counts)
    wins_k = [torch.empty(max(int(wst[r + 1] - wst[r]), 4), dtype=torch.int32, device=dev) for r in range(P)]
    wins_v = [torch.empty_like(w) for w in wins_k] if kv else None
    for r in range(P):
        delta, _ = dist_targets(P, r, m, counts)
        t = scatter_target([w.data_ptr() for w in wins_k], [w.data_ptr() for w in wins_v] if kv else None, wst, delta)
        plan, ws = plans[r]
        plan.postscan_scatter(shards_keys[r], scans[r][0], t, vals=shards_vals[r] if kv else None, workspace=ws)
    torch.cuda.synchronize()
    keys = torch.cat([wins_k[r][:int(wst[r + 1] - wst[r])] for r in range(P)])
    vals = torch.cat([wins_v[r][:int(wst[r + 1] - wst[r])] for r in range(P)]) if kv else None
    return keys, vals


class FusedDistPlan:
    """ms_dist_run_fused (include/ms.h): the sharded multisplit whose post-scan stores every run
    straight into the owners' windows.  The windows are torch symmetric-memory buffers (allocated
    and rendezvoused once per plan, mapped on every peer over NVLink / NVSwitch); `peer_windows`
    overrides them with explicit per-rank device pointers (e.g. virtual ranks on one GPU).
    m <= 32, computed bucket kinds."""

    def __init__(self, spec, comm: "NcclComm", max_local: int, max_total: int, with_values: bool = False,
                 group=None, peer_windows=None):
        import torch
        from .api import Plan
        if spec.m > 32 or spec.kind == "ids":
            raise NotImplementedError("the fused sharded scatter runs on K3 v2 (m <= 32, computed bucket ids)")
        self.spec, self.comm, self.kv = spec, comm, with_values
        self.plan = Plan(spec, max(int(max_local), 1), with_values=with_values, device=comm.device)
        b = ctypes.c_size_t()
        check(_abi.lib().ms_dist_workspace_size_fused(self.plan._h, max(int(max_local), 1), comm.nranks,
                                                      ctypes.byref(b)), "ms_dist_workspace_size_fused")
        dev = torch.device("cuda", comm.device)
        self.ws = torch.empty(max(b.value, 256), dtype=torch.uint8, device=dev)
        self.cap = -(-int(max_total) // comm.nranks) + 1
        if peer_windows is not None:
            kp, vp = peer_windows
            self.bufs = None
        else:
            import torch.distributed as dist
            import torch.distributed._symmetric_memory as symm_mem
            grp = group if group is not None else dist.group.WORLD
            self.bufs, ptrs = [], []
            for _ in range(2 if with_values else 1):
                buf = symm_mem.empty(self.cap, dtype=torch.int32, device=dev)
                h = symm_mem.rendezvous(buf, grp)
                self.bufs.append(buf)
                ptrs.append(list(h.buffer_ptrs))
            kp, vp = ptrs[0], (ptrs[1] if with_values else None)
        P = comm.nranks
        self._kp = (ctypes.c_void_p * P)(*[int(x) for x in kp])
        self._vp = (ctypes.c_void_p * P)(*[int(x) for x in vp]) if vp is not None else None

    def run(self, keys, vals=None, stream=None, copy_out=True):
        """Collective.  Returns (keys_window, vals_window, offsets_global u64[m+1] numpy, window_start);
        the windows are complete on return of the stream's work (the call ends with an NCCL barrier).
        copy_out=False returns views of this rank's symmetric window (overwritten by the next run)."""
        from .api import _ptr, _stream
        offg = np.zeros(self.spec.m + 1, dtype=np.uint64)
        ws0, wl = ctypes.c_uint64(), ctypes.c_uint64()
        check(_abi.lib().ms_dist_run_fused(self.plan._h, self.comm._h, _ptr(keys), _ptr(vals), keys.numel(),
                                           self._kp, self._vp if vals is not None else None, self.cap,
                                           offg.ctypes.data_as(ctypes.c_void_p), ctypes.byref(ws0), ctypes.byref(wl),
                                           _ptr(self.ws), self.ws.numel(), _stream(stream)), "ms_dist_run_fused")
        if self.bufs is None:
            return None, None, offg, ws0.value
        k = self.bufs[0][:wl.value]
        v = self.bufs[1][:wl.value] if vals is not None else None
        if copy_out:
            k = k.clone()
            v = v.clone() if v is not None else None
        return k, v, offg, ws0.value


_FUSED = {}


def dist_multisplit_fused(keys, vals=None, spec=None, group=None):
    """Collective, one process per GPU (NCCL process group): like dist_multisplit, but the
    exchange IS the post-scan kernel (ms_dist_run_fused into symmetric-memory windows).  Returns
    (keys_window, vals_window, window_start); the windows are copies the caller owns."""
    import torch.distributed as dist
    P = dist.get_world_size(group)
    n = keys.numel()
    key = (id(group), keys.device.index, vals is not None, spec.kind, spec.m, spec.shift, spec.delta,
           tuple(spec.splitters or ()))
    ent = _FUSED.get(key)
    if ent is None or ent[0] < n:
        comm = ent[1].comm if ent is not None else NcclComm(group, keys.device.index)
        # every rank sizes for the largest shard (max over ranks) and the global total
        import torch
        t = torch.tensor([n, n], dtype=torch.int64, device=keys.device)
        dist.all_reduce(t[:1], op=dist.ReduceOp.MAX, group=group)
        dist.all_reduce(t[1:], op=dist.ReduceOp.SUM, group=group)
        cap_local, total = int(t[0]), int(t[1])
        ent = _FUSED[key] = (cap_local, comm, FusedDistPlan(spec, comm, cap_local, max(total, cap_local * P),
                                                            vals is not None, group))
    k, v, _, w0 = ent[2].run(keys, vals)
    return k, v, w0


# ---------------------------------------------------------------------------
# ms_dist_run (include/ms.h): the whole sharded multisplit as one native collective call over an
# NCCL communicator that libms bootstraps itself (the 128-byte unique id is broadcast over the torch
# process group).  The count all-gather, the count differencing, the piece planning and the grouped
# NCCL send/recv all run inside libms.so.
class NcclComm:
    """An ncclComm_t for ms_dist_run, one per rank of `group` (collective constructor)."""

    def __init__(self, group=None, device=None):
        import torch
        import torch.distributed as dist
        self.rank = dist.get_rank(group)
        self.nranks = dist.get_world_size(group)
        self.device = torch.cuda.current_device() if device is None else int(device)
        uid = ctypes.create_string_buffer(128)
        if self.rank == 0:
            check(_abi.lib().ms_nccl_get_unique_id(uid), "ms_nccl_get_unique_id")
        box = [bytes(uid.raw) if self.rank == 0 else None]
        src = dist.get_global_rank(group, 0) if group is not None else 0
        dist.broadcast_object_list(box, src=src, group=group)
        uid = ctypes.create_string_buffer(box[0], 128)
        self._h = ctypes.c_void_p()
        check(_abi.lib().ms_nccl_comm_init(ctypes.byref(self._h), self.nranks, self.rank, uid, self.device),
              "ms_nccl_comm_init")

    @classmethod
    def single(cls, device=None):
        """A one-rank communicator (no process group needed): ms_dist_run then equals ms_run."""
        import torch
        self = cls.__new__(cls)
        self.rank, self.nranks = 0, 1
        self.device = torch.cuda.current_device() if device is None else int(device)
        uid = ctypes.create_string_buffer(128)
        check(_abi.lib().ms_nccl_get_unique_id(uid), "ms_nccl_get_unique_id")
        self._h = ctypes.c_void_p()
        check(_abi.lib().ms_nccl_comm_init(ctypes.byref(self._h), 1, 0, uid, self.device), "ms_nccl_comm_init")
        return self

    def close(self):
        if getattr(self, "_h", None):
            _abi.lib().ms_nccl_comm_destroy(self._h)
            self._h = ctypes.c_void_p()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


class DistPlan:
    """A plan + workspace + window buffers for repeated ms_dist_run calls on shards of up to
    max_local elements and a global total of up to max_total elements."""

    def __init__(self, spec, comm: NcclComm, max_local: int, max_total: int, with_values: bool = False):
        import torch
        from .api import Plan
        self.spec, self.comm = spec, comm
        self.plan = Plan(spec, max(int(max_local), 1), with_values=with_values, device=comm.device)
        b = ctypes.c_size_t()
        check(_abi.lib().ms_dist_workspace_size(self.plan._h, max(int(max_local), 1), comm.nranks, ctypes.byref(b)),
              "ms_dist_workspace_size")
        dev = torch.device("cuda", comm.device)
        self.ws = torch.empty(max(b.value, 256), dtype=torch.uint8, device=dev)
        self.cap = -(-int(max_total) // comm.nranks) + 1
        self.out_k = torch.empty(self.cap, dtype=torch.int32, device=dev)
        self.out_v = torch.empty(self.cap, dtype=torch.int32, device=dev) if with_values else None

    def run(self, keys, vals=None, ids=None, stream=None, copy_out=True):
        """Collective.  Returns (keys_window, vals_window, offsets_global u64[m+1] numpy, window_start).
        copy_out=False returns views of the reused window buffers (valid until the next run)."""
        from .api import _ptr, _stream
        offg = np.zeros(self.spec.m + 1, dtype=np.uint64)
        ws0, wl = ctypes.c_uint64(), ctypes.c_uint64()
        check(_abi.lib().ms_dist_run(self.plan._h, self.comm._h, _ptr(keys), _ptr(vals), _ptr(ids), keys.numel(),
                                     _ptr(self.out_k), _ptr(self.out_v if vals is not None else None), self.cap,
                                     offg.ctypes.data_as(ctypes.c_void_p), ctypes.byref(ws0), ctypes.byref(wl),
                                     _ptr(self.ws), self.ws.numel(), _stream(stream)), "ms_dist_run")
        k = self.out_k[:wl.value]
        v = self.out_v[:wl.value] if vals is not None else None
        if copy_out:
            k = k.clone()
            v = v.clone() if v is not None else None
        return k, v, offg, ws0.value
