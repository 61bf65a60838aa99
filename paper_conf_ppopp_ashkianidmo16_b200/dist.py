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
