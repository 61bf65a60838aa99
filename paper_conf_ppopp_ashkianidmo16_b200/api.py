"""Python surface of the B200 multisplit: same names as the C ABI (include/ms.h).

PyTorch is plumbing here (device memory, streams); every step of the
multisplit runs in libms.so's kernels.  Tensors are 4-byte (torch.int32 or
torch.uint32, treated as uint32 bit patterns), contiguous, on the GPU.
"""
from __future__ import annotations

import ctypes

from . import _abi
from ._abi import check

KINDS = {"lowbits": _abi.MS_LOWBITS, "delta": _abi.MS_DELTA, "splitters": _abi.MS_SPLITTERS,
         "ids": _abi.MS_IDS}


class BucketSpec:
    """whatBucket() as one of four kinds (readings 7-11)."""

    def __init__(self, kind: str, m: int, shift: int = 0, delta: int = 1, splitters=None, id_bytes: int = 1):
        self.kind = kind
        self.m = int(m)
        self.shift = int(shift)
        self.delta = int(delta)
        self.splitters = None if splitters is None else [int(x) for x in splitters]
        self.id_bytes = int(id_bytes)

    @classmethod
    def lowbits(cls, m, shift=0):
        return cls("lowbits", m, shift=shift)

    @classmethod
    def delta_range(cls, m, delta):
        return cls("delta", m, delta=delta)

    @classmethod
    def from_splitters(cls, splitters):
        s = [int(x) for x in splitters]
        return cls("splitters", len(s) + 1, splitters=s)

    @classmethod
    def precomputed(cls, m, id_bytes=1):
        return cls("ids", m, id_bytes=id_bytes)

    def _c(self):
        spec = _abi.ms_bucket_spec()
        spec.kind = KINDS[self.kind]
        spec.m = self.m
        spec.shift = self.shift
        spec.delta = self.delta & 0xFFFFFFFF
        spec.id_bytes = self.id_bytes
        self._keep = None
        if self.splitters is not None:
            arr = (ctypes.c_uint32 * max(1, len(self.splitters)))(*[x & 0xFFFFFFFF for x in self.splitters])
            self._keep = arr
            spec.splitters = ctypes.cast(arr, ctypes.POINTER(ctypes.c_uint32))
        return spec


def _ptr(t):
    return None if t is None else ctypes.c_void_p(t.data_ptr())


def _stream(stream):
    import torch
    if stream is None:
        stream = torch.cuda.current_stream()
    return ctypes.c_void_p(stream.cuda_stream)


def _check_tensor(t, name):
    import torch
    if t is None:
        return
    if not t.is_cuda:
        raise ValueError(f"{name} must be a CUDA tensor")
    if not t.is_contiguous():
        raise ValueError(f"{name} must be contiguous")


VARIANT_FLAGS = {None: 0, "3k": _abi.MS_VARIANT_3K, "tile": _abi.MS_VARIANT_3K, "ranged": _abi.MS_VARIANT_RANGED,
                 "one": _abi.MS_VARIANT_ONE, "direct": _abi.MS_ABLATION_DIRECT, "nw2": _abi.MS_ABLATION_NW2,
                 "nw4": _abi.MS_ABLATION_NW4, "ballot": _abi.MS_ABLATION_BALLOT, "warp": _abi.MS_ABLATION_WARP}


class Plan:
    """ms_plan_t with a cached device workspace.

    variant: None (chosen per run), "3k"/"tile", "ranged", "one" (MS_VARIANT_*), or an
    ablation: "direct", "nw2", "nw4", "ballot", "warp" (MS_ABLATION_*, include/ms.h).  device: CUDA
    ordinal (None = the current device)."""

    def __init__(self, spec: BucketSpec, max_n: int, with_values: bool = False, validate: bool = False,
                 variant: str | None = None, device: int | None = None):
        L = _abi.lib()
        if variant not in VARIANT_FLAGS:
            raise ValueError(f"unknown variant {variant!r}")
        flags = (_abi.MS_VALIDATE if validate else 0) | VARIANT_FLAGS[variant]
        self.spec = spec
        self.max_n = int(max_n)
        self.with_values = bool(with_values)
        self._h = ctypes.c_void_p()
        c = spec._c()
        check(L.ms_plan_create(ctypes.byref(self._h), ctypes.byref(c), self.max_n, int(with_values), flags,
                               -1 if device is None else int(device)), "ms_plan_create")
        self._ws = None

    def __del__(self):
        try:
            if self._h:
                _abi.lib().ms_plan_destroy(self._h)
                self._h = ctypes.c_void_p()
        except Exception:
            pass

    # ---------------------------------------------------------------- sizes
    def workspace_size(self, n: int) -> int:
        b = ctypes.c_size_t()
        check(_abi.lib().ms_plan_workspace_size(self._h, int(n), ctypes.byref(b)), "ms_plan_workspace_size")
        return b.value

    def workspace_size_host(self, n: int) -> int:
        b = ctypes.c_size_t()
        check(_abi.lib().ms_plan_workspace_size_host(self._h, int(n), ctypes.byref(b)),
              "ms_plan_workspace_size_host")
        return b.value

    def geometry(self, n: int):
        t, L, v = ctypes.c_uint32(), ctypes.c_uint64(), ctypes.c_int32()
        check(_abi.lib().ms_plan_geometry(self._h, int(n), ctypes.byref(t), ctypes.byref(L), ctypes.byref(v)),
              "ms_plan_geometry")
        return t.value, L.value, v.value

    def workspace(self, n: int, host: bool = False):
        import torch
        need = self.workspace_size_host(n) if host else self.workspace_size(n)
        if self._ws is None or self._ws.numel() < need:
            self._ws = torch.empty(max(need, 256), dtype=torch.uint8, device="cuda")
        return self._ws

    def last_launches(self) -> int:
        return int(_abi.lib().ms_plan_last_launches(self._h))

    def trace(self, enable=True):
        """ms_plan_trace: record CUDA events on every following run -- per stage
        (True / 1; kernels then launch without PDL) or whole run only ("run" / 2)."""
        mode = 2 if enable == "run" else int(bool(enable)) if not isinstance(enable, int) else enable
        check(_abi.lib().ms_plan_trace(self._h, mode), "ms_plan_trace")

    def trace_read(self, max_runs: int = 100000):
        """ms_plan_trace_read -> list of [stage0_ms, stage1_ms, stage2_ms, total_ms] per traced run."""
        import numpy as np
        buf = np.zeros(4 * max_runs, dtype=np.float32)
        runs, stages = ctypes.c_int32(), ctypes.c_int32()
        check(_abi.lib().ms_plan_trace_read(self._h, buf.ctypes.data_as(ctypes.c_void_p), max_runs,
                                            ctypes.byref(runs), ctypes.byref(stages)), "ms_plan_trace_read")
        return buf[:4 * runs.value].reshape(runs.value, 4).tolist()

    # ---------------------------------------------------------------- run
    def run(self, keys, vals=None, ids=None, keys_out=None, vals_out=None, offsets=None,
            want_offsets: bool = True, workspace=None, stream=None):
        """ms_run: returns (keys_out, vals_out, offsets[m+1] u32 as int32 tensor)."""
        import torch
        n = keys.numel()
        for t, nm in ((keys, "keys"), (vals, "vals"), (ids, "ids")):
            _check_tensor(t, nm)
        if keys_out is None:
            keys_out = torch.empty_like(keys)
        if vals is not None and vals_out is None:
            vals_out = torch.empty_like(vals)
        if offsets is None and want_offsets:
            offsets = torch.empty(self.spec.m + 1, dtype=torch.int32, device=keys.device)
        ws = self.workspace(n) if workspace is None else workspace
        check(_abi.lib().ms_run(self._h, _ptr(keys), _ptr(vals), _ptr(ids), _ptr(keys_out), _ptr(vals_out), n,
                                _ptr(offsets), _ptr(ws), ws.numel(), _stream(stream)), "ms_run")
        return keys_out, vals_out, offsets

    def run_host(self, keys, vals=None, ids=None, keys_out=None, vals_out=None, offsets=None,
                 workspace=None, stream=None):
        """ms_run_host over host (ideally pinned) CPU tensors; the stream is synchronised before return."""
        import torch
        n = keys.numel()
        if keys_out is None:
            keys_out = torch.empty_like(keys)
        if vals is not None and vals_out is None:
            vals_out = torch.empty_like(vals)
        if offsets is None:
            offsets = torch.empty(self.spec.m + 1, dtype=torch.int32)
        ws = self.workspace(n, host=True) if workspace is None else workspace
        s = torch.cuda.current_stream() if stream is None else stream
        check(_abi.lib().ms_run_host(self._h, _ptr(keys), _ptr(vals), _ptr(ids), _ptr(keys_out), _ptr(vals_out),
                                     n, _ptr(offsets), _ptr(ws), ws.numel(), _stream(s)), "ms_run_host")
        s.synchronize()
        return keys_out, vals_out, offsets

    # ---------------------------------------------------------------- stages
    def prescan(self, keys, ids=None, H=None, workspace=None, stream=None):
        import torch
        n = keys.numel()
        _, L, _ = self.geometry(n)
        if H is None:
            H = torch.empty(self.spec.m * L, dtype=torch.int32, device=keys.device)
        ws = self.workspace(n) if workspace is None else workspace
        check(_abi.lib().ms_prescan(self._h, _ptr(keys), _ptr(ids), n, _ptr(H), _ptr(ws), ws.numel(),
                                    _stream(stream)), "ms_prescan")
        return H

    def scan(self, HG, n, offsets=None, workspace=None, stream=None):
        ws = self.workspace(n) if workspace is None else workspace
        check(_abi.lib().ms_scan(self._h, _ptr(HG), int(n), _ptr(offsets), _ptr(ws), ws.numel(), _stream(stream)),
              "ms_scan")
        return HG

    def postscan(self, keys, G, vals=None, ids=None, keys_out=None, vals_out=None, workspace=None, stream=None):
        import torch
        n = keys.numel()
        if keys_out is None:
            keys_out = torch.empty_like(keys)
        if vals is not None and vals_out is None:
            vals_out = torch.empty_like(vals)
        ws = self.workspace(n) if workspace is None else workspace
        check(_abi.lib().ms_postscan(self._h, _ptr(keys), _ptr(vals), _ptr(ids), _ptr(G), _ptr(keys_out),
                                     _ptr(vals_out), n, _ptr(ws), ws.numel(), _stream(stream)), "ms_postscan")
        return keys_out, vals_out

    def postscan_scatter(self, keys, G, target, vals=None, workspace=None, stream=None):
        """ms_postscan_scatter: K3 storing every run into its owners' windows (`target`: an
        _abi.ms_scatter_target with window pointers valid on this GPU)."""
        n = keys.numel()
        ws = self.workspace(n) if workspace is None else workspace
        check(_abi.lib().ms_postscan_scatter(self._h, _ptr(keys), _ptr(vals), _ptr(G), n, ctypes.byref(target),
                                             _ptr(ws), ws.numel(), _stream(stream)), "ms_postscan_scatter")

    def bucket_ids(self, keys, out=None, stream=None):
        import torch
        if out is None:
            out = torch.empty_like(keys)
        check(_abi.lib().ms_bucket_ids(self._h, _ptr(keys), keys.numel(), _ptr(out), _stream(stream)),
              "ms_bucket_ids")
        return out

    def check(self, workspace=None, stream=None) -> int:
        """ms_plan_check: 0 if fine, MS_ERR_BUCKET_RANGE if the last run saw an id >= m."""
        ws = self._ws if workspace is None else workspace
        return int(_abi.lib().ms_plan_check(self._h, _ptr(ws), _stream(stream)))


def multisplit(keys, vals=None, spec: BucketSpec | None = None, ids=None, validate: bool = False):
    """One-shot stable multisplit of CUDA tensors: (keys_out, vals_out, offsets[m+1])."""
    plan = Plan(spec, max(1, keys.numel()), with_values=vals is not None, validate=validate)
    out = plan.run(keys, vals, ids)
    if validate and plan.check() != _abi.MS_OK:
        raise _abi.MultisplitError(_abi.MS_ERR_BUCKET_RANGE, "multisplit")
    return out
