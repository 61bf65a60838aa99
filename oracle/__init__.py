"""CPU oracle for the stable multisplit -- TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py`` (its
``cpu_baseline`` leg and ``--impl reference``) may import this package.  The
product package ``paper_conf_ppopp_ashkianidmo16_b200`` never imports it, and
the two share no code: the oracle is ``oracle.c`` (plain serial C, see its
header for the PAPER.md passages it follows) plus the pure-Python simulator of
the paper's warp procedures in ``warp_sim.py``.

Parity is pinned for every function here (tests/test_oracle.py); nothing is
"parity unpinned".
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

HERE = os.path.dirname(os.path.abspath(__file__))
SRC = os.path.join(HERE, "oracle.c")
LIB = os.path.join(HERE, "liboracle.so")

LOWBITS, DELTA, SPLITTERS, IDS = 0, 1, 2, 3
KIND_NAMES = {"lowbits": LOWBITS, "delta": DELTA, "splitters": SPLITTERS, "ids": IDS}

_lib = None


def build(force: bool = False) -> str:
    """Compile liboracle.so with gcc -O2 (serial, no OpenMP)."""
    if force or not os.path.exists(LIB) or os.path.getmtime(LIB) < os.path.getmtime(SRC):
        tmp = LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-std=c11", "-shared", "-fPIC", "-o", tmp, SRC])
        os.replace(tmp, LIB)
    return LIB


def lib():
    global _lib
    if _lib is None:
        build()
        L = ctypes.CDLL(LIB)
        P, U32, U64, I32 = ctypes.c_void_p, ctypes.c_uint32, ctypes.c_uint64, ctypes.c_int
        L.oracle_multisplit.argtypes = [I32, U32, U32, U32, P, P, U32, P, P, U64, P, P, P]
        L.oracle_multisplit.restype = I32
        L.oracle_bucket_ids.argtypes = [I32, U32, U32, U32, P, P, U32, P, U64, P]
        L.oracle_bucket_ids.restype = ctypes.c_int64
        L.oracle_tile_matrices.argtypes = [P, U64, U32, U64, P, P]
        L.oracle_tile_matrices.restype = I32
        L.oracle_threads.restype = I32
        _lib = L
    return _lib


def _ptr(a):
    return None if a is None else a.ctypes.data_as(ctypes.c_void_p)


class Spec:
    """Bucket spec mirror for the oracle (kept independent of the product's)."""

    def __init__(self, kind, m, shift=0, delta=1, splitters=None, id_bytes=1):
        self.kind = KIND_NAMES[kind] if isinstance(kind, str) else int(kind)
        self.m = int(m)
        self.shift = int(shift)
        self.delta = int(delta)
        self.splitters = None if splitters is None else np.ascontiguousarray(splitters, dtype=np.uint32)
        self.id_bytes = int(id_bytes)

    def _args(self):
        return (self.kind, self.m, self.shift, self.delta, _ptr(self.splitters))


def bucket_ids(spec: Spec, keys=None, ids=None, n=None) -> np.ndarray:
    """ids[i] = whatBucket(keys[i]) as uint32; raises if an id is >= m."""
    n = len(keys) if keys is not None else len(ids)
    keys = None if keys is None else np.ascontiguousarray(keys, dtype=np.uint32)
    if ids is not None:
        ids = np.ascontiguousarray(ids, dtype=np.uint8 if spec.id_bytes == 1 else np.uint32)
    out = np.empty(n, dtype=np.uint32)
    r = lib().oracle_bucket_ids(*spec._args(), _ptr(ids), spec.id_bytes, _ptr(keys), n, _ptr(out))
    if r >= 0:
        raise ValueError(f"bucket id out of range at index {r}")
    return out


def multisplit(spec: Spec, keys, vals=None, ids=None):
    """Stable multisplit (Eq. 1). Returns (keys_out, vals_out or None, offsets[m+1] uint64)."""
    keys = np.ascontiguousarray(keys, dtype=np.uint32)
    n = len(keys)
    if vals is not None:
        vals = np.ascontiguousarray(vals, dtype=np.uint32)
    if ids is not None:
        ids = np.ascontiguousarray(ids, dtype=np.uint8 if spec.id_bytes == 1 else np.uint32)
    ko = np.empty(n, dtype=np.uint32)
    vo = np.empty(n, dtype=np.uint32) if vals is not None else None
    off = np.empty(spec.m + 1, dtype=np.uint64)
    r = lib().oracle_multisplit(*spec._args(), _ptr(ids), spec.id_bytes, _ptr(keys), _ptr(vals), n,
                                _ptr(ko), _ptr(vo), _ptr(off))
    if r != 0:
        raise ValueError("oracle_multisplit failed (bucket id out of range?)")
    return ko, vo, off


def tile_matrices(ids_u32, m: int, T: int):
    """Eq. (2) H and G (bucket-major, m x L uint32) for subproblems of T elements."""
    ids_u32 = np.ascontiguousarray(ids_u32, dtype=np.uint32)
    n = len(ids_u32)
    L = (n + T - 1) // T
    H = np.empty(m * L, dtype=np.uint32)
    G = np.empty(m * L, dtype=np.uint32)
    if lib().oracle_tile_matrices(_ptr(ids_u32), n, m, T, _ptr(H), _ptr(G)) != 0:
        raise MemoryError
    return H.reshape(m, L), G.reshape(m, L)


def threads() -> int:
    return int(lib().oracle_threads())
