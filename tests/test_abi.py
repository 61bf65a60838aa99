"""C ABI on CPU: libms.so loads, exports every symbol include/ms.h declares, and rejects bad
arguments synchronously (before any CUDA call -- these tests run without a GPU)."""
import ctypes
import os
import re

import pytest

from paper_conf_ppopp_ashkianidmo16_b200 import _abi
from paper_conf_ppopp_ashkianidmo16_b200.api import BucketSpec

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "ms.h")


def _declared():
    src = open(HEADER).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(ms_[a-z_]+)\s*\(", src)))


def test_exports_every_declared_symbol():
    L = _abi.lib()
    names = _declared()
    assert len(names) >= 10
    for name in names:
        assert hasattr(L, name), f"libms.so does not export {name}"
    assert set(names) == set(_abi.EXPORTS)


def _create(spec: BucketSpec, max_n=1 << 20, kv=0, flags=0, device=-1):
    h = ctypes.c_void_p()
    c = spec._c()
    st = _abi.lib().ms_plan_create(ctypes.byref(h), ctypes.byref(c), max_n, kv, flags, device)
    return st, h


@pytest.mark.parametrize("spec,flags", [
    (BucketSpec("lowbits", 0), 0),
    (BucketSpec("lowbits", 257), 0),
    (BucketSpec("lowbits", 3), 0),                 # reading #10: low-bit needs 2^k buckets
    (BucketSpec("lowbits", 4, shift=31), 0),       # shift + log2 m > 32
    (BucketSpec("delta", 8, delta=0), 0),
    (BucketSpec("splitters", 3, splitters=[5, 4]), 0),   # not non-decreasing
    (BucketSpec("ids", 8, id_bytes=2), 0),
    (BucketSpec("delta", 8, delta=5), 2 | 4),      # two variants forced
    (BucketSpec("delta", 8, delta=5), 4 | 8),
    (BucketSpec("delta", 8, delta=5), 2 | 8),
    (BucketSpec("delta", 8, delta=1 << 29), 16 | 2),  # ablation + forced variant
    (BucketSpec("delta", 8, delta=5), 512),        # unknown flag
    (BucketSpec("delta", 64, delta=1 << 26), 128 | 256),  # two ablations
    (BucketSpec("delta", 8, delta=1 << 29), 32 | 64),  # two ablations
])
def test_plan_create_rejects(spec, flags):
    st, h = _create(spec, flags=flags)
    assert st == _abi.MS_ERR_INVALID_ARG and not h.value


def test_plan_create_rejects_huge_n():
    st, _ = _create(BucketSpec("delta", 8, delta=5), max_n=1 << 32)
    assert st == _abi.MS_ERR_INVALID_ARG


@pytest.mark.parametrize("spec", [BucketSpec("lowbits", 1), BucketSpec("lowbits", 256, shift=24),
                                  BucketSpec("delta", 256, delta=1 << 24),
                                  BucketSpec("splitters", 3, splitters=[7, 7]),
                                  BucketSpec("ids", 256, id_bytes=4)])
def test_plan_create_accepts(spec):
    st, h = _create(spec)
    assert st == _abi.MS_OK and h.value
    _abi.lib().ms_plan_destroy(h)


@pytest.mark.parametrize("spec,flags", [
    (BucketSpec("delta", 64, delta=1 << 26), 4),   # ranged needs m <= 32, ONE m <= 64 key-only
    (BucketSpec("delta", 128, delta=1 << 25), 8),
    (BucketSpec("ids", 64, id_bytes=4), 8),        # ONE above 32 buckets: computed or u8 ids
    (BucketSpec("delta", 8, delta=5), 16),         # Direct ablation: DELTA with m * delta = 2^32 only
    (BucketSpec("delta", 64, delta=1 << 26), 16),
    (BucketSpec("ids", 8), 16),
    (BucketSpec("delta", 8, delta=5), 32),         # NW ablations: the same one bucket kind
    (BucketSpec("delta", 64, delta=1 << 26), 64),
    (BucketSpec("delta", 8, delta=5), 128),        # ballot / warp-level ablations: SHIFT kind, 2 <= m <= 256
    (BucketSpec("delta", 1, delta=1 << 31), 256),
    (BucketSpec("lowbits", 64), 256),
])
def test_plan_create_unsupported(spec, flags):
    st, h = _create(spec, flags=flags)
    assert st == _abi.MS_ERR_UNSUPPORTED and not h.value


@pytest.mark.parametrize("m", [2, 32, 64, 256])
@pytest.mark.parametrize("flag", [128, 256])
def test_ballot_warp_ablations_tile_variant(m, flag):
    """MS_ABLATION_BALLOT / _WARP are accepted for the SHIFT kind at any 2 <= m <= 256 and run the
    tile variant (K1 -> K2 -> ballot K3)."""
    assert _variant(BucketSpec("delta", m, delta=(1 << 32) // m), 1 << 24, False, flags=flag) == _abi.VARIANT_TILE


def test_plan_create_device_argument():
    assert _create(BucketSpec("delta", 8, delta=5), device=-2)[0] == _abi.MS_ERR_INVALID_ARG
    st, h = _create(BucketSpec("delta", 8, delta=5), device=0)
    assert st == _abi.MS_OK
    _abi.lib().ms_plan_destroy(h)


def _variant(spec, n, kv, flags=0):
    st, h = _create(spec, max_n=1 << 28, kv=kv, flags=flags)
    assert st == _abi.MS_OK
    v = ctypes.c_int32()
    assert _abi.lib().ms_plan_geometry(h, n, None, None, ctypes.byref(v)) == _abi.MS_OK
    _abi.lib().ms_plan_destroy(h)
    return v.value


def test_variant_rule():
    """ms_plan_geometry reports the variant the run takes: ONE for key-only m <= 32;
    key-value: ranged from 8 (m <= 8), 16 (m <= 16, precomputed ids) or 65 (m <= 32) tiles per SM,
    ONE below; tile for m > 32; a MS_VARIANT_* flag always wins.  (Without a GPU the SM count is
    B200's 148.)"""
    T, ONE, RANGED, TILE = _abi.VARIANT_TILE, _abi.VARIANT_ONE, _abi.VARIANT_RANGED, _abi.VARIANT_TILE
    d8, d32, d256 = (BucketSpec("delta", 8, delta=1 << 29), BucketSpec("delta", 32, delta=1 << 27),
                     BucketSpec("delta", 256, delta=1 << 24))
    assert _variant(d8, 1 << 28, 0) == ONE and _variant(d32, 1 << 28, 0) == ONE
    assert _variant(d8, 1 << 25, 1) == RANGED and _variant(d32, 1 << 25, 1) == ONE  # 8192 tiles: 55 per SM
    assert _variant(d8, 1 << 22, 1) == ONE and _variant(d8, 1 << 23, 1) == RANGED   # 1024 / 2048 tiles
    assert _variant(d8, 1 << 28, 1) == RANGED and _variant(d32, 1 << 28, 1) == RANGED
    assert _variant(BucketSpec("ids", 32), 1 << 25, 1) == RANGED and _variant(BucketSpec("ids", 32), 1 << 23, 1) == ONE
    assert _variant(d256, 1 << 20, 0) == T and _variant(d256, 1 << 28, 1) == T
    d64 = BucketSpec("delta", 64, delta=1 << 26)  # 33..64 buckets: key-only ONE (8192-key tiles), else tile
    assert _variant(d64, 1 << 28, 0) == ONE and _variant(d64, 1000, 0) == ONE and _variant(d64, 1 << 28, 1) == T
    assert _variant(BucketSpec("delta", 33, delta=5), 1 << 24, 0) == ONE
    assert _variant(BucketSpec("ids", 64), 1 << 24, 0) == ONE
    assert _variant(BucketSpec("ids", 64, id_bytes=4), 1 << 24, 0) == T
    assert _variant(BucketSpec("delta", 65, delta=5), 1 << 24, 0) == T
    assert _variant(d64, 1 << 24, 0, 2) == T and _variant(d64, 1 << 24, 0, 8) == ONE
    for flags, want in ((2, TILE), (4, RANGED), (8, ONE)):
        assert _variant(d8, 1 << 28, 1, flags) == want and _variant(d32, 1000, 0, flags) == want
    assert _variant(d8, 1 << 20, 0, 16) == TILE      # the Direct ablation runs the tile variant


def test_geometry_and_workspace():
    L = _abi.lib()
    st, h = _create(BucketSpec("delta", 32, delta=1 << 27), max_n=1 << 28)
    for n in [1, 1 << 20, (1 << 25) + 1, 1 << 28]:
        t, nt, v = ctypes.c_uint32(), ctypes.c_uint64(), ctypes.c_int32()
        assert L.ms_plan_geometry(h, n, ctypes.byref(t), ctypes.byref(nt), ctypes.byref(v)) == 0
        assert nt.value == (n + t.value - 1) // t.value
        assert t.value % 256 == 0 and 2048 <= t.value <= 8192
        b = ctypes.c_size_t()
        assert L.ms_plan_workspace_size(h, n, ctypes.byref(b)) == 0
        assert b.value >= 32 * nt.value * 4                    # holds H (m x L u32)
        bh = ctypes.c_size_t()
        assert L.ms_plan_workspace_size_host(h, n, ctypes.byref(bh)) == 0 and bh.value >= b.value + 2 * 4 * n
    assert L.ms_plan_workspace_size(h, (1 << 28) + 1, ctypes.byref(ctypes.c_size_t())) == _abi.MS_ERR_INVALID_ARG
    L.ms_plan_destroy(h)


def test_run_argument_errors_without_gpu():
    """All of these must be refused before anything touches CUDA."""
    L = _abi.lib()
    st, h = _create(BucketSpec("delta", 8, delta=5), max_n=4096, kv=0)
    P = ctypes.c_void_p
    A, B, W = P(0x10000000), P(0x20000000), P(0x30000000)
    big = 1 << 20
    run = lambda k, v, i, ko, vo, n, off, ws, wsb: L.ms_run(h, k, v, i, ko, vo, n, off, ws, wsb, None)
    assert run(None, None, None, B, None, 100, None, W, big) == _abi.MS_ERR_INVALID_ARG      # null keys
    assert run(A, None, None, B, None, 5000, None, W, big) == _abi.MS_ERR_INVALID_ARG        # n > max_n
    assert run(P(0x10000004), None, None, B, None, 100, None, W, big) == _abi.MS_ERR_ALIGNMENT
    assert run(A, None, None, P(0x20000008), None, 100, None, W, big) == _abi.MS_ERR_ALIGNMENT
    assert run(A, None, None, P(0x10000010), None, 100, None, W, big) == _abi.MS_ERR_ALIAS    # overlaps keys_in
    assert run(A, A, None, B, B, 100, None, W, big) == _abi.MS_ERR_UNSUPPORTED             # values on KO plan
    assert run(A, A, None, B, None, 100, None, W, big) == _abi.MS_ERR_INVALID_ARG           # unpaired values
    assert run(A, None, None, B, None, 100, None, W, 16) == _abi.MS_ERR_WORKSPACE
    assert run(A, None, None, B, None, 100, None, None, big) == _abi.MS_ERR_WORKSPACE
    L.ms_plan_destroy(h)
    st, h2 = _create(BucketSpec("ids", 8, id_bytes=1), max_n=4096)
    assert L.ms_run(h2, A, None, None, B, None, 100, None, W, big, None) == _abi.MS_ERR_INVALID_ARG  # ids missing
    L.ms_plan_destroy(h2)


def test_postscan_scatter_argument_errors_without_gpu():
    """ms_postscan_scatter (fused sharded scatter) refuses bad targets before touching CUDA."""
    from paper_conf_ppopp_ashkianidmo16_b200.dist import scatter_target
    L = _abi.lib()
    P = ctypes.c_void_p
    A, B, W = P(0x10000000), P(0x20000000), P(0x30000000)
    big = 1 << 20
    st, h = _create(BucketSpec("delta", 8, delta=5), max_n=4096, kv=0)
    t = scatter_target([0x40000000, 0x50000000], None, [0, 50, 100], [0] * 8)
    call = lambda tg, n=100, k=A, g=B: L.ms_postscan_scatter(h, k, None, g, n, tg, W, big, None)
    assert call(None) == _abi.MS_ERR_INVALID_ARG                                   # no target
    assert call(ctypes.byref(t), k=None) == _abi.MS_ERR_INVALID_ARG                # null keys
    assert call(ctypes.byref(t), g=P(0x20000004)) == _abi.MS_ERR_ALIGNMENT         # misaligned G
    bad = scatter_target([0x40000000, 0], None, [0, 50, 100], [0] * 8)
    assert call(ctypes.byref(bad)) == _abi.MS_ERR_INVALID_ARG                      # non-empty window, no pointer
    bad = scatter_target([0x40000000, 0x50000004], None, [0, 50, 100], [0] * 8)
    assert call(ctypes.byref(bad)) == _abi.MS_ERR_ALIGNMENT                        # misaligned window
    bad = scatter_target([0x40000000, 0x50000000], None, [0, 60, 50], [0] * 8)
    assert call(ctypes.byref(bad)) == _abi.MS_ERR_INVALID_ARG                      # decreasing window starts
    t.nranks = 0
    assert call(ctypes.byref(t)) == _abi.MS_ERR_INVALID_ARG
    t.nranks = 9
    assert call(ctypes.byref(t)) == _abi.MS_ERR_INVALID_ARG
    L.ms_plan_destroy(h)
    for spec in (BucketSpec("delta", 64, delta=5), BucketSpec("ids", 8, id_bytes=1)):
        st, h = _create(spec, max_n=4096, kv=0)
        t = scatter_target([0x40000000], None, [0, 100], [0] * 32)
        assert L.ms_postscan_scatter(h, A, None, B, 100, ctypes.byref(t), W, big, None) == _abi.MS_ERR_UNSUPPORTED
        L.ms_plan_destroy(h)


def test_status_strings():
    for s in [0, -1, -2, -3, -4, -5, -6, -8]:
        assert _abi.status_string(s) and _abi.status_string(s) != "unknown status"


def test_product_path_has_no_oracle_or_fallback():
    """The product package never imports the oracle and has no CPU fallback."""
    pkg = os.path.join(ROOT, "paper_conf_ppopp_ashkianidmo16_b200")
    for dirpath, _, files in os.walk(pkg):
        for f in files:
            if f.endswith((".py", ".cu", ".cuh", ".h", ".cpp")):
                src = open(os.path.join(dirpath, f)).read()
                assert "import oracle" not in src and "from oracle" not in src and "liboracle" not in src, f


def test_dist_run_argument_errors_without_gpu():
    """ms_dist_run / the NCCL bootstrap refuse bad arguments before touching NCCL or CUDA."""
    L = _abi.lib()
    st, h = _create(BucketSpec("delta", 8, delta=5), max_n=4096)
    P = ctypes.c_void_p
    A, B, W = P(0x10000000), P(0x20000000), P(0x30000000)
    assert L.ms_dist_run(h, None, A, None, None, 100, B, None, 100, None, None, None, W, 1 << 20, None) == \
        _abi.MS_ERR_INVALID_ARG                                                   # no communicator
    assert L.ms_dist_run(h, P(0x40000000), A, A, None, 100, B, None, 100, None, None, None, W, 1 << 20, None) == \
        _abi.MS_ERR_INVALID_ARG                                                   # unpaired values
    assert L.ms_dist_run(h, P(0x40000000), A, A, None, 100, B, B, 100, None, None, None, W, 1 << 20, None) == \
        _abi.MS_ERR_UNSUPPORTED                                                   # values on a key-only plan
    b = ctypes.c_size_t()
    assert L.ms_dist_workspace_size(h, 4096, 4, ctypes.byref(b)) == _abi.MS_OK
    ws = ctypes.c_size_t()
    assert L.ms_plan_workspace_size(h, 4096, ctypes.byref(ws)) == _abi.MS_OK
    assert b.value >= ws.value + 4096 * 4 + 4 * 8 * 8                             # staging + counts
    assert L.ms_dist_workspace_size(h, 4096, 0, ctypes.byref(b)) == _abi.MS_ERR_INVALID_ARG
    wins = (ctypes.c_void_p * 1)(B)
    assert L.ms_dist_run_fused(h, None, A, None, 100, wins, None, 100, None, None, None, W, 1 << 20, None) == \
        _abi.MS_ERR_INVALID_ARG                                                   # no communicator
    assert L.ms_dist_run_fused(h, P(0x40000000), A, A, 100, wins, wins, 100, None, None, None, W, 1 << 20,
                               None) == _abi.MS_ERR_UNSUPPORTED                   # values on a key-only plan
    assert L.ms_dist_workspace_size_fused(h, 4096, 9, ctypes.byref(b)) == _abi.MS_ERR_INVALID_ARG  # > 8 ranks
    assert L.ms_dist_workspace_size_fused(h, 4096, 4, ctypes.byref(b)) == _abi.MS_OK
    cm = ctypes.c_void_p()
    assert L.ms_nccl_comm_init(ctypes.byref(cm), 2, 2, A, 0) == _abi.MS_ERR_INVALID_ARG   # rank >= nranks
    assert L.ms_nccl_comm_init(None, 2, 0, A, 0) == _abi.MS_ERR_INVALID_ARG
    assert L.ms_nccl_get_unique_id(None) == _abi.MS_ERR_INVALID_ARG
    spec = _abi.ms_bucket_spec()
    kv = ctypes.c_int32()
    assert L.ms_plan_spec(h, ctypes.byref(spec), ctypes.byref(kv)) == _abi.MS_OK
    assert spec.m == 8 and spec.delta == 5 and kv.value == 0
    L.ms_plan_destroy(h)


def test_wide_plans_without_gpu():
    """m in (256, 65536] (two-pass plans): accepted kinds, rejected ones, geometry and
    workspace (both pass temporaries)."""
    L = _abi.lib()
    for spec, kv in ((BucketSpec("lowbits", 65536), 0), (BucketSpec("delta", 1000, delta=4000037), 1),
                     (BucketSpec("delta", 300, delta=1 << 20), 0), (BucketSpec("ids", 4096, id_bytes=4), 1)):
        st, h = _create(spec, max_n=1 << 20, kv=kv)
        assert st == _abi.MS_OK, spec.kind
        v, b = ctypes.c_int32(), ctypes.c_size_t()
        assert L.ms_plan_geometry(h, 1 << 20, None, None, ctypes.byref(v)) == 0 and v.value == _abi.VARIANT_WIDE
        assert L.ms_plan_workspace_size(h, 1 << 20, ctypes.byref(b)) == 0
        assert b.value >= (1 << 20) * 4 * (1 + kv + (2 if spec.kind == "ids" else 0))
        P = ctypes.c_void_p
        # the stage-wise calls are for plans of m <= 256
        assert L.ms_prescan(h, P(0x10000000), P(0x20000000) if spec.kind == "ids" else None, 100, P(0x30000000),
                            P(0x40000000), 1 << 30, None) == _abi.MS_ERR_UNSUPPORTED
        L.ms_plan_destroy(h)
    assert _create(BucketSpec("lowbits", 65537 + 65535))[0] == _abi.MS_ERR_INVALID_ARG      # m > 65536
    assert _create(BucketSpec("delta", 65537, delta=3))[0] == _abi.MS_ERR_INVALID_ARG
    assert _create(BucketSpec("splitters", 300, splitters=list(range(299))))[0] == _abi.MS_ERR_UNSUPPORTED
    assert _create(BucketSpec("ids", 300, id_bytes=1))[0] == _abi.MS_ERR_UNSUPPORTED
    assert _create(BucketSpec("delta", 1000, delta=5), flags=2)[0] == _abi.MS_ERR_UNSUPPORTED
    assert _create(BucketSpec("lowbits", 1024, shift=23))[0] == _abi.MS_ERR_INVALID_ARG     # shift + log2 m > 32


def _build_c_example():
    import subprocess
    import tempfile
    out = os.path.join(tempfile.mkdtemp(), "c_multisplit")
    libdir = os.path.join(ROOT, "paper_conf_ppopp_ashkianidmo16_b200")
    cmd = ["gcc", "-O2", "-I", os.path.join(ROOT, "include"), "-I", "/usr/local/cuda/include",
           os.path.join(ROOT, "examples", "c_multisplit.c"), "-L", libdir, "-lms", "-L", "/usr/local/cuda/lib64",
           "-lcudart", f"-Wl,-rpath,{libdir}", "-o", out]
    subprocess.run(cmd, check=True, capture_output=True)
    return out


def test_c_example_builds():
    """The C ABI is usable from plain C: examples/c_multisplit.c compiles and links against libms.so."""
    assert os.path.exists(_build_c_example())


@pytest.mark.gpu
def test_c_example_runs():
    """examples/c_multisplit.c on the GPU: the invariants of a stable multisplit hold (its own check,
    no oracle, no Python on the data path)."""
    import subprocess
    exe = _build_c_example()
    for n, m in ((1 << 24) + 77, 16), ((1 << 20) + 3, 256), (5, 3):
        r = subprocess.run([exe, str(n), str(m)], capture_output=True, text=True, timeout=300)
        assert r.returncode == 0 and "C ABI OK" in r.stdout, r.stdout + r.stderr
