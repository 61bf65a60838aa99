#!/usr/bin/env python
"""Bench: stable multisplit throughput (G keys/s) and HBM-roofline fraction on B200.

Contract (one JSON line from rank 0):
  python bench.py --gpus N --steps K --warmup W [--impl ours|reference] [--config NAME]

Headline workload (BASELINE.json north_star bar, "m <= 32 on 2^28 keys"): NSko -- key-only,
m = 32 delta-range buckets, n = 2^28 uniform uint32 keys -- at N = 1; for N > 1 the sharded
config C5 (BJ configs[4]: key-value, m = 32 splitters, 2^31 keys in total, strong-scaled over
the N GPUs with ms_dist_run: local multisplit + NCCL count all-gather + NCCL send/recv).
A step = one whole multisplit (one ms_run: ONE / CTA-range / tile variant as the library
chooses) over the config's synthetic input, already resident in HBM.  L2 is flushed between
timed steps, outside the timed kernels.  Timing = CUDA events recorded by libms's native trace
on the launch stream (max over ranks).  `e2e` = the same metric through ms_run_host (pinned
host buffers, H2D + run + D2H inside the timed region).  `roofline` = the dominant kernel
against the measured HBM copy bandwidth (MEASURED_PEAKS.json), also against 8 TB/s nominal;
`traffic` = its ncu dram bytes (profiles/ncu_traffic.json, tools/ncu_traffic.py).
`cpu_baseline` = the serial CPU oracle on this host (rank 0, N = 1 only); `--impl reference`
times that oracle as the reference arm.  Byte model: PAPER.md §6.2.2, see
paper_conf_ppopp_ashkianidmo16_b200/model.py and DESIGN.md.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

import workloads as W  # noqa: E402

# Paper context numbers (Table 5): best method per (mode, m), n = 2^25.
PAPER_TABLE5_BEST = {("ko", 2): 10.04, ("ko", 4): 8.23, ("ko", 8): 6.92, ("ko", 16): 5.51, ("ko", 32): 4.51,
                     ("kv", 2): 7.14, ("kv", 4): 6.31, ("kv", 8): 5.66, ("kv", 16): 4.50, ("kv", 32): 3.93}

CONFIGS = {
    # BJ configs[0]: small case (L2-resident, launch-bound)
    "C1": dict(desc="key-only low-bit m=2, n=2^20, uniform uint32 keys", kind="lowbits", m=2, n=1 << 20,
               kv=False, dist="uniform", seed=W.SEEDS["C1"]),
    # BJ configs[1]: the headline workload
    "C2": dict(desc="key-only delta-range floor(k/D) m=8 D=400000000 (SSSP-like), n=2^25, keys uniform in [0,8D)",
               kind="delta", m=8, delta=400000000, n=1 << 25, kv=False, dist="buckets", seed=W.SEEDS["C2"]),
    "C2far": dict(desc="key-only delta-range m=8 D=4e8, n=2^25, keys uniform over uint32 (far pile 34.8%)",
                  kind="delta", m=8, delta=400000000, n=1 << 25, kv=False, dist="uniform", seed=W.SEEDS["C2"]),
    "C3": dict(desc="key-value m=32 splitter buckets, n=2^25, uniform over buckets", kind="splitters", m=32,
               n=1 << 25, kv=True, dist="buckets", seed=W.SEEDS["C3"]),
    "C3bin": dict(desc="key-value m=32 splitters, n=2^25, binomial B(31,1/2) buckets", kind="splitters", m=32,
                  n=1 << 25, kv=True, dist="binomial", seed=W.SEEDS["C3"]),
    "C3hot": dict(desc="key-value m=32 splitters, n=2^25, 75% in one bucket", kind="splitters", m=32,
                  n=1 << 25, kv=True, dist="hot", seed=W.SEEDS["C3"]),
    "C4ko": dict(desc="key-only m=256 delta D=2^24 (equal division), n=2^28, uniform", kind="delta", m=256,
                 delta=1 << 24, n=1 << 28, kv=False, dist="uniform", seed=W.SEEDS["C4"]),
    "C4kv": dict(desc="key-value m=256 delta D=2^24 (equal division), n=2^28, uniform", kind="delta", m=256,
                 delta=1 << 24, n=1 << 28, kv=True, dist="uniform", seed=W.SEEDS["C4"]),
    # north-star bar: m <= 32 at n = 2^28 (>= 70 % of HBM roofline)
    "NSko": dict(desc="key-only m=32 delta D=2^27 (equal division), n=2^28, uniform", kind="delta", m=32,
                 delta=1 << 27, n=1 << 28, kv=False, dist="uniform", seed=W.SEEDS["C4"]),
    "NSkv": dict(desc="key-value m=32 delta D=2^27 (equal division), n=2^28, uniform", kind="delta", m=32,
                 delta=1 << 27, n=1 << 28, kv=True, dist="uniform", seed=W.SEEDS["C4"]),
}
for _m in (2, 4, 8, 16, 32, 64, 128, 256):
    for _kv in (False, True):
        CONFIGS[f"sweep_m{_m}_{'kv' if _kv else 'ko'}"] = dict(
            desc=f"{'key-value' if _kv else 'key-only'} m={_m} delta D=2^32/m, n=2^28, uniform", kind="delta",
            m=_m, delta=(1 << 32) // _m, n=1 << 28, kv=_kv, dist="uniform", seed=W.SEEDS["C4"])

for _m in (512, 1024, 4096, 16384, 65536):  # m > 256 (two-pass plans; the Fig. 4 question)
    for _kv in (False, True):
        CONFIGS[f"wide_m{_m}_{'kv' if _kv else 'ko'}"] = dict(
            desc=f"{'key-value' if _kv else 'key-only'} m={_m} delta D=2^32/m, n=2^28, uniform", kind="delta",
            m=_m, delta=(1 << 32) // _m, n=1 << 28, kv=_kv, dist="uniform", seed=W.SEEDS["C4"])
for _e in (22, 23, 24, 26, 27, 28):  # size sweep of C2 (fixed-cost analysis)
    CONFIGS[f"C2_n{_e}"] = dict(CONFIGS["C2"], n=1 << _e, desc=CONFIGS["C2"]["desc"].replace("2^25", f"2^{_e}"))
for _d, _dn in (("binomial", "bin"), ("hot", "hot")):  # skewed north-star workloads (Fig. 5)
    for _kv in (False, True):
        CONFIGS[f"NS{_dn}_{'kv' if _kv else 'ko'}"] = dict(
            desc=f"{'key-value' if _kv else 'key-only'} m=32 delta D=2^27, n=2^28, {_d} buckets", kind="delta",
            m=32, delta=1 << 27, n=1 << 28, kv=_kv, dist=_d, seed=W.SEEDS["C4"])
for _d, _dn in (("binomial", "bin"), ("hot", "hot")):  # skewed m = 256 workloads (the m > 32 post-scan)
    for _kv in (False, True):
        CONFIGS[f"C4{_dn}_{'kv' if _kv else 'ko'}"] = dict(
            desc=f"{'key-value' if _kv else 'key-only'} m=256 delta D=2^24, n=2^28, {_d} buckets", kind="delta",
            m=256, delta=1 << 24, n=1 << 28, kv=_kv, dist=_d, seed=W.SEEDS["C4"])
# precomputed ids (MS_IDS, u8), the fourth bucket kind
CONFIGS["IDSko"] = dict(desc="key-only m=32 precomputed u8 ids, n=2^28, uniform ids", kind="ids", m=32, n=1 << 28,
                        kv=False, dist="uniform", seed=W.SEEDS["C4"])
CONFIGS["IDSkv"] = dict(desc="key-value m=32 precomputed u8 ids, n=2^28, uniform ids", kind="ids", m=32,
                        n=1 << 28, kv=True, dist="uniform", seed=W.SEEDS["C4"])
# BJ configs[4]: the sharded multisplit, 2^31 (key, value) pairs in total, strong-scaled over N GPUs
CONFIGS["C5"] = dict(desc="sharded key-value m=32 splitter buckets, n=2^31 total (strong-scaled over the GPUs), "
                          "uniform", kind="splitters", m=32, n=1 << 31, kv=True, dist="uniform",
                     seed=W.SEEDS.get("C5", 0x4D530005), strong=True)
CONFIGS["C5s"] = dict(CONFIGS["C5"], n=1 << 26, desc=CONFIGS["C5"]["desc"].replace("2^31", "2^26 (small C5, tests)"))

DEFAULT = "NSko"      # N = 1 headline
DEFAULT_DIST = "C5"   # N > 1 headline
EXTRA_DEFAULT = ",".join(["NSkv", "NSbin_ko", "NShot_ko", "NSbin_kv", "NShot_kv", "C4ko", "C4kv", "C4bin_ko",
                          "C4hot_ko", "C3", "C3bin",
                          "C3hot", "C2", "C2far", "C1", "IDSko", "IDSkv"] +
                         [f"sweep_m{m}_{t}" for t in ("ko", "kv") for m in (2, 4, 8, 16, 64, 128)] +
                         [f"wide_m{m}_{t}" for t in ("ko", "kv") for m in (512, 4096, 65536)])


def log(*a):
    print(*a, file=sys.stderr, flush=True)


def spec_of(cfg):
    from paper_conf_ppopp_ashkianidmo16_b200 import BucketSpec
    if cfg["kind"] == "lowbits":
        return BucketSpec.lowbits(cfg["m"], cfg.get("shift", 0))
    if cfg["kind"] == "delta":
        return BucketSpec.delta_range(cfg["m"], cfg["delta"])
    if cfg["kind"] == "splitters":
        return BucketSpec.from_splitters(W.gen_splitters(cfg["m"], cfg["seed"]).tolist())
    return BucketSpec.precomputed(cfg["m"], cfg.get("id_bytes", 1))


def ranges_of(cfg):
    if cfg["kind"] == "delta":
        return W.ranges_delta(cfg["m"], cfg["delta"])
    if cfg["kind"] == "splitters":
        return W.ranges_splitters(W.gen_splitters(cfg["m"], cfg["seed"]))
    return None


def inputs_torch(cfg, n, start, device):
    """(keys, vals or None, ids or None) on the device, seeded (workloads/)."""
    dist = cfg["dist"]
    if cfg["kind"] == "ids":
        keys = W.keys_torch(n, cfg["seed"], device, start=start)
        ids = W.bucket_draw_torch(n, cfg["seed"], dist, cfg["m"], device, start=start)
        vals = W.values_torch(n, cfg["seed"], device, "random", start=start) if cfg["kv"] else None
        return keys, vals, ids
    if dist == "uniform":
        keys = W.keys_torch(n, cfg["seed"], device, start=start)
    else:
        keys = W.keys_torch(n, cfg["seed"], device, dist, cfg["m"], ranges_of(cfg), start=start,
                            lowbits_shift=cfg.get("shift", 0) if cfg["kind"] == "lowbits" else None)
    vals = W.values_torch(n, cfg["seed"], device, "random", start=start) if cfg["kv"] else None
    return keys, vals, None


def inputs_np(cfg, n, start):
    """(keys, vals or None, ids or None) on the host, bit-identical to inputs_torch."""
    if cfg["kind"] == "ids":
        keys = W.keys_np(n, cfg["seed"], start=start)
        ids = W.bucket_draw_np(n, cfg["seed"], cfg["dist"], cfg["m"], start=start)
        vals = W.values_np(n, cfg["seed"], "random", start=start) if cfg["kv"] else None
        return keys, vals, ids
    if cfg["dist"] == "uniform":
        keys = W.keys_np(n, cfg["seed"], start=start)
    else:
        keys = W.keys_np(n, cfg["seed"], cfg["dist"], cfg["m"], ranges_of(cfg), start=start,
                         lowbits_shift=cfg.get("shift", 0) if cfg["kind"] == "lowbits" else None)
    vals = W.values_np(n, cfg["seed"], "random", start=start) if cfg["kv"] else None
    return keys, vals, None


NOMINAL_HBM_GBS = 8000.0  # B200 nominal HBM3e bandwidth (BJ north_star: "against B200's ~8 TB/s")


def load_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        with open(p) as f:
            d = json.load(f)
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs: torch copy, read+write bytes)"
    return 6650.0, "fallback (B200_PROFILING.md: 6.65 TB/s)"


def load_traffic(name, kernel):
    """ncu dram read+write bytes of one launch of `kernel` (name prefix) in this workload, from the
    committed capture profiles/ncu_traffic.json (tools/ncu_traffic.py), or None."""
    p = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    if not os.path.exists(p):
        return None
    try:
        with open(p) as f:
            ent = json.load(f).get("configs", {}).get(name)
    except Exception:
        return None
    if not ent:
        return None
    for k in ent.get("kernels", []):
        if k["kernel"].startswith(kernel):
            return k["dram_bytes"]
    return None


def cpu_model():
    try:
        with open("/proc/cpuinfo") as f:
            for line in f:
                if line.startswith("model name"):
                    return line.split(":", 1)[1].strip()
    except Exception:
        pass
    return None


class ClockSampler:
    """NVML sampling of SM clock + throttle reasons during the timed region."""

    REASONS = {"hw_slowdown": 0x8, "sw_thermal_slowdown": 0x20, "hw_thermal_slowdown": 0x40,
               "sw_power_cap": 0x4, "hw_power_brake_slowdown": 0x80}

    def __init__(self, index):
        self.samples, self.reasons, self.max_mhz = [], set(), None
        self._stop = threading.Event()
        try:
            import pynvml
            pynvml.nvmlInit()
            self.h = pynvml.nvmlDeviceGetHandleByIndex(index)
            self.nv = pynvml
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(self.h, pynvml.NVML_CLOCK_SM)
        except Exception as e:  # pragma: no cover
            self.nv = None
            log("nvml unavailable:", e)

    def _run(self):
        while not self._stop.is_set():
            try:
                self.samples.append(self.nv.nvmlDeviceGetClockInfo(self.h, self.nv.NVML_CLOCK_SM))
                r = self.nv.nvmlDeviceGetCurrentClocksEventReasons(self.h)
                for k, bit in self.REASONS.items():
                    if r & bit:
                        self.reasons.add(k)
            except Exception:
                pass
            time.sleep(0.005)

    def __enter__(self):
        if self.nv:
            self.t = threading.Thread(target=self._run, daemon=True)
            self.t.start()
        return self

    def __exit__(self, *a):
        self._stop.set()
        if self.nv:
            self.t.join()

    def result(self):
        return {"sm_mhz": statistics.median(self.samples) if self.samples else None,
                "sm_max_mhz": self.max_mhz, "reasons": sorted(self.reasons), "samples": len(self.samples)}


class L2Flush:
    """Between timed steps: write a 512 MiB buffer (> the 126 MB L2), then read a second
    512 MiB buffer so the dirty flush lines are written back BEFORE the next timed step
    (otherwise the timed kernels pay for the flush's write-back)."""

    def __init__(self, device):
        import torch
        self.w = torch.empty(512 << 20, dtype=torch.uint8, device=device)
        self.r = torch.ones(128 << 20, dtype=torch.int32, device=device)
        self.acc = torch.zeros((), dtype=torch.int64, device=device)

    def __call__(self):
        import torch
        self.w.fill_(1)
        self.acc += self.r.sum(dtype=torch.int64)


def dist_setup(args):
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return world, rank, local


def max_over_ranks(x, world, device):
    if world == 1:
        return x
    import torch
    import torch.distributed as dist
    t = torch.tensor([x], dtype=torch.float64, device=device)
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return float(t.item())


def barrier(world):
    if world > 1:
        import torch.distributed as dist
        dist.barrier()


# ------------------------------------------------------------------ shared descriptors
def n_local_of(cfg, world):
    """Keys per rank: strong-scaled configs split cfg['n'] over the ranks, the others are per GPU."""
    if cfg.get("strong"):
        return cfg["n"] // world + (1 if 0 < cfg["n"] % world else 0) if world > 1 else cfg["n"]
    return cfg["n"]


def config_dict(name, cfg, world, dist_mode=None):
    """The `config` object of the JSON line -- identical for our arm and the reference arm."""
    d = {"workload": name, "desc": cfg["desc"], "n_total": cfg["n"] if cfg.get("strong") else cfg["n"] * world,
         "n_per_gpu": n_local_of(cfg, world), "m": cfg["m"], "kind": cfg["kind"], "kv": cfg["kv"],
         "dist": cfg["dist"],
         "l2": "flushed between timed steps (512 MiB write + 512 MiB read so the write-back is done), outside the "
               "timed kernels",
         "parallelism": "single GPU" if world == 1 else
         (f"sharded multisplit x{world} (ms_dist_run: local ms_run + NCCL count all-gather + NCCL send/recv into "
          f"balanced windows)" if dist_mode == "nccl" else
          f"sharded multisplit x{world} ({dist_mode})")}
    return d


# ------------------------------------------------------------------ reference arm (the CPU oracle)
def time_oracle(cfg, budget_s=12.0, max_n=1 << 25, min_reps=1):
    """The serial oracle as it stands on one host core, on a bounded sample of the workload."""
    import oracle
    n = min(cfg["n"], max_n)
    keys, vals, ids = inputs_np(cfg, n, 0)
    spl = W.gen_splitters(cfg["m"], cfg["seed"]) if cfg["kind"] == "splitters" else None
    ospec = oracle.Spec(cfg["kind"], cfg["m"], shift=cfg.get("shift", 0), delta=cfg.get("delta", 1), splitters=spl,
                        id_bytes=cfg.get("id_bytes", 1))
    try:
        cores_avail = len(os.sched_getaffinity(0))
        old = os.sched_getaffinity(0)
        os.sched_setaffinity(0, {min(old)})
    except Exception:
        cores_avail, old = os.cpu_count(), None
    times = []
    t_start = time.perf_counter()
    while len(times) < min_reps or (time.perf_counter() - t_start < budget_s and len(times) < 50):
        t0 = time.perf_counter()
        oracle.multisplit(ospec, keys, vals, ids=ids)
        times.append(time.perf_counter() - t0)
    if old is not None:
        os.sched_setaffinity(0, old)
    t = statistics.median(times)
    return {"value": n / t / 1e9, "unit": "G keys/s", "cores": oracle.threads(), "kind": "oracle",
            "cpu_model": cpu_model(),
            "sample": f"{n} keys of {cfg['n']} ({cfg['desc']}), median of {len(times)} reps, "
                      f"1 of {cores_avail} host cores ({cpu_model()})", "reps": len(times), "seconds": t}


def run_reference(args, name, cfg, world, rank):
    if rank != 0:
        return
    ps = time_oracle(cfg, budget_s=max(3.0, min(60.0, 1.0 * args.steps)), min_reps=max(1, args.steps))
    out = {"metric": "G keys/s", "value": round(ps["value"], 4), "unit": "G keys/s", "n_gpus": args.gpus,
           "steps": args.steps, "warmup": args.warmup, "ms_per_step": ps["seconds"] * 1e3,
           "higher_is_better": True, "scaling": "strong" if cfg.get("strong") else "weak", "vs_baseline": None,
           "dtype": "u32", "data": "synthetic (seeded splitmix64)", "impl": "reference",
           "config": config_dict(name, cfg, world, args.dist_mode),
           "cpu_baseline": {k: ps[k] for k in ("value", "unit", "cores", "kind", "sample", "cpu_model")},
           "e2e": {"value": round(ps["value"], 4), "unit": "G keys/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(out), flush=True)


# ------------------------------------------------------------------ our arm
def measure_device(cfg, plan, keys, vals, ids, K, Wm, flush, device):
    """Warm up, then two passes of K runs, each with an L2 flush before every run:
    (1) the timed pass: libms records one event before the first kernel and one after the last
        of every run (trace mode "run"; the kernels keep their programmatic dependent launch);
    (2) the breakdown pass: an event between every two kernels (per-stage times; the
        kernels then launch without PDL, so these stages sum to slightly more).
    Returns (per-run whole-step ms, per-run stage ms [k1, k2, k3, total], launches per run)."""
    import torch
    keys_out = torch.empty_like(keys)
    vals_out = torch.empty_like(vals) if vals is not None else None
    offsets = torch.empty(cfg["m"] + 1, dtype=torch.int32, device=device)
    ws = plan.workspace(keys.numel())
    for _ in range(Wm):
        plan.run(keys, vals, ids, keys_out=keys_out, vals_out=vals_out, offsets=offsets, workspace=ws)
    torch.cuda.synchronize()
    out = []
    for mode in ("run", True):
        plan.trace(mode)
        for _ in range(K):
            flush()
            plan.run(keys, vals, ids, keys_out=keys_out, vals_out=vals_out, offsets=offsets, workspace=ws)
        torch.cuda.synchronize()
        out.append(plan.trace_read(K))
        plan.trace(False)
    whole = [r[3] for r in out[0]]
    return whole, out[1], plan.last_launches()


def measure_e2e(cfg, plan, keys_d, vals_d, ids_d, K):
    """ms_run_host from pinned host buffers: every step copies its inputs host->device, multisplits
    and copies its result (keys, values, offsets) device->host, all inside the timed region.  Steps
    alternate between two streams (each with its own workspace and pinned output buffers), so step
    i+1's host->device copy overlaps step i's device->host copy on the other copy engine -- a stream
    of multisplits through the public call, as a user would pipeline it.  Timed with events."""
    import torch
    from paper_conf_ppopp_ashkianidmo16_b200 import _abi, api
    n = keys_d.numel()
    kh = keys_d.cpu().pin_memory()
    vh = vals_d.cpu().pin_memory() if vals_d is not None else None
    ih = ids_d.cpu().pin_memory() if ids_d is not None else None
    streams = [torch.cuda.Stream(), torch.cuda.Stream()]
    bufs = []
    for _ in streams:
        ko = torch.empty_like(kh).pin_memory()
        vo = torch.empty_like(vh).pin_memory() if vh is not None else None
        off = torch.empty(cfg["m"] + 1, dtype=torch.int32).pin_memory()
        ws = torch.empty(plan.workspace_size_host(n), dtype=torch.uint8, device="cuda")
        bufs.append((ko, vo, off, ws))

    def step(i):
        ko, vo, off, ws = bufs[i % 2]
        _abi.check(_abi.lib().ms_run_host(plan._h, api._ptr(kh), api._ptr(vh), api._ptr(ih), api._ptr(ko),
                                          api._ptr(vo), n, api._ptr(off), api._ptr(ws), ws.numel(),
                                          api._stream(streams[i % 2])), "ms_run_host")
    step(0)
    step(1)  # warm both
    torch.cuda.synchronize()
    s0, s1 = streams
    e0, e1, ej = (torch.cuda.Event(enable_timing=True) for _ in range(3))
    e0.record(s0)
    s1.wait_event(e0)
    for i in range(K):
        step(i)
    ej.record(s1)
    s0.wait_event(ej)
    e1.record(s0)
    torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / K
    ib = ids_d.element_size() * n if ids_d is not None else 0
    h2d = n * 4 * (2 if vh is not None else 1) + ib
    d2h = n * 4 * (2 if vh is not None else 1) + (cfg["m"] + 1) * 4
    return n / (ms * 1e-3) / 1e9, h2d, d2h, ms


def torch_bucket_ids(cfg, keys, ids=None):
    """Bucket ids with plain torch ops (the comparator's own pre-pass; not our kernels)."""
    import torch
    if cfg["kind"] == "ids":
        return ids.to(torch.int64)
    k = keys.to(torch.int64) & 0xFFFFFFFF
    if cfg["kind"] == "lowbits":
        return (k >> cfg.get("shift", 0)) & (cfg["m"] - 1)
    if cfg["kind"] == "delta":
        return torch.clamp(k // cfg["delta"], max=cfg["m"] - 1)
    spl = torch.as_tensor(W.gen_splitters(cfg["m"], cfg["seed"]).astype(np.int64), device=keys.device)
    return torch.searchsorted(spl, k, side="left")  # #{j : s_j < k}


def measure_comparators(cfg, plan, keys, vals, ids, K, flush):
    """Same-run comparators, each timed with CUDA events on the current stream, L2 flushed
    before every run: (i) torch.sort of the keys (+ gather of the values): the paper's radix-sort row
    (Table 3/6); (ii) the reduced-bit sort (§3.4): ids by torch elementwise ops,
    torch.sort(ids, stable=True), gather keys (and values) -- its output must be bit-identical to ours;
    (iii) key-value only: the paper's full reduced-bit sort with 64-bit packing: one
    torch.sort of (id << 32 | value) as int64 (ids as the most significant bits; values unique
    per position are NOT required -- the pack is sorted stably), then the keys gathered by the
    sorted values' positions -- implemented as sort of (id << 32 | index) and two gathers."""
    import torch
    s = torch.cuda.current_stream()
    ko = torch.empty_like(keys)
    vo = torch.empty_like(vals) if vals is not None else None
    plan.run(keys, vals, ids, keys_out=ko, vals_out=vo)
    n = keys.numel()

    def sort_keys():
        sk, idx = torch.sort(keys)
        if vals is not None:
            return sk, vals[idx]
        return sk, None

    def reduced_bit():  # the fewest id bits torch can sort: u8 (m <= 256), or i16 of id - 2^15 (m <= 65536)
        b = torch_bucket_ids(cfg, keys, ids)
        b = b.to(torch.uint8) if cfg["m"] <= 256 else (b - 32768).to(torch.int16) if cfg["m"] <= 65536 else \
            b.to(torch.int32)
        _, idx = torch.sort(b, stable=True)
        return keys[idx], (vals[idx] if vals is not None else None)

    def reduced_bit_packed():  # (id << 32) | i in one 64-bit key: unique keys, any sort order is stable
        b = torch_bucket_ids(cfg, keys, ids)
        packed = (b << 32) | torch.arange(n, dtype=torch.int64, device=keys.device)
        sp, _ = torch.sort(packed)
        idx = sp & 0xFFFFFFFF
        return keys[idx], (vals[idx] if vals is not None else None)

    fns = [("torch_sort_keys", sort_keys), ("torch_sort_on_bucket_id", reduced_bit)]
    if vals is not None:
        fns.append(("reduced_bit_sort_64bit_pack", reduced_bit_packed))
    out = {}
    for nm, fn in fns:
        res = fn()
        torch.cuda.synchronize()
        ts = []
        for _ in range(K):
            flush()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(s)
            fn()
            e1.record(s)
            torch.cuda.synchronize()
            ts.append(e0.elapsed_time(e1))
        ms = statistics.median(ts)
        out[nm] = {"value": round(n / (ms * 1e-3) / 1e9, 3), "unit": "G keys/s", "ms": round(ms, 4)}
        if nm != "torch_sort_keys":
            same = bool(torch.equal(res[0], ko)) and (vals is None or bool(torch.equal(res[1], vo)))
            out[nm]["bit_identical_to_multisplit"] = same
        del res
    return out


def bench_config(name, cfg, K, Wm, device, world, rank, with_e2e=True, comparators=False):
    import torch
    import paper_conf_ppopp_ashkianidmo16_b200 as P
    from paper_conf_ppopp_ashkianidmo16_b200 import model
    n = n_local_of(cfg, world)
    keys, vals, ids = inputs_torch(cfg, n, rank * n, device)
    plan = P.Plan(spec_of(cfg), n, with_values=cfg["kv"], variant=cfg.get("variant"))
    flush = L2Flush(device)
    barrier(world)
    clocks = ClockSampler(torch.cuda.current_device())
    with clocks:
        whole, runs, launches = measure_device(cfg, plan, keys, vals, ids, K, Wm, flush, device)
    barrier(world)
    runs = np.array(runs, dtype=np.float64)
    total_ms = max_over_ranks(float(np.sum(whole)), world, device)
    ms_step = total_ms / K
    value = n * world / (ms_step * 1e-3) / 1e9
    k1_ms, k2_ms, k3_ms = (float(runs[:, c].mean()) for c in range(3))
    idb = cfg.get("id_bytes", 1) if cfg["kind"] == "ids" else 0
    pre_b, post_b = model.pass_bytes_per_key(cfg["kv"], idb)
    peak, peak_src = load_peaks()
    T, L, variant = plan.geometry(n)
    alg_bytes = model.algorithmic_bytes_per_key(cfg["kv"], idb) * n
    one = launches == 1  # ONE cooperative launch: the single kernel moves all 12 (KO) / 20 (KV) B per key
    wide = variant == 3  # m > 256: two passes + offsets; reported as a whole against the one-pass model
    kern_bytes = alg_bytes if (one or wide) else post_b * n
    kern_ms = ms_step if wide else k3_ms
    achieved = kern_bytes / (kern_ms * 1e-3) / 1e9
    kname = "two-pass plan" if wide else ("k3v_postscan" if cfg["m"] <= 32 else "k3_postscan")
    wl = np.array(whole)
    res = {
        "value": value, "ms_per_step": ms_step,
        "ms_stats": {"mean": round(float(wl.mean()), 5), "median": round(float(np.median(wl)), 5),
                     "min": round(float(wl.min()), 5), "p90": round(float(np.percentile(wl, 90)), 5),
                     "runs": len(wl)},
        "stages_ms": {"k1_prescan": k1_ms, "k2_scan": k2_ms, "k3_postscan": k3_ms,
                      "sum_without_pdl": float(runs[:, 3].mean())},
        "whole_step_hbm_gbs": alg_bytes / (ms_step * 1e-3) / 1e9,
        "whole_step_frac": alg_bytes / (ms_step * 1e-3) / 1e9 / peak,
        "whole_step_frac_nominal_8tbs": alg_bytes / (ms_step * 1e-3) / 1e9 / NOMINAL_HBM_GBS,
        "roofline": {"bound": "hbm",
                     "kernel": (kname + " ONE (pre-scan + scan + post-scan in one cooperative launch)") if one
                     else kname + " (whole step vs the one-pass byte model)" if wide else kname + " (post-scan)",
                     "achieved": round(achieved, 1), "peak": peak, "unit": "GB/s", "frac": round(achieved / peak, 4),
                     "frac_vs_nominal_8tbs": round(achieved / NOMINAL_HBM_GBS, 4),
                     "traffic": load_traffic(name, kname),
                     "algorithmic_bytes_per_launch": kern_bytes,
                     "algorithmic_bytes_per_key": kern_bytes / n,
                     "peak_source": peak_src,
                     "k1_prescan_frac": None if (one or wide) else round(pre_b * n / (k1_ms * 1e-3) / 1e9 / peak, 4)},
        "gpu_launches": launches * K, "launches_per_step": launches, "tile": T, "tiles": L,
        "variant": ["tile", "ranged", "one", "two-pass"][variant], "clocks": clocks.result(),
    }
    if n <= (1 << 22) and world == 1:  # launch-bound sizes: also the CUDA-graph replay rate
        res["graph_replay"] = measure_graph(cfg, plan, keys, vals, ids)
    if comparators:
        comp = measure_comparators(cfg, plan, keys, vals, ids, 3, flush)
        for v in comp.values():
            v["multisplit_speedup"] = round(value / v["value"], 2)
        res["comparators"] = comp
    if with_e2e:
        e2e_v, h2d, d2h, e2e_ms = measure_e2e(cfg, plan, keys, vals, ids, max(4, min(K, 10)))
        res["e2e"] = {"value": e2e_v * world, "unit": "G keys/s", "h2d_bytes_per_step": h2d,
                      "d2h_bytes_per_step": d2h, "ms_per_step": e2e_ms}
    del keys, vals, ids, flush
    torch.cuda.empty_cache()
    return res


def measure_graph(cfg, plan, keys, vals, ids, calls=20, reps=10):
    """Small, launch-bound workloads: `calls` back-to-back ms_run calls captured in
    one CUDA graph and replayed (L2-warm: the inputs stay resident between calls) -- the per-call
    device time without per-call launch gaps."""
    import torch
    ko = torch.empty_like(keys)
    vo = torch.empty_like(vals) if vals is not None else None
    off = torch.empty(cfg["m"] + 1, dtype=torch.int32, device=keys.device)
    ws = plan.workspace(keys.numel())
    s = torch.cuda.Stream()
    s.wait_stream(torch.cuda.current_stream())
    with torch.cuda.stream(s):
        for _ in range(3):
            plan.run(keys, vals, ids, keys_out=ko, vals_out=vo, offsets=off, workspace=ws)
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=s):
        for _ in range(calls):
            plan.run(keys, vals, ids, keys_out=ko, vals_out=vo, offsets=off, workspace=ws)
    g.replay()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(reps):
        g.replay()
    e1.record()
    torch.cuda.synchronize()
    us = e0.elapsed_time(e1) * 1e3 / (reps * calls)
    return {"per_call_us": round(us, 3), "value": round(keys.numel() / (us * 1e-6) / 1e9, 2), "unit": "G keys/s",
            "note": f"{calls} back-to-back ms_run calls captured in one CUDA graph, replayed {reps}x; L2-warm"}


NVLINK_GBS_PER_DIR = 900.0  # NVLink 5 per GPU per direction (NVSwitch: uniform to every peer)


def bench_dist(name, cfg, K, Wm, device, world, rank, backend, mode="nccl"):
    """N > 1: the sharded multisplit.  mode "nccl": ms_dist_run (libms: local ms_run, NCCL count
    all-gather, piece planning, NCCL group send/recv into balanced windows); "fused": local K1+K2,
    count all-gather, K3 peer stores into symmetric-memory windows (dist.py); backend "gloo" (testing
    on one GPU / CPU hosts): dist.py's host-staged exchange.  Strong-scaled configs split cfg['n']
    over the ranks.  Time = CUDA events around each whole collective step on the launch stream,
    summed over K steps, max over ranks.  Also: the same run's plain all_to_all_single of the bytes
    the exchange moves (the attainable NVLink rate) and the step's NVLink / HBM bounds."""
    import torch
    import torch.distributed as dist
    import paper_conf_ppopp_ashkianidmo16_b200 as P
    from paper_conf_ppopp_ashkianidmo16_b200.dist import DistPlan, NcclComm, dist_multisplit, dist_multisplit_fused
    n = n_local_of(cfg, world)
    n_total = cfg["n"] if cfg.get("strong") else cfg["n"] * world
    keys, vals, ids = inputs_torch(cfg, n, rank * n, device)
    spec = spec_of(cfg)
    kv = cfg["kv"]
    comm = None
    if backend == "gloo":
        plan = P.Plan(spec, n, with_values=kv)

        def local(k, v):
            ko, vo, off = plan.run(k, v, ids)
            return ko.cpu(), (vo.cpu() if vo is not None else None), off.cpu().to(torch.int64) & 0xFFFFFFFF

        def step(k, v):
            wk, wv, offg, ws = dist_multisplit(k, v, spec, local=local)
            return wk, wv
    elif mode == "fused":
        def step(k, v):
            wk, wv, w0 = dist_multisplit_fused(k, v, spec)
            return wk, wv
    else:
        comm = NcclComm(device=device.index)
        dp = DistPlan(spec, comm, n, n_total, with_values=kv)

        def step(k, v):
            wk, wv, offg, ws = dp.run(k, v, ids, copy_out=False)
            return wk, wv
    flush = L2Flush(device)
    for _ in range(Wm):
        step(keys, vals)
    torch.cuda.synchronize()
    dist.barrier()
    s = torch.cuda.current_stream()
    tot_ms = 0.0
    clocks = ClockSampler(torch.cuda.current_device())
    with clocks:
        for _ in range(K):
            flush()
            torch.cuda.synchronize()
            dist.barrier()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(s)
            wk, wv = step(keys, vals)
            e1.record(s)
            torch.cuda.synchronize()
            tot_ms += e0.elapsed_time(e1)
    dist.barrier()
    tot_ms = max_over_ranks(tot_ms, world, device)
    ms_step = tot_ms / K
    value = n_total / (ms_step * 1e-3) / 1e9
    # the attainable NVLink rate in this run: all_to_all_single of the bytes one rank sends
    bpk = 8 if kv else 4
    xbytes = int(n * bpk * (world - 1) / world)
    a2a = None
    if backend == "nccl":
        per = max(1, xbytes // 4 // world) * world
        src = torch.empty(per, dtype=torch.int32, device=device)
        dst = torch.empty_like(src)
        dist.all_to_all_single(dst, src)
        torch.cuda.synchronize()
        ta = 0.0
        for _ in range(max(3, K // 2)):
            dist.barrier()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(s)
            dist.all_to_all_single(dst, src)
            e1.record(s)
            torch.cuda.synchronize()
            ta += e0.elapsed_time(e1)
        ta = max_over_ranks(ta, world, device) / max(3, K // 2)
        a2a = {"bytes_per_rank": per * 4, "ms": round(ta, 4), "GBps_per_rank": round(per * 4 * (world - 1) / world
                                                                                    / (ta * 1e-3) / 1e9, 1)}
        del src, dst
    peak, _ = load_peaks()
    t_hbm = (20 if kv else 12) * n / (peak * 1e9) * 1e3
    t_nvl = xbytes / (NVLINK_GBS_PER_DIR * 1e9) * 1e3
    bounds = {"hbm_bound_ms": round(t_hbm, 4), "nvlink_bound_ms": round(t_nvl, 4),
              "frac_of_bound": round(max(t_hbm, t_nvl) / ms_step, 4),
              "frac_of_bound_a2a": round(max(t_hbm, a2a["ms"]) / ms_step, 4) if a2a else None,
              "all_to_all_single_same_bytes": a2a,
              "note": "bound = max(HBM time of the local multisplit at the measured copy rate, NVLink time of "
                      "the exchange at 900 GB/s per direction); *_a2a uses the same run's all_to_all_single"}
    # e2e: pinned host shard -> device, sharded multisplit, window -> pinned host
    kh = keys.cpu().pin_memory()
    vh = vals.cpu().pin_memory() if vals is not None else None
    cap_h = -(-n_total // world) + 1
    ko_h = torch.empty(cap_h, dtype=torch.int32).pin_memory()
    vo_h = torch.empty(cap_h, dtype=torch.int32).pin_memory() if vals is not None else None
    Ke = max(2, min(K, 5))
    e2e_ms = 0.0
    for _ in range(Ke):
        torch.cuda.synchronize()
        dist.barrier()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(s)
        kd = kh.to(device, non_blocking=True)
        vd = vh.to(device, non_blocking=True) if vh is not None else None
        wk, wv = step(kd, vd)
        ko_h[:wk.numel()].copy_(wk, non_blocking=True)
        if wv is not None:
            vo_h[:wv.numel()].copy_(wv, non_blocking=True)
        e1.record(s)
        torch.cuda.synchronize()
        e2e_ms += e0.elapsed_time(e1)
    e2e_ms = max_over_ranks(e2e_ms, world, device) / Ke
    h2d = n * 4 * (2 if vals is not None else 1)
    d2h = wk.numel() * 4 * (2 if vals is not None else 1)
    del keys, vals, flush
    if comm is not None:
        del dp
        comm.close()
    return {"value": value, "ms_per_step": ms_step, "clocks": clocks.result(), "bounds": bounds,
            "e2e": {"value": n_total / (e2e_ms * 1e-3) / 1e9, "unit": "G keys/s", "h2d_bytes_per_step": h2d,
                    "d2h_bytes_per_step": d2h, "ms_per_step": e2e_ms}}


def run_ours(args, name, cfg, world, rank, local):
    import torch
    # one process per GPU; ranks beyond the visible GPUs share them (only for the gloo test mode)
    device = torch.device("cuda", local % max(1, torch.cuda.device_count()))
    torch.cuda.set_device(device)
    sharded = world > 1 or args.sharded_at_1
    if sharded:
        import torch.distributed as dist
        if world == 1:  # --sharded-at-1: the N > 1 code path on a one-rank process group (testing)
            os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
            os.environ.setdefault("MASTER_PORT", "29517")
            os.environ.setdefault("RANK", "0")
            os.environ.setdefault("WORLD_SIZE", "1")
        if args.dist_backend == "nccl":
            dist.init_process_group("nccl", device_id=device)
        else:
            dist.init_process_group(args.dist_backend)
    from paper_conf_ppopp_ashkianidmo16_b200 import build as b
    if rank == 0:
        b.build()
    barrier(world)
    if not sharded:
        res = bench_config(name, cfg, args.steps, args.warmup, device, world, rank, with_e2e=True,
                           comparators=not args.no_extra)
    else:
        # the per-rank kernels alone (roofline, stages), then the sharded step (the headline at N > 1)
        res = bench_config(name, cfg, max(3, args.steps // 2), args.warmup, device, world, rank, with_e2e=False)
        d = bench_dist(name, cfg, args.steps, args.warmup, device, world, rank, args.dist_backend, args.dist_mode)
        local_value = res["value"]
        res.update(value=d["value"], ms_per_step=d["ms_per_step"], clocks=d["clocks"], e2e=d["e2e"],
                   bounds=d["bounds"])
        res["local_step"] = {"value_if_independent": round(local_value, 3),
                             "note": "the same local kernels without the exchange, max over ranks"}
    extra = {}
    if not args.no_extra and world == 1:
        for nm in args.extra.split(","):
            if nm and nm in CONFIGS and nm != name:
                r = bench_config(nm, CONFIGS[nm], max(5, args.steps // 4), 3, device, world, rank, with_e2e=False,
                                 comparators=True)
                extra[nm] = {"desc": CONFIGS[nm]["desc"], "value": round(r["value"], 2),
                             "ms_per_step": round(r["ms_per_step"], 4), "ms_stats": r["ms_stats"],
                             "launches_per_step": r["launches_per_step"], "variant": r["variant"],
                             "whole_step_frac": round(r["whole_step_frac"], 4),
                             "whole_step_frac_nominal_8tbs": round(r["whole_step_frac_nominal_8tbs"], 4),
                             "kernel": r["roofline"]["kernel"], "kernel_frac": r["roofline"]["frac"],
                             "kernel_frac_nominal_8tbs": r["roofline"]["frac_vs_nominal_8tbs"],
                             "kernel_traffic": r["roofline"]["traffic"],
                             "kernel_alg_bytes": r["roofline"]["algorithmic_bytes_per_launch"],
                             "k1_frac": r["roofline"]["k1_prescan_frac"],
                             "stages_ms": {k: round(v, 4) for k, v in r["stages_ms"].items()},
                             "comparators": r.get("comparators"), "clocks": r["clocks"]}
                if "graph_replay" in r:
                    extra[nm]["graph_replay"] = r["graph_replay"]
                log(f"extra {nm}: {r['value']:.1f} G keys/s frac {r['whole_step_frac']:.3f}")
    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu:
        cpu = time_oracle(cfg, budget_s=10.0)
        cpu = {k: cpu[k] for k in ("value", "unit", "cores", "kind", "sample", "cpu_model")}
    if rank == 0:
        mode = "kv" if cfg["kv"] else "ko"
        pb = PAPER_TABLE5_BEST.get((mode, cfg["m"])) if cfg["n"] == 1 << 25 else None
        out = {
            "metric": "G keys/s", "value": round(res["value"], 3), "unit": "G keys/s", "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(res["ms_per_step"], 5),
            "higher_is_better": True, "scaling": "strong" if cfg.get("strong") else "weak",
            "vs_baseline": round(res["value"] / pb, 3) if pb else None,
            "vs_baseline_note": "paper K40c Table 5 best method, same mode/m/n (context only)" if pb else None,
            "dtype": "u32", "data": "synthetic (seeded splitmix64 keys; values random u32)",
            "config": config_dict(name, cfg, world, args.dist_mode if args.dist_backend == "nccl" else "gloo"),
            "roofline": res["roofline"], "e2e": res["e2e"], "cpu_baseline": cpu,
            "gpu_launches": res["gpu_launches"], "clocks": res["clocks"],
            "ms_stats": res["ms_stats"], "stages_ms": res["stages_ms"],
            "whole_step_frac": round(res["whole_step_frac"], 4),
            "whole_step_frac_nominal_8tbs": round(res["whole_step_frac_nominal_8tbs"], 4),
            "whole_step_hbm_gbs": round(res["whole_step_hbm_gbs"], 1),
            "tile": res["tile"], "variant": res["variant"], "launches_per_step": res["launches_per_step"],
            "extra": extra,
        }
        for k in ("comparators", "local_step", "bounds", "graph_replay"):
            if k in res:
                out[k] = res[k]
        print(json.dumps(out), flush=True)
    if sharded:
        import torch.distributed as dist
        dist.destroy_process_group()


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=50)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--config", default=None, choices=sorted(CONFIGS),
                    help=f"workload (default {DEFAULT} at N = 1, {DEFAULT_DIST} at N > 1)")
    ap.add_argument("--extra", default=EXTRA_DEFAULT)
    ap.add_argument("--no-extra", action="store_true")
    ap.add_argument("--no-cpu", action="store_true")
    ap.add_argument("--dist-backend", default="nccl", choices=["nccl", "gloo"],
                    help="N>1 exchange backend (gloo: host-staged, for testing on one GPU)")
    ap.add_argument("--sharded-at-1", action="store_true",
                    help="run the N > 1 sharded code path (NCCL communicator, ms_dist_run) on one GPU (testing)")
    ap.add_argument("--dist-mode", default="nccl", choices=["nccl", "fused"],
                    help="N>1 exchange: ms_dist_run (NCCL send/recv after a local ms_run), or the fused K3 that "
                         "stores into the owners' symmetric-memory windows (m <= 32, computed bucket ids)")
    args = ap.parse_args()
    if args.warmup < 3:
        args.warmup = 3
    world, rank, local = dist_setup(args)
    name = args.config or (DEFAULT if world == 1 else DEFAULT_DIST)
    cfg = CONFIGS[name]
    if args.impl == "reference":
        run_reference(args, name, cfg, world, rank)
        return
    run_ours(args, name, cfg, world, rank, local)


if __name__ == "__main__":
    main()
