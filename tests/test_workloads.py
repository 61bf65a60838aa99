"""The seeded generators: numpy and torch twins agree bit for bit; distributions are as stated."""
import numpy as np
import pytest
import torch

import workloads as W


def _u32(t):
    return t.cpu().numpy().view(np.uint32)


@pytest.mark.parametrize("start", [0, 12345])
def test_twins_uniform(start):
    a = W.keys_np(10007, 0x4D530002, start=start)
    b = _u32(W.keys_torch(10007, 0x4D530002, "cpu", start=start))
    assert np.array_equal(a, b)
    assert np.array_equal(W.values_np(999, 3, "random", start), _u32(W.values_torch(999, 3, "cpu", "random", start)))
    assert np.array_equal(W.values_np(999, 3, "index", start), _u32(W.values_torch(999, 3, "cpu", "index", start)))


@pytest.mark.parametrize("dist", ["buckets", "binomial", "hot"])
@pytest.mark.parametrize("m", [2, 32, 65, 256])
def test_twins_bucket_targeted(dist, m):
    spl = W.gen_splitters(m, 9)
    rng = W.ranges_splitters(spl)
    a = W.keys_np(5003, 7, dist, m, rng)
    b = _u32(W.keys_torch(5003, 7, "cpu", dist, m, rng))
    assert np.array_equal(a, b)
    if m <= 256:
        sh = 32 - (m - 1).bit_length() if (m & (m - 1)) == 0 else None
        if sh is not None:
            a = W.keys_np(777, 7, dist, m, lowbits_shift=sh)
            b = _u32(W.keys_torch(777, 7, "cpu", dist, m, lowbits_shift=sh))
            assert np.array_equal(a, b)
    assert np.array_equal(W.bucket_draw_np(3000, 5, dist, m), W.bucket_draw_torch(3000, 5, dist, m, "cpu").numpy())


def test_distribution_shapes():
    n, m = 200000, 32
    b = W.draw_buckets_np("binomial", m, 1, 0, n).astype(np.float64)
    assert abs(b.mean() - (m - 1) / 2) < 0.05 and abs(b.var() - (m - 1) / 4) < 0.2   # B(m-1, 1/2)
    h = W.draw_buckets_np("hot", m, 1, 0, n)
    assert abs(np.mean(h == m // 2) - (0.75 + 0.25 / m)) < 0.01                      # 25 % uniform + rest hot
    u = W.draw_buckets_np("buckets", m, 1, 0, n)
    assert np.bincount(u, minlength=m).min() > n / m * 0.9


def test_keys_land_in_requested_ranges():
    m, delta = 8, 400000000
    rng = W.ranges_delta(m, delta)
    k = W.keys_np(50000, 2, "buckets", m, rng)
    b = W.draw_buckets_np("buckets", m, 2, 0, 50000)
    assert np.all(k >= rng.lo[b]) and np.all(k <= rng.hi[b])
    spl = W.gen_splitters(32, 4)
    assert np.all(np.diff(spl.astype(np.int64)) > 0) and spl[0] >= 1 and spl[-1] <= 0xFFFFFFFE
