// ms_wide.cu -- device helpers of the two-pass multisplit for m > 256 ("wide" plans, ms_api.cu;
// DESIGN.md §7b, §6.4).
//
// A wide plan splits every bucket id into a low and a high digit and runs two stable
// multisplits, by the low digit then by the high digit (the least-significant-digit order of
// the reduced-bit view, §3.4, with multisplit passes instead of radix-sort passes):
// the second pass is stable, so inside each high digit the order of the first pass -- ascending
// low digit, input order among equal ids -- survives, and the result is the stable multisplit by
// the full id.  Neither pass knows the per-bucket counts of the full id, so the m+1 offsets are
// read back from the output: it is sorted by id, so offsets[j] is the first position whose id
// is >= j, which one pass over the output finds at the positions where the id changes.
#include <cuda_runtime.h>

#include "ms_device.cuh"

namespace ms {

// offsets[j] = #{ i : id(src[i]) < j } for j = 0..m, with src sorted by id.  Each thread step
// owns 16 consecutive positions (four 128-bit loads in flight, plus the element before them); a
// position i whose id differs from its predecessor's writes offsets(prev_id, id], the first
// position writes offsets[0..id], the last writes offsets(id, m].  Every offset is written
// exactly once.
constexpr int kWideKeys = 16;
template <int KIND>
__global__ void __launch_bounds__(256)
k_wide_offsets(const uint32_t *__restrict__ src, uint64_t n, uint32_t *__restrict__ offsets,
               const __grid_constant__ BucketParams p) {
  const uint32_t m = p.m;
  for (uint64_t q = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; q * kWideKeys < n;
       q += (uint64_t)gridDim.x * blockDim.x) {
    const uint64_t i0 = q * kWideKeys;
    uint32_t v[kWideKeys];
    if (i0 + kWideKeys <= n) {
#pragma unroll
      for (int c = 0; c < kWideKeys / 4; ++c) {
        const uint4 x = __ldcs(reinterpret_cast<const uint4 *>(src + i0) + c);
        v[4 * c] = x.x; v[4 * c + 1] = x.y; v[4 * c + 2] = x.z; v[4 * c + 3] = x.w;
      }
    } else {
      for (int e = 0; e < kWideKeys; ++e) v[e] = i0 + e < n ? src[i0 + e] : 0u;
    }
    uint32_t prev = i0 ? bucket_of_key<KIND>(__ldg(src + i0 - 1), p, nullptr) : 0u;
#pragma unroll
    for (int e = 0; e < kWideKeys; ++e) {
      const uint64_t i = i0 + e;
      if (i >= n) break;
      const uint32_t id = bucket_of_key<KIND>(v[e], p, nullptr);
      if (i == 0) {
        for (uint32_t j = 0; j <= id; ++j) offsets[j] = 0u;
      } else if (id != prev) {
        for (uint32_t j = prev + 1; j <= id; ++j) offsets[j] = (uint32_t)i;
      }
      if (i == n - 1)
        for (uint32_t j = id + 1; j <= m; ++j) offsets[j] = (uint32_t)n;
      prev = id;
    }
  }
}

// MS_IDS validation of a wide plan: flag (bit 0) when some id >= m.
__global__ void __launch_bounds__(256)
k_ids_check(const uint32_t *__restrict__ ids, uint64_t n, uint32_t m, uint32_t *__restrict__ flag) {
  uint32_t bad = 0;
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x)
    bad |= __ldcs(ids + i) >= m;
  if (__any_sync(0xFFFFFFFFu, bad) && (threadIdx.x & 31) == 0) atomicOr(flag, 1u);
}

cudaError_t wide_offsets_launch(int kind, const uint32_t *src, uint64_t n, uint32_t *offsets,
                                const BucketParams &bp, int sms, cudaStream_t s) {
  const unsigned grid = (unsigned)umin64_host((n + 256 * kWideKeys - 1) / (256 * kWideKeys), (uint64_t)sms * 8);
  switch (kind) {
    case LOWBITS: k_wide_offsets<LOWBITS><<<grid, 256, 0, s>>>(src, n, offsets, bp); break;
    case SHIFTC: k_wide_offsets<SHIFTC><<<grid, 256, 0, s>>>(src, n, offsets, bp); break;
    case DELTA: k_wide_offsets<DELTA><<<grid, 256, 0, s>>>(src, n, offsets, bp); break;
    default: return cudaErrorInvalidValue;
  }
  return cudaGetLastError();
}

cudaError_t ids_check_launch(const uint32_t *ids, uint64_t n, uint32_t m, uint32_t *flag, int sms, cudaStream_t s) {
  const unsigned grid = (unsigned)umin64_host((n + 255) / 256, (uint64_t)sms * 8);
  k_ids_check<<<grid, 256, 0, s>>>(ids, n, m, flag);
  return cudaGetLastError();
}

}  // namespace ms
