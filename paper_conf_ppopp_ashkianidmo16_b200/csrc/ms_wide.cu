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

// offsets[j] = #{ i : id(src[i]) < j } for j = 0..m, with src sorted by id.  A warp step reads 512
// consecutive elements as four coalesced 128-bit loads (lane l holds elements 128c + 4l .. +3 of
// group c); an element's predecessor comes from the lane below (or, for lane 0, from the previous
// group's lane 31 / one scalar load before the span).  A position i whose id differs from its
// predecessor's writes offsets(prev_id, id], the first position writes offsets[0..id], the last
// writes offsets(id, m].  Every offset is written exactly once.
template <int KIND>
__global__ void __launch_bounds__(256)
k_wide_offsets(const uint32_t *__restrict__ src, uint64_t n, uint32_t *__restrict__ offsets,
               const __grid_constant__ BucketParams p) {
  const uint32_t m = p.m;
  const uint32_t lane = threadIdx.x & 31;
  const uint64_t warps = (uint64_t)gridDim.x * (blockDim.x / 32);
  auto idof = [&](uint32_t k) { return bucket_of_key<KIND>(k, p, nullptr); };
  auto mark = [&](uint64_t i, uint32_t prev_id, uint32_t id) {  // position i, id of i-1 (ignored for i == 0)
    if (i == 0) {
      for (uint32_t j = 0; j <= id; ++j) offsets[j] = 0u;
    } else if (id != prev_id) {
      for (uint32_t j = prev_id + 1; j <= id; ++j) offsets[j] = (uint32_t)i;
    }
    if (i == n - 1)
      for (uint32_t j = id + 1; j <= m; ++j) offsets[j] = (uint32_t)n;
  };
  for (uint64_t w = (uint64_t)blockIdx.x * (blockDim.x / 32) + (threadIdx.x >> 5); w * 512 < n; w += warps) {
    const uint64_t span = w * 512;
    if (span + 512 <= n) {
      uint32_t v[4][4];
#pragma unroll
      for (int c = 0; c < 4; ++c) {
        const uint4 x = __ldcs(reinterpret_cast<const uint4 *>(src + span + 128 * c) + lane);
        v[c][0] = x.x; v[c][1] = x.y; v[c][2] = x.z; v[c][3] = x.w;
      }
      uint32_t before = span ? __ldg(src + span - 1) : 0u;  // the element before the span (lane 0, group 0)
#pragma unroll
      for (int c = 0; c < 4; ++c) {
        const uint32_t up = __shfl_up_sync(0xFFFFFFFFu, v[c][3], 1);
        const uint32_t wrap = __shfl_sync(0xFFFFFFFFu, c ? v[c - 1][3] : 0u, 31);
        const uint32_t pv = lane ? up : (c ? wrap : before);
        uint32_t prev_id = idof(pv);
#pragma unroll
        for (int e = 0; e < 4; ++e) {
          const uint32_t id = idof(v[c][e]);
          if (id != prev_id || (span + 128 * c + 4 * lane + e == 0) || (span + 128 * c + 4 * lane + e == n - 1))
            mark(span + 128 * c + 4 * lane + e, prev_id, id);
          prev_id = id;
        }
      }
    } else {  // the ragged end: element by element
      for (uint64_t i = span + lane; i < n; i += 32) {
        const uint32_t id = idof(src[i]);
        const uint32_t prev_id = i ? idof(src[i - 1]) : 0u;
        if (id != prev_id || i == 0 || i == n - 1) mark(i, prev_id, id);
      }
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
  const unsigned grid = (unsigned)umin64_host((n + 8 * 512 - 1) / (8 * 512), (uint64_t)sms * 8);
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
