// ms_ranged.cuh -- the CTA-range form of Eq. (2): K1r range histograms (sm_100a).
//
// Eq. (2) holds for ANY partition of the input into
// consecutive subproblems.  The tile variant (ms_kernels.cuh) uses one
// subproblem per K3 tile, so H and G hold m x L words (L = n / T).  Here the
// subproblems are the C contiguous tile RANGES that the C persistent K3 CTAs
// own (range c = tiles [c*L/C, (c+1)*L/C), C = K3's resident grid, <= ~900):
//   K1r: HC[c][j] = #{keys of range c in bucket j}      (local step 1 of the range)
//   K3 prologue (range_base, ms_k3p_args.h): GB[c][j] = sum_{k<j} total_k + sum_{c'<c} HC[c'][j]
//        (terms 1+2 of Eq. 2), then K3 walks its range's tiles in order and keeps G_j for the current tile
//        as a running sum in registers (GB[c][j] + counts of the range's earlier
//        tiles), i.e. Eq. (2) once more one level down, with no H/G array.
// H/G traffic drops from 16 m / T bytes per key to 16 m C / n, and K2 becomes a
// scan of C x m words folded into K3's prologue instead of a grid-wide chained scan of m x L.
// Stable by construction: ranges, tiles and keys are all visited in input order.
#pragma once
#include "ms_k3p_args.h"

namespace ms {


// key span [k0, k1) of sub-range i (of k) of range c, for L tiles of T keys
// split over C ranges; sub-ranges split a range's tiles as evenly as possible
__device__ __forceinline__ void range_span(uint32_t c, uint32_t i, uint32_t k, uint32_t C, uint32_t L, uint32_t T,
                                           uint32_t n, uint64_t *k0, uint64_t *k1) {
  const uint64_t t0 = (uint64_t)c * L / C, t1 = (uint64_t)(c + 1) * L / C;
  const uint64_t s0 = t0 + (t1 - t0) * i / k, s1 = t0 + (t1 - t0) * (i + 1) / k;
  *k0 = s0 * T;
  *k1 = umin64(s1 * T, n);
}

// ============================================================== K1r
// One CTA per sub-range (k per range, so that >= ~8 CTAs of 256 threads per
// SM keep enough 128-bit loads in flight; row r = c*k + i of HC).  Every thread counts 16 keys per sub-tile (four coalesced
// 128-bit loads) into PRIVATE byte counters c8[j][slot(tid)] (bank-conflict-
// free slot layout as in K1); every 15 sub-tiles (<= 240 per byte) and at the
// end the counters are folded into 32-bit per-bucket sums with dp4a.
template <int NT1>
__device__ __forceinline__ uint32_t k1r_slot(uint32_t tid) {
  const uint32_t lane = tid & 31, warp = tid >> 5;
  return (warp >> 2) * 128 + lane * 4 + (warp & 3);  // NT1 bytes per row
}

template <int NT1>
__device__ __forceinline__ void k1r_flush(uint8_t *c8, uint32_t *acc, uint32_t m) {
  // row j = NT1 bytes = NT1/16 uint4; warp w folds rows w, w + NW, ...
  constexpr int NW = NT1 / 32, Q = NT1 / 16;  // Q <= 32 chunks per row
  const uint32_t lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  __syncthreads();
  for (uint32_t j = warp; j < m; j += NW) {
    uint4 *row = reinterpret_cast<uint4 *>(c8 + j * NT1);
    uint32_t s = 0;
    if (lane < (uint32_t)Q) {
      const uint4 w = row[lane];
      s = __dp4a(w.x, 0x01010101u, s);
      s = __dp4a(w.y, 0x01010101u, s);
      s = __dp4a(w.z, 0x01010101u, s);
      s = __dp4a(w.w, 0x01010101u, s);
      row[lane] = make_uint4(0, 0, 0, 0);
    }
    s = warp_sum(s);
    if (lane == 0) acc[j] += s;
  }
  __syncthreads();
}

template <int KIND, int NT1>
__global__ void __launch_bounds__(NT1)
k1r_prescan(const uint32_t *__restrict__ keys, const void *__restrict__ ids, uint32_t n, uint32_t L,
            uint32_t T, uint32_t C, uint32_t k, uint32_t *__restrict__ HC, const __grid_constant__ BucketParams p,
            uint32_t *__restrict__ err_flag) {
  constexpr int KPT = 16, S = NT1 * KPT, FLUSH = 255 / KPT;
  extern __shared__ __align__(16) uint32_t smem[];
  uint32_t *spl_s = smem;                                              // kMaxM words (SPLITTERS)
  uint32_t *tbl_s = smem + kMaxM;                                      // kSplBins words (SPLITTERS)
  uint32_t *acc = smem + (KIND == SPLITTERS ? kMaxM + kSplBins : 0);   // [32]
  uint8_t *c8 = reinterpret_cast<uint8_t *>(acc + 32);                // [m][NT1]
  const uint32_t tid = threadIdx.x, lane = tid & 31;
  const uint32_t m = p.m;
  uint64_t k0, k1;
  range_span(blockIdx.x / k, blockIdx.x % k, k, C, L, T, n, &k0, &k1);

  pdl_trigger();  // K3 (launched with PDL) may be scheduled once every K1r CTA has started
  uint4 *c4 = reinterpret_cast<uint4 *>(c8);
  for (uint32_t i = tid; i < m * (NT1 / 16); i += NT1) c4[i] = make_uint4(0, 0, 0, 0);
  if (tid < 32) acc[tid] = 0;
  if constexpr (KIND == SPLITTERS) {
    for (uint32_t i = tid; i < (1u << p.logm); i += NT1) spl_s[i] = p.spl[i];
    __syncthreads();
    build_spl_table<NT1>(tbl_s, spl_s, p.logm);
  }
  __syncthreads();
  uint8_t *mine = c8 + k1r_slot<NT1>(tid);
  uint32_t bad = 0;
  auto count = [&](uint32_t raw) {
    uint32_t id;
    if constexpr (KIND == IDS) {
      bad |= raw > p.mmask;
      id = min(raw, p.mmask);
    } else {
      id = KIND == SPLITTERS ? id_spl_table(raw, tbl_s, spl_s) : bucket_of_key<KIND>(raw, p, spl_s);
    }
    mine[id * NT1] += 1;
  };

  int since = 0;
  uint64_t base = k0;
  if constexpr (KIND == IDS) {
    for (; base + S <= k1; base += S) {  // full sub-tiles: chunk g = j*NT1 + tid holds keys 4g..4g+3
      if (p.id_bytes == 1) {  // 16 ids per thread = one 16-byte chunk
        const uint4 w = __ldg(reinterpret_cast<const uint4 *>((const uint8_t *)ids + base) + tid);
        const uint32_t ww[4] = {w.x, w.y, w.z, w.w};
#pragma unroll
        for (int q = 0; q < 16; ++q) count((ww[q >> 2] >> (8 * (q & 3))) & 255u);
      } else {
        uint4 v[KPT / 4];
        const uint4 *k4 = reinterpret_cast<const uint4 *>((const uint32_t *)ids + base);
#pragma unroll
        for (int j = 0; j < KPT / 4; ++j) v[j] = __ldg(k4 + j * NT1 + tid);
#pragma unroll
        for (int j = 0; j < KPT / 4; ++j) { count(v[j].x); count(v[j].y); count(v[j].z); count(v[j].w); }
      }
      if (++since == FLUSH) {
        k1r_flush<NT1>(c8, acc, m);
        since = 0;
      }
    }
  } else {
    for (; base + S <= k1; base += S) {  // full sub-tiles: chunk g = j*NT1 + tid holds keys 4g..4g+3
      uint4 v[KPT / 4];
      const uint4 *k4 = reinterpret_cast<const uint4 *>(keys + base);
#pragma unroll
      for (int j = 0; j < KPT / 4; ++j) v[j] = __ldg(k4 + j * NT1 + tid);
#pragma unroll
      for (int j = 0; j < KPT / 4; ++j) { count(v[j].x); count(v[j].y); count(v[j].z); count(v[j].w); }
      if (++since == FLUSH) {
        k1r_flush<NT1>(c8, acc, m);
        since = 0;
      }
    }
  }
  if (base < k1) {  // last, partial sub-tile: whole 16-byte chunks where they fit, scalar keys after
    if constexpr (KIND == IDS) {
      if (p.id_bytes == 1) {
        const uint64_t e = base + 16ull * tid;
        if (e + 16 <= k1) {
          const uint4 w = __ldg(reinterpret_cast<const uint4 *>((const uint8_t *)ids + e));
          const uint32_t ww[4] = {w.x, w.y, w.z, w.w};
#pragma unroll
          for (int q = 0; q < 16; ++q) count((ww[q >> 2] >> (8 * (q & 3))) & 255u);
        } else {
          for (uint64_t i = e; i < k1; ++i) count(((const uint8_t *)ids)[i]);
        }
      }
    }
    if (KIND != IDS || p.id_bytes == 4) {
      const uint32_t *src = KIND == IDS ? (const uint32_t *)ids : keys;
#pragma unroll
      for (int j = 0; j < KPT / 4; ++j) {
        const uint64_t e = base + 4ull * (j * NT1 + tid);
        if (e + 4 <= k1) {
          const uint4 v = __ldg(reinterpret_cast<const uint4 *>(src + e));
          count(v.x); count(v.y); count(v.z); count(v.w);
        } else {
          for (uint64_t i = e; i < k1; ++i) count(src[i]);
        }
      }
    }
  }
  if constexpr (KIND == IDS) {
    if (p.validate && __any_sync(0xFFFFFFFFu, bad) && lane == 0) atomicOr(err_flag, 1u);
  }
  k1r_flush<NT1>(c8, acc, m);
  if (tid < m) HC[(uint64_t)blockIdx.x * m + tid] = acc[tid];
}

inline size_t k1r_smem(uint32_t m, int kind, int nt1) {
  return (kind == SPLITTERS ? (kMaxM + kSplBins) * 4 : 0) + 32 * 4 + (size_t)m * nt1;
}

// Rows of K1r's range-count matrix: R = C * k <= max(C, 8 * SMs) on B200 (<= 1184).
constexpr uint32_t kMaxRangeRows = 1280;

}  // namespace ms
