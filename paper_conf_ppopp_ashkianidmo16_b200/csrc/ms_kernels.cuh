// ms_kernels.cuh -- the hot path: K1 pre-scan, K2 scan, K3 post-scan (sm_100a).
//
// PAPER.md §4 {prescan, scan, postscan}; Alg. 1;
// Eq. (2) with subproblems = tiles of T = 256*R consecutive keys
// (one CTA per tile, the paper's block-level granularity of Table 1
// P:714-744, but with R keys per thread so that L = n/T stays small).
#pragma once
#include "ms_device.cuh"

namespace ms {

// ============================================================== K1 pre-scan
// Per-tile bucket histogram -> column `tile` of H (bucket-major, H[j*L + l]).
// Local step 1 of the skeleton, Alg. 1 lines P:819-824.
//
// B200 design: 128-bit streaming loads (KPT keys per thread, all in flight
// before any use); per-thread PRIVATE byte counters in shared memory,
// c8[j][slot(tid)] (a thread counts <= KPT <= 32 keys, so a byte never
// overflows), laid out so the 32 lanes of a warp always hit 32 different
// banks whatever their bucket ids: 4 instructions per key, no atomics, no
// warp votes.  Thread j then sums row j (256 bytes) with dp4a, reading
// 16-byte chunks in a lane-rotated order (conflict-free).
__device__ __forceinline__ uint32_t k1_slot(uint32_t tid) {
  const uint32_t lane = tid & 31, warp = tid >> 5;
  return (warp >> 2) * 128 + lane * 4 + (warp & 3);
}

template <int KIND, int KPT, int SUBT>
__global__ void __launch_bounds__(kThreads)
k1_prescan(const uint32_t *__restrict__ keys, const void *__restrict__ ids, uint32_t n,
           uint32_t L, uint32_t *__restrict__ H, const __grid_constant__ BucketParams p,
           uint64_t *__restrict__ zero_ptr, uint32_t zero_words, uint32_t *__restrict__ err_flag) {
  // SUBT tiles per CTA: warps [h*8/SUBT, (h+1)*8/SUBT) count tile SUBT*blockIdx + h.
  // The byte-counter slot layout puts warps 0-3 in bytes [0,128) of every row and
  // warps 4-7 in [128,256), so each half-row is one tile's column.
  constexpr int NTS = kThreads / SUBT;   // threads per tile
  constexpr int T = NTS * KPT;           // keys per tile
  static_assert(KPT <= 255 && KPT % 4 == 0, "byte counters");
  extern __shared__ __align__(16) uint32_t smem[];
  uint32_t *spl_s = smem;                                     // kMaxM words (SPLITTERS)
  uint8_t *c8 = reinterpret_cast<uint8_t *>(smem + kMaxM);    // [m][256] bytes
  const uint32_t tid = threadIdx.x, lane = tid & 31;
  const uint32_t h = tid / NTS, tl = tid % NTS;
  const uint64_t tile = (uint64_t)blockIdx.x * SUBT + h;
  const uint64_t base = tile * T;
  const uint32_t nt = tile < L ? (uint32_t)umin64(T, n - base) : 0u;
  const uint32_t m = p.m;

  // issue this thread's loads first (they overlap the shared-memory setup)
  uint4 v[KPT / 4];
  const bool full = (nt == T);
  if (full) {
    const uint4 *k4 = reinterpret_cast<const uint4 *>(keys + base);
#pragma unroll
    for (int j = 0; j < KPT / 4; ++j) v[j] = __ldg(k4 + j * NTS + tl);  // coalesced 128-bit loads
  }
  pdl_trigger();  // K2 (launched with PDL) may be scheduled once every K1 CTA has started
  // K2's look-back status words are cleared here (K1 precedes K2 in the stream).
  for (uint32_t i = blockIdx.x * kThreads + tid; i < zero_words; i += gridDim.x * kThreads) zero_ptr[i] = 0;
  uint4 *c4 = reinterpret_cast<uint4 *>(c8);
  for (uint32_t i = tid; i < m * 16; i += kThreads) c4[i] = make_uint4(0, 0, 0, 0);
  if constexpr (KIND == SPLITTERS) {
    for (uint32_t i = tid; i < (1u << p.logm); i += kThreads) spl_s[i] = p.spl[i];
  }
  __syncthreads();

  uint8_t *mine = c8 + k1_slot(tid);
  uint32_t bad = 0;
  if (full) {
    if constexpr (KIND == IDS) {
#pragma unroll
      for (int j = 0; j < KPT / 4; ++j) {
        const uint64_t i0 = base + 4ull * (j * NTS + tl);
        uint32_t raw[4];
        if (p.id_bytes == 1) {
          uint32_t w = __ldg(reinterpret_cast<const uint32_t *>((const uint8_t *)ids + i0));
          raw[0] = w & 255u; raw[1] = (w >> 8) & 255u; raw[2] = (w >> 16) & 255u; raw[3] = w >> 24;
        } else {
          uint4 w = __ldg(reinterpret_cast<const uint4 *>((const uint32_t *)ids + i0));
          raw[0] = w.x; raw[1] = w.y; raw[2] = w.z; raw[3] = w.w;
        }
#pragma unroll
        for (int q = 0; q < 4; ++q) {
          bad |= raw[q] > p.mmask;
          mine[min(raw[q], p.mmask) * kThreads] += 1;
        }
      }
    } else {
#pragma unroll
      for (int j = 0; j < KPT / 4; ++j) {
        mine[bucket_of_key<KIND>(v[j].x, p, spl_s) * kThreads] += 1;
        mine[bucket_of_key<KIND>(v[j].y, p, spl_s) * kThreads] += 1;
        mine[bucket_of_key<KIND>(v[j].z, p, spl_s) * kThreads] += 1;
        mine[bucket_of_key<KIND>(v[j].w, p, spl_s) * kThreads] += 1;
      }
    }
  } else {
    for (uint32_t i = tl; i < nt; i += NTS) {
      uint32_t id;
      if constexpr (KIND == IDS) {
        uint32_t raw = p.id_bytes == 1 ? (uint32_t)((const uint8_t *)ids)[base + i]
                                       : ((const uint32_t *)ids)[base + i];
        bad |= raw > p.mmask;
        id = min(raw, p.mmask);
      } else {
        id = bucket_of_key<KIND>(keys[base + i], p, spl_s);
      }
      mine[id * kThreads] += 1;
    }
  }
  if constexpr (KIND == IDS) {
    if (p.validate && __any_sync(0xFFFFFFFFu, bad) && lane == 0) atomicOr(err_flag, 1u);
  }
  __syncthreads();

  // tile column j = the bytes of row j that belong to this tile's threads;
  // thread j (< m) of each half sums its 256/SUBT bytes with dp4a, reading
  // 16-byte chunks in a lane-rotated order (conflict-free)
  constexpr int CPH = 16 / SUBT;  // 16-byte chunks per half-row
  for (uint32_t b = tl; b < m && tile < L; b += NTS) {
    const uint4 *row = c4 + b * 16 + h * CPH;
    uint32_t acc = 0;
#pragma unroll
    for (int j = 0; j < CPH; ++j) {
      const uint4 w = row[(j + b) & (CPH - 1)];
      acc = __dp4a(w.x, 0x01010101u, acc);
      acc = __dp4a(w.y, 0x01010101u, acc);
      acc = __dp4a(w.z, 0x01010101u, acc);
      acc = __dp4a(w.w, 0x01010101u, acc);
    }
    H[(uint64_t)b * L + tile] = acc;
  }
}

// K1 for m > 32: one u32 histogram per tile in shared memory, updated by all
// its warps with shared-memory atomics (round 2: per-warp histograms summed
// per tile measured 6 % slower, C4 260 vs 243 us).  Bound by the atomics'
// throughput (about 4 lanes per clock per SM: C4 243 us for 1 GiB of keys,
// 0.67 of the copy rate).  Byte counters with 64 keys per thread (no atomics,
// 4 B of counter reduction per key) measured slower still (374 us).
template <int KIND, int KPT, int SUBT>
__global__ void __launch_bounds__(kThreads)
k1a_prescan(const uint32_t *__restrict__ keys, const void *__restrict__ ids, uint32_t n,
            uint32_t L, uint32_t *__restrict__ H, const __grid_constant__ BucketParams p,
            uint64_t *__restrict__ zero_ptr, uint32_t zero_words, uint32_t *__restrict__ err_flag) {
  constexpr int NTS = kThreads / SUBT;   // threads per tile
  constexpr int T = NTS * KPT;           // keys per tile
  extern __shared__ __align__(16) uint32_t smem[];
  uint32_t *spl_s = smem;                // kMaxM words (SPLITTERS)
  uint32_t *hist = smem + kMaxM;         // [SUBT][m]: one histogram per tile, all its warps' atomics
  const uint32_t tid = threadIdx.x, lane = tid & 31;
  const uint32_t h = tid / NTS, tl = tid % NTS;
  const uint64_t tile = (uint64_t)blockIdx.x * SUBT + h;
  const uint64_t base = tile * T;
  const uint32_t nt = tile < L ? (uint32_t)umin64(T, n - base) : 0u;
  const uint32_t m = p.m;

  uint4 v[KPT / 4];
  const bool full = (nt == T);
  if (full && KIND != IDS) {
    const uint4 *k4 = reinterpret_cast<const uint4 *>(keys + base);
#pragma unroll
    for (int j = 0; j < KPT / 4; ++j) v[j] = __ldg(k4 + j * NTS + tl);
  }
  pdl_trigger();
  for (uint32_t i = blockIdx.x * kThreads + tid; i < zero_words; i += gridDim.x * kThreads) zero_ptr[i] = 0;
  for (uint32_t i = tid; i < SUBT * m; i += kThreads) hist[i] = 0;
  if constexpr (KIND == SPLITTERS) {
    for (uint32_t i = tid; i < (1u << p.logm); i += kThreads) spl_s[i] = p.spl[i];
  }
  __syncthreads();
  uint32_t *hw = hist + h * m;
  uint32_t bad = 0;
  if (full) {
    if constexpr (KIND == IDS) {
#pragma unroll
      for (int j = 0; j < KPT / 4; ++j) {
        const uint64_t i0 = base + 4ull * (j * NTS + tl);
        uint32_t raw[4];
        if (p.id_bytes == 1) {
          uint32_t w = __ldg(reinterpret_cast<const uint32_t *>((const uint8_t *)ids + i0));
          raw[0] = w & 255u; raw[1] = (w >> 8) & 255u; raw[2] = (w >> 16) & 255u; raw[3] = w >> 24;
        } else {
          uint4 w = __ldg(reinterpret_cast<const uint4 *>((const uint32_t *)ids + i0));
          raw[0] = w.x; raw[1] = w.y; raw[2] = w.z; raw[3] = w.w;
        }
#pragma unroll
        for (int q = 0; q < 4; ++q) {
          bad |= raw[q] > p.mmask;
          atomicAdd(hw + min(raw[q], p.mmask), 1u);
        }
      }
    } else {
#pragma unroll
      for (int j = 0; j < KPT / 4; ++j) {
        atomicAdd(hw + bucket_of_key<KIND>(v[j].x, p, spl_s), 1u);
        atomicAdd(hw + bucket_of_key<KIND>(v[j].y, p, spl_s), 1u);
        atomicAdd(hw + bucket_of_key<KIND>(v[j].z, p, spl_s), 1u);
        atomicAdd(hw + bucket_of_key<KIND>(v[j].w, p, spl_s), 1u);
      }
    }
  } else {
    for (uint32_t i = tl; i < nt; i += NTS) {
      uint32_t id;
      if constexpr (KIND == IDS) {
        uint32_t raw = p.id_bytes == 1 ? (uint32_t)((const uint8_t *)ids)[base + i]
                                       : ((const uint32_t *)ids)[base + i];
        bad |= raw > p.mmask;
        id = min(raw, p.mmask);
      } else {
        id = bucket_of_key<KIND>(keys[base + i], p, spl_s);
      }
      atomicAdd(hw + id, 1u);
    }
  }
  if constexpr (KIND == IDS) {
    if (p.validate && __any_sync(0xFFFFFFFFu, bad) && lane == 0) atomicOr(err_flag, 1u);
  }
  __syncthreads();
  for (uint32_t b = tl; b < m && tile < L; b += NTS) {
    const uint32_t acc = hist[h * m + b];
    H[(uint64_t)b * L + tile] = acc;
  }
}

// Persistent form of K1 for MS_SPLITTERS: the bin table (ms_device.cuh) is
// built once per CTA, then the CTA walks tile groups with a stride of gridDim.x.
template <int KIND, int KPT, int SUBT>
__global__ void __launch_bounds__(kThreads)
k1s_prescan(const uint32_t *__restrict__ keys, const void *__restrict__ ids, uint32_t n,
           uint32_t L, uint32_t *__restrict__ H, const __grid_constant__ BucketParams p,
           uint64_t *__restrict__ zero_ptr, uint32_t zero_words, uint32_t *__restrict__ err_flag) {
  // SUBT tiles per CTA iteration: warps [h*8/SUBT, (h+1)*8/SUBT) count tile SUBT*group + h.
  // The byte-counter slot layout puts warps 0-3 in bytes [0,128) of every row and
  // warps 4-7 in [128,256), so each half-row is one tile's column.  CTAs walk
  // the tile groups with a stride of gridDim.x (one group per CTA unless the
  // launcher makes the grid persistent -- SPLITTERS, whose bin table is built
  // once per CTA).
  constexpr int NTS = kThreads / SUBT;   // threads per tile
  constexpr int T = NTS * KPT;           // keys per tile
  static_assert(KPT <= 255 && KPT % 4 == 0, "byte counters");
  extern __shared__ __align__(16) uint32_t smem[];
  uint32_t *spl_s = smem;                                     // kMaxM words (SPLITTERS)
  uint32_t *tbl_s = smem + kMaxM;                             // kSplBins words (SPLITTERS)
  uint8_t *c8 = reinterpret_cast<uint8_t *>(smem + kMaxM + (KIND == SPLITTERS ? kSplBins : 0));  // [m][256]
  const uint32_t tid = threadIdx.x, lane = tid & 31;
  const uint32_t h = tid / NTS, tl = tid % NTS;
  const uint32_t m = p.m;
  const uint64_t groups = ((uint64_t)L + SUBT - 1) / SUBT;

  if constexpr (KIND == SPLITTERS) {
    for (uint32_t i = tid; i < (1u << p.logm); i += kThreads) spl_s[i] = p.spl[i];
    __syncthreads();
    build_spl_table<kThreads>(tbl_s, spl_s, p.logm);
  }
  uint8_t *mine = c8 + k1_slot(tid);
  uint4 *c4 = reinterpret_cast<uint4 *>(c8);
  uint32_t bad = 0;
  auto id_of = [&](uint32_t k) -> uint32_t {
    if constexpr (KIND == SPLITTERS) return id_spl_table(k, tbl_s, spl_s);
    else return bucket_of_key<KIND>(k, p, spl_s);
  };

  for (uint64_t grp = blockIdx.x; grp < groups; grp += gridDim.x) {
    const uint64_t tile = grp * SUBT + h;
    const uint64_t base = tile * T;
    const uint32_t nt = tile < L ? (uint32_t)umin64(T, n - base) : 0u;
    // issue this thread's loads first (they overlap the counter reset)
    uint4 v[KPT / 4];
    const bool full = (nt == T);
    if (full) {
      const uint4 *k4 = reinterpret_cast<const uint4 *>(keys + base);
#pragma unroll
      for (int j = 0; j < KPT / 4; ++j) v[j] = __ldg(k4 + j * NTS + tl);  // coalesced 128-bit loads
    }
    if (grp == blockIdx.x) {
      pdl_trigger();  // K2 (launched with PDL) may be scheduled once every K1 CTA has started
      // K2's look-back status words are cleared here (K1 precedes K2 in the stream).
      for (uint32_t i = blockIdx.x * kThreads + tid; i < zero_words; i += gridDim.x * kThreads) zero_ptr[i] = 0;
    } else {
      __syncthreads();  // the previous group's row sums have read the counters
    }
    for (uint32_t i = tid; i < m * 16; i += kThreads) c4[i] = make_uint4(0, 0, 0, 0);
    __syncthreads();

    if (full) {
      if constexpr (KIND == IDS) {
#pragma unroll
        for (int j = 0; j < KPT / 4; ++j) {
          const uint64_t i0 = base + 4ull * (j * NTS + tl);
          uint32_t raw[4];
          if (p.id_bytes == 1) {
            uint32_t w = __ldg(reinterpret_cast<const uint32_t *>((const uint8_t *)ids + i0));
            raw[0] = w & 255u; raw[1] = (w >> 8) & 255u; raw[2] = (w >> 16) & 255u; raw[3] = w >> 24;
          } else {
            uint4 w = __ldg(reinterpret_cast<const uint4 *>((const uint32_t *)ids + i0));
            raw[0] = w.x; raw[1] = w.y; raw[2] = w.z; raw[3] = w.w;
          }
#pragma unroll
          for (int q = 0; q < 4; ++q) {
            bad |= raw[q] > p.mmask;
            mine[min(raw[q], p.mmask) * kThreads] += 1;
          }
        }
      } else {
#pragma unroll
        for (int j = 0; j < KPT / 4; ++j) {
          mine[id_of(v[j].x) * kThreads] += 1;
          mine[id_of(v[j].y) * kThreads] += 1;
          mine[id_of(v[j].z) * kThreads] += 1;
          mine[id_of(v[j].w) * kThreads] += 1;
        }
      }
    } else {
      for (uint32_t i = tl; i < nt; i += NTS) {
        uint32_t id;
        if constexpr (KIND == IDS) {
          uint32_t raw = p.id_bytes == 1 ? (uint32_t)((const uint8_t *)ids)[base + i]
                                         : ((const uint32_t *)ids)[base + i];
          bad |= raw > p.mmask;
          id = min(raw, p.mmask);
        } else {
          id = id_of(keys[base + i]);
        }
        mine[id * kThreads] += 1;
      }
    }
    __syncthreads();

    // tile column j = the bytes of row j that belong to this tile's threads;
    // thread j (< m) of each half sums its 256/SUBT bytes with dp4a, reading
    // 16-byte chunks in a lane-rotated order (conflict-free)
    constexpr int CPH = 16 / SUBT;  // 16-byte chunks per half-row
    for (uint32_t b = tl; b < m && tile < L; b += NTS) {
      const uint4 *row = c4 + b * 16 + h * CPH;
      uint32_t acc = 0;
#pragma unroll
      for (int j = 0; j < CPH; ++j) {
        const uint4 w = row[(j + b) & (CPH - 1)];
        acc = __dp4a(w.x, 0x01010101u, acc);
        acc = __dp4a(w.y, 0x01010101u, acc);
        acc = __dp4a(w.z, 0x01010101u, acc);
        acc = __dp4a(w.w, 0x01010101u, acc);
      }
      H[(uint64_t)b * L + tile] = acc;
    }
  }
  if constexpr (KIND == IDS) {
    if (p.validate && __any_sync(0xFFFFFFFFu, bad) && lane == 0) atomicOr(err_flag, 1u);
  }
}

// ============================================================== K2 scan
// G = exclusive scan of row-vectorised H (in place), Alg. 1 P:825-828:
// G[j][l] = sum_{k<j} sum_l' h_{k,l'} + sum_{l'<l} h_{j,l'} (terms 1+2 of
// Eq. 2).  Single pass, chained with a decoupled look-back over 64-bit
// status words (flag << 32 | value); status is zeroed by K1 (or by the host
// when the stage runs alone).  offsets[j] = G[j][0], offsets[m] = n.
constexpr int kScanItems = 16;
constexpr int kScanChunk = kThreads * kScanItems;
constexpr uint64_t kFlagA = 1ull << 32;  // aggregate available
constexpr uint64_t kFlagP = 2ull << 32;  // inclusive prefix available

__global__ void __launch_bounds__(kThreads)
k2_scan(uint32_t *__restrict__ data, uint64_t total, uint64_t *__restrict__ status,
        uint32_t *__restrict__ offsets, uint32_t L, uint32_t m, uint32_t n) {
  __shared__ uint32_t buf[kScanChunk + kScanChunk / 32];
  __shared__ uint32_t wsum[kWarps];
  __shared__ uint32_t prefix_s;
  const uint32_t tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const uint64_t chunk = blockIdx.x;
  const uint64_t base = chunk * kScanChunk;
  const uint32_t cnt = (uint32_t)umin64(kScanChunk, total - base);
  pdl_wait();     // K1's H and zeroed status words are complete and visible
  pdl_trigger();

#pragma unroll
  for (int j = 0; j < kScanItems; ++j) {
    uint32_t i = j * kThreads + tid;
    buf[i + (i >> 5)] = i < cnt ? data[base + i] : 0u;
  }
  __syncthreads();
  uint32_t v[kScanItems];
  uint32_t s = 0;
#pragma unroll
  for (int q = 0; q < kScanItems; ++q) {
    uint32_t i = tid * kScanItems + q;
    v[q] = buf[i + (i >> 5)];
    s += v[q];
  }
  uint32_t incl = warp_incl_scan(s, lane);
  if (lane == 31) wsum[warp] = incl;
  __syncthreads();
  uint32_t wpre = 0, agg = 0;
#pragma unroll
  for (int w = 0; w < kWarps; ++w) {
    uint32_t x = wsum[w];
    wpre += (w < (int)warp) ? x : 0u;
    agg += x;
  }
  uint32_t texcl = wpre + incl - s;

  if (chunk == 0) {
    if (tid == 0) {
      st_status(status, kFlagP | agg);
      prefix_s = 0;
    }
  } else {
    if (tid == 0) st_status(status + chunk, kFlagA | agg);
    if (warp == 0) {
      uint32_t excl = 0;
      int64_t pred = (int64_t)chunk - 1;
      while (true) {
        int64_t idx = pred - lane;
        uint64_t st = idx >= 0 ? ld_status(status + idx) : kFlagP;
        while (__any_sync(0xFFFFFFFFu, (st >> 32) == 0)) {
          if ((st >> 32) == 0) st = ld_status(status + idx);
        }
        uint32_t pmask = __ballot_sync(0xFFFFFFFFu, (st >> 32) == 2);
        uint32_t val = (uint32_t)st;
        if (pmask) {
          uint32_t first = __ffs(pmask) - 1;
          excl += warp_sum(lane <= first ? val : 0u);
          break;
        }
        excl += warp_sum(val);
        pred -= 32;
      }
      if (lane == 0) {
        st_status(status + chunk, kFlagP | (uint32_t)(excl + agg));
        prefix_s = excl;
      }
    }
  }
  __syncthreads();
  uint32_t run = prefix_s + texcl;
#pragma unroll
  for (int q = 0; q < kScanItems; ++q) {
    uint32_t i = tid * kScanItems + q;
    buf[i + (i >> 5)] = run;
    run += v[q];
  }
  __syncthreads();
#pragma unroll
  for (int j = 0; j < kScanItems; ++j) {
    uint32_t i = j * kThreads + tid;
    if (i < cnt) {
      uint64_t g = base + i;
      uint32_t out = buf[i + (i >> 5)];
      data[g] = out;
      if (offsets != nullptr && (g % L) == 0) offsets[g / L] = out;
    }
  }
  if (offsets != nullptr && chunk == 0 && tid == 0) offsets[m] = n;
}

// ============================================================== K2, row-parallel (m > 32)
// The same terms 1+2 of Eq. (2) split into their two sums: CTA j scans bucket row j of H alone
// (term 2: G'[j][l] = sum_{l'<l} h_{j,l'}, in place) and writes the row total; the last CTA to
// finish (atomic ticket, zeroed by K1) scans the m row totals -- term 1, rowbase[j] =
// sum_{k<j} tot_k -- and writes the offsets; K3 adds rowbase[j] to G'[j][tile] (k3_postscan's
// `rowbase` mode).  No look-back chain: m independent CTAs stream their rows (32 KB chunks staged
// in shared memory with a running carry), against the chained single-pass scan of m*L words that
// the look-back serialises (C4: 72 us).
constexpr int kRowThreads = 512;
constexpr int kRowItems = 16;
constexpr int kRowChunk = kRowThreads * kRowItems;  // 8192 words

__global__ void __launch_bounds__(kRowThreads)
k2w_rowscan(uint32_t *__restrict__ HG, uint32_t L, uint32_t m, uint32_t n, uint32_t *__restrict__ rowtot,
            uint32_t *__restrict__ rowbase, uint32_t *__restrict__ ticket, uint32_t *__restrict__ offsets) {
  __shared__ uint32_t buf[kRowChunk + kRowChunk / 32];
  __shared__ uint32_t wsum[kRowThreads / 32];
  __shared__ uint32_t last;
  const uint32_t tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  uint32_t *row = HG + (uint64_t)blockIdx.x * L;
  pdl_wait();  // K1's H is complete and visible
  pdl_trigger();
  uint32_t carry = 0;
  for (uint32_t base = 0; base < L; base += kRowChunk) {
    const uint32_t cnt = min(L - base, (uint32_t)kRowChunk);
#pragma unroll
    for (int j = 0; j < kRowItems; ++j) {
      const uint32_t i = j * kRowThreads + tid;
      buf[i + (i >> 5)] = i < cnt ? __ldcs(row + base + i) : 0u;
    }
    __syncthreads();
    uint32_t v[kRowItems], s = 0;
#pragma unroll
    for (int q = 0; q < kRowItems; ++q) {
      const uint32_t i = tid * kRowItems + q;
      v[q] = buf[i + (i >> 5)];
      s += v[q];
    }
    const uint32_t incl = warp_incl_scan(s, lane);
    if (lane == 31) wsum[warp] = incl;
    __syncthreads();
    uint32_t wpre = 0, agg = 0;
#pragma unroll
    for (int w = 0; w < kRowThreads / 32; ++w) {
      const uint32_t x = wsum[w];
      wpre += (w < (int)warp) ? x : 0u;
      agg += x;
    }
    uint32_t run = carry + wpre + incl - s;
#pragma unroll
    for (int q = 0; q < kRowItems; ++q) {
      const uint32_t i = tid * kRowItems + q;
      buf[i + (i >> 5)] = run;
      run += v[q];
    }
    __syncthreads();
#pragma unroll
    for (int j = 0; j < kRowItems; ++j) {
      const uint32_t i = j * kRowThreads + tid;
      if (i < cnt) __stcg(row + base + i, buf[i + (i >> 5)]);
    }
    carry += agg;
    __syncthreads();  // buf and wsum are reused by the next chunk
  }
  if (tid == 0) {
    rowtot[blockIdx.x] = carry;
    __threadfence();
    last = atomicAdd(ticket, 1u) == gridDim.x - 1;
  }
  __syncthreads();
  if (!last) return;
  // the last row CTA: term 1 = exclusive scan of the m (<= kRowThreads) row totals
  __threadfence();
  const uint32_t t = tid < m ? __ldcg(rowtot + tid) : 0u;
  const uint32_t incl = warp_incl_scan(t, lane);
  if (lane == 31) wsum[warp] = incl;
  __syncthreads();
  uint32_t start = incl - t;
#pragma unroll
  for (int w = 0; w < kRowThreads / 32; ++w) start += (w < (int)warp) ? wsum[w] : 0u;
  if (tid < m) {
    rowbase[tid] = start;
    if (offsets != nullptr) offsets[tid] = start;
  }
  if (tid == 0) {
    if (offsets != nullptr) offsets[m] = n;
    *ticket = 0;  // (K1 zeroes it again before the next K2)
  }
}

// ============================================================== whatBucket() only
template <int KIND>
__global__ void __launch_bounds__(kThreads)
k_bucket_ids(const uint32_t *__restrict__ keys, uint64_t n, uint32_t *__restrict__ out,
             const __grid_constant__ BucketParams p) {
  __shared__ uint32_t spl_s[kMaxM];
  __shared__ uint32_t tbl_s[KIND == SPLITTERS ? kSplBins : 1];
  if constexpr (KIND == SPLITTERS) {  // the same bin table as K1 / K3 (so the functor tests pin it)
    for (uint32_t i = threadIdx.x; i < (1u << p.logm); i += kThreads) spl_s[i] = p.spl[i];
    __syncthreads();
    build_spl_table<kThreads>(tbl_s, spl_s, p.logm);
    __syncthreads();
  }
  for (uint64_t i = (uint64_t)blockIdx.x * kThreads + threadIdx.x; i < n;
       i += (uint64_t)gridDim.x * kThreads) {
    if constexpr (KIND == SPLITTERS) out[i] = id_spl_table(keys[i], tbl_s, spl_s);
    else out[i] = bucket_of_key<KIND>(keys[i], p, spl_s);
  }
}

}  // namespace ms
