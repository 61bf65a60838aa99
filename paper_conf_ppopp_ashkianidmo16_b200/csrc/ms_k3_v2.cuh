// ms_k3_v2.cuh -- K3 post-scan for m <= 32, second generation (sm_100a).
//
// Same contract and the same paper steps as k3p_postscan (ms_k3_blocked.cuh):
// recompute ids (footnote 6), stable local offsets (term 3 of
// Eq. (2)) by an explicit, hierarchical H-bar scan,
// a local stable multisplit of the tile in shared memory (§4 reordering,
// P:689-713; §5.2.2), bucket runs written to G[j][tile] +
// (slot - S_t[j]).  What changes is how the SM spends its instructions and
// shared-memory wavefronts ("K3 v2"):
//  * tiles are staged by the TMA engine (cp.async.bulk.tensor.2d, one
//    instruction per array per tile, issued by one thread) with the 128-byte
//    swizzle, so every thread reads its contiguous 16-key block as four
//    conflict-free 128-bit loads with no address arithmetic per chunk;
//  * keys stay in registers from the counting pass to the scatter; the key
//    stage is handed back to the TMA right after counting, the value stage
//    (key-value) after the scatter -- separate mbarriers per array;
//  * the counter matrix is padded (16 B per 128 B) so that both the counting
//    and the 128-bit scan accesses are conflict-free with no per-lane
//    rotation, and the scan uses packed u16 arithmetic (3 instructions per
//    2 counters: IMAD, IMAD, IDP2A);
//  * counters and reordered keys are addressed by 32-bit shared-window
//    addresses (one IMAD per access);
//  * splitter ids come from a 1024-bin table in shared memory (one load and
//    a compare per key, ms_device.cuh id_spl_table).
// Tile walk: tile mode (tiles blockIdx.x, blockIdx.x + gridDim.x, ..., G from
// the global G column) or RANGED (contiguous range per CTA, running G, see
// ms_ranged.cuh).  The partial last tile (if any) is loaded with predicated
// plain loads straight into registers.
#pragma once
#include <cuda.h>
#include <cudaTypedefs.h>

#include <cooperative_groups.h>

#include <type_traits>

#include "ms_k3p_args.h"

#ifndef MS_K32_MINM
#define MS_K32_MINM 2  // key-only ONE with 8192-key tiles from this many buckets
#endif

namespace ms {

template <int LOGMP, bool KV, int NT, int STAGES, int KPT = 16>
struct K3vLayout {
  static constexpr int MP = 1 << LOGMP;         // bucket rows (m rounded up to a power of 2, >= 2)
  static constexpr int K = KPT;                 // keys per thread (one contiguous block): 16, or 32 with NT = 128
  static constexpr int T = NT * K;              // keys per tile
  static constexpr int TB = T * 4;              // bytes of one staged array (keys or values)
  static constexpr int KSR = (T + 3 * MP + 4 + 3) & ~3;  // reorder slots incl. alignment padding
  static constexpr int MW = 4 * MP + 8;         // per-tile metadata words: rowS[MP+4] P[MP] G[MP] D[MP]
  // u16 counter matrix c[j][beta], row-major; inside a row, 16 bytes of
  // padding after every 128 bytes (byte q of a plain row lives at
  // q + 16 * (q / 128)), and the row stride is rounded up to a multiple of
  // 128 bytes.  Counting (32 lanes, 32 consecutive words of their rows: bank =
  // lane whatever the row) and the scan (thread t reads the 4*WPT-byte
  // segment t with 128-bit loads) are then both free of bank conflicts,
  // without rotating any register order.
  static constexpr int RS = (2 * NT + 2 * NT / 8 + 127) / 128 * 128;  // padded row stride (bytes)
  static constexpr int CNTB = MP * RS;
  // byte offsets from the 1024-byte-aligned base (128B swizzle needs 1024 B alignment)
  static constexpr int O_SK = 0;                          // [STAGES][T] staged keys
  static constexpr int O_SV = O_SK + STAGES * TB;         // [STAGES][T] staged values
  static constexpr int O_KS = O_SV + (KV ? STAGES * TB : 0);  // reordered keys
  static constexpr int O_VS = O_KS + KSR * 4;             // reordered values
  static constexpr int O_CNT = O_VS + (KV ? KSR * 4 : 0); // counters
  static constexpr int O_META = O_CNT + CNTB;             // [2][MW] words (tile parity)
  static constexpr int O_WS = O_META + 2 * MW * 4;        // warp sums [16]
  static constexpr int O_TOT = O_WS + 16 * 4;             // ONE: this range's bucket totals [max(MP, 32)]
  static constexpr int O_BAR = (O_TOT + (MP > 32 ? MP : 32) * 4 + 7) & ~7;  // mbarriers: keys, values [STAGES]
  static constexpr int O_SPL = O_BAR + 2 * STAGES * 8;    // SPLITTERS: padded splitters [256] + bin table
  static constexpr int O_TBL = O_SPL + kMaxM * 4;
  static constexpr int BYTES = O_SPL;                     // + 1024 alignment slack at launch
  static constexpr int BYTES_SPL = O_TBL + kSplBins * 4;
};

// TMA 2-D tensor load (box = T/32 rows of 32 keys) into shared memory, completion on `bar`.
__device__ __forceinline__ void tma_load_2d(void *dst, const CUtensorMap *tm, int c0, int c1, uint64_t *bar) {
  asm volatile(
      "cp.async.bulk.tensor.2d.shared::cluster.global.tile.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], [%4];" ::"r"(
          smem_u32(dst)),
      "l"(tm), "r"(c0), "r"(c1), "r"(smem_u32(bar))
      : "memory");
}

// ONE (implies RANGED): the whole multisplit in ONE cooperative launch.  Phase 1
// counts this CTA's range (K1r's job) through the same TMA pipeline, the range
// counts are published to rs.HC, a grid-wide barrier, the range scan
// (range_base) -- then phase 2 walks the range's tiles in REVERSE (the first
// tiles it reads are the ones phase 1 read last, still in L2), with the running
// G counting down from the range's end.
// DIRECT (ablation, SURVEY NEXT-2 / the paper's "Direct" method of Table 4): no local reorder --
// every key is stored from registers straight to its global position G_j + local offset.
// IDS (precomputed ids, IDB = 1 or 4 bytes per id): the ids of a thread's block are read
// straight from global memory (16 B / 64 B per 16 keys, next to the TMA-staged keys), clamped
// to m-1 (a contract violation never indexes outside the counters) and flagged in *flag when
// p.validate; ONE's phase 1 counts from the ids alone (1 or 4 B per key instead of 4).
template <int KIND, bool KV, int LOGMP, int NT, int STAGES, bool RANGED, int MINB, int KPT, bool ONE = false,
          bool DIRECT = false, int IDB = 0>
__global__ void __launch_bounds__(NT, MINB)
k3v_postscan(const __grid_constant__ CUtensorMap tmk, const __grid_constant__ CUtensorMap tmv,
             const uint32_t *__restrict__ keys, const uint32_t *__restrict__ vals,
             const void *__restrict__ ids, uint32_t *__restrict__ flag,
             const uint32_t *__restrict__ G, uint32_t *__restrict__ keys_out, uint32_t *__restrict__ vals_out,
             uint32_t n, uint32_t L, const __grid_constant__ BucketParams p,
             const __grid_constant__ RangeScan rs, const __grid_constant__ DistTarget ds) {
  using Ly = K3vLayout<LOGMP, KV, NT, STAGES, KPT>;
  constexpr int MP = Ly::MP, K = Ly::K, T = Ly::T, TB = Ly::TB, RS = Ly::RS;
  constexpr int NW = NT / 32;
  constexpr int NCH = K / 4;  // 16-byte chunks per thread block
  constexpr int LOGNT = NT == 256 ? 8 : NT == 128 ? 7 : 6;
  static_assert(NT == 64 || NT == 128 || NT == 256, "NT");
  // multi-instruction (and precomputed) ids are kept in registers, one byte per key, not recomputed
  constexpr bool KEEP_ID = KIND == SPLITTERS || KIND == DELTA || KIND == IDS || KIND == SHIFTC_LO || KIND == DELTA_LO;
  static_assert(KIND != IDS || IDB == 1 || IDB == 4, "IDS needs IDB = 1 or 4");
  const uint32_t mm4 = p.mmask * 0x01010101u;  // IDS: per-byte clamp bound
  uint32_t bad = 0;                            // IDS: some raw id > m - 1 (validation)
  // IDS: clamp 4 raw u32 ids into one word of 4 byte ids
  auto clamp_pack = [&](uint32_t a, uint32_t b, uint32_t c, uint32_t d) -> uint32_t {
    bad |= (a > p.mmask) | (b > p.mmask) | (c > p.mmask) | (d > p.mmask);
    return min(a, p.mmask) | (min(b, p.mmask) << 8) | (min(c, p.mmask) << 16) | (min(d, p.mmask) << 24);
  };
  auto clamp4 = [&](uint32_t w) -> uint32_t {  // 4 raw u8 ids
    bad |= __vcmpgtu4(w, mm4);
    return __vminu4(w, mm4);
  };
  // IDS: byte ids of the nch4 * 4 keys from key index e (16-byte aligned, all valid) into w[]
  auto load_ids_full = [&](uint64_t e, uint32_t *w, int nch4) {
    if constexpr (IDB == 1) {
      const uint4 x = __ldcs(reinterpret_cast<const uint4 *>(static_cast<const uint8_t *>(ids) + e));
      const uint32_t xx[4] = {x.x, x.y, x.z, x.w};
#pragma unroll
      for (int c = 0; c < 4; ++c)
        if (c < nch4) w[c] = clamp4(xx[c]);
    } else {
#pragma unroll
      for (int c = 0; c < 4; ++c)
        if (c < nch4) {
          const uint4 x = __ldcs(reinterpret_cast<const uint4 *>(static_cast<const uint32_t *>(ids) + e) + c);
          w[c] = clamp_pack(x.x, x.y, x.z, x.w);
        }
    }
  };
  auto load_id1 = [&](uint64_t i) -> uint32_t {  // one id, clamped
    uint32_t v;
    if constexpr (IDB == 1) v = static_cast<const uint8_t *>(ids)[i];
    else v = static_cast<const uint32_t *>(ids)[i];
    bad |= v > p.mmask;
    return min(v, p.mmask);
  };
  extern __shared__ uint8_t smraw[];
  // align to 1024 B by offsetting the shared pointer itself (an integer round
  // trip would turn every access below into a generic LD/ST)
  uint8_t *sm = smraw + ((1024u - (smem_u32(smraw) & 1023u)) & 1023u);
  uint32_t *keys_s = reinterpret_cast<uint32_t *>(sm + Ly::O_KS);
  uint32_t *vals_s = reinterpret_cast<uint32_t *>(sm + Ly::O_VS);
  uint8_t *cnt = sm + Ly::O_CNT;
  uint32_t *wsum = reinterpret_cast<uint32_t *>(sm + Ly::O_WS);
  uint64_t *bar_k = reinterpret_cast<uint64_t *>(sm + Ly::O_BAR);
  uint64_t *bar_v = bar_k + STAGES;
  uint32_t *spl_s = reinterpret_cast<uint32_t *>(sm + Ly::O_SPL);
  uint32_t *tbl_s = reinterpret_cast<uint32_t *>(sm + Ly::O_TBL);

  const uint32_t tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  // block beta of this thread: the 32 lanes of a warp own 32 consecutive
  // counter words of a row (32 banks) whatever their ids; the staged block is
  // row beta >> 1, half beta & 1 of the swizzled 128-byte rows
  const uint32_t beta = 2 * lane + (warp & 1) + 64 * (warp >> 1);
  // (K = 32: the block is the whole swizzled row beta)
  const uint32_t srow = K == 16 ? beta >> 1 : beta, shalf = K == 16 ? beta & 1 : 0;
  // K = 32: the lanes of a quarter warp read rows 2 apart, which the 128B swizzle maps onto only 4
  // chunk positions; lanes 4..7 (mod 8) read their chunks rotated by one (step c -> chunk c + 1),
  // so every 128-bit stage load is conflict-free, and phase 2 rotates the registers back
  const uint32_t rot = K == 32 ? (lane >> 2) & 1u : 0u;
  uint32_t choff[NCH];  // byte offsets of the block's chunks inside a stage (128B swizzle)
#pragma unroll
  for (int c = 0; c < NCH; ++c)
    choff[c] = srow * 128 + 16 * ((NCH * shalf + ((c + rot) & (NCH - 1))) ^ (srow & 7));
  const uint32_t m = p.m;
  const uint32_t b0 = beta * K;
  // c[j][beta] at shared address ccol + j * RS
  const uint32_t ccol = smem_u32(cnt) + 2 * beta + 16 * (beta >> 6);
  const uint32_t ks32 = smem_u32(keys_s), vs32 = smem_u32(vals_s);

  const uint64_t r0 = RANGED ? (uint64_t)blockIdx.x * L / gridDim.x : 0;
  const uint32_t iters = RANGED ? (uint32_t)((uint64_t)(blockIdx.x + 1) * L / gridDim.x - r0)
                                : (blockIdx.x < L ? (L - 1 - blockIdx.x) / gridDim.x + 1 : 0);
  auto tile_of = [&](uint32_t it) -> uint64_t {
    if constexpr (ONE) return r0 + iters - 1 - it;  // phase 2: reverse walk
    return RANGED ? r0 + it : (uint64_t)blockIdx.x + (uint64_t)it * gridDim.x;
  };
  const uint64_t Lfull = n / T;  // tiles the TMA loads; a partial last tile is loaded by hand
  // ONE: full tiles of the range, and whether the range ends with the partial tile
  const uint32_t nf = ONE ? (uint32_t)(umin64(r0 + iters, Lfull) > r0 ? umin64(r0 + iters, Lfull) - r0 : 0) : 0;
  const uint32_t ptail = ONE ? iters - nf : 0;  // 0 or 1
  // ONE, key-only (two stages): phase 1 reads the keys through the TMA stages too (measured
  // better than plain loads: C2 389 vs 371 G keys/s); key-value (one stage): plain coalesced loads
  constexpr bool P1TMA = ONE && !KV && KIND != IDS;
  // ... and with a single key stage (the 8192-key tiles) phase 1 double-buffers through the reorder
  // buffer, which phase 2 needs only later: odd phase-1 tiles land there, on the (unused key-only)
  // value mbarrier, so one tile's load is in flight while the previous one is counted
#ifndef MS_P1X
#define MS_P1X 1
#endif
  constexpr bool P1X = MS_P1X && P1TMA && STAGES == 1;
  // TMA sequence numbers: ONE keys: [P1TMA: phase 1 forward over the nf full tiles, then] phase 2
  // reverse; ONE values: phase 2 only.  Otherwise sequence = iteration.
  auto seq_tile = [&](uint32_t sq, bool values) -> uint64_t {
    if constexpr (ONE) {
      if (P1TMA && !values && sq < nf) return r0 + sq;
      const uint32_t j = (P1TMA && !values) ? sq - nf : sq;
      return r0 + nf - 1 - j;
    }
    return tile_of(sq);
  };
  auto issue = [&](uint32_t it, bool values) {  // one thread: TMA of sequence `it` into its stage
    const uint64_t tile = seq_tile(it, values);
    if (tile >= Lfull) return;
    const int st = (int)(it % STAGES);
    if (!values) {
      mbar_arrive_expect_tx(bar_k + st, TB);
      tma_load_2d(sm + Ly::O_SK + st * TB, &tmk, 0, (int)(tile * (T / 32)), bar_k + st);
    } else {
      mbar_arrive_expect_tx(bar_v + st, TB);
      tma_load_2d(sm + Ly::O_SV + st * TB, &tmv, 0, (int)(tile * (T / 32)), bar_v + st);
    }
  };

  if (tid == 0) {
#pragma unroll
    for (int s = 0; s < STAGES; ++s) {
      mbar_init(bar_k + s, 1);
      mbar_init(bar_v + s, 1);
    }
    fence_mbar_init();
    const uint32_t nk = ONE ? (P1TMA ? 2 * nf : nf) : iters, nv = ONE ? nf : iters;
    for (uint32_t s = 0; s < (uint32_t)STAGES; ++s) {
      if (s < nk) issue(s, false);
      if constexpr (KV) {
        if (s < nv) issue(s, true);
      }
    }
    if constexpr (P1X) {
      if (nf >= 2) {
        mbar_arrive_expect_tx(bar_v, TB);
        tma_load_2d(sm + Ly::O_KS, &tmk, 0, (int)((r0 + 1) * (T / 32)), bar_v);
      }
    }
  }
  if constexpr (KIND == SPLITTERS) {
    for (uint32_t i = tid; i < (1u << p.logm); i += NT) spl_s[i] = p.spl[i];
    __syncthreads();
    build_spl_table<NT>(tbl_s, spl_s, p.logm);
  }
  auto id_of = [&](uint32_t key) -> uint32_t {
    if constexpr (KIND == SPLITTERS) return id_spl_table(key, tbl_s, spl_s);
    else return bucket_of_key<KIND>(key, p, spl_s);
  };

  pdl_wait();  // K2's G / GB is complete (the first tiles' loads above are already in flight)
  uint32_t gnext = 0;  // tile mode: the next tile's G column
  uint32_t grun = 0;   // RANGED: G_row of the current tile (all threads of bucket row `row`)
  const uint32_t row = tid >> (LOGNT - LOGMP);
  uint32_t *tot_s = reinterpret_cast<uint32_t *>(sm + Ly::O_TOT);
  if constexpr (ONE) {
    // ---- phase 1: this range's bucket counts (private u16 counter columns,
    // folded into tot_s every 32768 / K tiles so that no counter exceeds 32768)
    constexpr uint32_t FOLDT = 32768u / K;
    if (tid < (MP > 32 ? MP : 32)) tot_s[tid] = 0;
    auto zero_cnt = [&]() {
      uint4 *c4 = reinterpret_cast<uint4 *>(cnt);
      for (int idx = tid; idx < Ly::CNTB / 16; idx += NT) c4[idx] = make_uint4(0, 0, 0, 0);
    };
    auto fold = [&]() {  // row sums of the counter matrix -> tot_s (then zero it)
      __syncthreads();
      constexpr uint32_t SEGS1 = NT >> LOGMP;  // threads per row, each 2*MP... plain bytes
      constexpr uint32_t BPT = 2 * NT / SEGS1;  // bytes of a row per thread (= 2 * MP)
      const uint32_t rr = tid / SEGS1, q = BPT * (tid % SEGS1);
      uint32_t sum = 0;
      for (uint32_t bq = 0; bq < BPT; bq += 4) {
        const uint32_t o = q + bq;
        sum = __dp2a_lo(*reinterpret_cast<const uint32_t *>(cnt + rr * RS + o + 16 * (o >> 7)), 0x0101u, sum);
      }
      if (rr < m && sum) atomicAdd(tot_s + rr, sum);
      __syncthreads();
      zero_cnt();
      __syncthreads();
    };
    zero_cnt();
    __syncthreads();
    auto count_id = [&](uint32_t id) {
      const uint32_t a = ccol + id * RS;
      red_inc_u16(a);
    };
    auto count1 = [&](uint32_t key) { count_id(id_of(key)); };
    // counting needs no key-to-thread order: coalesced 128-bit loads (chunk j*NT + tid of the
    // tile), the next tile's loads issued before this one is counted (register double buffer)
    auto ld = [&](uint32_t sq, uint4 *dst) {
      const uint4 *t4 = reinterpret_cast<const uint4 *>(keys + (r0 + sq) * T);
#pragma unroll
      for (int c = 0; c < NCH; ++c) dst[c] = __ldg(t4 + c * NT + tid);
    };
    auto cnt4 = [&](const uint4 *x) {
#pragma unroll
      for (int c = 0; c < NCH; ++c) {
        count1(x[c].x); count1(x[c].y); count1(x[c].z); count1(x[c].w);
      }
    };
    if constexpr (P1TMA) {
      for (uint32_t sq = 0; sq < nf; ++sq) {
        const bool odd = P1X && (sq & 1u);
        if (P1X) mbar_wait(odd ? bar_v : bar_k, (sq >> 1) & 1u);
        else mbar_wait(bar_k + sq % STAGES, (sq / STAGES) & 1u);
        const uint8_t *sk = odd ? sm + Ly::O_KS : sm + Ly::O_SK + (sq % STAGES) * TB;
        uint4 kx[NCH];
#pragma unroll
        for (int c = 0; c < NCH; ++c) kx[c] = *reinterpret_cast<const uint4 *>(sk + choff[c]);
        cnt4(kx);
        // the stage may be refilled only once every thread's loads of it have
        // RETURNED (values consumed above), not merely been issued
        __syncthreads();
        if constexpr (P1X) {
          if (tid == 0) {
            if (sq + 2 < nf) {  // the next tile of this buffer
              mbar_arrive_expect_tx(odd ? bar_v : bar_k, TB);
              tma_load_2d(odd ? sm + Ly::O_KS : sm + Ly::O_SK, &tmk, 0, (int)((r0 + sq + 2) * (T / 32)),
                          odd ? bar_v : bar_k);
            } else if (!odd) {
              issue(nf, false);  // phase 2's first tile into the key stage (exactly one of the last two)
            }
          }
        } else {
          if (tid == 0 && sq + STAGES < 2 * nf) issue(sq + STAGES, false);
        }
        if ((sq & (FOLDT - 1)) == FOLDT - 1) fold();
      }
    }
    if constexpr (KIND == IDS) {  // precomputed ids: phase 1 reads only the ids (coalesced 16-byte chunks)
      constexpr int CH = IDB == 1 ? K / 16 : NCH;  // 16-byte chunks per thread per tile
      for (uint32_t sq = 0; sq < nf; ++sq) {
        const uint64_t tb = (r0 + sq) * T;
#pragma unroll
        for (int c = 0; c < CH; ++c) {
          uint32_t w[4];
          load_ids_full(tb + (uint64_t)(IDB == 1 ? 16 : 4) * (c * NT + tid), w, IDB == 1 ? 4 : 1);
#pragma unroll
          for (int q = 0; q < (IDB == 1 ? 4 : 1); ++q) {
            count_id(w[q] & 255u); count_id((w[q] >> 8) & 255u);
            count_id((w[q] >> 16) & 255u); count_id(w[q] >> 24);
          }
        }
        if ((sq & (FOLDT - 1)) == FOLDT - 1) fold();
      }
    }
    constexpr bool P1LD = !P1TMA && KIND != IDS;  // key-value, computed ids: plain loads of the keys
    uint4 xa[P1LD ? NCH : 1], xb[P1LD ? NCH : 1];
    if (P1LD && nf) ld(0, xa);
    for (uint32_t sq = 0; P1LD && sq < nf;) {
      if (sq + 1 < nf) ld(sq + 1, xb);
      cnt4(xa);
      if ((sq & (FOLDT - 1)) == FOLDT - 1) fold();
      if (++sq >= nf) break;
      if (sq + 1 < nf) ld(sq + 1, xa);
      cnt4(xb);
      if ((sq & (FOLDT - 1)) == FOLDT - 1) fold();
      ++sq;
    }
    if (ptail) {  // the partial last tile of the input
      const uint64_t base = (r0 + nf) * T;
      const uint32_t nt = (uint32_t)(n - base);
      for (uint32_t q = 0; q < (uint32_t)K; ++q)
        if (b0 + q < nt) {
          if constexpr (KIND == IDS) count_id(load_id1(base + b0 + q));
          else count1(__ldg(keys + base + b0 + q));
        }
    }
    fold();
    if (tid < m) const_cast<uint32_t *>(rs.HC)[(uint64_t)blockIdx.x * m + tid] = tot_s[tid];
    __threadfence();
    cooperative_groups::this_grid().sync();
    RangeScan r1 = rs;  // one row per CTA range
    r1.R = gridDim.x;
    r1.k = 1;
    grun = range_base<NT, LOGMP>(r1, m, blockIdx.x, n, keys_s, row);
    if (row < m) grun += tot_s[row];  // the reverse walk counts down from the range's end
    __syncthreads();
  } else if constexpr (RANGED) {
    // the range scan (Eq. (2) terms 1+2 over ranges) from K1r's rows (keys_s is free until tile 0)
    grun = range_base<NT, LOGMP>(rs, m, blockIdx.x, n, keys_s, row);
    __syncthreads();
  } else {
    if (iters && tid < m) gnext = __ldg(G + (uint64_t)tid * L + tile_of(0));
  }

  // one tile; FULL (compile time): all T keys valid, TMA-staged.  The partial
  // tile (at most one, the last of its CTA) is peeled off the loop
  // MS_IDS with u8 ids: the next full tile's K ids of this thread are loaded one tile ahead
  // (a register double buffer), so their HBM latency overlaps a whole tile instead of stalling the
  // counting pass
  uint4 idpre[K / 16] = {};
  auto id_prefetch = [&](uint32_t it) {
    if constexpr (KIND == IDS && IDB == 1) {
      if (it < iters && tile_of(it) < Lfull) {
        const uint4 *src = reinterpret_cast<const uint4 *>(static_cast<const uint8_t *>(ids) + tile_of(it) * T + b0);
#pragma unroll
        for (int q = 0; q < K / 16; ++q) idpre[q] = __ldcs(src + q);
      }
    }
  };
  id_prefetch(ONE ? ptail : 0u);  // the first full tile of the walk
  auto tile_body = [&](uint32_t it, auto fullc) {
    constexpr bool FULL = decltype(fullc)::value;
    const uint64_t tile = tile_of(it);
    const uint64_t base = tile * T;
    const uint32_t nt = FULL ? (uint32_t)T : (uint32_t)(n - base);
    // key / value TMA sequence numbers of this tile (ONE: phase 1 used keys 0..nf-1;
    // a partial tile, processed first in the reverse walk, has none)
    const uint32_t kq = ONE ? (P1TMA ? nf : 0u) + it - ptail : it, vq = ONE ? it - ptail : it;
    const int st = (int)(kq % STAGES);
    // (P1X: the key mbarrier completed (nf + 1) / 2 phase-1 loads before phase 2's first)
    const uint32_t ph = P1X ? ((nf + 1) / 2 + kq - nf) & 1u : (kq / STAGES) & 1u;
    const int vst = (int)(vq % STAGES);
    const uint32_t vph = (vq / STAGES) & 1u;
    uint32_t *meta = reinterpret_cast<uint32_t *>(sm + Ly::O_META) + (it & 1) * Ly::MW;
    uint32_t *rowS = meta;          // [MP+4]
    uint32_t *Pj = meta + MP + 4;   // [MP]
    uint32_t *Gj = Pj + MP;         // [MP]
    uint32_t *Dj = Gj + MP;         // [MP] DIRECT: G_j - P_j

    // ---- 0. zero the counters (last read by the previous tile's scatter,
    // before its final barrier) -- the plain 16-byte chunks only, not the
    // padding (chunk c of row r at r * RS + 16 * (c + c / 8)); publish this
    // tile's G column
    {
      constexpr int CPR = 2 * NT / 16, PCH = MP * CPR;
#pragma unroll
      for (int i = 0; i < (PCH + NT - 1) / NT; ++i) {
        const int idx = i * NT + tid;
        const int r = idx / CPR, c = idx % CPR;
        if (idx < PCH) *reinterpret_cast<uint4 *>(cnt + r * RS + 16 * (c + (c >> 3))) = make_uint4(0, 0, 0, 0);
      }
    }
    if constexpr (!RANGED) {
      if (tid < m) Gj[tid] = gnext;
      if (it + 1 < iters && tid < m) gnext = __ldg(G + (uint64_t)tid * L + tile_of(it + 1));
    }
    __syncthreads();

    // ---- 1. this thread's block -> registers; sequential counting into the
    // private counter column (the value read is the key's rank in the block)
    uint4 kx[NCH];
    if constexpr (FULL) {
      mbar_wait(bar_k + st, ph);
      const uint8_t *sk = sm + Ly::O_SK + st * TB;
      uint4 raw[NCH];
#pragma unroll
      for (int c = 0; c < NCH; ++c) raw[c] = *reinterpret_cast<const uint4 *>(sk + choff[c]);
#pragma unroll
      for (int c = 0; c < NCH; ++c) kx[c] = rot ? raw[(c + NCH - 1) & (NCH - 1)] : raw[c];
    } else {
      uint32_t t[K];
#pragma unroll
      for (int q = 0; q < K; ++q) t[q] = b0 + q < nt ? __ldg(keys + base + b0 + q) : 0u;
#pragma unroll
      for (int c = 0; c < NCH; ++c) kx[c] = make_uint4(t[4 * c], t[4 * c + 1], t[4 * c + 2], t[4 * c + 3]);
    }
    uint32_t rk[NCH];                   // ranks (< K), one byte each
    uint32_t idk[KEEP_ID ? NCH : 1];    // kept ids, one byte each
    if constexpr (KIND == IDS) {
      if constexpr (FULL && IDB == 1) {
#pragma unroll
        for (int q = 0; q < K / 16; ++q) {
          idk[4 * q] = clamp4(idpre[q].x); idk[4 * q + 1] = clamp4(idpre[q].y);
          idk[4 * q + 2] = clamp4(idpre[q].z); idk[4 * q + 3] = clamp4(idpre[q].w);
        }
        id_prefetch(it + 1);
      } else if constexpr (FULL) {
        load_ids_full(base + b0, idk, 4);
      } else {
#pragma unroll
        for (int c = 0; c < NCH; ++c) {
          uint32_t t4[4];
#pragma unroll
          for (int j = 0; j < 4; ++j) t4[j] = b0 + 4 * c + j < nt ? load_id1(base + b0 + 4 * c + j) : 0u;
          idk[c] = t4[0] | (t4[1] << 8) | (t4[2] << 16) | (t4[3] << 24);
        }
      }
    }
#pragma unroll
    for (int c = 0; c < NCH; ++c) {
      const uint32_t kk[4] = {kx[c].x, kx[c].y, kx[c].z, kx[c].w};
      rk[c] = 0u;
      if constexpr (KEEP_ID && KIND != IDS) idk[c] = 0u;
#pragma unroll
      for (int j = 0; j < 4; ++j) {
        if (FULL || b0 + 4 * c + j < nt) {
          uint32_t id;
          if constexpr (KIND == IDS) id = __byte_perm(idk[c], 0u, 0x4440u + j);
          else id = id_of(kk[j]);
          const uint32_t a = ccol + id * RS;
          const uint32_t r = atom_inc_u16(a);
          rk[c] |= r << (8 * j);
          if constexpr (KEEP_ID && KIND != IDS) idk[c] |= id << (8 * j);
        }
      }
    }
    __syncthreads();
    // the key stage is free again (keys are in registers): refill it
    if (FULL && tid == 0 && kq + STAGES < (ONE ? (P1TMA ? 2 * nf : nf) : iters)) issue(kq + STAGES, false);

    // ---- 2. CTA exclusive scan of the row-vectorised counter matrix:
    // thread t owns plain words [t*WPT, (t+1)*WPT) (inside one bucket row)
    constexpr int WPT = MP / 2;
    constexpr int NC = WPT >= 4 ? WPT / 4 : 1;
    constexpr int CWD = WPT >= 4 ? 4 : WPT;
    constexpr uint32_t SEGS = 2 * NT / (4 * WPT);  // segments per row
    const uint32_t q = 4 * WPT * (tid % SEGS);     // plain byte offset inside row tid / SEGS
    uint8_t *seg = cnt + (tid / SEGS) * RS + q + 16 * (q >> 7);
    uint32_t w[NC][CWD];
    uint32_t s = 0;
#pragma unroll
    for (int i = 0; i < NC; ++i) {
      const uint8_t *src = seg + 16 * i;
      if constexpr (CWD == 4) {
        const uint4 x = *reinterpret_cast<const uint4 *>(src);
        w[i][0] = x.x; w[i][1] = x.y; w[i][2] = x.z; w[i][3] = x.w;
      } else if constexpr (CWD == 2) {
        const uint2 x = *reinterpret_cast<const uint2 *>(src);
        w[i][0] = x.x; w[i][1] = x.y;
      } else {
        w[i][0] = *reinterpret_cast<const uint32_t *>(src);
      }
#pragma unroll
      for (int j = 0; j < CWD; ++j) s = __dp2a_lo(w[i][j], 0x0101u, s);  // += lo + hi
    }
    const uint32_t incl = warp_incl_scan(s, lane);
    if (lane == 31) wsum[warp] = incl;
    __syncthreads();
    uint32_t wpre = 0, tot = 0;
#pragma unroll
    for (int i = 0; i < NW; ++i) {
      const uint32_t x = wsum[i];
      wpre += (i < (int)warp) ? x : 0u;
      tot += x;
    }
    const uint32_t excl = wpre + incl - s;
    constexpr uint32_t TPR = NT >> LOGMP;  // threads per bucket row
    uint32_t Sr;                           // S_row = excl of the row's first thread
    if constexpr (TPR < 32) {
      Sr = __shfl_sync(0xFFFFFFFFu, excl, lane & ~(TPR - 1));
    } else {
      Sr = 0;
      const uint32_t w0 = (row * TPR) >> 5;
#pragma unroll
      for (int i = 0; i < NW; ++i) Sr += ((uint32_t)i < w0) ? wsum[i] : 0u;
    }
    if ((tid & (TPR - 1)) == 0) rowS[row] = excl;
    if (tid == 0) rowS[MP] = tot;
    uint32_t Gr;
    if constexpr (RANGED) {
      if constexpr (!ONE) Gr = grun;
      uint32_t rtot;  // this tile's count of bucket `row`
      if constexpr (TPR < 32) {
        rtot = __shfl_sync(0xFFFFFFFFu, excl + s, lane | (TPR - 1)) - Sr;
      } else {
        rtot = 0;
        const uint32_t w0 = (row * TPR) >> 5;
#pragma unroll
        for (int i = 0; i < NW; ++i) rtot += ((uint32_t)i >= w0 && (uint32_t)i < w0 + TPR / 32) ? wsum[i] : 0u;
      }
      if constexpr (ONE) {
        grun -= rtot;
        Gr = grun;
      } else {
        grun += rtot;
      }
      if ((tid & (TPR - 1)) == 0) Gj[row] = Gr;
    } else {
      Gr = row < m ? Gj[row] : 0u;  // (fused sharded scatter: replaced by the destination offset below)
    }
    if constexpr (!RANGED) {
      // fused sharded scatter: align the run to its destination offset in the
      // window that owns its first key (global position G_j + delta_j)
      if (ds.P > 0 && row < m) {
        const uint64_t gs = (uint64_t)Gr + ds.delta[row];
        uint32_t r = 0;
        for (int i = 1; i < ds.P; ++i) r += gs >= ds.wst[i] ? 1u : 0u;
        Gr = (uint32_t)(gs - ds.wst[r]);
      }
    }
    // padded run start P_j = S_j + 3j + ((G_j - S_j - 3j) & 3): P_j = G_j (mod 4)
    // and P_j >= P_{j-1} + h_{j-1}; closed form, no serial dependency over j
    const uint32_t pad = 3 * row + ((Gr - Sr - 3 * row) & 3u);
    uint32_t run = excl + pad;
#pragma unroll
    for (int i = 0; i < NC; ++i) {
#pragma unroll
      for (int j = 0; j < CWD; ++j) {
        const uint32_t x = w[i][j];
        w[i][j] = x * 0x10000u + run * 0x10001u;  // (run, run + lo)
        run = __dp2a_lo(x, 0x0101u, run);         // run + lo + hi
      }
      uint8_t *dst = seg + 16 * i;
      if constexpr (CWD == 4) *reinterpret_cast<uint4 *>(dst) = make_uint4(w[i][0], w[i][1], w[i][2], w[i][3]);
      else if constexpr (CWD == 2) *reinterpret_cast<uint2 *>(dst) = make_uint2(w[i][0], w[i][1]);
      else *reinterpret_cast<uint32_t *>(dst) = w[i][0];
    }
    if ((tid & (TPR - 1)) == 0) Pj[row] = Sr + pad;
    if constexpr (DIRECT) {
      if ((tid & (TPR - 1)) == 0) Dj[row] = Gr - (Sr + pad);
    }
    bulk_wait_read0();  // this thread's bulk stores of the previous tile have read keys_s/vals_s
    __syncthreads();

    // ---- 3. local multisplit of the tile into shared memory
    uint4 vy[KV ? NCH : 1];
    if constexpr (KV) {
      if constexpr (FULL) {
        mbar_wait(bar_v + vst, vph);
        const uint8_t *sv = sm + Ly::O_SV + vst * TB;
#pragma unroll
        for (int c = 0; c < NCH; ++c) vy[c] = *reinterpret_cast<const uint4 *>(sv + choff[c]);
        if (rot) {  // (K = 32) back to block order
          const uint4 last = vy[NCH - 1];
#pragma unroll
          for (int c = NCH - 1; c > 0; --c) vy[c] = vy[c - 1];
          vy[0] = last;
        }
      } else {
        uint32_t t[K];
#pragma unroll
        for (int q = 0; q < K; ++q) t[q] = b0 + q < nt ? __ldg(vals + base + b0 + q) : 0u;
#pragma unroll
        for (int c = 0; c < NCH; ++c) vy[c] = make_uint4(t[4 * c], t[4 * c + 1], t[4 * c + 2], t[4 * c + 3]);
      }
    }
#pragma unroll
    for (int c = 0; c < NCH; ++c) {
      const uint32_t kk[4] = {kx[c].x, kx[c].y, kx[c].z, kx[c].w};
      uint32_t vv[4];
      if constexpr (KV) {
        vv[0] = vy[c].x; vv[1] = vy[c].y; vv[2] = vy[c].z; vv[3] = vy[c].w;
      }
      uint32_t sl[4], idv[4];
#pragma unroll
      for (int j = 0; j < 4; ++j) {
        uint32_t id;
        if constexpr (KEEP_ID) id = __byte_perm(idk[c], 0u, 0x4440u + j);
        else id = id_of(kk[j]);
        idv[j] = id;
        sl[j] = (FULL || b0 + 4 * c + j < nt) ? lds_u16(ccol + id * RS) : 0u;
      }
#pragma unroll
      for (int j = 0; j < 4; ++j) {
        if (FULL || b0 + 4 * c + j < nt) {
          const uint32_t slot = sl[j] + __byte_perm(rk[c], 0u, 0x4440u + j);
          if constexpr (DIRECT) {
            const uint32_t dst = Dj[idv[j]] + slot;
            keys_out[dst] = kk[j];
            if constexpr (KV) vals_out[dst] = vv[j];
          } else {
            sts_u32(ks32 + 4 * slot, kk[j]);
            if constexpr (KV) sts_u32(vs32 + 4 * slot, vv[j]);
          }
        }
      }
    }
    fence_proxy_async_smem();  // generic-proxy writes -> visible to the TMA (async proxy)
    __syncthreads();
    if constexpr (KV) {  // the value stage is free again: refill it
      if (FULL && tid == 0 && vq + STAGES < (ONE ? nf : iters)) issue(vq + STAGES, true);
    }

    // ---- 4. bucket runs: SPB threads per bucket share its <= 3 head keys,
    // <= 3 tail keys and the TMA bulk store(s) of the 16-byte-aligned body
    if (DIRECT) {
      // (stored in step 3)
    } else if (!RANGED && ds.P > 0) {
      // fused sharded scatter: the run [gs, gs + len) of global positions is
      // cut at window boundaries; each piece goes to its owner's window, the
      // 16-byte-aligned body by one TMA bulk store per array (peer memory is
      // plain global memory to the TMA), the rest by the SPB threads
      constexpr uint32_t SPB = NT / 32;
      const uint32_t b = tid / SPB, sub = tid % SPB;
      if (b < m) {
        uint32_t left = rowS[b + 1] - rowS[b];
        uint32_t src = Pj[b];
        uint64_t gs = (uint64_t)Gj[b] + ds.delta[b];
        while (left) {
          if (gs >= ds.wst[ds.P]) {  // inconsistent target (a run past the last window): store nothing
            atomicOr(flag, 2u);      // more, report it through ms_plan_check
            break;
          }
          uint32_t r = 0;
          for (int i = 1; i < ds.P; ++i) r += gs >= ds.wst[i] ? 1u : 0u;
          const uint64_t room = ds.wst[r + 1] - gs;
          const uint32_t len = room < left ? (uint32_t)room : left;
          const uint64_t doff = gs - ds.wst[r];
          uint32_t *dk = ds.keys[r] + doff;
          uint32_t *dv = KV ? ds.vals[r] + doff : nullptr;
          uint32_t head = min(len, (4u - (uint32_t)(doff & 3u)) & 3u);
          uint32_t body = (len - head) & ~3u;
          if (((src + head) & 3u) != 0u) {  // source and destination disagree mod 16 B: no bulk copy
            head = len;
            body = 0;
          }
          for (uint32_t i = sub; i < head; i += SPB) {
            dk[i] = keys_s[src + i];
            if constexpr (KV) dv[i] = vals_s[src + i];
          }
          for (uint32_t i = head + body + sub; i < len; i += SPB) {
            dk[i] = keys_s[src + i];
            if constexpr (KV) dv[i] = vals_s[src + i];
          }
          if (body && (sub == SPB - 1 || (KV && sub == SPB - 2))) {
            if (sub == SPB - 1) bulk_s2g(dk + head, keys_s + src + head, body * 4u);
            else bulk_s2g(dv + head, vals_s + src + head, body * 4u);
            bulk_commit();
          }
          gs += len;
          src += len;
          left -= len;
        }
      }
    } else {
      constexpr uint32_t SPB = NT / (MP > 32 ? MP : 32);  // threads per bucket run
      const uint32_t b = tid / SPB, sub = tid % SPB;
      if (b < m) {
        const uint32_t len = rowS[b + 1] - rowS[b];
        const uint32_t P = Pj[b], Gd = Gj[b];
        const uint32_t head = min(len, (4u - (Gd & 3u)) & 3u);
        const uint32_t body = (len - head) & ~3u;
        if constexpr (SPB == 8) {
          if (sub < 6) {
            const uint32_t i = sub < 3 ? sub : head + body + (sub - 3);
            if ((sub < 3 && sub < head) || (sub >= 3 && i < len)) {
              keys_out[Gd + i] = keys_s[P + i];
              if constexpr (KV) vals_out[Gd + i] = vals_s[P + i];
            }
          } else if (body && (sub == 6 || KV)) {
            if (sub == 6) bulk_s2g(keys_out + Gd + head, keys_s + P + head, body * 4u);
            else bulk_s2g(vals_out + Gd + head, vals_s + P + head, body * 4u);
            bulk_commit();
          }
        } else if constexpr (SPB == 2) {  // (NT = 64) sub 0: head, tail, keys body; sub 1: values body
          if (sub == 0) {
            for (uint32_t i = 0; i < head; ++i) {
              keys_out[Gd + i] = keys_s[P + i];
              if constexpr (KV) vals_out[Gd + i] = vals_s[P + i];
            }
            for (uint32_t i = head + body; i < len; ++i) {
              keys_out[Gd + i] = keys_s[P + i];
              if constexpr (KV) vals_out[Gd + i] = vals_s[P + i];
            }
          }
          if (body && (sub == 0 || KV)) {
            if (sub == 0) bulk_s2g(keys_out + Gd + head, keys_s + P + head, body * 4u);
            else bulk_s2g(vals_out + Gd + head, vals_s + P + head, body * 4u);
            bulk_commit();
          }
        } else {  // SPB == 4: head / tail / keys body / values body
          if (sub < 2) {
            const uint32_t i0 = sub == 0 ? 0u : head + body, i1 = sub == 0 ? head : len;
            for (uint32_t i = i0; i < i1; ++i) {
              keys_out[Gd + i] = keys_s[P + i];
              if constexpr (KV) vals_out[Gd + i] = vals_s[P + i];
            }
          } else if (body && (sub == 2 || KV)) {
            if (sub == 2) bulk_s2g(keys_out + Gd + head, keys_s + P + head, body * 4u);
            else bulk_s2g(vals_out + Gd + head, vals_s + P + head, body * 4u);
            bulk_commit();
          }
        }
      }
    }
  };
  if constexpr (ONE) {  // reverse walk: the partial tile (if any) comes first
    if (ptail) tile_body(0u, std::false_type{});
    for (uint32_t it = ptail; it < iters; ++it) tile_body(it, std::true_type{});
  } else {
    const bool has_tail = iters && tile_of(iters - 1) >= Lfull;
    const uint32_t iters_full = iters - (has_tail ? 1u : 0u);
    for (uint32_t it = 0; it < iters_full; ++it) tile_body(it, std::true_type{});
    if (has_tail) tile_body(iters_full, std::false_type{});
  }
  if constexpr (KIND == IDS) {
    if (p.validate && __any_sync(0xFFFFFFFFu, bad != 0) && lane == 0) atomicOr(flag, 1u);
  }
  if (ds.P > 0) bulk_wait0();  // peer stores complete before the grid ends (made visible by the stream order)
  else bulk_wait_read0();
}

// ------------------------------------------------------------------ host launcher
inline PFN_cuTensorMapEncodeTiled_v12000 tensor_map_encoder() {
  static PFN_cuTensorMapEncodeTiled_v12000 fn = nullptr;
  if (!fn) {
    void *f = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &f, cudaEnableDefault, &q) == cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      fn = reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(f);
  }
  return fn;
}

// keys (or values) of the `full` tiles as a [rows][32] u32 tensor, box = T/32 rows, 128B swizzle
inline bool make_tile_map(CUtensorMap *tm, const uint32_t *ptr, uint64_t rows, uint32_t T) {
  memset(tm, 0, sizeof(*tm));
  if (!ptr || rows == 0) return true;  // no full tile: the map is never used
  auto enc = tensor_map_encoder();
  if (!enc) return false;
  const cuuint64_t dims[2] = {32, rows};
  const cuuint64_t strides[1] = {128};
  const cuuint32_t box[2] = {32, T / 32};
  const cuuint32_t es[2] = {1, 1};
  return enc(tm, CU_TENSOR_MAP_DATA_TYPE_UINT32, 2, const_cast<uint32_t *>(ptr), dims, strides, box, es,
             CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
             CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

template <int KIND, bool KV, int LOGMP, int NT, int STAGES, bool RANGED, bool ONE = false, bool DIRECT = false,
          int IDB = 0, int KPT = 16>
inline cudaError_t k3v_launch_one(const K3pArgs &a) {
  using Ly = K3vLayout<LOGMP, KV, NT, STAGES, KPT>;
  // CTAs per SM the register budget is sized for: key-value 2, key-only 3 -- and 4 for the
  // two-stage key-only m <= 8 form used on smaller inputs (k3v_launch_n)
  // (32 keys per thread: one key stage, 2 CTAs/SM)
  constexpr int MINB = KPT == 32 ? 2 : (KV ? 2 : (STAGES == 2 && LOGMP <= 3 ? 4 : 3)) * (256 / NT);
  auto k = k3v_postscan<KIND, KV, LOGMP, NT, STAGES, RANGED, MINB, KPT, ONE, DIRECT, IDB>;
  const size_t smem = (size_t)(KIND == SPLITTERS ? Ly::BYTES_SPL : Ly::BYTES) + 1024;
  cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  int per_sm = 0;
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k, NT, smem);
  if (per_sm <= 0) per_sm = 1;
  uint64_t g = umin64_host(a.L, (uint64_t)a.sms * per_sm);
  if (a.ranged) g = umin64_host(g, kMaxRanges);
  const unsigned grid = (unsigned)g;
  if (a.grid_out) {
    *a.grid_out = grid;
    return cudaSuccess;
  }
  const uint64_t rows = (uint64_t)(a.n / Ly::T) * (Ly::T / 32);
  CUtensorMap tmk, tmv;
  if (!make_tile_map(&tmk, a.keys, rows, Ly::T) || !make_tile_map(&tmv, KV ? a.vals : nullptr, rows, Ly::T))
    return cudaErrorInvalidValue;
  const cudaError_t e = ONE ? launch_coop(k, dim3(grid), dim3(NT), smem, a.stream, tmk, tmv, a.keys, a.vals, a.ids,
                                          a.flag, a.G, a.keys_out, a.vals_out, a.n, a.L, *a.bp, a.rs, DistTarget{})
                            : launch_ex(a.pdl != 0, k, dim3(grid), dim3(NT), smem, a.stream, tmk, tmv, a.keys,
                                        a.vals, a.ids, a.flag, a.G, a.keys_out, a.vals_out, a.n, a.L, *a.bp, a.rs,
                                        a.ds ? *a.ds : DistTarget{});
  return e != cudaSuccess ? e : cudaGetLastError();
}

template <int KIND, bool KV, int LOGMP, int IDB>
inline cudaError_t k3v_launch_n(const K3pArgs &a) {
  constexpr int NT = 256;
  if constexpr (LOGMP == 6) {  // 33..64 buckets: only the key-only ONE with 8192-key tiles
    if constexpr (!KV && (KIND != IDS || IDB == 1)) {
      if (a.ranged == 2 && a.kpt == 32 && a.nt == 256 && !a.direct)
        return k3v_launch_one<KIND, KV, LOGMP, NT, 1, true, true, false, IDB, 32>(a);
    }
    return cudaErrorNotSupported;
  } else {
  constexpr int STAGES = KV ? 1 : (LOGMP <= 3 ? 3 : 2);  // m <= 8 key-only: 3 stages still fit 3 CTAs/SM
  if (a.nt != 256) {  // ablation (NW sweep): 2 or 4 warps per CTA, ranged variant, one bucket kind
    if constexpr (KIND == SHIFT) {
      if (a.ranged != 1) return cudaErrorNotSupported;
      return a.nt == 128 ? k3v_launch_one<KIND, KV, LOGMP, 128, STAGES, true>(a)
                         : k3v_launch_one<KIND, KV, LOGMP, 64, STAGES, true>(a);
    }
    return cudaErrorNotSupported;
  }
  if (a.ranged == 2) {
    // key-only ONE with 8192-key tiles (32 per thread, one key stage, 2 CTAs per SM): half the
    // zeroing and scan of the counter matrix per key; ms_run passes kpt = 32 for every key-only run
    // of computed or u8 ids
    if (a.kpt == 32) {
      if constexpr (!KV && (KIND != IDS || IDB == 1) && (1 << LOGMP) >= MS_K32_MINM)
        return k3v_launch_one<KIND, KV, LOGMP, NT, 1, true, true, false, IDB, 32>(a);
      return cudaErrorInvalidValue;
    }
    // ONE, key-only, m <= 8 with 4096-key tiles (u32 ids): up to 64 tiles per SM two key stages at
    // 4 CTAs/SM (more CTAs to share the fixed cost and the tail), above that three stages at 3
    // CTAs/SM (the deeper prefetch wins for long streams)
    if constexpr (!KV && LOGMP <= 3) {
      if (a.L <= 64ull * (uint64_t)a.sms) return k3v_launch_one<KIND, KV, LOGMP, NT, 2, true, true, false, IDB>(a);
    }
    return k3v_launch_one<KIND, KV, LOGMP, NT, STAGES, true, true, false, IDB>(a);
  }
  if (a.direct) {  // ablation: instantiated for the one-shift bucket kind only (SHIFT: DELTA with m*delta = 2^32)
    if constexpr (KIND == SHIFT) return k3v_launch_one<KIND, KV, LOGMP, NT, STAGES, false, false, true>(a);
    return cudaErrorNotSupported;
  }
  return a.ranged ? k3v_launch_one<KIND, KV, LOGMP, NT, STAGES, true, false, false, IDB>(a)
                  : k3v_launch_one<KIND, KV, LOGMP, NT, STAGES, false, false, false, IDB>(a);
  }
}

template <int KIND, bool KV, int IDB>
inline cudaError_t k3v_launch_kv(const K3pArgs &a) {
  uint32_t l = 1;
  while ((1u << l) < a.m) ++l;
  switch (l) {
    case 1: return k3v_launch_n<KIND, KV, 1, IDB>(a);
    case 2: return k3v_launch_n<KIND, KV, 2, IDB>(a);
    case 3: return k3v_launch_n<KIND, KV, 3, IDB>(a);
    case 4: return k3v_launch_n<KIND, KV, 4, IDB>(a);
    case 5: return k3v_launch_n<KIND, KV, 5, IDB>(a);
    default: return k3v_launch_n<KIND, KV, 6, IDB>(a);
  }
}

template <int KIND>
inline cudaError_t k3v_launch(const K3pArgs &a) {
  if constexpr (KIND == IDS) {
    if (a.id_bytes == 1) return a.vals ? k3v_launch_kv<KIND, true, 1>(a) : k3v_launch_kv<KIND, false, 1>(a);
    return a.vals ? k3v_launch_kv<KIND, true, 4>(a) : k3v_launch_kv<KIND, false, 4>(a);
  } else {
    return a.vals ? k3v_launch_kv<KIND, true, 0>(a) : k3v_launch_kv<KIND, false, 0>(a);
  }
}

}  // namespace ms
