// ms_k3_lsd.cuh -- K3 post-scan for 32 < m <= 256: two-digit local multisplit (sm_100a).
//
// Same contract and paper steps as the other K3s: recompute ids (footnote 6,
// P:857-859), stable tile-local offsets (term 3 of Eq. (2)), a
// local stable multisplit of the tile in shared memory (§4 "reordering",
// P:689-713; §5.2.2 block-level reordering P:1262-1301), then every key goes
// to G[j][tile] + (slot - S_t[j]).
//
// What differs ("K3 for m > 32"): the tile-local multisplit by
// the 8-bit id is done as TWO stable local multisplits by 4-bit digits,
// least significant first -- by lo = id & 15, then by hi = id >> 4 -- which
// is the paper's own observation that a multisplit can be composed from
// stable multisplits on parts of the id (the reduced-bit / LSD view of §3.4,
// P:432-464), applied inside one tile.  Each digit pass is the blocked
// private-counter scheme of K3 v2 (ms_k3_v2.cuh) at 16 rows: thread beta
// counts its contiguous 16-key block into its own u16 counter column (the
// value read is the key's rank in the block), one CTA scan of the
// row-vectorised 16 x NT counter matrix gives every (digit, block) its start,
// and slot = start + rank.  Stable by construction (blocks are contiguous
// and ordered by beta; digit passes are stable), so pass 2 of the stable
// pass-1 order is the stable order by the whole id.  Per key this costs two
// counter read-modify-writes, two scatters and ~2 counter words of scan,
// instead of the 8 ballot rounds (~40 instructions) of Alg. 3.
//
// The tile histogram (256 buckets) is not counted at all: G is the exclusive
// scan of the row-vectorised H, so H[j][t] = G_flat[j*L + t + 1] - G_flat[j*L + t]
// (G_flat[m*L] = n), two adjacent words of the G matrix (one 32-byte sector).
// Its exclusive scan over j gives the tile's bucket starts S_t[j]; D[j] =
// G[j][t] - S_t[j], and the key in final slot i goes to D[id] + i.
//
// Tile = 256 threads x 16 keys = 4096 keys, persistent CTAs walking tiles
// blockIdx.x, blockIdx.x + gridDim.x, ...; keys (and values) staged by the
// TMA tensor engine with the 128-byte swizzle (as K3 v2); the pass-1 result
// is written with the same swizzle so that pass 2 reads each thread's
// 16-key block as four conflict-free 128-bit loads.
#pragma once
#include <cuda.h>
#include <cudaTypedefs.h>

#include <type_traits>

#include "ms_k3_v2.cuh"  // tma_load_2d, make_tile_map

namespace ms {

template <int LOGM, bool KV, int STAGES>
struct K3hLayout {
  static constexpr int NT = 256, K = 16, T = NT * K, TB = T * 4;
  static constexpr int LB = 4, HB = LOGM - LB;  // digit bits: lo (16 rows), hi (2^HB rows, 4..16)
  static constexpr int RA = 1 << LB, RB = 1 << HB;
  static constexpr int RS = (2 * NT + 2 * NT / 8 + 127) / 128 * 128;  // padded counter row stride (bytes)
  static constexpr int O_SK = 0;                                // [STAGES][T] staged keys (1024-B aligned)
  static constexpr int O_SV = O_SK + STAGES * TB;               // [STAGES][T] staged values
  static constexpr int O_X = O_SV + (KV ? STAGES * TB : 0);     // [T] keys after pass 1 (swizzled), pass 2 (linear)
  static constexpr int O_XV = O_X + TB;                         // [T] values
  static constexpr int O_XI = O_XV + (KV ? TB : 0);             // [T] u8 ids
  static constexpr int O_CA = O_XI + T;                         // pass-1 counters [RA][RS]
  static constexpr int O_CB = O_CA + RA * RS;                   // pass-2 counters [RB][RS]
  static constexpr int O_D = O_CB + RB * RS;                    // [256] D[j] = G[j][t] - S_t[j]
  static constexpr int O_WS = O_D + 256 * 4;                    // warp sums [3][8]
  static constexpr int O_BAR = (O_WS + 3 * 8 * 4 + 7) & ~7;     // mbarriers: keys [STAGES], values [STAGES]
  static constexpr int O_SPL = O_BAR + 2 * STAGES * 8;          // SPLITTERS: padded splitters [256] + bin table
  static constexpr int O_TBL = O_SPL + kMaxM * 4;
  static constexpr int BYTES = O_SPL;
  static constexpr int BYTES_SPL = O_TBL + kSplBins * 4;
};

__device__ __forceinline__ void sts_u8(uint32_t a, uint32_t v) {
  asm volatile("st.shared.u8 [%0], %1;" ::"r"(a), "h"((uint16_t)v) : "memory");
}

// CTA exclusive scan of a row-vectorised u16 counter matrix of 2^LR rows x 256
// columns (padded rows, see K3vLayout), in place: counter (j, beta) becomes the
// number of counted keys before it in row-major order.  Thread t owns plain
// words [t*WPT, (t+1)*WPT) of row t / SEGS.  Two barriers (one inside, one at
// the end).
template <int LR>
__device__ __forceinline__ void scan_counters(uint8_t *cnt, uint32_t *wsum, uint32_t tid) {
  constexpr int NT = 256, NW = NT / 32, RS = (2 * NT + 2 * NT / 8 + 127) / 128 * 128;
  constexpr int WPT = (1 << LR) / 2;
  constexpr int NC = WPT >= 4 ? WPT / 4 : 1;
  constexpr int CWD = WPT >= 4 ? 4 : WPT;
  constexpr uint32_t SEGS = 2 * NT / (4 * WPT);
  const uint32_t lane = tid & 31, warp = tid >> 5;
  const uint32_t q = 4 * WPT * (tid % SEGS);
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
    for (int j = 0; j < CWD; ++j) s = __dp2a_lo(w[i][j], 0x0101u, s);
  }
  const uint32_t incl = warp_incl_scan(s, lane);
  if (lane == 31) wsum[warp] = incl;
  __syncthreads();
  uint32_t run = incl - s;
#pragma unroll
  for (int i = 0; i < NW; ++i) run += (i < (int)warp) ? wsum[i] : 0u;
#pragma unroll
  for (int i = 0; i < NC; ++i) {
#pragma unroll
    for (int j = 0; j < CWD; ++j) {
      const uint32_t x = w[i][j];
      w[i][j] = x * 0x10000u + run * 0x10001u;  // (run, run + lo)
      run = __dp2a_lo(x, 0x0101u, run);
    }
    uint8_t *dst = seg + 16 * i;
    if constexpr (CWD == 4) *reinterpret_cast<uint4 *>(dst) = make_uint4(w[i][0], w[i][1], w[i][2], w[i][3]);
    else if constexpr (CWD == 2) *reinterpret_cast<uint2 *>(dst) = make_uint2(w[i][0], w[i][1]);
    else *reinterpret_cast<uint32_t *>(dst) = w[i][0];
  }
  __syncthreads();
}

template <int KIND, bool KV, int LOGM, int STAGES, int MINB>
__global__ void __launch_bounds__(256, MINB)
k3h_postscan(const __grid_constant__ CUtensorMap tmk, const __grid_constant__ CUtensorMap tmv,
             const uint32_t *__restrict__ keys, const uint32_t *__restrict__ vals,
             const uint32_t *__restrict__ G, uint32_t *__restrict__ keys_out, uint32_t *__restrict__ vals_out,
             uint32_t n, uint32_t L, const __grid_constant__ BucketParams p) {
  using Ly = K3hLayout<LOGM, KV, STAGES>;
  constexpr int NT = Ly::NT, K = Ly::K, T = Ly::T, TB = Ly::TB, RS = Ly::RS;
  constexpr int NW = NT / 32;
  // ids kept in registers from the counting pass; the store phase re-derives the
  // id from the key when that is one instruction, else reads the stored byte
  constexpr bool ID8 = !(KIND == SHIFT || KIND == LOWBITS);
  constexpr bool RECOMP = !ID8;  // one-instruction ids: recomputed in pass 2 and the stores, no id bytes
  extern __shared__ uint8_t smraw[];
  uint8_t *sm = smraw + ((1024u - (smem_u32(smraw) & 1023u)) & 1023u);
  uint32_t *wsum = reinterpret_cast<uint32_t *>(sm + Ly::O_WS);
  uint64_t *bar_k = reinterpret_cast<uint64_t *>(sm + Ly::O_BAR);
  uint64_t *bar_v = bar_k + STAGES;
  uint32_t *spl_s = reinterpret_cast<uint32_t *>(sm + Ly::O_SPL);
  uint32_t *tbl_s = reinterpret_cast<uint32_t *>(sm + Ly::O_TBL);

  const uint32_t tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const uint32_t beta = 2 * lane + (warp & 1) + 64 * (warp >> 1);
  const uint32_t srow = beta >> 1, shalf = beta & 1;
  uint32_t choff[4];  // byte offsets of block beta's 4 chunks in a swizzled [T] array
#pragma unroll
  for (int c = 0; c < 4; ++c) choff[c] = srow * 128 + 16 * ((4 * shalf + c) ^ (srow & 7));
  const uint32_t m = p.m;
  const uint32_t b0 = beta * K;
  const uint32_t colA = smem_u32(sm + Ly::O_CA) + 2 * beta + 16 * (beta >> 6);
  const uint32_t colB = smem_u32(sm + Ly::O_CB) + 2 * beta + 16 * (beta >> 6);
  const uint32_t x32 = smem_u32(sm + Ly::O_X), xv32 = smem_u32(sm + Ly::O_XV), xi32 = smem_u32(sm + Ly::O_XI);

  auto tile_of = [&](uint32_t it) -> uint64_t { return (uint64_t)blockIdx.x + (uint64_t)it * gridDim.x; };
  const uint32_t iters = blockIdx.x < L ? (L - 1 - blockIdx.x) / gridDim.x + 1 : 0;
  const uint64_t Lfull = n / T;
  const uint64_t mL = (uint64_t)m * L;
  auto issue = [&](uint32_t it, bool values) {
    const uint64_t tile = tile_of(it);
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
    for (uint32_t s = 0; s < (uint32_t)STAGES && s < iters; ++s) {
      issue(s, false);
      if constexpr (KV) issue(s, true);
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

  pdl_wait();  // K2's G is complete (the first tiles' TMA loads are already in flight)
  // G pair (G[j][t], next word of the flat G) of the next tile, for bucket j = tid
  auto load_gpair = [&](uint64_t tile, uint32_t &g0, uint32_t &g1) {
    g0 = g1 = 0;
    if (tid < m) {
      const uint64_t f = (uint64_t)tid * L + tile;
      g0 = __ldg(G + f);
      g1 = f + 1 < mL ? __ldg(G + f + 1) : n;
    }
  };
  uint32_t gn0 = 0, gn1 = 0;
  if (iters) load_gpair(tile_of(0), gn0, gn1);

  auto tile_body = [&](uint32_t it, auto fullc) {
    constexpr bool FULL = decltype(fullc)::value;
    const uint64_t tile = tile_of(it);
    const uint64_t base = tile * T;
    const uint32_t nt = FULL ? (uint32_t)T : (uint32_t)(n - base);
    const int st = (int)(it % STAGES);
    const uint32_t ph = (it / STAGES) & 1u;
    uint32_t *D = reinterpret_cast<uint32_t *>(sm + Ly::O_D);  // written in step 1, read in step 5

    // ---- 0. zero both counter matrices; this tile's histogram column
    // h_j = G_flat[f+1] - G_flat[f] and its scan (first half)
    {
      uint4 *c4 = reinterpret_cast<uint4 *>(sm + Ly::O_CA);
      constexpr int N16 = (Ly::RA + Ly::RB) * RS / 16;
#pragma unroll
      for (int i = 0; i < (N16 + NT - 1) / NT; ++i) {
        const int idx = i * NT + tid;
        if (idx < N16) c4[idx] = make_uint4(0, 0, 0, 0);
      }
    }
    const uint32_t g0 = gn0, hj = gn1 - gn0;
    if (it + 1 < iters) load_gpair(tile_of(it + 1), gn0, gn1);
    const uint32_t hincl = warp_incl_scan(hj, lane);
    if (lane == 31) wsum[16 + warp] = hincl;
    __syncthreads();

    // ---- 1. pass 1 (lo digit): block -> registers, private counting
    uint4 kx[4];
    if constexpr (FULL) {
      mbar_wait(bar_k + st, ph);
      const uint8_t *sk = sm + Ly::O_SK + st * TB;
#pragma unroll
      for (int c = 0; c < 4; ++c) kx[c] = *reinterpret_cast<const uint4 *>(sk + choff[c]);
    } else {
      uint32_t t[K];
#pragma unroll
      for (int q = 0; q < K; ++q) t[q] = b0 + q < nt ? __ldg(keys + base + b0 + q) : 0u;
#pragma unroll
      for (int c = 0; c < 4; ++c) kx[c] = make_uint4(t[4 * c], t[4 * c + 1], t[4 * c + 2], t[4 * c + 3]);
    }
    uint32_t rk[4], idk[4];  // one byte per key: rank in block (< 16), id
#pragma unroll
    for (int c = 0; c < 4; ++c) {
      const uint32_t kk[4] = {kx[c].x, kx[c].y, kx[c].z, kx[c].w};
      rk[c] = 0u;
      idk[c] = 0u;
#pragma unroll
      for (int j = 0; j < 4; ++j) {
        if (FULL || b0 + 4 * c + j < nt) {
          const uint32_t id = id_of(kk[j]);
          const uint32_t a = colA + (id & 15u) * RS;
          const uint32_t r = lds_u16(a);
          sts_u16(a, r + 1);
          rk[c] |= r << (8 * j);
          idk[c] |= id << (8 * j);
        }
      }
    }
    // D[j] for this tile (S_t = exclusive scan of h over j); read only in step 6
    if (tid < m) {
      uint32_t wpre = 0;
#pragma unroll
      for (int i = 0; i < NW; ++i) wpre += (i < (int)warp) ? wsum[16 + i] : 0u;
      D[tid] = g0 - (wpre + hincl - hj);
    }
    __syncthreads();
    if (tid == 0 && it + STAGES < iters) issue(it + STAGES, false);  // key stage free again

    scan_counters<Ly::LB>(sm + Ly::O_CA, wsum, tid);

    // ---- 2. pass-1 scatter into X (128-B swizzled), values and id bytes alongside
    uint4 vy[KV ? 4 : 1];
    if constexpr (KV) {
      if constexpr (FULL) {
        mbar_wait(bar_v + st, ph);
        const uint8_t *sv = sm + Ly::O_SV + st * TB;
#pragma unroll
        for (int c = 0; c < 4; ++c) vy[c] = *reinterpret_cast<const uint4 *>(sv + choff[c]);
      } else {
        uint32_t t[K];
#pragma unroll
        for (int q = 0; q < K; ++q) t[q] = b0 + q < nt ? __ldg(vals + base + b0 + q) : 0u;
#pragma unroll
        for (int c = 0; c < 4; ++c) vy[c] = make_uint4(t[4 * c], t[4 * c + 1], t[4 * c + 2], t[4 * c + 3]);
      }
    }
#pragma unroll
    for (int c = 0; c < 4; ++c) {
      const uint32_t kk[4] = {kx[c].x, kx[c].y, kx[c].z, kx[c].w};
      uint32_t vv[4];
      if constexpr (KV) {
        vv[0] = vy[c].x; vv[1] = vy[c].y; vv[2] = vy[c].z; vv[3] = vy[c].w;
      }
      uint32_t sl[4];  // the 4 counter loads first (independent), then the stores
#pragma unroll
      for (int j = 0; j < 4; ++j)
        sl[j] = (FULL || b0 + 4 * c + j < nt) ? lds_u16(colA + (__byte_perm(idk[c], 0u, 0x4440u + j) & 15u) * RS)
                                              : 0u;
#pragma unroll
      for (int j = 0; j < 4; ++j) {
        if (FULL || b0 + 4 * c + j < nt) {
          const uint32_t slot = sl[j] + __byte_perm(rk[c], 0u, 0x4440u + j);
          const uint32_t o = (slot << 2) ^ ((slot >> 1) & 0x70u);  // 128-B swizzle: chunk ^= row & 7
          sts_u32(x32 + o, kk[j]);
          if constexpr (KV) sts_u32(xv32 + o, vv[j]);
          if constexpr (!RECOMP) sts_u8(xi32 + slot, __byte_perm(idk[c], 0u, 0x4440u + j));
        }
      }
    }
    __syncthreads();
    if constexpr (KV) {
      if (tid == 0 && it + STAGES < iters) issue(it + STAGES, true);  // value stage free again
    }

    // ---- 3. pass 2 (hi digit): block beta of the pass-1 order -> registers
    // (keys in place of the staged ones), private counting by hi
    {
      const uint8_t *xs = sm + Ly::O_X;
#pragma unroll
      for (int c = 0; c < 4; ++c) kx[c] = *reinterpret_cast<const uint4 *>(xs + choff[c]);
      if constexpr (KV) {
        const uint8_t *xv = sm + Ly::O_XV;
#pragma unroll
        for (int c = 0; c < 4; ++c) vy[c] = *reinterpret_cast<const uint4 *>(xv + choff[c]);
      }
      if constexpr (!RECOMP) {
        const uint4 iw = *reinterpret_cast<const uint4 *>(sm + Ly::O_XI + b0);
        idk[0] = iw.x; idk[1] = iw.y; idk[2] = iw.z; idk[3] = iw.w;
      }
    }
#pragma unroll
    for (int c = 0; c < 4; ++c) {
      rk[c] = 0u;
      const uint32_t kk[4] = {kx[c].x, kx[c].y, kx[c].z, kx[c].w};
#pragma unroll
      for (int j = 0; j < 4; ++j) {
        if (FULL || b0 + 4 * c + j < nt) {
          const uint32_t hi = (RECOMP ? id_of(kk[j]) : __byte_perm(idk[c], 0u, 0x4440u + j)) >> 4;
          const uint32_t a = colB + hi * RS;
          const uint32_t r = lds_u16(a);
          sts_u16(a, r + 1);
          rk[c] |= r << (8 * j);
        }
      }
    }
    __syncthreads();  // every thread holds its block: X may be overwritten below
    scan_counters<Ly::HB>(sm + Ly::O_CB, wsum + 8, tid);

    // ---- 4. pass-2 scatter into X (linear): the tile in stable id order
#pragma unroll
    for (int c = 0; c < 4; ++c) {
      const uint32_t kk[4] = {kx[c].x, kx[c].y, kx[c].z, kx[c].w};
      uint32_t vv[4];
      if constexpr (KV) {
        vv[0] = vy[c].x; vv[1] = vy[c].y; vv[2] = vy[c].z; vv[3] = vy[c].w;
      }
      uint32_t sl[4];
#pragma unroll
      for (int j = 0; j < 4; ++j) {
        const uint32_t hi = (RECOMP ? id_of(kk[j]) : __byte_perm(idk[c], 0u, 0x4440u + j)) >> 4;
        sl[j] = (FULL || b0 + 4 * c + j < nt) ? lds_u16(colB + hi * RS) : 0u;
      }
#pragma unroll
      for (int j = 0; j < 4; ++j) {
        if (FULL || b0 + 4 * c + j < nt) {
          const uint32_t slot = sl[j] + __byte_perm(rk[c], 0u, 0x4440u + j);
          sts_u32(x32 + 4 * slot, kk[j]);
          if constexpr (KV) sts_u32(xv32 + 4 * slot, vv[j]);
          if constexpr (!RECOMP) sts_u8(xi32 + slot, __byte_perm(idk[c], 0u, 0x4440u + j));
        }
      }
    }
    __syncthreads();

    // ---- 5. stores: final slot i -> D[id] + i (runs of a bucket are consecutive slots);
    // plain shared loads (no stores in this phase), so they can be batched
    const uint32_t *xk = reinterpret_cast<const uint32_t *>(sm + Ly::O_X);
    const uint32_t *xv = reinterpret_cast<const uint32_t *>(sm + Ly::O_XV);
    const uint8_t *xi = sm + Ly::O_XI;
    auto store = [&](uint32_t i) {
      const uint32_t k = xk[i];
      const uint32_t id = RECOMP ? id_of(k) : (uint32_t)xi[i];
      const uint32_t dst = D[id] + i;
      __stcs(keys_out + dst, k);
      if constexpr (KV) __stcs(vals_out + dst, xv[i]);
    };
    if constexpr (FULL) {
#pragma unroll 8
      for (int q = 0; q < K; ++q) store(q * NT + tid);
    } else {
      for (uint32_t i = tid; i < nt; i += NT) store(i);
    }
  };
  const bool has_tail = iters && tile_of(iters - 1) >= Lfull;
  const uint32_t iters_full = iters - (has_tail ? 1u : 0u);
  for (uint32_t it = 0; it < iters_full; ++it) tile_body(it, std::true_type{});
  if (has_tail) tile_body(iters_full, std::false_type{});
}

// ------------------------------------------------------------------ host launcher
template <int KIND, bool KV, int LOGM>
inline cudaError_t k3h_launch_l(const K3pArgs &a) {
  constexpr int STAGES = KV ? 1 : 2;
  using Ly = K3hLayout<LOGM, KV, STAGES>;
  constexpr int MINB = KV ? 2 : 3;
  auto k = k3h_postscan<KIND, KV, LOGM, STAGES, MINB>;
  const size_t smem = (size_t)(KIND == SPLITTERS ? Ly::BYTES_SPL : Ly::BYTES) + 1024;
  cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  int per_sm = 0;
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k, Ly::NT, smem);
  if (per_sm <= 0) per_sm = 1;
  const unsigned grid = (unsigned)umin64_host(a.L, (uint64_t)a.sms * per_sm);
  if (a.grid_out) {
    *a.grid_out = grid;
    return cudaSuccess;
  }
  const uint64_t rows = (uint64_t)(a.n / Ly::T) * (Ly::T / 32);
  CUtensorMap tmk, tmv;
  if (!make_tile_map(&tmk, a.keys, rows, Ly::T) || !make_tile_map(&tmv, KV ? a.vals : nullptr, rows, Ly::T))
    return cudaErrorInvalidValue;
  const cudaError_t e = launch_ex(a.pdl != 0, k, dim3(grid), dim3(Ly::NT), smem, a.stream, tmk, tmv, a.keys, a.vals,
                                  a.G, a.keys_out, a.vals_out, a.n, a.L, *a.bp);
  return e != cudaSuccess ? e : cudaGetLastError();
}

template <int KIND, bool KV>
inline cudaError_t k3h_launch_kv(const K3pArgs &a) {
  if (a.m <= 64) return k3h_launch_l<KIND, KV, 6>(a);
  if (a.m <= 128) return k3h_launch_l<KIND, KV, 7>(a);
  return k3h_launch_l<KIND, KV, 8>(a);
}

template <int KIND>
inline cudaError_t k3h_launch(const K3pArgs &a) {
  return a.vals ? k3h_launch_kv<KIND, true>(a) : k3h_launch_kv<KIND, false>(a);
}

}  // namespace ms
