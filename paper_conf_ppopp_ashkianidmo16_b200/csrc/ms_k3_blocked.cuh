// ms_k3_blocked.cuh -- K3 post-scan for m <= 32: persistent, blocked ranks, TMA bulk stores (sm_100a).
//
// Same contract as k3_postscan (ms_kernels.cuh): recompute ids (footnote 6,
// P:857-859), stable local offsets (term 3 of Eq. (2)), a local
// stable multisplit of the tile in shared memory (§4 reordering, P:689-713;
// block-level reordering §5.2.2), then bucket runs written to
// G[j][tile] + (slot - S_t[j]).
//
// B200 design: no warp votes at all.  The paper's local
// offsets come from an explicit H-bar scan (§4 "explicit" local offsets,
// P:650-666) done hierarchically:
//  * thread t owns the contiguous block beta(t) of 16 keys and counts them
//    sequentially into a private column of u16 counters c[j][beta] in shared
//    memory -- the count it reads before incrementing IS the key's stable
//    rank inside the block; beta(t) = 2*lane + (warp & 1) + 64*(warp >> 1)
//    puts the 32 lanes of a warp in 32 different banks whatever their ids;
//  * one CTA-wide exclusive scan over the row-vectorised counter matrix
//    (bucket-major, blocks in input order -- the same "row-vectorised" scan
//    as the global one, Alg. 1) turns every counter into the
//    key's slot in the locally multisplit tile;
//  * bucket j's run is placed at a slot P_j congruent to its global start
//    G_j modulo 4 keys (<= 3 padding slots per bucket), so the run body is
//    one TMA bulk store (cp.async.bulk, UBLKCP) shared -> global; only the
//    <= 3 + 3 unaligned head/tail keys use plain stores.
// Persistent CTAs walk tiles with a stride of gridDim.x; each thread
// prefetches its own next blocks with cp.async (LDGSTS) into a chunk-major
// staging ring, so loads for the next STAGES tiles are in flight while the
// current tile is ranked and stored, and no barrier guards the staging data.
#include "ms_k3p_args.h"

namespace ms {

template <int LOGMP, bool KV, bool IDS8, int KPT, int NT = kThreads>
struct K3pLayout {
  static constexpr int MP = 1 << LOGMP;        // bucket rows (m rounded up to a power of 2, >= 2)
  static constexpr int K = KPT;                // keys per thread (16 or 32)
  static constexpr int CH = K / 4;             // 16-byte chunks per thread per array
  static constexpr int T = NT * K;             // keys per tile (NT threads per CTA)
  static constexpr int STAGES = (KV || K > 16) ? 1 : 2;  // tiles prefetched ahead
  static constexpr int CW = MP * NT / 2;       // counter words (MP x NT u16)
  static constexpr int KSR = (T + 3 * MP + 4 + 3) & ~3;  // key slots incl. alignment padding
  static constexpr int WPT = MP / 2;           // counter words per thread in the scan
  static constexpr int MW = 3 * MP + 8;        // per-tile metadata words: rowS[MP+4] P[MP] G[MP]
  static constexpr int IW = IDS8 ? T / 4 : 0;  // staged u8 ids per stage (words)
  // word offsets
  static constexpr int O_CNT = 0;
  static constexpr int O_KEYS = O_CNT + CW;
  static constexpr int O_VALS = O_KEYS + KSR;
  static constexpr int O_STK = O_VALS + (KV ? KSR : 0);           // [STAGES][T] keys
  static constexpr int O_STV = O_STK + STAGES * T;                // [STAGES][T] vals
  static constexpr int O_STI = O_STV + (KV ? STAGES * T : 0);     // [STAGES][T/4] u8 ids
  static constexpr int O_META = O_STI + STAGES * IW;              // [2][MW] (tile parity)
  static constexpr int O_WS = O_META + 2 * MW;
  static constexpr int O_SPL = O_WS + 12;
  static constexpr int WORDS = O_SPL + kMaxM;
  static constexpr size_t BYTES = (size_t)WORDS * 4;
};

__device__ __forceinline__ void cp_async16(void *smem_dst, const void *src, uint32_t src_bytes) {
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;" ::"r"(smem_u32(smem_dst)), "l"(src),
               "r"(src_bytes)
               : "memory");
}
__device__ __forceinline__ void cp_async16_full(void *smem_dst, const void *src) {
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(smem_u32(smem_dst)), "l"(src) : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void cp_async_wait() {
  asm volatile("cp.async.wait_group %0;" ::"n"(N) : "memory");
}

// Stage this thread's chunks of tile `tile` (keys: CH x 16 B; vals likewise;
// u8 ids: K/16 x 16 B) into stage slot `st`, chunk-major ([c][tid]) so the
// later 128-bit reads are conflict-free.  Bytes past n are zero-filled.
// owner thread of block beta (inverse of beta(t) = 2*lane + (warp & 1) + 64*(warp >> 1))
__device__ __forceinline__ uint32_t k3p_owner(uint32_t beta) {
  const uint32_t lane = (beta >> 1) & 31u, warp = ((beta >> 6) << 1) | (beta & 1u);
  return warp * 32u + lane;
}

// Copies are COALESCED: thread t fetches the tile's 16-byte chunks t, t+256,
// ... (consecutive threads, consecutive chunks -- whole 128-byte lines per
// warp instruction) and drops chunk g = 4*beta + c (keys 4g..4g+3 of block
// beta) at the owner's chunk-major slot [c][owner(beta)].  Owners read their
// chunks only after the begin-of-tile barrier, and a stage is refilled only
// after the tile's last barrier, so the cross-thread handoff is ordered.
template <bool KV, bool IDS8, int T, int K, int NT>
__device__ __forceinline__ void k3p_prefetch(uint32_t *stk, uint32_t *stv, uint32_t *sti, int st,
                                             const uint32_t *keys, const uint32_t *vals, const void *ids,
                                             uint64_t tile, uint32_t n, uint32_t /*beta*/) {
  constexpr int CH = K / 4;                 // chunks per block; the tile has NT*CH chunks
  const uint32_t tid = threadIdx.x;
  const uint64_t t0 = tile * T;
  const bool full = t0 + T <= n;
#pragma unroll
  for (int i = 0; i < CH; ++i) {
    const uint32_t g = i * NT + tid;  // chunk index within the tile
    const uint32_t beta = g / CH, c = g % CH;
    const uint32_t dst = (c * NT + k3p_owner(beta)) * 4;
    const uint64_t e = t0 + 4ull * g;
    if (full) {
      cp_async16_full(stk + st * T + dst, keys + e);
      if constexpr (KV) cp_async16_full(stv + st * T + dst, vals + e);
    } else {
      const uint32_t bytes = e >= n ? 0u : (uint32_t)(umin64(4, n - e) * 4);
      const uint64_t src = bytes ? e : 0;
      cp_async16(stk + st * T + dst, keys + src, bytes);
      if constexpr (KV) cp_async16(stv + st * T + dst, vals + src, bytes);
    }
  }
  if constexpr (IDS8) {  // u8 ids: block beta's K bytes = K/16 chunks, chunk-major by owner
#pragma unroll
    for (int i = 0; i < K / 16; ++i) {
      const uint32_t g = i * NT + tid;
      const uint32_t beta = g / (K / 16), c = g % (K / 16);
      uint32_t *d = sti + st * (T / 4) + (c * NT + k3p_owner(beta)) * 4;
      const uint64_t e = t0 + 16ull * g;
      if (full) {
        cp_async16_full(d, (const uint8_t *)ids + e);
      } else {
        const uint32_t bytes = e >= n ? 0u : (uint32_t)umin64(16, n - e);
        cp_async16(d, (const uint8_t *)ids + (bytes ? e : 0), bytes);
      }
    }
  }
}

// One tile, already staged.  FULL: all T keys valid (no per-key predicates).
// RANGED (ms_ranged.cuh): G_j of this tile is the running sum `grun` held by
// the threads of bucket row j (advanced here by the tile's row total) instead
// of a column of the global G array.
template <int KIND, bool KV, int LOGMP, bool IDS8, int KPT, int NT, bool FULL, bool RANGED>
__device__ __forceinline__ void k3p_tile(const uint32_t *sm_k, const uint32_t *sm_v, const uint32_t *sm_i,
                                         const void *__restrict__ ids, uint32_t *__restrict__ keys_out,
                                         uint32_t *__restrict__ vals_out, uint64_t base, uint32_t nt,
                                         const BucketParams &p, uint32_t *sm, uint32_t beta, uint32_t *meta,
                                         uint32_t &grun) {
  using Ly = K3pLayout<LOGMP, KV, IDS8, KPT, NT>;
  constexpr int MP = Ly::MP, K = Ly::K, CH = Ly::CH;
  constexpr int NW = NT / 32;
  constexpr int LOGNT = NT == 256 ? 8 : 7;
  // ids are recomputed from the key where that is cheaper than keeping them
  constexpr bool KEEP_ID = (KIND == SPLITTERS) || (KIND == IDS && !IDS8);
  uint32_t *cnt32 = sm + Ly::O_CNT;
  uint32_t *keys_s = sm + Ly::O_KEYS;
  uint32_t *vals_s = sm + Ly::O_VALS;
  uint32_t *rowS = meta;            // [MP+4]
  uint32_t *Pj = meta + MP + 4;     // [MP]
  uint32_t *Gj = Pj + MP;           // [MP]
  uint32_t *wsum = sm + Ly::O_WS;
  const uint32_t *spl_s = sm + Ly::O_SPL;
  const uint32_t tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const uint32_t m = p.m;
  const uint32_t b0 = beta * K;
  // this thread's counter column: byte address of c[0][beta]; c[j][beta] is j*2*NT bytes further
  uint8_t *cb = reinterpret_cast<uint8_t *>(cnt32) + 2 * beta;

  // Keys (and values) are read from this thread's own staged chunks twice --
  // for counting and again for the scatter -- instead of being held in
  // registers across the scan (no spills at 3 CTAs/SM).
  auto chunk = [&](const uint32_t *st, int c) -> uint4 {
    return *reinterpret_cast<const uint4 *>(st + (c * NT + tid) * 4);
  };
  uint32_t idw[IDS8 ? K / 4 : 1];
  if constexpr (IDS8) {
#pragma unroll
    for (int c = 0; c < K / 16; ++c) {
      const uint4 x = chunk(sm_i, c);
      idw[4 * c] = x.x; idw[4 * c + 1] = x.y; idw[4 * c + 2] = x.z; idw[4 * c + 3] = x.w;
    }
  }
  auto id_of = [&](uint32_t key, int q) -> uint32_t {
    if constexpr (KIND == IDS) {
      if constexpr (IDS8) return min(__byte_perm(idw[q >> 2], 0u, 0x4440u + (q & 3)), p.mmask);
      else return (FULL || b0 + q < nt) ? load_id(ids, base + b0 + q, p) : 0u;
    } else {
      return bucket_of_key<KIND>(key, p, spl_s);
    }
  };

  // ---- 1. sequential per-block counting: the rank within the block, by an
  // in-order read-modify-write of the thread's private counter column in
  // shared memory.  Keys past the tail (partial tile only) are skipped.
  // (Measured alternatives: a register histogram for m <= 8 and
  // grouped counter loads with compare corrections were both slower.)
  uint32_t rk[K / 4];                        // ranks (< K), one byte each
  uint32_t idk[KEEP_ID ? K / 4 : 1];         // kept ids, one byte each
  uint4 kx[CH];  // all staged chunks first: no chunk load waits behind a counter store
#pragma unroll
  for (int c = 0; c < CH; ++c) kx[c] = chunk(sm_k, c);
#pragma unroll
  for (int c = 0; c < CH; ++c) {
    const uint32_t kk[4] = {kx[c].x, kx[c].y, kx[c].z, kx[c].w};
    uint32_t id[4], r[4];
    bool ok[4];
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      id[j] = id_of(kk[j], 4 * c + j);
      ok[j] = FULL || (b0 + 4 * c + j < nt);
    }
    rk[c] = 0u;
    if constexpr (KEEP_ID) idk[c] = 0u;
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      if (ok[j]) {
        uint16_t *cp = reinterpret_cast<uint16_t *>(cb + id[j] * (2 * NT));
        if (p.dbg != 7 && p.dbg != 8) {
          r[j] = *cp;
          *cp = (uint16_t)(r[j] + 1);
        } else {
          r[j] = 0u;  // ablation: no counting
        }
        rk[c] |= r[j] << (8 * j);
        if constexpr (KEEP_ID) idk[c] |= id[j] << (8 * j);
      }
    }
  }
  __syncthreads();

  // ---- 2. CTA exclusive scan of the row-vectorised counter matrix
  // Thread t owns words [t*WPT, (t+1)*WPT) (one bucket row).  With >= 2
  // 16-byte chunks per thread, the chunk order is rotated per lane so the
  // 128-bit accesses of every 8-lane phase hit 8 different bank groups.
  const uint32_t row = tid >> (LOGNT - LOGMP);
  constexpr int WPT = Ly::WPT;
  constexpr int NC = WPT >= 4 ? WPT / 4 : 1;       // 16-byte chunks per thread
  constexpr int CWD = WPT >= 4 ? 4 : WPT;          // words per chunk
  const uint32_t rot = NC == 4 ? ((tid >> 1) & 3) : NC == 2 ? ((tid >> 2) & 1) : 0;
  uint32_t w[NC][CWD];
  uint32_t csum[NC];
#pragma unroll
  for (int i = 0; i < NC; ++i) {
    const uint32_t pc = (i + rot) & (NC - 1);   // physical chunk held in register slot i
    const uint32_t *src = cnt32 + tid * WPT + pc * CWD;
    if (p.dbg >= 6 && p.dbg <= 8) {  // ablation: no scan traffic
#pragma unroll
      for (int j = 0; j < CWD; ++j) w[i][j] = 0u;
    } else if constexpr (CWD == 4) {
      const uint4 x = *reinterpret_cast<const uint4 *>(src);
      w[i][0] = x.x; w[i][1] = x.y; w[i][2] = x.z; w[i][3] = x.w;
    } else if constexpr (CWD == 2) {
      const uint2 x = *reinterpret_cast<const uint2 *>(src);
      w[i][0] = x.x; w[i][1] = x.y;
    } else {
      w[i][0] = src[0];
    }
    uint32_t s2 = 0;  // packed (lo-sum, hi-sum), each <= T/2 + ... < 2^16
#pragma unroll
    for (int j = 0; j < CWD; ++j) s2 += w[i][j];
    csum[i] = (s2 & 0xFFFFu) + (s2 >> 16);
  }
  uint32_t s = 0;
#pragma unroll
  for (int i = 0; i < NC; ++i) s += csum[i];
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
  // S_row = excl of the row's first thread: a lane of this warp (rows < 32
  // threads) or lane 0 of warp row*TPR/32, whose excl is the warp prefix.
  uint32_t Sr;
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
  // padded run start P_j = S_j + 3j + ((G_j - S_j - 3j) & 3): P_j = G_j (mod 4)
  // and P_j >= P_{j-1} + h_{j-1}; closed form, no serial dependency over j.
  uint32_t Gr;
  if constexpr (RANGED) {
    Gr = grun;
    uint32_t rtot;  // this tile's count of bucket `row`
    if constexpr (TPR < 32) {
      rtot = __shfl_sync(0xFFFFFFFFu, excl + s, lane | (TPR - 1)) - Sr;
    } else {
      rtot = 0;
      const uint32_t w0 = (row * TPR) >> 5;
#pragma unroll
      for (int i = 0; i < NW; ++i) rtot += ((uint32_t)i >= w0 && (uint32_t)i < w0 + TPR / 32) ? wsum[i] : 0u;
    }
    grun += rtot;
    if ((tid & (TPR - 1)) == 0) Gj[row] = Gr;
  } else {
    Gr = row < m ? Gj[row] : 0u;
  }
  const uint32_t pad = 3 * row + ((Gr - Sr - 3 * row) & 3u);
#pragma unroll
  for (int i = 0; i < NC; ++i) {
    const uint32_t pc = (i + rot) & (NC - 1);
    uint32_t run = excl + pad;  // + sum of the chunks physically before pc
#pragma unroll
    for (int i2 = 0; i2 < NC; ++i2) run += (((i2 + rot) & (NC - 1)) < pc) ? csum[i2] : 0u;
#pragma unroll
    for (int j = 0; j < CWD; ++j) {
      const uint32_t x = w[i][j];
      w[i][j] = run * 0x10001u + (x << 16);      // (run, run + lo)
      run += (x * 0x10001u) >> 16;               // lo + hi (< 2^16, no carry into bit 32)
    }
    uint32_t *dst = cnt32 + tid * WPT + pc * CWD;
    if (p.dbg >= 6 && p.dbg <= 8) {
    } else if constexpr (CWD == 4) *reinterpret_cast<uint4 *>(dst) = make_uint4(w[i][0], w[i][1], w[i][2], w[i][3]);
    else if constexpr (CWD == 2) *reinterpret_cast<uint2 *>(dst) = make_uint2(w[i][0], w[i][1]);
    else dst[0] = w[i][0];
  }
  if ((tid & (TPR - 1)) == 0) Pj[row] = Sr + pad;
  bulk_wait_read0();  // keys_s may still be read by this thread's bulk stores of the previous tile
  __syncthreads();

  // ---- 3. local multisplit of the tile into shared memory, one staged
  // chunk (4 keys) at a time: its 4 slot bases are loaded before its stores
  uint4 sx[CH];  // staged keys (and values) first, then the per-chunk slot loads and stores
  uint4 sy[KV ? CH : 1];
#pragma unroll
  for (int c = 0; c < CH; ++c) {
    sx[c] = chunk(sm_k, c);
    if constexpr (KV) sy[c] = chunk(sm_v, c);
  }
#pragma unroll
  for (int c = 0; c < CH; ++c) {
    const uint32_t kk[4] = {sx[c].x, sx[c].y, sx[c].z, sx[c].w};
    uint32_t vv[4];
    if constexpr (KV) {
      vv[0] = sy[c].x; vv[1] = sy[c].y; vv[2] = sy[c].z; vv[3] = sy[c].w;
    }
    uint32_t sl[4];
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      const int q = 4 * c + j;
      uint32_t id;
      if constexpr (KEEP_ID) id = __byte_perm(idk[c], 0u, 0x4440u + j);
      else id = id_of(kk[j], q);
      sl[j] = (FULL || b0 + q < nt) ? *reinterpret_cast<const uint16_t *>(cb + id * (2 * NT)) : 0u;
    }
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      const int q = 4 * c + j;
      if (FULL || b0 + q < nt) {
        const uint32_t slot = sl[j] + __byte_perm(rk[c], 0u, 0x4440u + j);
        if (p.dbg != 8) keys_s[slot] = kk[j];
        if constexpr (KV) vals_s[slot] = vv[j];
      }
    }
  }
  fence_proxy_async_smem();  // generic-proxy writes -> visible to the TMA (async proxy)
  __syncthreads();

  // ---- 4. bucket runs: NT/32 threads per bucket (m <= 32) share its
  //         <= 3 head keys, <= 3 tail keys and the TMA bulk store(s) of the
  //         16-byte-aligned body
  if (p.dbg == 1 || (p.dbg >= 6 && p.dbg <= 8)) return;  // ablation: no stores
  {
    constexpr uint32_t SPB = NT / 32;
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
        } else if (body) {
          if (sub == 6) bulk_s2g(keys_out + Gd + head, keys_s + P + head, body * 4u);
          else if (KV) bulk_s2g(vals_out + Gd + head, vals_s + P + head, body * 4u);
          bulk_commit();
        }
      } else {  // SPB == 4: head / tail / keys body / values body
        if (sub < 2) {
          const uint32_t i0 = sub == 0 ? 0u : head + body, i1 = sub == 0 ? head : len;
          for (uint32_t i = i0; i < i1; ++i) {
            keys_out[Gd + i] = keys_s[P + i];
            if constexpr (KV) vals_out[Gd + i] = vals_s[P + i];
          }
        } else if (body) {
          if (sub == 2) bulk_s2g(keys_out + Gd + head, keys_s + P + head, body * 4u);
          else if (KV) bulk_s2g(vals_out + Gd + head, vals_s + P + head, body * 4u);
          bulk_commit();
        }
      }
    }
  }
}

template <int KIND, bool KV, int LOGMP, bool IDS8, int KPT, int NT, bool RANGED>
__global__ void __launch_bounds__(NT, NT == 256 ? (KV ? 2 : 3) : (KV ? 4 : 6))
k3p_postscan(const uint32_t *__restrict__ keys, const uint32_t *__restrict__ vals,
             const void *__restrict__ ids, const uint32_t *__restrict__ G,
             uint32_t *__restrict__ keys_out, uint32_t *__restrict__ vals_out, uint32_t n,
             uint32_t L, const __grid_constant__ BucketParams p, const __grid_constant__ RangeScan rs) {
  using Ly = K3pLayout<LOGMP, KV, IDS8, KPT, NT>;
  constexpr int T = Ly::T, STAGES = Ly::STAGES, CW = Ly::CW, MP = Ly::MP, K = Ly::K;
  constexpr int LOGNT = NT == 256 ? 8 : 7;
  extern __shared__ __align__(128) uint32_t sm[];
  uint32_t *stk = sm + Ly::O_STK;
  uint32_t *stv = sm + Ly::O_STV;
  uint32_t *sti = sm + Ly::O_STI;
  const uint32_t tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const uint32_t beta = 2 * lane + (warp & 1) + 64 * (warp >> 1);
  const uint32_t m = p.m;
  // Tile mode: tiles blockIdx.x, blockIdx.x + gridDim.x, ...; the partial
  // tile (if any) is the last one overall, hence the last of its CTA: it is
  // peeled off the loop so its predicated code does not raise the loop's
  // registers.  p.reverse: walk tiles last-to-first, so the first tiles K3
  // reads are the ones K1 read last (still in the 126 MB L2); the partial
  // tile is then the FIRST tile of CTA 0 instead of the last of its CTA.
  // RANGED: CTA c walks its contiguous range [c*L/C, (c+1)*L/C) in order
  // (G = GB[c][:], the range's bucket starts; the partial tile, if any, is
  // the last tile of the last range).
  const bool rev = !RANGED && p.reverse != 0;
  const uint64_t r0 = RANGED ? (uint64_t)blockIdx.x * L / gridDim.x : 0;
  auto tile_of = [&](uint32_t it) -> uint64_t {
    if constexpr (RANGED) return r0 + it;
    const uint64_t t = (uint64_t)blockIdx.x + (uint64_t)it * gridDim.x;
    return rev ? (uint64_t)L - 1 - t : t;
  };
  const uint32_t iters = RANGED ? (uint32_t)((uint64_t)(blockIdx.x + 1) * L / gridDim.x - r0)
                                : (blockIdx.x < L ? (L - 1 - blockIdx.x) / gridDim.x + 1 : 0);
  const bool partial = (uint64_t)n < (uint64_t)L * T;
  const bool tail_first = partial && rev && iters && blockIdx.x == 0;
  const bool has_tail = partial && !rev && iters && tile_of(iters - 1) == L - 1;
  const uint32_t iters_full = iters - (has_tail ? 1 : 0);

  if constexpr (KIND == SPLITTERS) {
    if (tid < (1u << p.logm)) sm[Ly::O_SPL + tid] = p.spl[tid];
  }
  // prologue: STAGES tiles in flight
#pragma unroll
  for (int s = 0; s < STAGES; ++s) {
    if ((uint32_t)s < iters) k3p_prefetch<KV, IDS8, T, K, NT>(stk, stv, sti, s, keys, vals, ids, tile_of(s), n, beta);
    cp_async_commit();
  }
  pdl_wait();  // K2's G / GB is complete (the first tiles' loads above are already in flight)
  uint32_t gnext = 0;  // tile mode: the next tile's G column
  uint32_t grun = 0;   // RANGED: G_row of the current tile (all threads of bucket row `row`)
  if constexpr (RANGED) {
    const uint32_t row = tid >> (LOGNT - LOGMP);
    if (rs.HC != nullptr) {  // K2r folded in (the reorder slots are free until tile 0)
      grun = range_base<NT, LOGMP>(rs, m, blockIdx.x, n, sm + Ly::O_KEYS, row);
      __syncthreads();
    } else if (iters && row < m) {
      grun = __ldg(G + (uint64_t)blockIdx.x * m + row);
    }
  } else {
    if (iters && tid < m) gnext = __ldg(G + (uint64_t)tid * L + tile_of(0));
  }

  // per-iteration prologue: zero the counters (last read by the previous
  // tile's scatter, before a barrier), publish G[:, tile] into this parity's
  // metadata, prefetch the next G column, wait for this thread's staged chunks
  auto begin_tile = [&](uint32_t it, uint32_t *meta) {
    {
      uint4 *c4 = reinterpret_cast<uint4 *>(sm + Ly::O_CNT);
#pragma unroll
      for (int i = 0; i < (CW / 4 + NT - 1) / NT; ++i) {
        const int idx = i * NT + tid;
        if (idx < CW / 4) c4[idx] = make_uint4(0, 0, 0, 0);
      }
    }
    if constexpr (!RANGED) {
      if (tid < m) meta[MP + 4 + MP + tid] = gnext;
      if (it + 1 < iters && tid < m) gnext = __ldg(G + (uint64_t)tid * L + tile_of(it + 1));
    }
    cp_async_wait<STAGES - 1>();
    __syncthreads();
  };

  uint32_t it = 0;
  if (tail_first) {
    const uint64_t tile = tile_of(0);
    uint32_t *meta = sm + Ly::O_META;
    begin_tile(0, meta);
    k3p_tile<KIND, KV, LOGMP, IDS8, KPT, NT, false, RANGED>(stk, stv, sti, ids, keys_out, vals_out, tile * T,
                                                (uint32_t)(n - tile * T), p, sm, beta, meta, grun);
    if (STAGES < iters) k3p_prefetch<KV, IDS8, T, K, NT>(stk, stv, sti, 0, keys, vals, ids, tile_of(STAGES), n, beta);
    cp_async_commit();
    it = 1;
  }
  for (; it < iters_full; ++it) {
    const uint64_t tile = tile_of(it);
    const int st = (int)(it % STAGES);
    uint32_t *meta = sm + Ly::O_META + (it & 1) * Ly::MW;
    begin_tile(it, meta);
    k3p_tile<KIND, KV, LOGMP, IDS8, KPT, NT, true, RANGED>(stk + st * T, stv + st * T, sti + st * Ly::IW, ids,
                                                       keys_out, vals_out, tile * T, T, p, sm, beta, meta, grun);
    // refill this stage with tile it + STAGES (own chunks only; already consumed)
    if (it + STAGES < iters)
      k3p_prefetch<KV, IDS8, T, K, NT>(stk, stv, sti, st, keys, vals, ids, tile_of(it + STAGES), n, beta);
    cp_async_commit();
  }
  if (has_tail) {
    const uint64_t tile = tile_of(it);
    const int st = (int)(it % STAGES);
    uint32_t *meta = sm + Ly::O_META + (it & 1) * Ly::MW;
    begin_tile(it, meta);
    k3p_tile<KIND, KV, LOGMP, IDS8, KPT, NT, false, RANGED>(stk + st * T, stv + st * T, sti + st * Ly::IW, ids,
                                                        keys_out, vals_out, tile * T, (uint32_t)(n - tile * T), p,
                                                        sm, beta, meta, grun);
  }
  bulk_wait_read0();
}

// ------------------------------------------------------------------ host launcher
template <int NT, typename Kern>
inline cudaError_t k3p_launch_one(Kern k, size_t smem, const K3pArgs &a) {
  if (smem > 48 * 1024) cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  int per_sm = 0;
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k, NT, smem);
  if (per_sm <= 0) per_sm = 1;
  if (a.bp->dbg >= 10 && (int)(a.bp->dbg - 10) < per_sm) per_sm = (int)(a.bp->dbg - 10);  // ablation: CTAs/SM
  uint64_t g = umin64_host(a.L, (uint64_t)a.sms * per_sm);
  if (a.ranged) g = umin64_host(g, kMaxRanges);
  const unsigned grid = (unsigned)g;
  if (a.grid_out) {
    *a.grid_out = grid;
    return cudaSuccess;
  }
  const cudaError_t e = launch_ex(a.pdl != 0, k, dim3(grid), dim3(NT), smem, a.stream, a.keys, a.vals, a.ids, a.G,
                                  a.keys_out, a.vals_out, a.n, a.L, *a.bp, a.rs);
  return e != cudaSuccess ? e : cudaGetLastError();
}

template <int KIND, bool KV, int LOGMP, int KPT, int NT, bool RANGED>
inline cudaError_t k3p_launch_r(const K3pArgs &a) {
  if constexpr (KIND == IDS) {
    if (a.id_bytes == 1)
      return k3p_launch_one<NT>(k3p_postscan<KIND, KV, LOGMP, true, KPT, NT, RANGED>,
                                K3pLayout<LOGMP, KV, true, KPT, NT>::BYTES, a);
  }
  return k3p_launch_one<NT>(k3p_postscan<KIND, KV, LOGMP, false, KPT, NT, RANGED>,
                            K3pLayout<LOGMP, KV, false, KPT, NT>::BYTES, a);
}

template <int KIND, bool KV, int LOGMP, int KPT, int NT>
inline cudaError_t k3p_launch_n(const K3pArgs &a) {
  return a.ranged ? k3p_launch_r<KIND, KV, LOGMP, KPT, NT, true>(a) : k3p_launch_r<KIND, KV, LOGMP, KPT, NT, false>(a);
}

template <int KIND, bool KV, int LOGMP, int KPT>
inline cudaError_t k3p_launch_l(const K3pArgs &a) {
  return a.nt == 128 ? k3p_launch_n<KIND, KV, LOGMP, KPT, 128>(a) : k3p_launch_n<KIND, KV, LOGMP, KPT, 256>(a);
}

template <int KIND, bool KV, int KPT>
inline cudaError_t k3p_launch_kv(const K3pArgs &a) {
  uint32_t l = 1;
  while ((1u << l) < a.m) ++l;
  switch (l) {
    case 1: return k3p_launch_l<KIND, KV, 1, KPT>(a);
    case 2: return k3p_launch_l<KIND, KV, 2, KPT>(a);
    case 3: return k3p_launch_l<KIND, KV, 3, KPT>(a);
    case 4: return k3p_launch_l<KIND, KV, 4, KPT>(a);
    default: return k3p_launch_l<KIND, KV, 5, KPT>(a);
  }
}

template <int KIND>
inline cudaError_t k3p_launch(const K3pArgs &a) {
  return a.vals ? k3p_launch_kv<KIND, true, 16>(a) : k3p_launch_kv<KIND, false, 16>(a);
}

}  // namespace ms
