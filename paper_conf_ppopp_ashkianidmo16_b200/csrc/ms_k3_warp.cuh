// ms_k3_warp.cuh -- K3 post-scan for m > 32: warp-striped rounds, Alg. 3 ballot ranks (sm_100a).
#pragma once
#include "ms_k3p_args.h"

namespace ms {

// ============================================================== K3 post-scan
// Recompute ids (footnote 6), stable tile-local ranks, a local
// stable multisplit of the tile in shared memory (§4 "reordering",
// P:689-713; §5.2.2 block-level reordering P:1262-1301) and coalesced stores
// of each bucket run to G[j][tile] + (slot - S_t[j]).
//
// Tile = 8 warps x R rounds x 32 keys; warp w owns the contiguous segment
// [w*32R, (w+1)*32R) and walks it in rounds of 32 consecutive keys, so
// (warp, round, lane) order IS input order and ranks are stable.
// Per round the LOGM ballots of Alg. 3 (one ballot per id bit,
// compile-time LOGM) give each lane the mask of same-bucket lanes (on sm_100
// __match_any_sync is ~2x dearer than 8 ballots when lanes hold distinct ids:
// it runs on the ADU pipe), popc(mask & lanemask_lt) is the
// exclusive rank (reading #4), and the highest lane of each group advances
// the warp's shared-memory counter for that bucket.  Cross-warp exclusive prefixes +
// the tile's bucket starts S_t then give each key its shared-memory slot
// (Eq. (2) one level down).  Keys (and values) arrive by one TMA
// bulk copy per array (UBLKCP) on an mbarrier.
template <int KIND, bool KV, int R, int LOGM, bool FULL, bool WL>
__device__ __forceinline__ uint32_t k3_tile(const uint32_t *__restrict__ vals_g, const void *__restrict__ ids,
                                        uint32_t *__restrict__ keys_out, uint32_t *__restrict__ vals_out,
                                        uint64_t base, uint32_t nt, const BucketParams &p,
                                        uint32_t *keys_s, uint32_t *vals_s, uint32_t *cnt_s,
                                        uint32_t *gD_s, const uint32_t *spl_s, uint8_t *id8_s,
                                        uint32_t *wsum, uint32_t gcol) {
  constexpr int SEG = 32 * R;
  constexpr bool ID8 = (KIND != LOWBITS && KIND != SHIFTC && KIND != SHIFT);
  const uint32_t tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const uint32_t m = p.m;
  const uint32_t lt = lanemask_lt(), gt = lanemask_gt();
  uint32_t *cnt_w = cnt_s + warp * kMaxM;
  const uint32_t seg0 = warp * SEG + lane;

  uint32_t idr[KIND == IDS ? R : 1];
  if constexpr (KIND == IDS) {
#pragma unroll
    for (int r = 0; r < R; ++r) {
      const uint32_t pos = seg0 + r * 32;
      idr[r] = (FULL || pos < nt) ? load_id(ids, base + pos, p) : 0xFFFFFFFFu;
    }
  }

  // ---- phase 1: stable ranks within the warp's segment
  uint32_t kreg[R];
  uint32_t vreg[KV ? R : 1];
  uint32_t pk[R];  // (rank within warp segment) << 8 | id
#pragma unroll
  for (int r = 0; r < R; ++r) {
    const uint32_t pos = seg0 + r * 32;
    const bool valid = FULL || pos < nt;
    const uint32_t key = keys_s[pos];
    uint32_t id;
    if constexpr (KIND == IDS) id = idr[r];
    else id = valid ? bucket_of_key<KIND>(key, p, spl_s) : 0xFFFFFFFFu;
    // lanes whose id differs from mine in bit b = vote_b XOR sext(my bit b);
    // one shifted copy of the id feeds both the vote predicate (its sign) and
    // the sign-extension, and one LOP3 accumulates the difference mask
    uint32_t peers;
    {
      uint32_t diff = FULL ? 0u : ~__ballot_sync(0xFFFFFFFFu, valid);
#pragma unroll
      for (int b = 0; b < LOGM; ++b) {
        if constexpr (!KV) {
          // 4 instructions per id bit: predicate from the bit (LOP3.P), ballot, predicated NOT,
          // OR (measured: C4ko 213 -> 236 G keys/s, m64 KO 286 -> 340)
          asm("{\n\t.reg .pred p;\n\t.reg .b32 t;\n\t"
              "setp.ne.u32 p, %1, 0;\n\t"
              "vote.sync.ballot.b32 t, p, 0xffffffff;\n\t"
              "@p not.b32 t, t;\n\t"
              "or.b32 %0, %0, t;\n\t}"
              : "+r"(diff)
              : "r"(id & (1u << b)));
        } else {
          // key-value: the compiler's 5-instruction form schedules better around the value
          // registers (the inline form measured 10-15 % slower for KV)
          const int32_t sh = (int32_t)(id << (31 - b));
          const uint32_t vote = __ballot_sync(0xFFFFFFFFu, sh < 0);
          diff |= vote ^ (uint32_t)(sh >> 31);
        }
      }
      peers = ~diff;
    }
    const uint32_t rank = __popc(peers & lt);
    uint32_t before = 0;
    if (valid) before = cnt_w[id];
    __syncwarp();
    if (valid && (peers & gt) == 0) cnt_w[id] = before + __popc(peers);
    __syncwarp();
    kreg[r] = key;
    if constexpr (KV) vreg[r] = vals_s[pos];
    pk[r] = ((before + rank) << 8) | (id & 255u);
  }
  __syncthreads();

  // ---- per-bucket cross-warp exclusive prefix, tile bucket starts S_t
  uint32_t tot = 0;
  if (tid < m) {
#pragma unroll
    for (int w = 0; w < kWarps; ++w) {
      const uint32_t c = cnt_s[w * kMaxM + tid];
      cnt_s[w * kMaxM + tid] = tot;
      tot += c;
    }
  }
  const uint32_t incl = warp_incl_scan(tot, lane);
  if (lane == 31) wsum[warp] = incl;
  __syncthreads();
  uint32_t wpre = 0;
#pragma unroll
  for (int w = 0; w < kWarps; ++w) wpre += (w < (int)warp) ? wsum[w] : 0u;
  const uint32_t S = wpre + incl - tot;  // exclusive scan of the tile histogram
  if (tid < m) {
#pragma unroll
    for (int w = 0; w < kWarps; ++w) cnt_s[w * kMaxM + tid] += S;
    gD_s[tid] = gcol - S;
  }
  __syncthreads();

  if constexpr (WL) {
    // ---- ablation (MS_ABLATION_WARP): the paper's Warp-level MS (§5.2.1) -- every
    // warp reorders only its own segment (SEG consecutive keys) and writes its bucket runs:
    // a warp-wide exclusive scan of the warp's bucket counts (shuffles) gives each key its
    // position inside the segment, and cnt_w (the warp's tile slot start per bucket, above)
    // its global position G_j + (slot - S_j).
    constexpr int BPL = ((1 << LOGM) + 31) / 32;  // buckets per lane
    uint32_t cw[BPL], st[BPL], sum = 0;
#pragma unroll
    for (int b = 0; b < BPL; ++b) {
      const uint32_t j = lane * BPL + b;
      cw[b] = st[b] = 0;
      if (j < m) {
        st[b] = cnt_w[j];
        const uint32_t next = warp + 1 < (uint32_t)kWarps ? cnt_s[(warp + 1) * kMaxM + j]
                              : (j + 1 < m ? cnt_s[j + 1] : nt);  // S_{j+1} = cnt_s[0][j+1]
        cw[b] = next - st[b];
      }
      sum += cw[b];
    }
    const uint32_t wincl = warp_incl_scan(sum, lane);
    const uint32_t wcount = __shfl_sync(0xFFFFFFFFu, wincl, 31);
    uint32_t ws[BPL], run = wincl - sum;
#pragma unroll
    for (int b = 0; b < BPL; ++b) {
      ws[b] = run;
      run += cw[b];
    }
    __syncthreads();  // every warp has read its successor's cnt_s row
#pragma unroll
    for (int b = 0; b < BPL; ++b)
      if (lane * BPL + b < m) cnt_w[lane * BPL + b] = ws[b];
    __syncwarp();
    const uint32_t wbase = warp * SEG;
#pragma unroll
    for (int r = 0; r < R; ++r) {
      if (FULL || seg0 + r * 32 < nt) {
        const uint32_t id = pk[r] & 255u;
        const uint32_t pos = wbase + cnt_w[id] + (pk[r] >> 8);
        keys_s[pos] = kreg[r];
        if constexpr (KV) vals_s[pos] = vreg[r];
        if constexpr (ID8) id8_s[pos] = (uint8_t)id;
      }
    }
    __syncwarp();
#pragma unroll
    for (int b = 0; b < BPL; ++b)  // global position of segment slot i = G_j + st_j - S_j + (i - ws_j)
      if (lane * BPL + b < m) cnt_w[lane * BPL + b] = gD_s[lane * BPL + b] + st[b] - ws[b];
    __syncwarp();
    for (uint32_t i = lane; i < wcount; i += 32) {
      const uint32_t k = keys_s[wbase + i];
      uint32_t id;
      if constexpr (ID8) id = id8_s[wbase + i];
      else id = bucket_of_key<KIND>(k, p, spl_s);
      const uint32_t dst = cnt_w[id] + i;
      __stcs(keys_out + dst, k);
      if constexpr (KV) __stcs(vals_out + dst, vals_s[wbase + i]);
    }
    return tot;
  }

  // ---- local multisplit of the tile into shared memory (in place)
#pragma unroll
  for (int r = 0; r < R; ++r) {
    if (FULL || seg0 + r * 32 < nt) {
      const uint32_t id = pk[r] & 255u;
      const uint32_t slot = cnt_w[id] + (pk[r] >> 8);
      keys_s[slot] = kreg[r];
      if constexpr (KV) vals_s[slot] = vreg[r];
      if constexpr (ID8) id8_s[slot] = (uint8_t)id;
    }
  }
  __syncthreads();

  // ---- coalesced stores of the bucket runs
  auto store = [&](uint32_t i) {
    const uint32_t k = keys_s[i];
    uint32_t id;
    if constexpr (ID8) id = id8_s[i];
    else id = bucket_of_key<KIND>(k, p, spl_s);
    const uint32_t dst = gD_s[id] + i;
    __stcs(keys_out + dst, k);
    if constexpr (KV) __stcs(vals_out + dst, vals_s[i]);
  };
  if constexpr (FULL) {
#pragma unroll 4
    for (int j = 0; j < R; ++j) store(j * kThreads + tid);
  } else {
    for (uint32_t i = tid; i < nt; i += kThreads) store(i);
  }
  return tot;  // this tile's count of bucket tid (tid < m)
}

// TPC reorder windows of T keys per subproblem (Eq. (2)'s column of G): with TPC = 2 the
// subproblems are 8192 keys (half the H / G words, K1 and K2 work) while the local reorder keeps
// 4096-key windows; the CTA walks its windows in order with a running G (the first window's
// bucket counts added before the second).  Key-only: both windows' TMA loads are issued up front
// (two buffers); key-value: one buffer, the second window loaded after the first has left.
template <int KIND, bool KV, int R, int LOGM, bool WL = false, int TPC = 1>
__global__ void __launch_bounds__(kThreads, KV ? 3 : 4)  // 4 / 3 CTAs per SM (64 / 85 registers)
k3_postscan(const uint32_t *__restrict__ keys, const uint32_t *__restrict__ vals,
            const void *__restrict__ ids, const uint32_t *__restrict__ G,
            uint32_t *__restrict__ keys_out, uint32_t *__restrict__ vals_out, uint32_t n,
            uint32_t L, const __grid_constant__ BucketParams p, const uint32_t *__restrict__ rowbase) {
  // G: the full Eq. (2) terms 1+2 (K2 = k2_scan), or -- rowbase != nullptr (K2 = k2w_rowscan) --
  // term 2 only, row by row, with term 1 in rowbase[j]
  constexpr int T = kThreads * R;
  constexpr int NB = (TPC > 1 && !KV) ? TPC : 1;  // window buffers
  extern __shared__ __align__(128) uint8_t smem_raw[];
  uint32_t *keys_s0 = reinterpret_cast<uint32_t *>(smem_raw);  // [NB][T]
  uint32_t *vals_s = keys_s0 + NB * T;
  uint32_t *cnt_s = vals_s + (KV ? T : 0);     // [8][256] per-warp counters
  uint32_t *gD_s = cnt_s + kWarps * kMaxM;     // [256] G[j][tile] - S_t[j]
  uint32_t *spl_s = gD_s + kMaxM;              // [256] padded splitters
  uint8_t *id8_s = reinterpret_cast<uint8_t *>(spl_s + kMaxM);  // [T]
  __shared__ __align__(8) uint64_t bar[TPC];
  __shared__ uint32_t wsum[kWarps];

  const uint32_t tid = threadIdx.x;
  const uint32_t tile = blockIdx.x;
  const uint32_t m = p.m;
  auto wbase = [&](int w) -> uint64_t { return ((uint64_t)tile * TPC + w) * T; };
  auto wnt = [&](int w) -> uint32_t { return wbase(w) < n ? (uint32_t)umin64(T, n - wbase(w)) : 0u; };
  auto load = [&](int w, uint32_t *ks) {  // window w into ks (+ vals_s): TMA when full, else by hand
    const uint64_t base = wbase(w);
    const uint32_t nt = wnt(w);
    if (nt == T) {
      if (tid == 0) {
        mbar_arrive_expect_tx(&bar[w], (KV ? 2u : 1u) * T * 4u);
        bulk_g2s(ks, keys + base, T * 4u, &bar[w]);
        if constexpr (KV) bulk_g2s(vals_s, vals + base, T * 4u, &bar[w]);
      }
    } else {
      for (uint32_t i = tid; i < nt; i += kThreads) {
        ks[i] = keys[base + i];
        if constexpr (KV) vals_s[i] = vals[base + i];
      }
    }
  };
  if (tid == 0) {  // (thread 0 also issues the TMA loads: no barrier needed before them)
#pragma unroll
    for (int w = 0; w < TPC; ++w) mbar_init(&bar[w], 1);
    fence_mbar_init();
  }
  load(0, keys_s0);
  if constexpr (NB > 1) {
#pragma unroll
    for (int w = 1; w < TPC; ++w) load(w, keys_s0 + w * T);
  }
  // per-bucket setup while the copy is in flight
  uint32_t gcol = 0;
  pdl_wait();  // K2's G is complete (the tile's TMA load above is already in flight)
  if (tid < m) gcol = __ldg(G + (uint64_t)tid * L + tile);
  if (rowbase != nullptr && tid < m) gcol += __ldg(rowbase + tid);
  if constexpr (KIND == SPLITTERS) {
    if (tid < (1u << p.logm)) spl_s[tid] = p.spl[tid];
  }
#pragma unroll 1
  for (int w = 0; w < TPC; ++w) {
    const uint32_t nt = wnt(w);
    if (nt == 0) break;
    uint32_t *keys_s = keys_s0 + (NB > 1 ? w * T : 0);
    if (NB == 1 && w > 0) load(w, keys_s);  // (the previous window's stores have read the buffer)
#pragma unroll
    for (int q = 0; q < kWarps; ++q) cnt_s[q * kMaxM + tid] = 0;  // kThreads == kMaxM
    __syncthreads();
    uint32_t tot;
    if (nt == T) {
      mbar_wait(&bar[w], 0);
      tot = k3_tile<KIND, KV, R, LOGM, true, WL>(vals, ids, keys_out, vals_out, wbase(w), nt, p, keys_s, vals_s,
                                                 cnt_s, gD_s, spl_s, id8_s, wsum, gcol);
    } else {
      tot = k3_tile<KIND, KV, R, LOGM, false, WL>(vals, ids, keys_out, vals_out, wbase(w), nt, p, keys_s, vals_s,
                                                  cnt_s, gD_s, spl_s, id8_s, wsum, gcol);
    }
    gcol += tot;  // the next window's bucket starts (running G)
    if (TPC > 1) __syncthreads();  // cnt_s / gD_s / id8_s / the buffers are reused by the next window
  }
}

// ------------------------------------------------------------------ host launcher (m > 32)
inline size_t k3w_smem(int R, bool kv, bool id8, int nb = 1) {
  const size_t T = 256u * R;
  return T * 4 * (kv ? 2 : nb) + (kWarps * kMaxM + 2 * kMaxM) * 4 + (id8 ? T : 0);
}

template <int KIND, bool KV, int R, int LOGM, bool WL = false, int TPC = 1>
inline cudaError_t k3w_launch_l(const K3pArgs &a) {
  constexpr bool id8 = (KIND != LOWBITS && KIND != SHIFTC && KIND != SHIFT);
  // ballot ranks (__match_any_sync measured 1.6x slower at m = 256 on B200: MATCH.ANY is
  // ADU-bound)
  auto k = k3_postscan<KIND, KV, R, LOGM, WL, TPC>;
  const size_t smem = k3w_smem(R, KV, id8, (TPC > 1 && !KV) ? TPC : 1);
  if (smem > 48 * 1024) cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  const cudaError_t e = launch_ex(a.pdl != 0, k, dim3(a.L), dim3(kThreads), smem, a.stream, a.keys, a.vals, a.ids,
                                  a.G, a.keys_out, a.vals_out, a.n, a.L, *a.bp, a.rowtot);
  return e != cudaSuccess ? e : cudaGetLastError();
}

template <int KIND, bool KV, int R, int TPC = 1>
inline cudaError_t k3w_launch_r(const K3pArgs &a) {
  if (a.k3w != 0) {  // ablations (MS_ABLATION_BALLOT / _WARP), one-shift bucket kind only, 2 <= m <= 256
    if constexpr (KIND == SHIFT) {
      uint32_t l = 1;
      while ((1u << l) < a.m) ++l;
      const bool wl = a.k3w == 2;
#define MS_K3W_ABL(LG) \
  return wl ? k3w_launch_l<KIND, KV, R, LG, true, TPC>(a) : k3w_launch_l<KIND, KV, R, LG, false, TPC>(a)
      switch (l) {
        case 1: MS_K3W_ABL(1);
        case 2: MS_K3W_ABL(2);
        case 3: MS_K3W_ABL(3);
        case 4: MS_K3W_ABL(4);
        case 5: MS_K3W_ABL(5);
        case 6: MS_K3W_ABL(6);
        case 7: MS_K3W_ABL(7);
        default: MS_K3W_ABL(8);
      }
#undef MS_K3W_ABL
    }
    return cudaErrorNotSupported;
  }
  if (a.m <= 64) return k3w_launch_l<KIND, KV, R, 6, false, TPC>(a);
  if (a.m <= 128) return k3w_launch_l<KIND, KV, R, 7, false, TPC>(a);
  return k3w_launch_l<KIND, KV, R, 8, false, TPC>(a);
}

template <int KIND>
inline cudaError_t k3w_launch(const K3pArgs &a) {
  if (a.kpt == 8) return a.vals ? k3w_launch_r<KIND, true, 8>(a) : k3w_launch_r<KIND, false, 8>(a);
  // 8192-key subproblems (kpt = 32): two 4096-key reorder windows per CTA
  if (a.kpt == 32) return a.vals ? k3w_launch_r<KIND, true, 16, 2>(a) : k3w_launch_r<KIND, false, 16, 2>(a);
  return a.vals ? k3w_launch_r<KIND, true, 16>(a) : k3w_launch_r<KIND, false, 16>(a);
}

}  // namespace ms
