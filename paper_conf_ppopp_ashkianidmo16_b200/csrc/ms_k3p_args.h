// ms_k3p_args.h -- host-side entry points of the persistent K3 (m <= 32), one TU per bucket kind.
#pragma once
#include <cuda_runtime.h>

#include <cstdint>
#include <cstdlib>
#include <cstring>
#include <utility>

#include "ms_device.cuh"

namespace ms {

// Ranged variant with the range scan folded into K3 (range_base below):
// HC = K1r's R = C*k sub-range rows of m counts; offsets written by CTA 0.
struct RangeScan {
  const uint32_t *HC;
  uint32_t *offsets;
  uint32_t R, k;
};

// Fused sharded scatter: K3 stores every bucket
// run straight into its owners' output windows -- peer memory over NVLink on a
// multi-GPU box (pointers from CUDA IPC / symmetric memory), or any device
// pointers.  Rank r owns global positions [wst[r], wst[r+1]); the local run of
// bucket j at local position x goes to global position x + delta[j].  P = 0:
// plain local output (keys_out / vals_out).
constexpr int kMaxPeers = 8;
struct DistTarget {
  uint32_t *keys[kMaxPeers];
  uint32_t *vals[kMaxPeers];
  uint64_t wst[kMaxPeers + 1];
  uint64_t delta[32];  // m <= 32 (K3 v2)
  int32_t P;
};

struct K3pArgs {
  const uint32_t *keys, *vals;
  const void *ids;
  const uint32_t *G;
  uint32_t *keys_out, *vals_out;
  uint32_t n, L, m, id_bytes, kpt;
  uint32_t nt;              // K3 v2 threads per CTA (256); tile = nt * 16 keys
  const BucketParams *bp;  // host copy, passed by value to the kernel
  int sms;
  cudaStream_t stream;
  int ranged = 0;               // 1: CTA-range mode (G = GB[C][m], ms_ranged.cuh); 2: one cooperative launch; m <= 32
  int pdl = 0;                  // 1: programmatic dependent launch after K2 (ms_device.cuh pdl_wait)
  uint32_t *grid_out = nullptr;  // non-null: only compute the grid C (no launch)
  RangeScan rs = {nullptr, nullptr, 0, 0};  // ranged / ONE: the range scan's input (K3's prologue)
  const DistTarget *ds = nullptr;           // fused sharded scatter (K3 v2, tile variant only)
  int direct = 0;                           // ablation: K3 v2 without the local reorder (MS_ABLATION_DIRECT)
  int k3w = 0;                              // ablation: the ballot K3 (ms_k3_warp.cuh) for any m, block-level (1,
                                            // MS_ABLATION_BALLOT) or warp-level (2, MS_ABLATION_WARP) reorder
  uint32_t *flag = nullptr;                 // IDS + validation: set to 1 when some id >= m
  const uint32_t *rowtot = nullptr;         // m > 32: G holds row-local scans, term 1 in rowtot[j] (row base)
};

// Launch with cudaLaunchAttributeProgrammaticStreamSerialization when `pdl`:
// the kernel may begin while its stream predecessor finishes, and must call
// pdl_wait() before touching the predecessor's output.
template <typename... KArgs, typename... Args>
inline cudaError_t launch_ex(bool pdl, void (*kern)(KArgs...), dim3 grid, dim3 block, size_t smem, cudaStream_t s,
                             Args &&...args) {
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = grid;
  cfg.blockDim = block;
  cfg.dynamicSmemBytes = smem;
  cfg.stream = s;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  at[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = at;
  cfg.numAttrs = pdl ? 1 : 0;
  return cudaLaunchKernelEx(&cfg, kern, std::forward<Args>(args)...);
}

// ============================================================== range scan folded into K3
// Terms 1+2 of Eq. (2) for range c, computed redundantly by every K3 CTA from
// K1r's rows (no separate scan launch or hand-off; the R x m words are
// L2-resident, R*m*4 <= 76 KB for m <= 16):
//   pre_j = sum_{r < c*k} HC[r][j],  tot_j = sum_r HC[r][j],
//   GB[c][j] = sum_{i<j} tot_i + pre_j,  offsets[j] = sum_{i<j} tot_i (CTA 0).
// Thread (s, j) (j = tid mod MP) sums rows s, s + NS, ... of column j, so one
// warp load covers 32/MP consecutive rows (contiguous words when m = MP).
// Every thread of the CTA must call it; `red` is 2*NT + 2*(NT/32)*max(MP, 32)
// words of scratch shared memory that nothing else touches until the caller's
// next __syncthreads().  m <= 64 (MP = 64: the key-only ONE of 33..64 buckets).
// Returns GB[c][row] (0 for row >= m).
template <int NT, int LOGMP>
__device__ __forceinline__ uint32_t range_base(const RangeScan &rs, uint32_t m, uint32_t c, uint32_t n,
                                               uint32_t *red, uint32_t row) {
  constexpr uint32_t MP = 1u << LOGMP, NS = NT / MP;
  static_assert(MP <= 64 && NT >= 2 * MP, "range_base: up to 64 buckets");
  const uint32_t tid = threadIdx.x, j = tid & (MP - 1), s = tid >> LOGMP;
  const uint32_t cut = c * rs.k;
  // red[0 .. MP): per-bucket sums of the rows before `cut` (pre), red[NT .. NT + MP): from `cut` on
  if (MP >= 4 && m == MP) {
    // m a power of two >= 4: 128-bit loads (thread t always reads column group t mod MP/4 of
    // rows t/(MP/4), (t+NT)/(MP/4), ...), lane-shuffle reduction per warp, then the warps' partials
    constexpr uint32_t Q4 = MP >= 4 ? MP / 4 : 1, NW = NT / 32, WS = MP > 32 ? MP : 32;
    const uint32_t lane = tid & 31, warp = tid >> 5, cg = tid & (Q4 - 1);
    uint32_t pr[4] = {0u, 0u, 0u, 0u}, po[4] = {0u, 0u, 0u, 0u};
    const uint4 *h4 = reinterpret_cast<const uint4 *>(rs.HC);
    const uint32_t tot4 = rs.R * Q4;
#pragma unroll 4
    for (uint32_t u = tid; u < tot4; u += NT) {
      const uint4 v = __ldcg(h4 + u);
      const uint32_t vv[4] = {v.x, v.y, v.z, v.w};
      const bool before = u / Q4 < cut;
#pragma unroll
      for (int e = 0; e < 4; ++e) {
        pr[e] += before ? vv[e] : 0u;
        po[e] += before ? 0u : vv[e];
      }
    }
#pragma unroll
    for (uint32_t off = 16; off >= Q4; off >>= 1) {
#pragma unroll
      for (int e = 0; e < 4; ++e) {
        pr[e] += __shfl_xor_sync(0xFFFFFFFFu, pr[e], off);
        po[e] += __shfl_xor_sync(0xFFFFFFFFu, po[e], off);
      }
    }
    uint32_t *part = red + 2 * NT;  // [2][NW][WS] the warps' partials
    if (lane < Q4) {
#pragma unroll
      for (int e = 0; e < 4; ++e) {
        part[warp * WS + cg * 4 + e] = pr[e];
        part[NW * WS + warp * WS + cg * 4 + e] = po[e];
      }
    }
    __syncthreads();
    if (tid < m) {
      uint32_t pj = 0, qj = 0;
#pragma unroll
      for (uint32_t w = 0; w < NW; ++w) {
        pj += part[w * WS + tid];
        qj += part[NW * WS + w * WS + tid];
      }
      red[tid] = pj;
      red[NT + tid] = qj;
    }
    __syncthreads();
  } else {
    uint32_t pre = 0, post = 0;
    if (j < m) {
      const uint32_t *col = rs.HC + j;
#pragma unroll 8
      for (uint32_t r = s; r < rs.R; r += NS) {
        const uint32_t v = __ldcg(col + (uint64_t)r * m);
        if (r < cut) pre += v;
        else post += v;
      }
    }
    red[tid] = pre;
    red[NT + tid] = post;
    __syncthreads();
#pragma unroll
    for (uint32_t d = NS / 2; d >= 1; d >>= 1) {
      if (s < d) {
        red[tid] += red[tid + d * MP];
        red[NT + tid] += red[NT + tid + d * MP];
      }
      __syncthreads();
    }
  }
  // one warp scans the m <= 64 bucket totals, two buckets per lane: bucket start + the pre part
  if (tid < 32) {
    const uint32_t b0 = 2 * tid, b1 = b0 + 1;
    const uint32_t p0 = b0 < m ? red[b0] : 0u, t0 = b0 < m ? p0 + red[NT + b0] : 0u;
    const uint32_t p1 = b1 < m ? red[b1] : 0u, t1 = b1 < m ? p1 + red[NT + b1] : 0u;
    const uint32_t st0 = warp_incl_scan(t0 + t1, tid) - t0 - t1, st1 = st0 + t0;
    __syncwarp();
    if (b0 < m) red[NT + b0] = st0 + p0;
    if (b1 < m) red[NT + b1] = st1 + p1;
    if (c == 0 && rs.offsets != nullptr) {
      if (b0 < m) rs.offsets[b0] = st0;
      if (b1 < m) rs.offsets[b1] = st1;
      if (tid == 0) rs.offsets[m] = n;
    }
  }
  __syncthreads();
  return row < m ? red[NT + row] : 0u;
}


// Cooperative launch (all CTAs co-resident; grid-wide barrier inside the kernel).
template <typename... KArgs, typename... Args>
inline cudaError_t launch_coop(void (*kern)(KArgs...), dim3 grid, dim3 block, size_t smem, cudaStream_t s,
                               Args &&...args) {
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = grid;
  cfg.blockDim = block;
  cfg.dynamicSmemBytes = smem;
  cfg.stream = s;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeCooperative;
  at[0].val.cooperative = 1;
  cfg.attrs = at;
  cfg.numAttrs = 1;
  return cudaLaunchKernelEx(&cfg, kern, std::forward<Args>(args)...);
}

constexpr uint32_t kMaxRanges = 1024;  // upper bound on the CTA-range count C (workspace sizing)

// m <= 32 (ms_k3_v2.cuh): TMA-tensor staging, keys in registers, blocked private counters
cudaError_t k3v_launch_lowbits(const K3pArgs &a);
cudaError_t k3v_launch_shiftc(const K3pArgs &a);
cudaError_t k3v_launch_shift(const K3pArgs &a);
cudaError_t k3v_launch_delta(const K3pArgs &a);
cudaError_t k3v_launch_splitters(const K3pArgs &a);
cudaError_t k3v_launch_ids(const K3pArgs &a);
cudaError_t k3v_launch_shiftc_lo(const K3pArgs &a);
cudaError_t k3v_launch_delta_lo(const K3pArgs &a);
// m > 32: warp-ballot K3 (ms_k3_warp.cuh); kpt carries the rounds per warp R (8 or 16)
cudaError_t k3w_launch_lowbits(const K3pArgs &a);
cudaError_t k3w_launch_shiftc(const K3pArgs &a);
cudaError_t k3w_launch_shift(const K3pArgs &a);
cudaError_t k3w_launch_delta(const K3pArgs &a);
cudaError_t k3w_launch_splitters(const K3pArgs &a);
cudaError_t k3w_launch_ids(const K3pArgs &a);
cudaError_t k3w_launch_shiftc_lo(const K3pArgs &a);
cudaError_t k3w_launch_delta_lo(const K3pArgs &a);
// m > 256 (ms_wide.cu): offsets from the id-sorted output, MS_IDS range check
cudaError_t wide_offsets_launch(int kind, const uint32_t *src, uint64_t n, uint32_t *offsets,
                                const BucketParams &bp, int sms, cudaStream_t s);
cudaError_t ids_check_launch(const uint32_t *ids, uint64_t n, uint32_t m, uint32_t *flag, int sms, cudaStream_t s);

}  // namespace ms
