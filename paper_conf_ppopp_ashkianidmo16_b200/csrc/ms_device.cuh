// ms_device.cuh -- device primitives of the B200 multisplit (sm_100a).
//
// Bucket functors (whatBucket()), warp
// helpers and the TMA bulk-copy + mbarrier wrappers used to stage tiles in
// shared memory.
#pragma once
#include <cstdint>

namespace ms {

// Kernel-level bucket-function kinds.  The public kinds (ms.h) map onto
// these; MS_DELTA becomes SHIFTC when delta is a power of two (incl. 1), and
// SHIFT when in addition m * delta >= 2^32 (the clamp can never fire: the
// paper's "buckets equally divide the 32-bit domain").
// SHIFTC_LO / DELTA_LO: the LOW digit of a clamped id, (min(q, clamp) & mmask)
// with q = k >> shift or floor(k / delta) -- the first pass of the two-pass
// multisplit for m > 256 (ms_api.cu "wide plans").
enum Kind : int { LOWBITS = 0, DELTA = 1, SPLITTERS = 2, IDS = 3, SHIFTC = 4, SHIFT = 5, SHIFTC_LO = 6,
                  DELTA_LO = 7 };

constexpr int kThreads = 256;  // CTA = 8 warps (the paper's NW = 8)
constexpr int kWarps = kThreads / 32;
constexpr int kMaxM = 256;

// Bucket-function constants, passed by value as a kernel parameter (constant
// bank; no device allocation).  spl[] holds the splitters padded to
// Q = 2^logm entries with 0xFFFFFFFF (never "< key"), so the branchless
// search below always runs exactly logm steps.
struct BucketParams {
  uint32_t m;         // number of buckets (1..256)
  uint32_t mmask;     // m - 1
  uint32_t shift;     // LOWBITS bit offset; SHIFTC: log2(delta)
  uint32_t magic_lo;  // DELTA: c = ceil(2^64 / delta) (Lemire-Kaser-Kurz), low word
  uint32_t magic_hi;  //        high word
  uint32_t logm;      // ceil(log2 m): splitter search steps
  uint32_t id_bytes;  // IDS: 1 or 4
  uint32_t validate;  // IDS: flag ids >= m
  uint32_t clamp;     // SHIFTC_LO / DELTA_LO: the full id's clamp (m_full - 1)
  uint32_t spl[kMaxM];
};

// id = (k >> shift) & (m - 1)
__device__ __forceinline__ uint32_t id_lowbits(uint32_t k, const BucketParams &p) {
  return (k >> p.shift) & p.mmask;
}

// id = min(k >> log2(delta), m - 1): delta a power of two
__device__ __forceinline__ uint32_t id_shiftc(uint32_t k, const BucketParams &p) {
  return min(k >> p.shift, p.mmask);
}

// id = min(floor(k / delta), m - 1) for 1 < delta < 2^32, not a power of two:
// floor(k * c / 2^64) with c = ceil(2^64 / delta) is exact for every 32-bit k
// (F = 64 >= N + log2(delta) = 32 + 32).  Two 32x32->64 multiply-adds.
__device__ __forceinline__ uint32_t div_delta(uint32_t k, const BucketParams &p) {
  const uint64_t lo = (uint64_t)p.magic_lo * k;
  const uint64_t hi = (uint64_t)p.magic_hi * k + (lo >> 32);
  return (uint32_t)(hi >> 32);
}
__device__ __forceinline__ uint32_t id_delta(uint32_t k, const BucketParams &p) {
  return min(div_delta(k, p), p.mmask);
}

// id = #{ j : s_j < k }: branchless binary search over the padded table.
template <int LOGM_MAX = 8>
__device__ __forceinline__ uint32_t id_splitters(uint32_t k, const uint32_t *S, uint32_t logm) {
  uint32_t pos = 0;
#pragma unroll
  for (int s = LOGM_MAX - 1; s >= 0; --s) {
    if ((uint32_t)s < logm) {
      uint32_t h = 1u << s;
      pos += (S[pos + h - 1] < k) ? h : 0u;
    }
  }
  return pos;
}

// ---- SPLITTERS through a bin table (DESIGN.md §7 "splitter bin table").
// The key domain is cut into 1024 bins of W = 2^22 keys.  For bin b
// (keys [b*W, (b+1)*W)) let lo = #{j : s_j < b*W} and c = the number of
// splitters in [b*W, b*W + W - 2] (a splitter equal to the bin's last key is
// never < a key of the bin).  Then for k in bin b, #{j : s_j < k} =
//   c == 0: lo;   c == 1: lo + ((k - b*W) > (s_lo - b*W));   c >= 2: lo + #{...}
// Entry: bit 31 = (c >= 2), bits 23..30 = lo, bits 0..22 = s_lo - b*W when
// c == 1, else 0x7FFFFF (larger than any in-bin offset: the compare is false).
// The c >= 2 case (rare for random splitters) walks the splitters from lo.
constexpr int kSplBins = 1024;
constexpr uint32_t kSplBinShift = 22;
constexpr uint32_t kSplOffMask = (1u << kSplBinShift) - 1;

__device__ __forceinline__ uint32_t id_spl_table(uint32_t k, const uint32_t *tbl, const uint32_t *S) {
  const uint32_t e = tbl[k >> kSplBinShift];
  uint32_t id = ((e >> 23) & 0xFFu) + ((k & kSplOffMask) > (e & 0x7FFFFFu) ? 1u : 0u);
  if ((int32_t)e < 0) {
    while (S[id] < k) ++id;  // S is padded with 0xFFFFFFFF: the walk stops by id = m - 1
  }
  return id;
}

// Build the bin table in shared memory from the padded splitters S (already
// in shared memory); NT threads, each computes kSplBins / NT entries with two
// branchless searches (lo and lo + c).
template <int NT>
__device__ __forceinline__ void build_spl_table(uint32_t *tbl, const uint32_t *S, uint32_t logm) {
  for (uint32_t b = threadIdx.x; b < (uint32_t)kSplBins; b += NT) {
    const uint32_t bs = b << kSplBinShift;
    const uint32_t lo = id_splitters(bs, S, logm);
    const uint32_t hi = id_splitters(bs + kSplOffMask, S, logm);  // #{s_j < bs + W - 1}
    const uint32_t c = hi - lo;
    tbl[b] = c == 0 ? (lo << 23) | 0x7FFFFFu
                    : c == 1 ? (lo << 23) | (S[lo] - bs) : 0x80000000u | (lo << 23) | 0x7FFFFFu;
  }
}

template <int KIND>
__device__ __forceinline__ uint32_t bucket_of_key(uint32_t k, const BucketParams &p,
                                                  const uint32_t *spl_s) {
  if constexpr (KIND == LOWBITS) return id_lowbits(k, p);
  else if constexpr (KIND == SHIFT) return k >> p.shift;  // m * delta >= 2^32: always < m
  else if constexpr (KIND == SHIFTC) return id_shiftc(k, p);
  else if constexpr (KIND == DELTA) return id_delta(k, p);
  else if constexpr (KIND == SHIFTC_LO) return min(k >> p.shift, p.clamp) & p.mmask;
  else if constexpr (KIND == DELTA_LO) return min(div_delta(k, p), p.clamp) & p.mmask;
  else if constexpr (KIND == SPLITTERS) return id_splitters(k, spl_s, p.logm);
  else return 0u;
}

// Precomputed id (MS_IDS), clamped so that a contract violation can never
// index outside the tile's counters (the output is then unspecified, and
// flagged when validation is on).
__device__ __forceinline__ uint32_t load_id(const void *ids, uint64_t i, const BucketParams &p) {
  uint32_t v = p.id_bytes == 1 ? (uint32_t)__ldg((const uint8_t *)ids + i)
                               : __ldg((const uint32_t *)ids + i);
  return min(v, p.mmask);
}

// ------------------------------------------------------------------ PTX helpers
// Programmatic dependent launch (sm_90+): a kernel launched with
// cudaLaunchAttributeProgrammaticStreamSerialization may start while its
// predecessor in the stream is still running; pdl_wait() blocks until the
// predecessor grid has completed and its memory is visible (a no-op without
// the attribute); pdl_trigger() lets the successor's CTAs be scheduled.
__device__ __forceinline__ void pdl_wait() { asm volatile("griddepcontrol.wait;" ::: "memory"); }
__device__ __forceinline__ void pdl_trigger() { asm volatile("griddepcontrol.launch_dependents;" ::: "memory"); }

__device__ __forceinline__ uint32_t smem_u32(const void *p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}

__device__ __forceinline__ void mbar_init(uint64_t *bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count));
}

__device__ __forceinline__ void fence_mbar_init() {
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}

// order generic-proxy shared-memory writes before later async-proxy (TMA) reads
__device__ __forceinline__ void fence_proxy_async_smem() {
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}

__device__ __forceinline__ void mbar_arrive_expect_tx(uint64_t *bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)),
               "r"(bytes)
               : "memory");
}

__device__ __forceinline__ void mbar_wait(uint64_t *bar, uint32_t parity) {
  uint32_t done = 0;
  while (!done) {
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n\t"
        "selp.u32 %0, 1, 0, p;\n\t}"
        : "=r"(done)
        : "r"(smem_u32(bar)), "r"(parity)
        : "memory");
  }
}

// TMA 1-D bulk copy global -> shared (UBLKCP), completion counted on `bar`.
// src, dst 16-byte aligned, bytes a multiple of 16.
__device__ __forceinline__ void bulk_g2s(void *dst_smem, const void *src, uint32_t bytes,
                                         uint64_t *bar) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
          smem_u32(dst_smem)),
      "l"(src), "r"(bytes), "r"(smem_u32(bar))
      : "memory");
}

// TMA 1-D bulk copy shared -> global (bulk-group completion).  dst, src
// 16-byte aligned, bytes a multiple of 16.
__device__ __forceinline__ void bulk_s2g(void *dst, const void *src_smem, uint32_t bytes) {
  asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(dst),
               "r"(smem_u32(src_smem)), "r"(bytes)
               : "memory");
}
__device__ __forceinline__ void bulk_commit() { asm volatile("cp.async.bulk.commit_group;" ::: "memory"); }
// wait until the committed bulk stores have finished READING shared memory
__device__ __forceinline__ void bulk_wait_read0() {
  asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory");
}
__device__ __forceinline__ void bulk_wait0() { asm volatile("cp.async.bulk.wait_group 0;" ::: "memory"); }

// shared-memory accesses by 32-bit shared-window address (one IMAD/LEA per
// address, in program order: the counting read-modify-write depends on it)
__device__ __forceinline__ uint32_t lds_u16(uint32_t a) {
  uint16_t v;
  asm volatile("ld.shared.u16 %0, [%1];" : "=h"(v) : "r"(a) : "memory");
  return v;
}
__device__ __forceinline__ void sts_u16(uint32_t a, uint32_t v) {
  asm volatile("st.shared.u16 [%0], %1;" ::"r"(a), "h"((uint16_t)v) : "memory");
}
__device__ __forceinline__ void sts_u32(uint32_t a, uint32_t v) {
  asm volatile("st.shared.u32 [%0], %1;" ::"r"(a), "r"(v) : "memory");
}
// u16 counter at shared address a (2-byte aligned) incremented by a 32-bit shared atomic on its
// word (the other half belongs to another thread and never carries: counts stay < 2^16); returns
// the counter's old value.  No load -> add -> store round trip in the issuing thread, so
// consecutive increments pipeline.
__device__ __forceinline__ uint32_t atom_inc_u16(uint32_t a) {
  const uint32_t sh = (a & 2u) * 8u;
  uint32_t old;
  asm volatile("atom.shared.add.u32 %0, [%1], %2;" : "=r"(old) : "r"(a & ~3u), "r"(1u << sh) : "memory");
  return (old >> sh) & 0xFFFFu;
}
__device__ __forceinline__ void red_inc_u16(uint32_t a) {  // the same, old value not needed
  asm volatile("red.shared.add.u32 [%0], %1;" ::"r"(a & ~3u), "r"(1u << ((a & 2u) * 8u)) : "memory");
}

__device__ __forceinline__ uint64_t umin64(uint64_t a, uint64_t b) { return a < b ? a : b; }
inline uint64_t umin64_host(uint64_t a, uint64_t b) { return a < b ? a : b; }

__device__ __forceinline__ uint32_t lanemask_lt() {
  uint32_t r;
  asm("mov.u32 %0, %%lanemask_lt;" : "=r"(r));
  return r;
}
__device__ __forceinline__ uint32_t lanemask_gt() {
  uint32_t r;
  asm("mov.u32 %0, %%lanemask_gt;" : "=r"(r));
  return r;
}

// 64-bit status words of the decoupled look-back: (flag << 32) | value.
__device__ __forceinline__ uint64_t ld_status(const uint64_t *p) {
  uint64_t v;
  asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_status(uint64_t *p, uint64_t v) {
  asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}

__device__ __forceinline__ uint32_t warp_incl_scan(uint32_t v, uint32_t lane) {
#pragma unroll
  for (int d = 1; d < 32; d <<= 1) {
    uint32_t t = __shfl_up_sync(0xFFFFFFFFu, v, d);
    if (lane >= (uint32_t)d) v += t;
  }
  return v;
}

__device__ __forceinline__ uint32_t warp_sum(uint32_t v) { return __reduce_add_sync(0xFFFFFFFFu, v); }

}  // namespace ms
