// ms_api.cu -- host plan + C ABI of libms.so (see include/ms.h).
//
// The plan is host metadata only: validated bucket spec, the bucket-function
// constants (BucketParams, passed to every kernel by value) and the tile
// geometry rule.  ms_run enqueues K1 -> K2 -> K3 on the caller's stream with
// no allocation and no synchronisation.
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdint>
#include <cstdlib>
#include <cstring>
#include <new>
#include <vector>

#include "../../include/ms.h"
#include "ms_kernels.cuh"
#include "ms_k3p_args.h"
#include "ms_ranged.cuh"

using namespace ms;

// Variants (include/ms.h): which kernels one ms_run enqueues.
enum Variant : int { V_TILE = 0, V_RANGED = 1, V_ONE = 2 };

struct ms_plan_s {
  ms_bucket_spec spec;
  uint64_t max_n;
  int kv;
  uint32_t flags;
  BucketParams bp;
  int kkind;  // kernel-level Kind (ms_device.cuh)
  int device;  // CUDA ordinal every call of this plan runs on
  int sms;     // its SM count
  uint32_t kpt = 16;    // K3 (m <= 32): keys per thread (32 for key-only ONE runs)
  uint32_t k3nt = 256;  // K3 (m <= 32): threads per CTA; tile T = k3nt * kpt = 4096
  int forced = -1;      // MS_VARIANT_* flag: the variant every run uses (-1: chosen per run)
  int direct = 0;       // MS_ABLATION_DIRECT: K3 stores keys straight to global, no local reorder
  int k3w = 0;          // MS_ABLATION_BALLOT (1) / _WARP (2): the ballot K3 for any m, block / warp reorder
  uint32_t k1s_per_sm = 8;  // splitter K1: persistent CTAs per SM (each builds the bin table once)
  int32_t last_launches;
  // m > 256 ("wide"): two stable passes, by the low then the high digit of the id;
  // wa / wb are the passes' plans (wb null when the high digit is always 0), wkind / wbp the full
  // id's bucket function for the offsets pass over the sorted output
  int wide = 0;  // 0 no, 1 computed ids (recomputed from the keys in each pass), 2 MS_IDS (u32 ids)
  ms_plan_s *wa = nullptr, *wb = nullptr;
  int wkind = 0;
  BucketParams wbp;
  // per-stage trace (ms_plan_trace): one set of 4 events per traced run
  int tracing = 0;     // 0 off, 1 per-stage events, 2 whole-run events only
  int trace_mode = 1;  // mode of the recorded runs (kept after tracing stops)
  size_t trace_runs = 0;
  std::vector<cudaEvent_t> trace_ev;  // 4 * capacity
};

#ifndef MS_K32_MINM
#define MS_K32_MINM 2
#endif
namespace {
// returns the 4 events for the next traced run (nullptr when not tracing)
cudaEvent_t *trace_next(ms_plan_s *p) {
  if (!p->tracing) return nullptr;
  size_t need = 4 * (p->trace_runs + 1);
  while (p->trace_ev.size() < need) {
    cudaEvent_t e;
    if (cudaEventCreate(&e) != cudaSuccess) return nullptr;
    p->trace_ev.push_back(e);
  }
  return &p->trace_ev[4 * p->trace_runs++];
}
}  // namespace

namespace {

constexpr size_t kAlign = 256;
inline size_t align_up(size_t x) { return (x + kAlign - 1) / kAlign * kAlign; }

uint32_t ceil_log2(uint32_t m) {
  uint32_t l = 0;
  while ((1ull << l) < m) ++l;
  return l;
}

// Division by an invariant 32-bit delta that is not a power of two (so
// delta >= 3): c = ceil(2^64 / delta) = floor((2^64 - 1) / delta) + 1, and
// floor(k / delta) = floor(k * c / 2^64) for every 32-bit k (Lemire, Kaser &
// Kurz: exact when the magic has >= 32 + log2(delta) fractional bits).
uint64_t delta_magic(uint32_t d) { return ~0ull / d + 1; }

// Rounds per warp R (subproblem T = 256 R keys): kpt for the blocked-rank K3 (m <= 32, and the
// key-only ONE up to 64 buckets); for the ballot K3 of m > 32, 32 on key-only plans (8192-key
// subproblems reordered as two 4096-key windows per CTA: half the H / G words and K1 / K2 work,
// C4ko 247 -> 259 G keys/s) and 16 on key-value plans (the second window's serialised load costs
// more there: C4kv 177 -> 155) -- halved while the grid would not fill two waves of 148 SMs (small
// n is launch / latency bound, not HBM bound).
int rounds_for(uint32_t m, uint64_t n, uint32_t kpt, bool kv_plan) {
  if (m <= 32 || (kpt == 32 && m <= 64)) return (int)kpt;  // blocked-rank K3: T = 256 * kpt for every n
  int R = kv_plan ? 16 : 32;
  while (R > 8 && (n + 256ull * R - 1) / (256ull * R) < 2 * 148) R >>= 1;
  return R;
}

struct Geometry {
  int R;
  uint32_t T;
  uint64_t L;
  uint64_t hg_words;   // m * L
  uint64_t chunks;     // K2 CTAs
  size_t off_hg, off_status, off_flag, off_rowtot, bytes;
  size_t off_hc;          // CTA-range / ONE variants: range counts HC[R][m], over the H/G region
};

Geometry geometry(const ms_plan_s *p, uint64_t n, uint32_t kpt = 0) {
  Geometry g{};
  g.R = rounds_for(p->spec.m, n, (kpt ? kpt : p->kpt) * p->k3nt / 256, p->kv != 0);
  g.T = 256u * g.R;
  g.L = (n + g.T - 1) / g.T;
  g.hg_words = (uint64_t)p->spec.m * g.L;
  g.chunks = (g.hg_words + kScanChunk - 1) / kScanChunk;
  // [flag | H/G | look-back status]; the flag sits at offset 0 for every n
  g.off_flag = 0;
  g.off_hg = kAlign;
  g.off_status = g.off_hg + align_up(g.hg_words * 4);
  // m > 32: K2's row totals [kMaxM], row bases [kMaxM] and its ticket
  g.off_rowtot = g.off_status + align_up(std::max<uint64_t>(g.chunks, 1) * 8);
  g.bytes = g.off_rowtot + align_up((size_t)(2 * kMaxM + 2) * 4);
  if (p->spec.m <= 32) {  // the range counts reuse the tile arrays' space (never live together)
    g.off_hc = g.off_hg;
    g.bytes = std::max(g.bytes, g.off_hc + align_up((size_t)kMaxRangeRows * p->spec.m * 4));
  }
  return g;
}

bool misaligned(const void *ptr) { return ptr && (reinterpret_cast<uintptr_t>(ptr) & 15u); }

bool overlap(const void *a, size_t abytes, const void *b, size_t bbytes) {
  if (!a || !b || !abytes || !bbytes) return false;
  uintptr_t x = (uintptr_t)a, y = (uintptr_t)b;
  return x < y + bbytes && y < x + abytes;
}

template <typename K>
void set_smem(K kernel, size_t bytes) {
  if (bytes > 48 * 1024) cudaFuncSetAttribute(kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)bytes);
}

// Every call of a plan runs on the plan's device: switch to it for the call's
// duration when the calling thread is on another one.
struct DeviceGuard {
  int prev = -1;
  explicit DeviceGuard(int dev) {
    int cur = -1;
    if (cudaGetDevice(&cur) == cudaSuccess && cur != dev && cudaSetDevice(dev) == cudaSuccess) prev = cur;
  }
  ~DeviceGuard() {
    if (prev >= 0) cudaSetDevice(prev);
  }
};

size_t k1_smem(uint32_t m, int kind) {
  return kMaxM * 4 + (kind == SPLITTERS ? kSplBins * 4 : 0) + (size_t)m * kThreads;
}


// ---------------------------------------------------------------- dispatch
template <int KIND>
cudaError_t launch_k1(const ms_plan_s *p, const Geometry &g, const uint32_t *keys, const void *ids,
                      uint32_t n, uint32_t *H, uint64_t *zero_ptr, uint32_t zero_words,
                      uint32_t *flag, cudaStream_t s) {
  const size_t smem = p->spec.m > 32 ? (kMaxM + 2 * (size_t)p->spec.m) * 4 : k1_smem(p->spec.m, KIND);
  // one CTA per tile group; SPLITTERS: k1s_prescan on a persistent grid (8 CTAs
  // per SM) so the bin table is built once per CTA
#define MS_K1(KPT, SUBT)                                                                          \
  {                                                                                                \
    auto k = p->spec.m > 32     ? k1a_prescan<KIND, KPT, SUBT>                                     \
             : KIND == SPLITTERS ? k1s_prescan<KIND, KPT, SUBT>                                     \
                                 : k1_prescan<KIND, KPT, SUBT>;                                     \
    set_smem(k, smem);                                                                             \
    uint64_t grid = (g.L + SUBT - 1) / SUBT;                                                       \
    if (KIND == SPLITTERS && p->spec.m <= 32) grid = std::min<uint64_t>(grid, (uint64_t)p->k1s_per_sm * p->sms); \
    k<<<(unsigned)grid, kThreads, smem, s>>>(keys, ids, n, (uint32_t)g.L, H, p->bp, zero_ptr, zero_words, \
                                             flag);                                                \
  }
  switch (g.R) {  // 16 keys per thread; T = 2048 tiles are counted two per CTA
    case 8: MS_K1(16, 2) break;
    case 16: MS_K1(16, 1) break;
    default: MS_K1(32, 1) break;
  }
#undef MS_K1
  return cudaGetLastError();
}

cudaError_t dispatch_k1(const ms_plan_s *p, const Geometry &g, const uint32_t *keys, const void *ids,
                        uint32_t n, uint32_t *H, uint64_t *zp, uint32_t zw, uint32_t *flag,
                        cudaStream_t s) {
  switch (p->kkind) {
    case LOWBITS: return launch_k1<LOWBITS>(p, g, keys, ids, n, H, zp, zw, flag, s);
    case SHIFTC: return launch_k1<SHIFTC>(p, g, keys, ids, n, H, zp, zw, flag, s);
    case SHIFT: return launch_k1<SHIFT>(p, g, keys, ids, n, H, zp, zw, flag, s);
    case SHIFTC_LO: return launch_k1<SHIFTC_LO>(p, g, keys, ids, n, H, zp, zw, flag, s);
    case DELTA_LO: return launch_k1<DELTA_LO>(p, g, keys, ids, n, H, zp, zw, flag, s);
    case DELTA: return launch_k1<DELTA>(p, g, keys, ids, n, H, zp, zw, flag, s);
    case SPLITTERS: return launch_k1<SPLITTERS>(p, g, keys, ids, n, H, zp, zw, flag, s);
    default: return launch_k1<IDS>(p, g, keys, ids, n, H, zp, zw, flag, s);
  }
}


cudaError_t dispatch_k3(const ms_plan_s *p, const Geometry &g, const uint32_t *keys,
                        const uint32_t *vals, const void *ids, const uint32_t *G, uint32_t *ko,
                        uint32_t *vo, uint32_t n, uint32_t *flag, cudaStream_t s, int ranged = 0,
                        uint32_t *grid_out = nullptr, int pdl = 0, const RangeScan *rs = nullptr,
                        const uint32_t *rowtot = nullptr) {
  K3pArgs a{keys, vals, ids, G, ko, vo, n, (uint32_t)g.L, p->spec.m, p->spec.id_bytes,
            p->spec.m <= 32 ? g.T / 256 : (uint32_t)g.R, p->k3nt, &p->bp, p->sms, s};
  a.ranged = ranged;
  a.grid_out = grid_out;
  a.pdl = pdl;
  a.direct = p->direct;
  a.k3w = p->k3w;
  a.flag = flag;
  a.rowtot = rowtot;
  if (rs) a.rs = *rs;
  if ((p->spec.m <= 32 || ranged == 2) && !p->k3w) {  // K3 v2 (ms_k3_v2.cuh), one TU per kind
    switch (p->kkind) {
      case LOWBITS: return k3v_launch_lowbits(a);
      case SHIFTC: return k3v_launch_shiftc(a);
      case SHIFT: return k3v_launch_shift(a);
      case SHIFTC_LO: return k3v_launch_shiftc_lo(a);
      case DELTA_LO: return k3v_launch_delta_lo(a);
      case DELTA: return k3v_launch_delta(a);
      case SPLITTERS: return k3v_launch_splitters(a);
      default: return k3v_launch_ids(a);
    }
  }
  switch (p->kkind) {  // m > 32: warp-ballot K3 (ms_k3_warp.cuh)
    case LOWBITS: return k3w_launch_lowbits(a);
    case SHIFTC: return k3w_launch_shiftc(a);
    case SHIFT: return k3w_launch_shift(a);
    case SHIFTC_LO: return k3w_launch_shiftc_lo(a);
    case DELTA_LO: return k3w_launch_delta_lo(a);
    case DELTA: return k3w_launch_delta(a);
    case SPLITTERS: return k3w_launch_splitters(a);
    default: return k3w_launch_ids(a);
  }
}

// K1r: k sub-ranges per range so that the grid has ~8 CTAs of 256 threads per SM
uint32_t k1r_split(const ms_plan_s *p, uint32_t C) {
  return std::max<uint32_t>(1u, std::min<uint32_t>(8u * (uint32_t)p->sms / C, kMaxRangeRows / C));
}

template <int KIND>
cudaError_t launch_k1r(const ms_plan_s *p, const Geometry &g, uint32_t C, const uint32_t *keys, const void *ids,
                       uint32_t n, uint32_t *HC, uint32_t *flag, cudaStream_t s) {
  const uint32_t k = k1r_split(p, C);
  auto kern = k1r_prescan<KIND, 256>;
  const size_t smem = k1r_smem(p->spec.m, KIND, 256);
  set_smem(kern, smem);
  kern<<<C * k, 256, smem, s>>>(keys, ids, n, (uint32_t)g.L, g.T, C, k, HC, p->bp, flag);
  return cudaGetLastError();
}

cudaError_t dispatch_k1r(const ms_plan_s *p, const Geometry &g, uint32_t C, const uint32_t *keys, const void *ids,
                         uint32_t n, uint32_t *HC, uint32_t *flag, cudaStream_t s) {
  switch (p->kkind) {
    case LOWBITS: return launch_k1r<LOWBITS>(p, g, C, keys, ids, n, HC, flag, s);
    case SHIFTC: return launch_k1r<SHIFTC>(p, g, C, keys, ids, n, HC, flag, s);
    case SHIFT: return launch_k1r<SHIFT>(p, g, C, keys, ids, n, HC, flag, s);
    case SHIFTC_LO: return launch_k1r<SHIFTC_LO>(p, g, C, keys, ids, n, HC, flag, s);
    case DELTA_LO: return launch_k1r<DELTA_LO>(p, g, C, keys, ids, n, HC, flag, s);
    case DELTA: return launch_k1r<DELTA>(p, g, C, keys, ids, n, HC, flag, s);
    case SPLITTERS: return launch_k1r<SPLITTERS>(p, g, C, keys, ids, n, HC, flag, s);
    default: return launch_k1r<IDS>(p, g, C, keys, ids, n, HC, flag, s);
  }
}

// The variant a run of L tiles uses (measured on B200 with tools/variant_sweep.py,
// profiles/r02_variants.md).  m > 32 and the Direct ablation: tile.  Forced by a MS_VARIANT_* plan
// flag: that one.  Key-only: ONE (m32 KO at 2^27: 407 vs 400 ranged vs 390 tile).  Key-value: the
// CTA-range variant once the input spans enough tiles per SM -- >= 8 for m <= 8 (m2 KV at 2^25:
// 294 vs 283 ONE), >= 16 for m <= 16 and precomputed ids (IDS m=32 KV at 2^25: 236 vs 224),
// > 64 above (C3 at 2^27: 234 vs 232 ONE vs 224 tile; at 2^25 ONE 212 vs 205) -- ONE below.
int choose_variant(const ms_plan_s *p, uint64_t L, bool kv) {
  if (p->direct || p->k3w) return V_TILE;
  if (p->spec.m > 32) {  // key-only 33..64 buckets (computed or u8 ids): ONE with 8192-key tiles (§7)
    const bool one = p->spec.m <= 64 && !kv && (p->kkind != IDS || p->spec.id_bytes == 1);
    return one && p->forced != V_TILE ? V_ONE : V_TILE;
  }
  if (p->forced >= 0) return p->forced;
  if (!kv) return V_ONE;
  const uint64_t per_sm = p->spec.m <= 8 ? 8 : (p->spec.m <= 16 || p->kkind == IDS) ? 16 : 65;
  return L >= per_sm * (uint64_t)p->sms ? V_RANGED : V_ONE;
}

ms_status check_ws(const ms_plan_s *p, uint64_t n, void *ws, size_t ws_bytes, Geometry *g) {
  *g = geometry(p, n);
  if (p->wide) return MS_ERR_UNSUPPORTED;  // the stage-wise calls: plans of m <= 256 only
  if (!ws || ws_bytes < g->bytes) return MS_ERR_WORKSPACE;
  if (misaligned(ws)) return MS_ERR_ALIGNMENT;
  return MS_OK;
}

ms_status check_common(const ms_plan_s *p, const uint32_t *keys_in, const void *ids, uint64_t n) {
  if (!p) return MS_ERR_INVALID_ARG;
  if (n > p->max_n || n >= (1ull << 32)) return MS_ERR_INVALID_ARG;
  if (n > 0 && !keys_in) return MS_ERR_INVALID_ARG;
  if (n > 0 && p->spec.kind == MS_IDS && !ids) return MS_ERR_INVALID_ARG;
  if (misaligned(keys_in) || misaligned(ids)) return MS_ERR_ALIGNMENT;
  return MS_OK;
}

}  // namespace

extern "C" ms_status ms_plan_create(ms_plan_t *plan, const ms_bucket_spec *spec, uint64_t max_n, int with_values,
                                    uint32_t flags, int device);
extern "C" ms_status ms_plan_destroy(ms_plan_t plan);

namespace {

constexpr uint32_t kMaxWideM = 65536;

// m in (256, 65536]: a plan of two passes.  The id has e <= 16 significant bits;
// pass A splits by its low bA = ceil(e/2) bits, pass B by the high e - bA bits (both <= 256
// buckets, so each pass is an ordinary plan: <= 32 buckets take K3 v2, 33..256 the ballot K3).
//   LOWBITS(s), and DELTA with delta = 2^s and m * delta >= 2^32 (id = k >> s):
//        A = LOWBITS(s, 2^bA), B = LOWBITS(s + bA, 2^(e - bA));
//   DELTA with delta = 2^s, m * delta < 2^32 (id = min(k >> s, m-1)):
//        A = SHIFTC_LO (min(k >> s, m-1) & (2^bA - 1)), B = DELTA(delta * 2^bA, ((m-1) >> bA) + 1)
//        since floor(min(q, m-1) / 2^bA) = min(floor(q / 2^bA), (m-1) >> bA);
//   DELTA otherwise: A = DELTA_LO (the same with floor(k / delta)), B = DELTA(delta * 2^bA, ...)
//        (floor(floor(k/delta) / 2^bA) = floor(k / (delta * 2^bA)));
//   MS_IDS (u32 ids): the ids ride as the KEYS of two key-value passes, A = LOWBITS(0, 2^bA),
//        B = LOWBITS(bA, 2^(e - bA)), the caller's keys (and values) as the payload.
// B is omitted when the high digit is 0 for every key (delta * 2^bA >= 2^32).  MS_SPLITTERS
// (more than 255 splitters) and the variant / ablation flags are not supported here.
ms_status create_wide(ms_plan_t *plan, const ms_bucket_spec *spec, uint64_t max_n, int with_values, uint32_t flags,
                      int device) {
  const uint32_t m = spec->m;
  if (flags & ~MS_VALIDATE) return MS_ERR_UNSUPPORTED;
  uint32_t e = ceil_log2(m), s = 0;
  int how = 0;  // 0 bit field, 1 SHIFTC_LO, 2 DELTA_LO, 3 ids
  switch (spec->kind) {
    case MS_LOWBITS:
      if (m & (m - 1)) return MS_ERR_INVALID_ARG;
      if (spec->shift > 31 || spec->shift + e > 32) return MS_ERR_INVALID_ARG;
      s = spec->shift;
      break;
    case MS_DELTA:
      if (spec->delta < 1) return MS_ERR_INVALID_ARG;
      if ((spec->delta & (spec->delta - 1)) == 0) {
        s = ceil_log2(spec->delta);
        if (((uint64_t)m << s) >= (1ull << 32)) e = 32 - s;  // id = k >> s < 2^(32-s) <= m: a bit field
        else how = 1;
      } else {
        how = 2;
      }
      break;
    case MS_IDS:
      if (spec->id_bytes != 4) return spec->id_bytes == 1 ? MS_ERR_UNSUPPORTED : MS_ERR_INVALID_ARG;
      how = 3;
      break;
    case MS_SPLITTERS: return MS_ERR_UNSUPPORTED;
    default: return MS_ERR_INVALID_ARG;
  }
  const uint32_t bA = e > 8 ? (e + 1) / 2 : e, bB = e - bA;
  const int kvsub = how == 3 ? 1 : with_values;
  ms_plan_s *a = nullptr, *b = nullptr;
  ms_bucket_spec sa{}, sb{};
  ms_status st;
  if (how == 0 || how == 3) {
    sa.kind = MS_LOWBITS;
    sa.m = 1u << bA;
    sa.shift = s;
    sb.kind = MS_LOWBITS;
    sb.m = 1u << bB;
    sb.shift = s + bA;
  } else {
    sa.kind = MS_DELTA;
    sa.m = 1u << bA;
    sa.delta = spec->delta;
    const uint64_t db = (uint64_t)spec->delta << bA;
    sb.kind = MS_DELTA;
    sb.m = db < (1ull << 32) ? ((m - 1) >> bA) + 1 : 1u;
    sb.delta = db < (1ull << 32) ? (uint32_t)db : 1u;
  }
  if ((st = ms_plan_create(&a, &sa, max_n, kvsub, 0, device)) != MS_OK) return st;
  if (how == 1 || how == 2) {  // pass A: the low digit of the CLAMPED id
    a->kkind = how == 1 ? SHIFTC_LO : DELTA_LO;
    a->bp.shift = s;
    a->bp.clamp = m - 1;
    a->bp.mmask = (1u << bA) - 1;
  }
  if (sb.m > 1 && (st = ms_plan_create(&b, &sb, max_n, kvsub, 0, device)) != MS_OK) {
    ms_plan_destroy(a);
    return st;
  }
  ms_plan_s *p = new (std::nothrow) ms_plan_s;
  if (!p) {
    ms_plan_destroy(a);
    ms_plan_destroy(b);
    return MS_ERR_INVALID_ARG;
  }
  p->spec = *spec;
  p->spec.splitters = nullptr;
  p->max_n = max_n;
  p->kv = with_values ? 1 : 0;
  p->flags = flags;
  memset(&p->bp, 0, sizeof(p->bp));
  p->bp.m = m;
  p->bp.mmask = m - 1;
  p->bp.logm = e;
  p->bp.validate = (flags & MS_VALIDATE) ? 1u : 0u;
  p->kkind = spec->kind == MS_IDS ? IDS : spec->kind == MS_LOWBITS ? LOWBITS : DELTA;
  p->device = a->device;
  p->sms = a->sms;
  p->last_launches = 0;
  p->wide = how == 3 ? 2 : 1;
  p->wa = a;
  p->wb = b;
  // the full id for the offsets pass: a bit field, min(k >> s, m-1), min(k / delta, m-1), or
  // min(id, m-1) over the sorted ids
  memset(&p->wbp, 0, sizeof(p->wbp));
  p->wbp.m = m;
  if (how == 0) {
    p->wkind = LOWBITS;
    p->wbp.shift = s;
    p->wbp.mmask = e >= 32 ? 0xFFFFFFFFu : (1u << e) - 1;
  } else if (how == 1 || how == 3) {
    p->wkind = SHIFTC;
    p->wbp.shift = s;
    p->wbp.mmask = m - 1;
  } else {
    p->wkind = DELTA;
    p->wbp.magic_lo = a->bp.magic_lo;
    p->wbp.magic_hi = a->bp.magic_hi;
    p->wbp.mmask = m - 1;
  }
  *plan = p;
  return MS_OK;
}

// workspace of a wide run: [the larger pass workspace | temporaries]
struct WideWs {
  size_t sub, off_tk, off_tv, off_ti, off_si, bytes;
};
WideWs wide_ws(const ms_plan_s *p, uint64_t n) {
  WideWs w{};
  w.sub = geometry(p->wa, n).bytes;
  if (p->wb) w.sub = std::max(w.sub, geometry(p->wb, n).bytes);
  w.sub = align_up(w.sub);
  const size_t arr = align_up(n * 4);
  w.off_tk = w.sub;
  w.off_tv = w.off_tk + arr;
  w.off_ti = w.off_tv + (p->kv ? arr : 0);
  w.off_si = w.off_ti + (p->wide == 2 ? arr : 0);
  w.bytes = w.off_si + (p->wide == 2 ? arr : 0);
  return w;
}

size_t plan_ws_bytes(const ms_plan_s *p, uint64_t n) { return p->wide ? wide_ws(p, n).bytes : geometry(p, n).bytes; }

}  // namespace

extern "C" ms_status ms_run(ms_plan_t p, const uint32_t *keys_in, const uint32_t *vals_in, const void *ids,
                            uint32_t *keys_out, uint32_t *vals_out, uint64_t n, uint32_t *offsets, void *ws,
                            size_t ws_bytes, void *stream);

namespace {

// ms_run of a wide plan (arguments already checked by ms_run): pass A into temporaries of the
// workspace, pass B into the outputs, then the offsets from the sorted output.
ms_status run_wide(ms_plan_s *p, const uint32_t *keys_in, const uint32_t *vals_in, const void *ids,
                   uint32_t *keys_out, uint32_t *vals_out, uint64_t n, uint32_t *offsets, void *ws, size_t ws_bytes,
                   void *stream) {
  const WideWs L = wide_ws(p, n);
  if (!ws || ws_bytes < L.bytes) return MS_ERR_WORKSPACE;
  if (misaligned(ws)) return MS_ERR_ALIGNMENT;
  DeviceGuard dg(p->device);
  cudaStream_t s = (cudaStream_t)stream;
  p->last_launches = 0;
  if (n == 0) {
    if (offsets && cudaMemsetAsync(offsets, 0, ((size_t)p->spec.m + 1) * 4, s) != cudaSuccess) return MS_ERR_CUDA;
    return MS_OK;
  }
  char *w = (char *)ws;
  uint32_t *tk = (uint32_t *)(w + L.off_tk), *tv = p->kv ? (uint32_t *)(w + L.off_tv) : nullptr;
  uint32_t *ti = (uint32_t *)(w + L.off_ti), *si = (uint32_t *)(w + L.off_si);
  cudaEvent_t *ev = trace_next(p);
  if (ev) cudaEventRecord(ev[0], s);
  int32_t launches = 0;
  ms_status st = MS_OK;
  auto run = [&](ms_plan_s *q, const uint32_t *k, const uint32_t *v, uint32_t *ko, uint32_t *vo) {
    if (st != MS_OK) return;
    st = ms_run(q, k, v, nullptr, ko, vo, n, nullptr, ws, L.sub, stream);
    launches += q->last_launches;
  };
  const uint32_t *sorted;  // the id-sorted array the offsets are read from
  if (p->wide == 1) {      // computed ids: recomputed from the keys by both passes
    if (p->wb) {
      run(p->wa, keys_in, vals_in, tk, tv);
      if (ev) cudaEventRecord(ev[1], s);
      run(p->wb, tk, tv, keys_out, vals_out);
    } else {
      run(p->wa, keys_in, vals_in, keys_out, vals_out);
      if (ev) cudaEventRecord(ev[1], s);
    }
    sorted = keys_out;
  } else {  // MS_IDS: the ids are the keys of both passes, the caller's keys (values) the payload
    const uint32_t *id32 = (const uint32_t *)ids;
    if (p->flags & MS_VALIDATE) {
      if (cudaMemsetAsync(ws, 0, 4, s) != cudaSuccess ||
          ids_check_launch(id32, n, p->spec.m, (uint32_t *)ws, p->sms, s) != cudaSuccess)
        return MS_ERR_CUDA;
      ++launches;
    }
    // (e >= 9 id bits for m > 256, so both digits are non-empty: wb exists)
    run(p->wa, id32, keys_in, ti, tk);
    if (vals_in) run(p->wa, id32, vals_in, si, tv);  // the same stable permutation (same ids)
    if (ev) cudaEventRecord(ev[1], s);
    run(p->wb, ti, tk, si, keys_out);
    if (vals_in) run(p->wb, ti, tv, tk, vals_out);
    sorted = si;
  }
  if (st != MS_OK) return st;
  if (ev) cudaEventRecord(ev[2], s);
  if (offsets) {
    if (wide_offsets_launch(p->wkind, sorted, n, offsets, p->wbp, p->sms, s) != cudaSuccess) return MS_ERR_CUDA;
    ++launches;
  }
  if (ev) cudaEventRecord(ev[3], s);
  p->last_launches = launches;
  return MS_OK;
}

}  // namespace

// ====================================================================== C ABI
extern "C" {

const char *ms_status_string(ms_status s) {
  switch (s) {
    case MS_OK: return "ok";
    case MS_ERR_INVALID_ARG: return "invalid argument";
    case MS_ERR_UNSUPPORTED: return "unsupported";
    case MS_ERR_ALIGNMENT: return "pointer not 16-byte aligned";
    case MS_ERR_ALIAS: return "output overlaps input";
    case MS_ERR_WORKSPACE: return "workspace missing or too small";
    case MS_ERR_CUDA: return "CUDA error";
    case MS_ERR_NCCL: return "NCCL error";
    case MS_ERR_BUCKET_RANGE: return "bucket id >= m";
    default: return "unknown status";
  }
}

ms_status ms_plan_create(ms_plan_t *plan, const ms_bucket_spec *spec, uint64_t max_n,
                         int with_values, uint32_t flags, int device) {
  if (!plan || !spec) return MS_ERR_INVALID_ARG;
  *plan = nullptr;
  const uint32_t m = spec->m;
  if (m < 1 || m > kMaxWideM) return MS_ERR_INVALID_ARG;
  if (max_n >= (1ull << 32)) return MS_ERR_INVALID_ARG;
  if (m > (uint32_t)kMaxM) return create_wide(plan, spec, max_n, with_values, flags, device);
  constexpr uint32_t kVariants = MS_VARIANT_3K | MS_VARIANT_RANGED | MS_VARIANT_ONE;
  constexpr uint32_t kAblations =
      MS_ABLATION_DIRECT | MS_ABLATION_NW2 | MS_ABLATION_NW4 | MS_ABLATION_BALLOT | MS_ABLATION_WARP;
  if (flags & ~(MS_VALIDATE | kVariants | kAblations)) return MS_ERR_INVALID_ARG;
  const uint32_t vf = flags & kVariants, af = flags & kAblations;
  if (vf & (vf - 1)) return MS_ERR_INVALID_ARG;  // at most one variant flag
  if (af & (af - 1)) return MS_ERR_INVALID_ARG;  // at most one ablation
  if (af && vf) return MS_ERR_INVALID_ARG;
  if ((flags & MS_VARIANT_RANGED) && m > 32) return MS_ERR_UNSUPPORTED;
  // ONE above 32 buckets: key-only, m <= 64, computed or u8 ids
  if ((flags & MS_VARIANT_ONE) && m > 32 &&
      (m > 64 || with_values || (spec->kind == MS_IDS && spec->id_bytes != 1)))
    return MS_ERR_UNSUPPORTED;
  BucketParams bp;
  memset(&bp, 0, sizeof(bp));
  int kkind = spec->kind;
  bp.m = m;
  bp.mmask = m - 1;
  bp.logm = ceil_log2(m);
  bp.validate = (flags & MS_VALIDATE) ? 1u : 0u;
  switch (spec->kind) {
    case MS_LOWBITS:
      if (m & (m - 1)) return MS_ERR_INVALID_ARG;  // reading #10
      if (spec->shift > 31 || spec->shift + bp.logm > 32) return MS_ERR_INVALID_ARG;
      bp.shift = spec->shift;
      break;
    case MS_DELTA:
      if (spec->delta < 1) return MS_ERR_INVALID_ARG;
      if ((spec->delta & (spec->delta - 1)) == 0) {  // power of two (incl. 1): a shift
        bp.shift = ceil_log2(spec->delta);
        // m * delta >= 2^32: k >> shift < m for every key, the clamp is dead
        kkind = ((uint64_t)m << bp.shift) >= (1ull << 32) ? SHIFT : SHIFTC;
      } else {
        kkind = DELTA;
        const uint64_t c = delta_magic(spec->delta);
        bp.magic_lo = (uint32_t)c;
        bp.magic_hi = (uint32_t)(c >> 32);
      }
      break;
    case MS_SPLITTERS: {
      if (m > 1 && !spec->splitters) return MS_ERR_INVALID_ARG;
      for (uint32_t j = 0; j < (1u << bp.logm); ++j) bp.spl[j] = 0xFFFFFFFFu;
      for (uint32_t j = 0; j + 1 < m; ++j) {
        if (j > 0 && spec->splitters[j] < spec->splitters[j - 1]) return MS_ERR_INVALID_ARG;
        bp.spl[j] = spec->splitters[j];
      }
      break;
    }
    case MS_IDS:
      if (spec->id_bytes != 1 && spec->id_bytes != 4) return MS_ERR_INVALID_ARG;
      bp.id_bytes = spec->id_bytes;
      break;
    default: return MS_ERR_INVALID_ARG;
  }
  // the ablations are instantiated for one bucket kind only (DELTA with m * delta = 2^32); the
  // ballot-K3 ablations for 2 <= m <= 256, the others for m <= 32
  const bool any_m = (af & (MS_ABLATION_BALLOT | MS_ABLATION_WARP)) != 0;
  if (af && (kkind != SHIFT || (any_m ? m < 2 : m > 32))) return MS_ERR_UNSUPPORTED;
  if (device < -1) return MS_ERR_INVALID_ARG;
  if (device == -1 && cudaGetDevice(&device) != cudaSuccess) {
    cudaGetLastError();
    device = 0;  // no usable device yet (host-only use of the plan): ordinal 0
  }
  int sms = 0;
  if (cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, device) != cudaSuccess || sms <= 0) {
    cudaGetLastError();
    sms = 148;  // B200
  }
  ms_plan_s *p = new (std::nothrow) ms_plan_s;
  if (!p) return MS_ERR_INVALID_ARG;
  p->spec = *spec;
  p->spec.splitters = nullptr;  // copied into bp.spl
  p->max_n = max_n;
  p->kv = with_values ? 1 : 0;
  p->flags = flags;
  p->bp = bp;
  p->kkind = kkind;
  p->device = device;
  p->sms = sms;
  p->last_launches = 0;
  p->forced = (flags & MS_VARIANT_3K) ? V_TILE : (flags & MS_VARIANT_RANGED) ? V_RANGED
            : (flags & MS_VARIANT_ONE) ? V_ONE : -1;
  p->direct = (flags & MS_ABLATION_DIRECT) ? 1 : 0;
  p->k3w = (flags & MS_ABLATION_BALLOT) ? 1 : (flags & MS_ABLATION_WARP) ? 2 : 0;
  if (flags & (MS_ABLATION_NW2 | MS_ABLATION_NW4)) {  // 2 / 4 warps per K3 CTA: T = 1024 / 2048, ranged
    p->k3nt = (flags & MS_ABLATION_NW2) ? 64u : 128u;
    p->forced = V_RANGED;
  }
  *plan = p;
  return MS_OK;
}

ms_status ms_plan_destroy(ms_plan_t plan) {
  if (plan) {
    for (cudaEvent_t e : plan->trace_ev) cudaEventDestroy(e);
    ms_plan_destroy(plan->wa);
    ms_plan_destroy(plan->wb);
  }
  delete plan;
  return MS_OK;
}

ms_status ms_plan_workspace_size(ms_plan_t p, uint64_t n, size_t *bytes) {
  if (!p || !bytes || n > p->max_n) return MS_ERR_INVALID_ARG;
  *bytes = plan_ws_bytes(p, n);
  return MS_OK;
}

ms_status ms_plan_geometry(ms_plan_t p, uint64_t n, uint32_t *tile, uint64_t *num_tiles,
                           int32_t *variant) {
  if (!p || n > p->max_n) return MS_ERR_INVALID_ARG;
  if (p->wide) {  // the first pass's tiles; variant 3 = two passes
    Geometry g = geometry(p->wa, n);
    if (tile) *tile = g.T;
    if (num_tiles) *num_tiles = g.L;
    if (variant) *variant = 3;
    return MS_OK;
  }
  Geometry g = geometry(p, n);
  if (tile) *tile = g.T;
  if (num_tiles) *num_tiles = g.L;
  if (variant) *variant = choose_variant(p, g.L, p->kv != 0);
  return MS_OK;
}

int32_t ms_plan_last_launches(ms_plan_t p) { return p ? p->last_launches : -1; }

ms_status ms_plan_spec(ms_plan_t p, ms_bucket_spec *spec, int32_t *with_values) {
  if (!p) return MS_ERR_INVALID_ARG;
  if (spec) *spec = p->spec;  // splitters: NULL (the plan keeps its own copy)
  if (with_values) *with_values = p->kv;
  return MS_OK;
}

ms_status ms_plan_trace(ms_plan_t p, int enable) {
  if (!p) return MS_ERR_INVALID_ARG;
  if (enable) p->trace_runs = 0;
  p->tracing = enable == 2 ? 2 : (enable ? 1 : 0);
  if (enable) p->trace_mode = p->tracing;
  return MS_OK;
}

ms_status ms_plan_trace_read(ms_plan_t p, float *stage_ms, int32_t max_runs, int32_t *runs, int32_t *stages) {
  if (!p || (!stage_ms && max_runs > 0)) return MS_ERR_INVALID_ARG;
  int32_t r = (int32_t)std::min<size_t>(p->trace_runs, (size_t)std::max(max_runs, 0));
  for (int32_t i = 0; i < r; ++i) {
    cudaEvent_t *ev = &p->trace_ev[4 * i];
    if (cudaEventSynchronize(ev[3]) != cudaSuccess) return MS_ERR_CUDA;
    for (int s = 0; s < 3; ++s) {
      stage_ms[4 * i + s] = 0.f;  // whole-run mode (2): no per-stage events
      if (p->trace_mode != 2 && cudaEventElapsedTime(&stage_ms[4 * i + s], ev[s], ev[s + 1]) != cudaSuccess)
        return MS_ERR_CUDA;
    }
    if (cudaEventElapsedTime(&stage_ms[4 * i + 3], ev[0], ev[3]) != cudaSuccess) return MS_ERR_CUDA;
  }
  if (runs) *runs = r;
  if (stages) *stages = 3;
  return MS_OK;
}

ms_status ms_prescan(ms_plan_t p, const uint32_t *keys_in, const void *ids, uint64_t n,
                     uint32_t *H, void *ws, size_t ws_bytes, void *stream) {
  ms_status st = check_common(p, keys_in, ids, n);
  if (st != MS_OK) return st;
  if (!H && n > 0) return MS_ERR_INVALID_ARG;
  if (misaligned(H)) return MS_ERR_ALIGNMENT;
  Geometry g;
  if ((st = check_ws(p, n, ws, ws_bytes, &g)) != MS_OK) return st;
  if (n == 0) return MS_OK;
  DeviceGuard dg(p->device);
  char *w = (char *)ws;
  cudaError_t e = dispatch_k1(p, g, keys_in, ids, (uint32_t)n, H, nullptr, 0,
                              (uint32_t *)(w + g.off_flag), (cudaStream_t)stream);
  return e == cudaSuccess ? MS_OK : MS_ERR_CUDA;
}

ms_status ms_scan(ms_plan_t p, uint32_t *HG, uint64_t n, uint32_t *offsets, void *ws,
                  size_t ws_bytes, void *stream) {
  if (!p || n > p->max_n) return MS_ERR_INVALID_ARG;
  if (misaligned(HG) || misaligned(offsets)) return MS_ERR_ALIGNMENT;
  Geometry g;
  ms_status st = check_ws(p, n, ws, ws_bytes, &g);
  if (st != MS_OK) return st;
  if (n > 0 && !HG) return MS_ERR_INVALID_ARG;
  DeviceGuard dg(p->device);
  cudaStream_t s = (cudaStream_t)stream;
  if (n == 0) {
    if (offsets && cudaMemsetAsync(offsets, 0, (p->spec.m + 1) * 4, s) != cudaSuccess) return MS_ERR_CUDA;
    return MS_OK;
  }
  char *w = (char *)ws;
  uint64_t *status = (uint64_t *)(w + g.off_status);
  if (cudaMemsetAsync(status, 0, g.chunks * 8, s) != cudaSuccess) return MS_ERR_CUDA;
  k2_scan<<<(unsigned)g.chunks, kThreads, 0, s>>>(HG, g.hg_words, status, offsets, (uint32_t)g.L,
                                                 p->spec.m, (uint32_t)n);
  return cudaGetLastError() == cudaSuccess ? MS_OK : MS_ERR_CUDA;
}

ms_status ms_postscan(ms_plan_t p, const uint32_t *keys_in, const uint32_t *vals_in,
                      const void *ids, const uint32_t *G, uint32_t *keys_out, uint32_t *vals_out,
                      uint64_t n, void *ws, size_t ws_bytes, void *stream) {
  ms_status st = check_common(p, keys_in, ids, n);
  if (st != MS_OK) return st;
  if ((vals_in == nullptr) != (vals_out == nullptr)) return MS_ERR_INVALID_ARG;
  if (vals_in && !p->kv) return MS_ERR_UNSUPPORTED;
  if (n > 0 && (!G || !keys_out)) return MS_ERR_INVALID_ARG;
  if (misaligned(vals_in) || misaligned(G) || misaligned(keys_out) || misaligned(vals_out))
    return MS_ERR_ALIGNMENT;
  Geometry g;
  if ((st = check_ws(p, n, ws, ws_bytes, &g)) != MS_OK) return st;
  if (n == 0) return MS_OK;
  DeviceGuard dg(p->device);
  cudaError_t e = dispatch_k3(p, g, keys_in, vals_in, ids, G, keys_out, vals_out, (uint32_t)n,
                              (uint32_t *)((char *)ws + g.off_flag), (cudaStream_t)stream);
  return e == cudaSuccess ? MS_OK : MS_ERR_CUDA;
}

ms_status ms_postscan_scatter(ms_plan_t p, const uint32_t *keys_in, const uint32_t *vals_in, const uint32_t *G,
                              uint64_t n, const ms_scatter_target *t, void *ws, size_t ws_bytes, void *stream) {
  if (!p) return MS_ERR_INVALID_ARG;
  if (p->spec.m > 32 || p->kkind == IDS || p->direct || p->k3w) return MS_ERR_UNSUPPORTED;
  ms_status st = check_common(p, keys_in, nullptr, n);
  if (st != MS_OK) return st;
  if (!t || t->nranks < 1 || t->nranks > MS_MAX_PEERS) return MS_ERR_INVALID_ARG;
  if (vals_in && !p->kv) return MS_ERR_UNSUPPORTED;
  if (misaligned(vals_in) || misaligned(G)) return MS_ERR_ALIGNMENT;
  for (int32_t r = 0; r < t->nranks; ++r) {
    if (t->win_start[r + 1] < t->win_start[r]) return MS_ERR_INVALID_ARG;
    const bool empty = t->win_start[r + 1] == t->win_start[r];
    if (!empty && (!t->keys_dst[r] || (vals_in && !t->vals_dst[r]))) return MS_ERR_INVALID_ARG;
    if (misaligned(t->keys_dst[r]) || misaligned(t->vals_dst[r])) return MS_ERR_ALIGNMENT;
  }
  Geometry g;
  if ((st = check_ws(p, n, ws, ws_bytes, &g)) != MS_OK) return st;
  if (n == 0) return MS_OK;
  if (!G) return MS_ERR_INVALID_ARG;
  DeviceGuard dg(p->device);
  DistTarget d{};
  d.P = t->nranks;
  for (int32_t r = 0; r < t->nranks; ++r) {
    d.keys[r] = t->keys_dst[r];
    d.vals[r] = t->vals_dst[r];
  }
  for (int32_t r = 0; r <= t->nranks; ++r) d.wst[r] = t->win_start[r];
  for (uint32_t b = 0; b < p->spec.m; ++b) d.delta[b] = t->delta[b];
  K3pArgs a{keys_in, vals_in, nullptr, G, nullptr, nullptr, (uint32_t)n, (uint32_t)g.L, p->spec.m,
            p->spec.id_bytes, p->kpt, p->k3nt, &p->bp, p->sms, (cudaStream_t)stream};
  a.ds = &d;
  a.flag = (uint32_t *)((char *)ws + g.off_flag);  // a run past win_start[P] sets bit 1 (ms_plan_check)
  cudaError_t e;
  switch (p->kkind) {
    case LOWBITS: e = k3v_launch_lowbits(a); break;
    case SHIFTC: e = k3v_launch_shiftc(a); break;
    case SHIFT: e = k3v_launch_shift(a); break;
    case DELTA: e = k3v_launch_delta(a); break;
    default: e = k3v_launch_splitters(a); break;
  }
  return e == cudaSuccess ? MS_OK : MS_ERR_CUDA;
}

ms_status ms_run(ms_plan_t p, const uint32_t *keys_in, const uint32_t *vals_in, const void *ids,
                 uint32_t *keys_out, uint32_t *vals_out, uint64_t n, uint32_t *offsets, void *ws,
                 size_t ws_bytes, void *stream) {
  ms_status st = check_common(p, keys_in, ids, n);
  if (st != MS_OK) return st;
  if ((vals_in == nullptr) != (vals_out == nullptr)) return MS_ERR_INVALID_ARG;
  if (vals_in && !p->kv) return MS_ERR_UNSUPPORTED;
  if (n > 0 && !keys_out) return MS_ERR_INVALID_ARG;
  if (misaligned(vals_in) || misaligned(keys_out) || misaligned(vals_out) || misaligned(offsets))
    return MS_ERR_ALIGNMENT;
  const size_t nb = n * 4;
  if (overlap(keys_out, nb, keys_in, nb) || overlap(keys_out, nb, vals_in, nb) ||
      overlap(vals_out, nb, keys_in, nb) || overlap(vals_out, nb, vals_in, nb) ||
      overlap(keys_out, nb, vals_out, nb) ||
      overlap(keys_out, nb, ids, n * p->spec.id_bytes) || overlap(vals_out, nb, ids, n * p->spec.id_bytes))
    return MS_ERR_ALIAS;
  if (p->wide) return run_wide(p, keys_in, vals_in, ids, keys_out, vals_out, n, offsets, ws, ws_bytes, stream);
  Geometry g;
  if ((st = check_ws(p, n, ws, ws_bytes, &g)) != MS_OK) return st;
  DeviceGuard dg(p->device);
  cudaStream_t s = (cudaStream_t)stream;
  p->last_launches = 0;
  if (n == 0) {
    if (offsets && cudaMemsetAsync(offsets, 0, (p->spec.m + 1) * 4, s) != cudaSuccess) return MS_ERR_CUDA;
    return MS_OK;
  }
  char *w = (char *)ws;
  uint32_t *HG = (uint32_t *)(w + g.off_hg);
  uint64_t *status = (uint64_t *)(w + g.off_status);
  uint32_t *flag = (uint32_t *)(w + g.off_flag);
  uint32_t *HC = (uint32_t *)(w + g.off_hc);
  if ((p->flags & MS_VALIDATE) && p->spec.kind == MS_IDS &&
      cudaMemsetAsync(flag, 0, 4, s) != cudaSuccess)
    return MS_ERR_CUDA;
  cudaEvent_t *ev = trace_next(p);
  if (ev) cudaEventRecord(ev[0], s);
  // K2 and K3 use programmatic dependent launch unless per-stage events sit
  // between the kernels (tracing == 1)
  const bool pdl = p->tracing != 1;
  int variant = choose_variant(p, g.L, vals_in != nullptr);
  if (variant == V_ONE) {  // ONE cooperative launch: counts, grid barrier, range scan, post-scan
    const RangeScan rs{HC, offsets, 0, 1};
    if (ev && p->tracing == 1) {
      cudaEventRecord(ev[1], s);
      cudaEventRecord(ev[2], s);
    }
    // key-only (computed or u8 ids): tiles of 8192 keys, 32 per thread (half the
    // counter-matrix work per key, phase 1 double-buffered; NSko 440 -> 507, m16 500 -> 526, C2
    // 420 -> 440 G keys/s)
    const bool k32 = vals_in == nullptr && p->spec.m >= MS_K32_MINM &&
                     (p->kkind != IDS || p->spec.id_bytes == 1) && p->k3nt == 256 && !p->direct;
    const cudaError_t e1 = dispatch_k3(p, k32 ? geometry(p, n, 32) : g, keys_in, vals_in, ids, nullptr, keys_out,
                                       vals_out, (uint32_t)n, flag, s, 2, nullptr, 0, &rs);
    if (e1 == cudaSuccess) {
      if (ev) cudaEventRecord(ev[3], s);
      p->last_launches = 1;
      return MS_OK;
    }
    // the grid could not be made co-resident (e.g. the GPU is partitioned / shared): unless ONE
    // was forced, clear the launch error and take the two-launch ranged variant (same result)
    if (e1 != cudaErrorCooperativeLaunchTooLarge || p->forced == V_ONE) return MS_ERR_CUDA;
    cudaGetLastError();
    variant = p->spec.m > 32 ? V_TILE : V_RANGED;
  }
  if (variant == V_RANGED) {  // K1r -> K3 over C contiguous tile ranges (ms_ranged.cuh); the range
                              // scan runs in K3's prologue
    uint32_t C = 0;
    if (dispatch_k3(p, g, keys_in, vals_in, ids, nullptr, keys_out, vals_out, (uint32_t)n, flag, s, 1, &C) !=
            cudaSuccess ||
        C == 0)
      return MS_ERR_CUDA;
    if (dispatch_k1r(p, g, C, keys_in, ids, (uint32_t)n, HC, flag, s) != cudaSuccess) return MS_ERR_CUDA;
    if (ev && p->tracing == 1) {
      cudaEventRecord(ev[1], s);
      cudaEventRecord(ev[2], s);
    }
    const uint32_t ksub = k1r_split(p, C);
    const RangeScan rs{HC, offsets, C * ksub, ksub};
    if (dispatch_k3(p, g, keys_in, vals_in, ids, nullptr, keys_out, vals_out, (uint32_t)n, flag, s, 1, nullptr, pdl,
                    &rs) != cudaSuccess)
      return MS_ERR_CUDA;
    if (ev) cudaEventRecord(ev[3], s);
    p->last_launches = 2;
    return MS_OK;
  }
  // m > 32: K2 row by row (k2w_rowscan, no look-back; term 1 of Eq. (2) folded into K3)
  const bool rowk2 = p->spec.m > 32;
  uint32_t *rowtot = (uint32_t *)(w + g.off_rowtot), *rowbase = rowtot + kMaxM, *ticket = rowbase + kMaxM;
  // K1 zeroes K2's look-back status words, or (row K2) its 8-byte ticket word
  cudaError_t e = dispatch_k1(p, g, keys_in, ids, (uint32_t)n, HG, rowk2 ? (uint64_t *)ticket : status,
                              rowk2 ? 1u : (uint32_t)g.chunks, flag, s);
  if (e != cudaSuccess) return MS_ERR_CUDA;
  if (ev && p->tracing == 1) cudaEventRecord(ev[1], s);
  if (rowk2) {
    if (launch_ex(pdl, k2w_rowscan, dim3(p->spec.m), dim3(kRowThreads), 0, s, HG, (uint32_t)g.L, p->spec.m,
                  (uint32_t)n, rowtot, rowbase, ticket, offsets) != cudaSuccess ||
        cudaGetLastError() != cudaSuccess)
      return MS_ERR_CUDA;
  } else if (launch_ex(pdl, k2_scan, dim3((unsigned)g.chunks), dim3(kThreads), 0, s, HG, (uint64_t)g.hg_words,
                       status, offsets, (uint32_t)g.L, p->spec.m, (uint32_t)n) != cudaSuccess ||
             cudaGetLastError() != cudaSuccess) {
    return MS_ERR_CUDA;
  }
  if (ev && p->tracing == 1) cudaEventRecord(ev[2], s);
  // K3 after the many-CTA K2 of the tile variant: PDL only for key-only runs
  // (measured: an early-resident key-value K3 -- 2 CTAs with
  // the whole register file per SM -- costs ~6 % at n = 2^28)
  e = dispatch_k3(p, g, keys_in, vals_in, ids, HG, keys_out, vals_out, (uint32_t)n, flag, s, 0, nullptr,
                  pdl && vals_in == nullptr, nullptr, rowk2 ? rowbase : nullptr);
  if (e != cudaSuccess) return MS_ERR_CUDA;
  if (ev) cudaEventRecord(ev[3], s);
  p->last_launches = 3;
  return MS_OK;
}

ms_status ms_plan_workspace_size_host(ms_plan_t p, uint64_t n, size_t *bytes) {
  if (!p || !bytes || n > p->max_n) return MS_ERR_INVALID_ARG;
  size_t ws = plan_ws_bytes(p, n);
  size_t arr = align_up(n * 4);
  size_t stage = arr * (p->kv ? 4 : 2) + (p->spec.kind == MS_IDS ? align_up(n * p->spec.id_bytes) : 0) +
                 align_up((p->spec.m + 1) * 4);
  *bytes = ws + stage;
  return MS_OK;
}

ms_status ms_run_host(ms_plan_t p, const uint32_t *keys_h, const uint32_t *vals_h, const void *ids_h,
                      uint32_t *keys_out_h, uint32_t *vals_out_h, uint64_t n, uint32_t *offsets_h,
                      void *ws, size_t ws_bytes, void *stream) {
  if (!p || n > p->max_n) return MS_ERR_INVALID_ARG;
  if ((vals_h == nullptr) != (vals_out_h == nullptr)) return MS_ERR_INVALID_ARG;
  if (vals_h && !p->kv) return MS_ERR_UNSUPPORTED;
  if (n > 0 && (!keys_out_h || !keys_h || (p->spec.kind == MS_IDS && !ids_h)))
    return MS_ERR_INVALID_ARG;
  size_t need = 0;
  ms_plan_workspace_size_host(p, n, &need);
  if (!ws || ws_bytes < need) return MS_ERR_WORKSPACE;
  if (misaligned(ws)) return MS_ERR_ALIGNMENT;
  DeviceGuard dg(p->device);
  cudaStream_t s = (cudaStream_t)stream;
  const size_t wsb = plan_ws_bytes(p, n);
  char *w = (char *)ws + wsb;
  size_t arr = align_up(n * 4);
  uint32_t *dk = (uint32_t *)w; w += arr;
  uint32_t *dko = (uint32_t *)w; w += arr;
  uint32_t *dv = nullptr, *dvo = nullptr;
  if (p->kv) { dv = (uint32_t *)w; w += arr; dvo = (uint32_t *)w; w += arr; }
  void *did = nullptr;
  if (p->spec.kind == MS_IDS) { did = w; w += align_up(n * p->spec.id_bytes); }
  uint32_t *doff = (uint32_t *)w;
  if (n > 0) {
    if (keys_h && cudaMemcpyAsync(dk, keys_h, n * 4, cudaMemcpyHostToDevice, s) != cudaSuccess) return MS_ERR_CUDA;
    if (vals_h && cudaMemcpyAsync(dv, vals_h, n * 4, cudaMemcpyHostToDevice, s) != cudaSuccess) return MS_ERR_CUDA;
    if (did && cudaMemcpyAsync(did, ids_h, n * p->spec.id_bytes, cudaMemcpyHostToDevice, s) != cudaSuccess)
      return MS_ERR_CUDA;
  }
  ms_status st = ms_run(p, keys_h ? dk : nullptr, vals_h ? dv : nullptr, did, dko, vals_h ? dvo : nullptr, n,
                        offsets_h ? doff : nullptr, ws, wsb, stream);
  if (st != MS_OK) return st;
  if (n > 0) {
    if (cudaMemcpyAsync(keys_out_h, dko, n * 4, cudaMemcpyDeviceToHost, s) != cudaSuccess) return MS_ERR_CUDA;
    if (vals_out_h && cudaMemcpyAsync(vals_out_h, dvo, n * 4, cudaMemcpyDeviceToHost, s) != cudaSuccess)
      return MS_ERR_CUDA;
  }
  if (offsets_h && cudaMemcpyAsync(offsets_h, doff, (p->spec.m + 1) * 4, cudaMemcpyDeviceToHost, s) != cudaSuccess)
    return MS_ERR_CUDA;
  return MS_OK;
}

ms_status ms_bucket_ids(ms_plan_t p, const uint32_t *keys_in, uint64_t n, uint32_t *out_ids, void *stream) {
  if (!p || !keys_in || !out_ids) return MS_ERR_INVALID_ARG;
  if (p->spec.kind == MS_IDS) return MS_ERR_UNSUPPORTED;
  if (misaligned(keys_in) || misaligned(out_ids)) return MS_ERR_ALIGNMENT;
  if (n == 0) return MS_OK;
  DeviceGuard dg(p->device);
  cudaStream_t s = (cudaStream_t)stream;
  unsigned grid = (unsigned)std::min<uint64_t>((n + kThreads - 1) / kThreads, 148ull * 16);
  switch (p->kkind) {
    case LOWBITS: k_bucket_ids<LOWBITS><<<grid, kThreads, 0, s>>>(keys_in, n, out_ids, p->bp); break;
    case SHIFTC: k_bucket_ids<SHIFTC><<<grid, kThreads, 0, s>>>(keys_in, n, out_ids, p->bp); break;
    case SHIFT: k_bucket_ids<SHIFT><<<grid, kThreads, 0, s>>>(keys_in, n, out_ids, p->bp); break;
    case DELTA: k_bucket_ids<DELTA><<<grid, kThreads, 0, s>>>(keys_in, n, out_ids, p->bp); break;
    default: k_bucket_ids<SPLITTERS><<<grid, kThreads, 0, s>>>(keys_in, n, out_ids, p->bp); break;
  }
  return cudaGetLastError() == cudaSuccess ? MS_OK : MS_ERR_CUDA;
}

ms_status ms_plan_check(ms_plan_t p, void *ws, void *stream) {
  if (!p || !ws) return MS_ERR_INVALID_ARG;
  DeviceGuard dg(p->device);
  cudaStream_t s = (cudaStream_t)stream;
  uint32_t host = 0;
  if (cudaMemcpyAsync(&host, ws, 4, cudaMemcpyDeviceToHost, s) != cudaSuccess) return MS_ERR_CUDA;
  if (cudaStreamSynchronize(s) != cudaSuccess) return MS_ERR_CUDA;
  if (host) {
    if (cudaMemsetAsync(ws, 0, 4, s) != cudaSuccess) return MS_ERR_CUDA;
    return (host & 2u) ? MS_ERR_INVALID_ARG : MS_ERR_BUCKET_RANGE;
  }
  return MS_OK;
}

}  // extern "C"
