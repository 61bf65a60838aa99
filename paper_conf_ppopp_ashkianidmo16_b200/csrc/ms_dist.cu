// ms_dist.cu -- host-side planning of the sharded multisplit (include/ms.h, ms_dist_pieces).
//
// Eq. (2) one level up: the P ranks are the outermost
// subproblems.  Pure host arithmetic on the all-gathered m x P count matrix;
// the data path is the local ms_run plus the exchange of the pieces computed here.
#include <cstdint>
#include <vector>

#include "../../include/ms.h"

namespace {

struct Windows {
  uint64_t q, rem;
  uint64_t start(int32_t r) const { return (uint64_t)r * q + (uint64_t)(r < (int64_t)rem ? r : rem); }
  // rank owning global position x (0 <= x < N)
  int32_t owner(uint64_t x) const {
    const uint64_t big = (q + 1) * rem;  // the first `rem` windows hold q+1 elements
    if (x < big) return (int32_t)(x / (q + 1));
    return (int32_t)(rem + (x - big) / (q ? q : 1));
  }
};

}  // namespace

extern "C" ms_status ms_dist_pieces(int32_t P, int32_t rank, uint32_t m, const uint64_t *counts,
                                    ms_piece *send, int32_t send_cap, int32_t *n_send, ms_piece *recv,
                                    int32_t recv_cap, int32_t *n_recv, uint64_t *offsets_global,
                                    uint64_t *win_start, uint64_t *win_len) {
  if (P < 1 || rank < 0 || rank >= P || m < 1 || !counts || !n_send || !n_recv) return MS_ERR_INVALID_ARG;
  // B[b] = sum_{b'<b} sum_g h[g][b'];  prefix[g][b] = sum_{g'<g} h[g'][b]
  std::vector<uint64_t> B(m + 1, 0), pref((size_t)P * m, 0);
  for (uint32_t b = 0; b < m; ++b) {
    uint64_t col = 0;
    for (int32_t g = 0; g < P; ++g) {
      pref[(size_t)g * m + b] = col;
      col += counts[(size_t)g * m + b];
    }
    B[b + 1] = B[b] + col;
  }
  const uint64_t N = B[m];
  if (offsets_global)
    for (uint32_t b = 0; b <= m; ++b) offsets_global[b] = B[b];
  const Windows W{N / (uint64_t)P, N % (uint64_t)P};
  if (win_start) *win_start = W.start(rank);
  if (win_len) *win_len = W.start(rank + 1) - W.start(rank);

  // sends: my local bucket b occupies local [off[b], off[b] + h[rank][b]) and
  // global [B[b] + pref[rank][b], ...); cut it at window boundaries
  int32_t ns = 0;
  uint64_t local_off = 0;
  for (uint32_t b = 0; b < m; ++b) {
    const uint64_t h = counts[(size_t)rank * m + b];
    uint64_t gs = B[b] + pref[(size_t)rank * m + b];
    const uint64_t ge = gs + h;
    uint64_t lo = local_off;
    while (gs < ge) {
      const int32_t r = W.owner(gs);
      const uint64_t wend = W.start(r + 1);
      const uint64_t e = ge < wend ? ge : wend;
      if (ns >= send_cap || !send) return MS_ERR_INVALID_ARG;
      send[ns++] = ms_piece{lo, e - gs, r, 0, gs - W.start(r)};
      lo += e - gs;
      gs = e;
    }
    local_off += h;
  }
  // receives: for every source rank s (ascending) and bucket b (ascending),
  // the part of s's bucket-b range that falls in my window, in the order s sends it
  int32_t nr = 0;
  const uint64_t ws = W.start(rank), we = W.start(rank + 1);
  for (int32_t s = 0; s < P; ++s) {
    uint64_t s_local = 0;
    for (uint32_t b = 0; b < m; ++b) {
      const uint64_t h = counts[(size_t)s * m + b];
      const uint64_t gs = B[b] + pref[(size_t)s * m + b], ge = gs + h;
      const uint64_t a = gs > ws ? gs : ws, e = ge < we ? ge : we;
      if (a < e) {
        if (nr >= recv_cap || !recv) return MS_ERR_INVALID_ARG;
        recv[nr++] = ms_piece{s_local + (a - gs), e - a, s, 0, a - ws};
      }
      s_local += h;
    }
  }
  *n_send = ns;
  *n_recv = nr;
  return MS_OK;
}

extern "C" ms_status ms_dist_targets(int32_t P, int32_t rank, uint32_t m, const uint64_t *counts, uint64_t *delta,
                                     uint64_t *win_start) {
  if (P < 1 || P > MS_MAX_PEERS || rank < 0 || rank >= P || m < 1 || !counts || !delta || !win_start)
    return MS_ERR_INVALID_ARG;
  // B[b] + sum_{g'<rank} h[g'][b] - off_rank[b], off_rank = exclusive scan of h[rank]
  uint64_t B = 0, off = 0;
  for (uint32_t b = 0; b < m; ++b) {
    uint64_t col = 0, pref = 0;
    for (int32_t g = 0; g < P; ++g) {
      if (g == rank) pref = col;
      col += counts[(size_t)g * m + b];
    }
    delta[b] = B + pref - off;  // >= 0: B >= off (all ranks' lower buckets include mine)
    B += col;
    off += counts[(size_t)rank * m + b];
  }
  const Windows W{B / (uint64_t)P, B % (uint64_t)P};
  for (int32_t r = 0; r <= P; ++r) win_start[r] = W.start(r);
  return MS_OK;
}

// =========================================================================
// ms_dist_run: the sharded multisplit as ONE stream-ordered collective call
// over an NCCL communicator.  Eq. (2) with the ranks
// as the outermost subproblems (hierarchical split P:667-674):
//   1. local stable multisplit of the shard (ms_run) into staging buffers
//      carved from the workspace; its m+1 local offsets;
//   2. counts h_g[b] = off[b+1] - off[b] (u64, device), NCCL all-gather of the
//      P x m count matrix, copied to the host (the ONE synchronisation: the
//      piece sizes are host arguments of the point-to-point calls);
//   3. ms_dist_pieces: global bucket starts, this rank's balanced window and
//      the <= m+P-1 contiguous pieces it sends / the pieces it receives;
//   4. one NCCL group of send/recv (pieces to self: device-to-device copies)
//      landing every piece at its final offset in the owner's window.
// NCCL is loaded at run time (dlopen of libnccl.so.2 -- the process's NCCL,
// e.g. the one torch already loaded), so libms.so has no link-time NCCL
// dependency and loads on machines without it.
// =========================================================================
#include <cuda_runtime.h>
#include <dlfcn.h>
#include <nccl.h>

#include <cstring>
#include <mutex>

namespace {

struct Nccl {
  bool ok = false;
  ncclResult_t (*GetUniqueId)(ncclUniqueId *);
  ncclResult_t (*CommInitRank)(ncclComm_t *, int, ncclUniqueId, int);
  ncclResult_t (*CommDestroy)(ncclComm_t);
  ncclResult_t (*CommCount)(const ncclComm_t, int *);
  ncclResult_t (*CommUserRank)(const ncclComm_t, int *);
  ncclResult_t (*CommCuDevice)(const ncclComm_t, int *);
  ncclResult_t (*AllGather)(const void *, void *, size_t, ncclDataType_t, ncclComm_t, cudaStream_t);
  ncclResult_t (*Send)(const void *, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t);
  ncclResult_t (*Recv)(void *, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t);
  ncclResult_t (*GroupStart)();
  ncclResult_t (*GroupEnd)();
  ncclResult_t (*AllReduce)(const void *, void *, size_t, ncclDataType_t, ncclRedOp_t, ncclComm_t, cudaStream_t);
};

const Nccl &nccl() {
  static Nccl N;
  static std::once_flag once;
  std::call_once(once, [] {
    void *h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
    if (!h) h = dlopen("libnccl.so", RTLD_NOW | RTLD_GLOBAL);
    if (!h) return;
    bool all = true;
    auto sym = [&](auto &fn, const char *name) {
      fn = reinterpret_cast<std::remove_reference_t<decltype(fn)>>(dlsym(h, name));
      all = all && fn != nullptr;
    };
    sym(N.GetUniqueId, "ncclGetUniqueId");
    sym(N.CommInitRank, "ncclCommInitRank");
    sym(N.CommDestroy, "ncclCommDestroy");
    sym(N.CommCount, "ncclCommCount");
    sym(N.CommUserRank, "ncclCommUserRank");
    sym(N.CommCuDevice, "ncclCommCuDevice");
    sym(N.AllGather, "ncclAllGather");
    sym(N.Send, "ncclSend");
    sym(N.Recv, "ncclRecv");
    sym(N.GroupStart, "ncclGroupStart");
    sym(N.GroupEnd, "ncclGroupEnd");
    sym(N.AllReduce, "ncclAllReduce");
    N.ok = all;
  });
  return N;
}

constexpr size_t kDAlign = 256;
inline size_t dalign(size_t x) { return (x + kDAlign - 1) / kDAlign * kDAlign; }

// counts[b] = off[b+1] - off[b] as u64 (local bucket sizes of this rank's shard)
__global__ void k_counts_from_offsets(const uint32_t *off, uint64_t *counts, uint32_t m) {
  for (uint32_t b = threadIdx.x; b < m; b += blockDim.x) counts[b] = (uint64_t)(off[b + 1] - off[b]);
}

struct DistLayout {
  size_t local_ws, off_keys, off_vals, off_loff, off_cnt, off_gath, bytes;
};

DistLayout dist_layout(ms_plan_t plan, uint32_t m, int kv, uint64_t n_local, int nranks, ms_status *st) {
  DistLayout d{};
  size_t ws = 0;
  *st = ms_plan_workspace_size(plan, n_local, &ws);
  d.local_ws = dalign(ws);
  d.off_keys = d.local_ws;
  d.off_vals = d.off_keys + dalign(n_local * 4);
  d.off_loff = d.off_vals + (kv ? dalign(n_local * 4) : 0);
  d.off_cnt = d.off_loff + dalign((size_t)(m + 1) * 4);
  d.off_gath = d.off_cnt + dalign((size_t)m * 8);
  d.bytes = d.off_gath + dalign((size_t)nranks * m * 8);
  return d;
}

}  // namespace

extern "C" ms_status ms_nccl_get_unique_id(void *id) {
  if (!id) return MS_ERR_INVALID_ARG;
  const Nccl &N = nccl();
  if (!N.ok) return MS_ERR_NCCL;
  ncclUniqueId u;
  if (N.GetUniqueId(&u) != ncclSuccess) return MS_ERR_NCCL;
  memcpy(id, &u, sizeof(u));
  return MS_OK;
}

extern "C" ms_status ms_nccl_comm_init(void **comm, int32_t nranks, int32_t rank, const void *id, int device) {
  if (!comm || !id || nranks < 1 || rank < 0 || rank >= nranks || device < 0) return MS_ERR_INVALID_ARG;
  const Nccl &N = nccl();
  if (!N.ok) return MS_ERR_NCCL;
  if (cudaSetDevice(device) != cudaSuccess) return MS_ERR_CUDA;
  ncclUniqueId u;
  memcpy(&u, id, sizeof(u));
  ncclComm_t c = nullptr;
  if (N.CommInitRank(&c, nranks, u, rank) != ncclSuccess) return MS_ERR_NCCL;
  *comm = c;
  return MS_OK;
}

extern "C" ms_status ms_nccl_comm_destroy(void *comm) {
  if (!comm) return MS_OK;
  const Nccl &N = nccl();
  if (!N.ok) return MS_ERR_NCCL;
  return N.CommDestroy((ncclComm_t)comm) == ncclSuccess ? MS_OK : MS_ERR_NCCL;
}

extern "C" ms_status ms_dist_workspace_size(ms_plan_t plan, uint64_t n_local, int32_t nranks, size_t *bytes) {
  if (!plan || !bytes || nranks < 1) return MS_ERR_INVALID_ARG;
  ms_bucket_spec spec;
  int32_t kv = 0;
  ms_status st = ms_plan_spec(plan, &spec, &kv);
  if (st != MS_OK) return st;
  DistLayout d = dist_layout(plan, spec.m, kv, n_local, nranks, &st);
  if (st != MS_OK) return st;
  *bytes = d.bytes;
  return MS_OK;
}

extern "C" ms_status ms_dist_run(ms_plan_t plan, void *comm, const uint32_t *keys_in, const uint32_t *vals_in,
                                 const void *ids, uint64_t n_local, uint32_t *keys_out, uint32_t *vals_out,
                                 uint64_t out_capacity, uint64_t *offsets_global, uint64_t *win_start,
                                 uint64_t *win_len, void *workspace, size_t workspace_bytes, void *stream) {
  if (!plan || !comm) return MS_ERR_INVALID_ARG;
  if ((vals_in == nullptr) != (vals_out == nullptr)) return MS_ERR_INVALID_ARG;
  if (!keys_out || !workspace) return MS_ERR_INVALID_ARG;
  ms_bucket_spec spec;
  int32_t kv = 0;
  ms_status st = ms_plan_spec(plan, &spec, &kv);
  if (st != MS_OK) return st;
  if (vals_in && !kv) return MS_ERR_UNSUPPORTED;
  const Nccl &N = nccl();
  if (!N.ok) return MS_ERR_NCCL;
  ncclComm_t c = (ncclComm_t)comm;
  int P = 0, rank = 0, dev = 0;
  if (N.CommCount(c, &P) != ncclSuccess || N.CommUserRank(c, &rank) != ncclSuccess ||
      N.CommCuDevice(c, &dev) != ncclSuccess)
    return MS_ERR_NCCL;
  const uint32_t m = spec.m;
  DistLayout d = dist_layout(plan, m, vals_in != nullptr, n_local, P, &st);
  if (st != MS_OK) return st;
  if (workspace_bytes < d.bytes) return MS_ERR_WORKSPACE;
  if (reinterpret_cast<uintptr_t>(workspace) & 15u) return MS_ERR_ALIGNMENT;
  int prev = -1;
  if (cudaGetDevice(&prev) != cudaSuccess) return MS_ERR_CUDA;
  if (prev != dev && cudaSetDevice(dev) != cudaSuccess) return MS_ERR_CUDA;
  struct Restore {
    int prev, dev;
    ~Restore() {
      if (prev != dev) cudaSetDevice(prev);
    }
  } restore{prev, dev};
  cudaStream_t s = (cudaStream_t)stream;
  char *w = (char *)workspace;
  uint32_t *lk = (uint32_t *)(w + d.off_keys), *lv = vals_in ? (uint32_t *)(w + d.off_vals) : nullptr;
  uint32_t *loff = (uint32_t *)(w + d.off_loff);
  uint64_t *cnt = (uint64_t *)(w + d.off_cnt), *gath = (uint64_t *)(w + d.off_gath);
  // 1. local stable multisplit of the shard
  st = ms_run(plan, keys_in, vals_in, ids, lk, lv, n_local, loff, workspace, d.local_ws, stream);
  if (st != MS_OK) return st;
  // 2. per-rank bucket counts, all-gathered (rows in rank order)
  k_counts_from_offsets<<<1, 256, 0, s>>>(loff, cnt, m);
  if (cudaGetLastError() != cudaSuccess) return MS_ERR_CUDA;
  if (N.AllGather(cnt, gath, m, ncclUint64, c, s) != ncclSuccess) return MS_ERR_NCCL;
  std::vector<uint64_t> counts((size_t)P * m);
  if (cudaMemcpyAsync(counts.data(), gath, counts.size() * 8, cudaMemcpyDeviceToHost, s) != cudaSuccess ||
      cudaStreamSynchronize(s) != cudaSuccess)
    return MS_ERR_CUDA;
  // 3. pieces
  std::vector<ms_piece> send(m + P), recv((size_t)m * P + 1);
  std::vector<uint64_t> offg(m + 1);
  int32_t ns = 0, nr = 0;
  uint64_t ws0 = 0, wl = 0;
  st = ms_dist_pieces(P, rank, m, counts.data(), send.data(), (int32_t)send.size(), &ns, recv.data(),
                      (int32_t)recv.size(), &nr, offg.data(), &ws0, &wl);
  if (st != MS_OK) return st;
  if (wl > out_capacity) return MS_ERR_INVALID_ARG;  // the caller's window buffers are too small
  if (offsets_global) memcpy(offsets_global, offg.data(), offg.size() * 8);
  if (win_start) *win_start = ws0;
  if (win_len) *win_len = wl;
  // 4. the exchange: local pieces by copy, the rest by one NCCL group of send/recv
  for (int32_t i = 0; i < ns; ++i) {
    const ms_piece &q = send[i];
    if (q.peer != rank || q.len == 0) continue;
    if (cudaMemcpyAsync(keys_out + q.dst_off, lk + q.src_off, q.len * 4, cudaMemcpyDeviceToDevice, s) != cudaSuccess)
      return MS_ERR_CUDA;
    if (lv && cudaMemcpyAsync(vals_out + q.dst_off, lv + q.src_off, q.len * 4, cudaMemcpyDeviceToDevice, s) !=
                  cudaSuccess)
      return MS_ERR_CUDA;
  }
  if (N.GroupStart() != ncclSuccess) return MS_ERR_NCCL;
  ncclResult_t r = ncclSuccess;
  for (int a = 0; a < (lv ? 2 : 1) && r == ncclSuccess; ++a) {
    const uint32_t *src = a ? lv : lk;
    uint32_t *dst = a ? vals_out : keys_out;
    for (int32_t i = 0; i < ns && r == ncclSuccess; ++i)
      if (send[i].peer != rank && send[i].len)
        r = N.Send(src + send[i].src_off, send[i].len, ncclUint32, send[i].peer, c, s);
    for (int32_t i = 0; i < nr && r == ncclSuccess; ++i)
      if (recv[i].peer != rank && recv[i].len)
        r = N.Recv(dst + recv[i].dst_off, recv[i].len, ncclUint32, recv[i].peer, c, s);
  }
  const ncclResult_t r2 = N.GroupEnd();
  return (r == ncclSuccess && r2 == ncclSuccess) ? MS_OK : MS_ERR_NCCL;
}

// =========================================================================
// ms_dist_run_fused: the sharded multisplit with the exchange fused into the
// post-scan: local K1 + K2 (ms_prescan / ms_scan), the count
// all-gather, the host targets (ms_dist_targets), then ONE K3 that stores every
// bucket run straight into the owners' windows (ms_postscan_scatter; TMA bulk
// stores over NVLink / NVSwitch when the windows are peer mappings), and a
// one-word NCCL all-reduce on the stream as the barrier after which every
// window is complete.
// =========================================================================
namespace {

struct FusedLayout {
  size_t local_ws, off_hg, off_loff, off_cnt, off_gath, off_bar, bytes;
};

FusedLayout fused_layout(ms_plan_t plan, uint32_t m, uint64_t n_local, int nranks, ms_status *st) {
  FusedLayout d{};
  size_t ws = 0;
  uint32_t T = 0;
  uint64_t L = 0;
  *st = ms_plan_workspace_size(plan, n_local, &ws);
  if (*st == MS_OK) *st = ms_plan_geometry(plan, n_local, &T, &L, nullptr);
  d.local_ws = dalign(ws);
  d.off_hg = d.local_ws;
  d.off_loff = d.off_hg + dalign((size_t)m * L * 4);
  d.off_cnt = d.off_loff + dalign((size_t)(m + 1) * 4);
  d.off_gath = d.off_cnt + dalign((size_t)m * 8);
  d.off_bar = d.off_gath + dalign((size_t)nranks * m * 8);
  d.bytes = d.off_bar + dalign(4);
  return d;
}

}  // namespace

extern "C" ms_status ms_dist_workspace_size_fused(ms_plan_t plan, uint64_t n_local, int32_t nranks, size_t *bytes) {
  if (!plan || !bytes || nranks < 1 || nranks > MS_MAX_PEERS) return MS_ERR_INVALID_ARG;
  ms_bucket_spec spec;
  ms_status st = ms_plan_spec(plan, &spec, nullptr);
  if (st != MS_OK) return st;
  FusedLayout d = fused_layout(plan, spec.m, n_local, nranks, &st);
  if (st != MS_OK) return st;
  *bytes = d.bytes;
  return MS_OK;
}

extern "C" ms_status ms_dist_run_fused(ms_plan_t plan, void *comm, const uint32_t *keys_in, const uint32_t *vals_in,
                                       uint64_t n_local, uint32_t *const *keys_windows,
                                       uint32_t *const *vals_windows, uint64_t window_capacity,
                                       uint64_t *offsets_global, uint64_t *win_start, uint64_t *win_len,
                                       void *workspace, size_t workspace_bytes, void *stream) {
  if (!plan || !comm || !keys_windows || !workspace) return MS_ERR_INVALID_ARG;
  ms_bucket_spec spec;
  int32_t kv = 0;
  ms_status st = ms_plan_spec(plan, &spec, &kv);
  if (st != MS_OK) return st;
  if (vals_in && (!kv || !vals_windows)) return vals_windows ? MS_ERR_UNSUPPORTED : MS_ERR_INVALID_ARG;
  if (spec.m > 32 || spec.kind == MS_IDS) return MS_ERR_UNSUPPORTED;
  const Nccl &N = nccl();
  if (!N.ok) return MS_ERR_NCCL;
  ncclComm_t c = (ncclComm_t)comm;
  int P = 0, rank = 0, dev = 0;
  if (N.CommCount(c, &P) != ncclSuccess || N.CommUserRank(c, &rank) != ncclSuccess ||
      N.CommCuDevice(c, &dev) != ncclSuccess)
    return MS_ERR_NCCL;
  if (P > MS_MAX_PEERS) return MS_ERR_UNSUPPORTED;
  const uint32_t m = spec.m;
  FusedLayout d = fused_layout(plan, m, n_local, P, &st);
  if (st != MS_OK) return st;
  if (workspace_bytes < d.bytes) return MS_ERR_WORKSPACE;
  if (reinterpret_cast<uintptr_t>(workspace) & 15u) return MS_ERR_ALIGNMENT;
  int prev = -1;
  if (cudaGetDevice(&prev) != cudaSuccess) return MS_ERR_CUDA;
  if (prev != dev && cudaSetDevice(dev) != cudaSuccess) return MS_ERR_CUDA;
  struct Restore {
    int prev, dev;
    ~Restore() {
      if (prev != dev) cudaSetDevice(prev);
    }
  } restore{prev, dev};
  cudaStream_t s = (cudaStream_t)stream;
  char *w = (char *)workspace;
  uint32_t *HG = (uint32_t *)(w + d.off_hg), *loff = (uint32_t *)(w + d.off_loff), *bar = (uint32_t *)(w + d.off_bar);
  uint64_t *cnt = (uint64_t *)(w + d.off_cnt), *gath = (uint64_t *)(w + d.off_gath);
  // 1. local K1 + K2 (tiles; G stays in the workspace for K3)
  if ((st = ms_prescan(plan, keys_in, nullptr, n_local, HG, workspace, d.local_ws, stream)) != MS_OK) return st;
  if ((st = ms_scan(plan, HG, n_local, loff, workspace, d.local_ws, stream)) != MS_OK) return st;
  // 2. counts, all-gathered, on the host
  k_counts_from_offsets<<<1, 256, 0, s>>>(loff, cnt, m);
  if (cudaGetLastError() != cudaSuccess) return MS_ERR_CUDA;
  if (N.AllGather(cnt, gath, m, ncclUint64, c, s) != ncclSuccess) return MS_ERR_NCCL;
  std::vector<uint64_t> counts((size_t)P * m);
  if (cudaMemcpyAsync(counts.data(), gath, counts.size() * 8, cudaMemcpyDeviceToHost, s) != cudaSuccess ||
      cudaStreamSynchronize(s) != cudaSuccess)
    return MS_ERR_CUDA;
  // 3. targets: global - local position per local bucket, the window starts
  ms_scatter_target t{};
  t.nranks = P;
  if ((st = ms_dist_targets(P, rank, m, counts.data(), t.delta, t.win_start)) != MS_OK) return st;
  for (int r = 0; r < P; ++r) {
    if (t.win_start[r + 1] - t.win_start[r] > window_capacity) return MS_ERR_INVALID_ARG;
    t.keys_dst[r] = keys_windows[r];
    t.vals_dst[r] = vals_in ? vals_windows[r] : nullptr;
  }
  if (offsets_global) {
    uint64_t B = 0;
    for (uint32_t b = 0; b < m; ++b) {
      offsets_global[b] = B;
      for (int g = 0; g < P; ++g) B += counts[(size_t)g * m + b];
    }
    offsets_global[m] = B;
  }
  if (win_start) *win_start = t.win_start[rank];
  if (win_len) *win_len = t.win_start[rank + 1] - t.win_start[rank];
  // 4. the post-scan storing into the owners' windows
  if ((st = ms_postscan_scatter(plan, keys_in, vals_in, HG, n_local, &t, workspace, d.local_ws, stream)) != MS_OK)
    return st;
  // 5. barrier: every rank's scatter kernel precedes its all-reduce on its stream
  if (cudaMemsetAsync(bar, 0, 4, s) != cudaSuccess) return MS_ERR_CUDA;
  if (N.AllReduce == nullptr || N.AllReduce(bar, bar, 1, ncclUint32, ncclSum, c, s) != ncclSuccess) return MS_ERR_NCCL;
  return MS_OK;
}
