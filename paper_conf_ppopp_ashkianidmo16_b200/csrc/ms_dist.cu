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
