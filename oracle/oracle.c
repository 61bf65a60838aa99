/*
 * oracle.c -- CPU oracle for the stable multisplit (TEST INFRASTRUCTURE ONLY).
 *
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
 * --impl reference legs may load this library.  The product path
 * (paper_conf_ppopp_ashkianidmo16_b200, libms.so) never links, imports or
 * calls it, and this file shares no code, header, table or constant
 * generator with the CUDA path.
 *
 * What it computes is the plain definition of the paper, serially, in the
 * paper's order and notation (PAPER.md = /root/reference/PAPER.md, "P:<line>"):
 *
 *   multisplit (§3.1): a permutation of the n input keys (or
 *   key-value pairs) such that all elements of a bucket are contiguous and
 *   buckets appear in ascending bucket-id order; "stable" keeps
 *   input order inside a bucket; optionally the start of each bucket is
 *   returned.  Stable multisplit is exactly Eq. (1) (§4,
 *   P:565-586):
 *        p(i) = sum_{k<j} h_k + |{u_r : u_r in B_j, r < i}|,  u_i in B_j
 *   computed as ids -> histogram h -> exclusive scan -> in-order scatter
 *   (a serial stable counting sort by bucket id).
 *
 *   oracle_tile_matrices: the matrices H (m x L, h_{j,l} = count of bucket j
 *   in subproblem l) and G (the exclusive scan of row-vectorised H, i.e. the
 *   first two terms of Eq. (2), §4 P:587-649 and §5.1) for
 *   subproblems of T consecutive keys.
 *
 * Bucket functions (whatBucket()) -- readings listed in
 * DESIGN.md "Readings of the paper":
 *   MS_LOWBITS   id = (k >> shift) & (m-1)                      (m a power of 2)
 *   MS_DELTA     id = min(floor(k / delta), m-1)   (reading 8: last bucket is
 *                                                   the far pile)
 *   MS_SPLITTERS id = #{ j : s_j < k }             (reading 9: a key equal to a
 *                                                   splitter is in the lower
 *                                                   bucket, Fig. 1(2))
 *   MS_IDS       id = ids[i]                        (precomputed, u8 or u32)
 *
 * Parity pins: tests/test_oracle.py (Fig. 1 golden vectors, brute force over
 * all id sequences, closed forms, invariants, reductions to sort/partition).
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

enum { O_LOWBITS = 0, O_DELTA = 1, O_SPLITTERS = 2, O_IDS = 3 };

/* #{ j < cnt : s[j] < k } for non-decreasing s: plain lower_bound. */
static uint32_t count_less(const uint32_t *s, uint32_t cnt, uint32_t k) {
  uint32_t lo = 0, hi = cnt; /* invariant: s[0..lo) < k, s[hi..cnt) >= k */
  while (lo < hi) {
    uint32_t mid = lo + (hi - lo) / 2;
    if (s[mid] < k) lo = mid + 1; else hi = mid;
  }
  return lo;
}

/* whatBucket() for one element. */
static uint32_t what_bucket(int kind, uint32_t m, uint32_t shift, uint32_t delta,
                            const uint32_t *splitters, const void *ids, uint32_t id_bytes,
                            uint32_t key, uint64_t i) {
  switch (kind) {
    case O_LOWBITS: return (key >> shift) & (m - 1u);
    case O_DELTA: { uint32_t q = key / delta; return q < m - 1u ? q : m - 1u; }
    case O_SPLITTERS: return count_less(splitters, m - 1u, key);
    default:
      return id_bytes == 1 ? (uint32_t)((const uint8_t *)ids)[i] : ((const uint32_t *)ids)[i];
  }
}

/* Step 1: ids[i] = whatBucket(key[i]).  Returns -1 if every id < m, else the
 * first index whose id is out of range (a partition violation). */
int64_t oracle_bucket_ids(int kind, uint32_t m, uint32_t shift, uint32_t delta,
                          const uint32_t *splitters, const void *ids, uint32_t id_bytes,
                          const uint32_t *keys, uint64_t n, uint32_t *out_ids) {
  for (uint64_t i = 0; i < n; ++i) {
    uint32_t b = what_bucket(kind, m, shift, delta, splitters, ids, id_bytes, keys ? keys[i] : 0u, i);
    if (b >= m) return (int64_t)i;
    out_ids[i] = b;
  }
  return -1;
}

/* Stable multisplit, Eq. (1).  vals / vals_out may be NULL (key-only);
 * offsets (m+1 entries) may be NULL.  Returns 0, or -1 if an id is >= m or
 * memory runs out. */
int oracle_multisplit(int kind, uint32_t m, uint32_t shift, uint32_t delta,
                      const uint32_t *splitters, const void *ids, uint32_t id_bytes,
                      const uint32_t *keys, const uint32_t *vals, uint64_t n,
                      uint32_t *keys_out, uint32_t *vals_out, uint64_t *offsets) {
  uint32_t *id = (uint32_t *)malloc((n ? n : 1) * sizeof(uint32_t));
  uint64_t *h = (uint64_t *)calloc(m + 1u, sizeof(uint64_t));
  uint64_t *cur = (uint64_t *)calloc(m + 1u, sizeof(uint64_t));
  if (!id || !h || !cur) { free(id); free(h); free(cur); return -1; }
  /* 1. ids */
  if (oracle_bucket_ids(kind, m, shift, delta, splitters, ids, id_bytes, keys, n, id) >= 0) {
    free(id); free(h); free(cur); return -1;
  }
  /* 2. histogram h_0..h_{m-1} */
  for (uint64_t i = 0; i < n; ++i) h[id[i]]++;
  /* 3. exclusive scan: first term of Eq. (1), sum_{k<j} h_k */
  cur[0] = 0;
  for (uint32_t b = 0; b < m; ++b) cur[b + 1] = cur[b] + h[b];
  if (offsets) for (uint32_t b = 0; b <= m; ++b) offsets[b] = cur[b];
  /* 4. in-order scatter: second term of Eq. (1), |{u_r in B_j : r < i}| */
  for (uint64_t i = 0; i < n; ++i) {
    uint64_t p = cur[id[i]]++;
    if (keys_out && keys) keys_out[p] = keys[i];
    if (vals_out && vals) vals_out[p] = vals[i];
  }
  free(id); free(h); free(cur);
  return 0;
}

/* Eq. (2) intermediates for subproblems of T consecutive elements
 * (L = ceil(n/T)), given ids (u32, each < m):
 *   H[j*L + l] = h_{j,l} = |{ i in subproblem l : id_i = j }|
 *   G[j*L + l] = sum_{k<j} sum_{l'} h_{k,l'} + sum_{l'<l} h_{j,l'}    (terms 1+2 of Eq. 2)
 * Both row-vectorised (bucket-major), as in Alg. 1 P:825-828.  G is written
 * out from its two-term definition (not by scanning H) so that a test can
 * pin "G = exclusive scan of row-vectorised H" independently. */
int oracle_tile_matrices(const uint32_t *ids, uint64_t n, uint32_t m, uint64_t T,
                         uint32_t *H, uint32_t *G) {
  uint64_t L = (n + T - 1) / T;
  uint64_t *tot = (uint64_t *)calloc(m ? m : 1, sizeof(uint64_t));
  if (!tot) return -1;
  memset(H, 0, (size_t)(m * L) * sizeof(uint32_t));
  for (uint64_t i = 0; i < n; ++i) H[(uint64_t)ids[i] * L + i / T]++;
  for (uint32_t j = 0; j < m; ++j)
    for (uint64_t l = 0; l < L; ++l) tot[j] += H[(uint64_t)j * L + l];
  for (uint32_t j = 0; j < m; ++j) {
    uint64_t term1 = 0;
    for (uint32_t k = 0; k < j; ++k) term1 += tot[k];
    uint64_t term2 = 0;
    for (uint64_t l = 0; l < L; ++l) {
      G[(uint64_t)j * L + l] = (uint32_t)(term1 + term2);
      term2 += H[(uint64_t)j * L + l];
    }
  }
  free(tot);
  return 0;
}

/* Number of host threads this library uses (it is serial). */
int oracle_threads(void) { return 1; }
