/*
 * ms.h -- C ABI of the B200-native stable multisplit (libms.so).
 *
 * Multisplit (§3.1): a permutation of n 32-bit keys, or
 * key-value pairs, into m contiguous buckets in ascending bucket-id order;
 * this library is always STABLE (input order kept inside a bucket,
 * P:358-363), so the output is unique and is defined by Eq. (1) (§4,
 * P:565-586):  p(i) = sum_{k<j} h_k + |{u_r in B_j : r < i}|  for u_i in B_j.
 * Optionally the start of every bucket is returned; this library
 * returns m+1 offsets (the last one is n).
 *
 * The hot path is the paper's {pre-scan, scan, post-scan} (§4 P:538-550,
 * Alg. 1) on tiles of T keys (subproblems of Eq. (2)):
 *   K1 pre-scan   per-tile bucket histograms H (m x L, bucket-major)
 *   K2 scan       G = exclusive scan of row-vectorised H, offsets = G[:,0]
 *   K3 post-scan  recompute ids, stable tile-local multisplit in shared
 *                 memory, coalesced scatter to G[j][l] + local offset
 * Variants (ms_plan_geometry reports tile (0), ranged (1), ONE (2) or
 * two-pass (3); ms_plan_last_launches how many kernels the last ms_run
 * enqueued):
 *   "tile"   subproblems = the L tiles (H, G are m x L words): K1, K2, K3
 *            (the default for key-value 32 < m <= 256, key-only 64 < m <= 256,
 *            and key-only u32 ids above 32 buckets);
 *   "ranged" (m <= 32) subproblems = the C <= 1024 contiguous tile ranges of
 *            K3's persistent CTAs: K1 writes per-range histograms (C x k x m),
 *            K3 folds their scan into its prologue and keeps each tile's G_j as
 *            a running sum inside its range (Eq. (2) applied twice): 2 kernels
 *            (the default for key-value runs of >= 8 (m <= 8), >= 16 (m <= 16,
 *            MS_IDS) or > 64 (m <= 32) tiles per SM);
 *   "ONE"    (m <= 32 every other run; key-only 33..64 buckets with computed
 *            or u8 ids) the ranged form in ONE cooperative launch: range
 *            counts, grid barrier, range scan, post-scan (reverse tile walk)
 *            -- 1 kernel; key-only runs use 8192-key tiles.  DESIGN.md §7-8;
 *   "two-pass" (m > 256) two stable multisplits by the low and the high digit
 *            of the id, then the offsets from the sorted output (§7b).
 * Every variant computes the same (unique, stable) result.  The MS_VARIANT_*
 * plan flags force one.  The stage-wise calls (ms_prescan / ms_scan /
 * ms_postscan) always use tiles.
 *
 * Conventions for every call below:
 *  - Pointers named *_in/*_out/ids/offsets/workspace/H/G are CUDA DEVICE
 *    pointers unless the function name ends in _host.  They must be 16-byte
 *    aligned (MS_ERR_ALIGNMENT otherwise).  Sizes are element counts.
 *  - Ownership: the caller owns every buffer; a plan owns only host metadata.
 *    Nothing here allocates device memory or synchronises, except
 *    ms_plan_check (synchronises `stream`).
 *  - `stream` is a cudaStream_t passed as void* (NULL = legacy default stream).
 *    All work is enqueued on it; results are valid when it completes.
 *  - Argument errors are returned synchronously before anything is enqueued.
 *    CUDA launch failures return MS_ERR_CUDA.
 *  - Out-of-place only: keys_out must not overlap keys_in.
 */
#ifndef MS_H
#define MS_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef int32_t ms_status;
#define MS_OK                 0
#define MS_ERR_INVALID_ARG   (-1) /* null pointer, m out of 1..256, bad kind, n > max_n, ... */
#define MS_ERR_UNSUPPORTED   (-2) /* e.g. values requested on a key-only plan                 */
#define MS_ERR_ALIGNMENT     (-3) /* a device pointer is not 16-byte aligned                   */
#define MS_ERR_ALIAS         (-4) /* an output overlaps an input                               */
#define MS_ERR_WORKSPACE     (-5) /* workspace NULL or smaller than ms_plan_workspace_size()   */
#define MS_ERR_CUDA          (-6) /* a CUDA runtime call failed                                */
#define MS_ERR_NCCL          (-7) /* an NCCL call failed (ms_dist_run)                          */
#define MS_ERR_BUCKET_RANGE  (-8) /* MS_VALIDATE: some precomputed id was >= m                 */

/* Bucket identifier kinds: the programmer's whatBucket() (P:353-357,
 * P:810-813) restricted to an enumerated set (readings 7-11). */
typedef enum {
  MS_LOWBITS = 0,   /* id = (key >> shift) & (m-1); m must be a power of two            */
  MS_DELTA = 1,     /* id = min(floor(key / delta), m-1); delta >= 1 (delta-stepping,
                       P:100-111; the last bucket is the far pile)                       */
  MS_SPLITTERS = 2, /* id = #{ j : splitters[j] < key } over m-1 non-decreasing splitters
                       (a key equal to a splitter goes to the lower bucket, Fig. 1(2))    */
  MS_IDS = 3        /* id = ids[i], precomputed, id_bytes = 1 (u8) or 4 (u32) per id      */
} ms_bucket_kind;

typedef struct {
  int32_t kind;               /* ms_bucket_kind                                          */
  uint32_t m;                 /* number of buckets, 1..256                               */
  uint32_t shift;             /* MS_LOWBITS: bit offset, shift + log2(m) <= 32           */
  uint32_t delta;             /* MS_DELTA: bucket width >= 1                             */
  const uint32_t *splitters;  /* MS_SPLITTERS: HOST pointer to m-1 non-decreasing values,
                                 copied at ms_plan_create (may be freed afterwards)       */
  uint32_t id_bytes;          /* MS_IDS: 1 or 4                                          */
} ms_bucket_spec;

typedef struct ms_plan_s *ms_plan_t;

/* plan flags.  Without a MS_VARIANT_* flag every run picks its variant from
 * (m, n, key-only / key-value) by the measured rule of DESIGN.md §7; a
 * MS_VARIANT_* flag makes every run use that one (at most one may be set):
 *   MS_VARIANT_3K      tile variant  K1 -> K2 -> K3     (3 launches, any m)
 *   MS_VARIANT_RANGED  CTA ranges    K1r -> K3          (2 launches, m <= 32)
 *   MS_VARIANT_ONE     cooperative   one kernel         (1 launch,  m <= 32, or
 *                      key-only m <= 64 with computed or u8 ids; a
 *                      grid that cannot be co-resident fails with MS_ERR_CUDA
 *                      instead of falling back to the ranged variant)
 * MS_ABLATION_DIRECT: the paper's "Direct" post-scan (Table 4):
 * no local reorder, every key stored straight to its global position (tile
 * variant; implemented for MS_DELTA with m <= 32 and m * delta = 2^32 only,
 * else MS_ERR_UNSUPPORTED) -- a design-space ablation, same result.
 * MS_ABLATION_NW2 / MS_ABLATION_NW4: the post-scan CTA has 2 / 4 warps instead
 * of 8 (tile T = 1024 / 2048 keys; the local reorder then spans fewer warps,
 * the B200 analogue of the paper's NW sweep and of warp- vs block-level
 * reordering); ranged variant, same kinds as
 * MS_ABLATION_DIRECT.
 * MS_ABLATION_BALLOT / MS_ABLATION_WARP: the post-scan of 32 < m <= 256 (Alg. 3
 * ballot ranks over warp-striped 32-key rounds, ms_k3_warp.cuh) used for any
 * 2 <= m <= 256, with the block-level reorder of the whole tile (BALLOT,
 * §5.2.2) or the paper's Warp-level MS (WARP, §5.2.1
 * every warp reorders only its own 512-key segment, a warp-wide
 * shuffle scan of its bucket counts giving the positions, and stores its
 * runs); tile variant, MS_DELTA with m * delta = 2^32 only (else
 * MS_ERR_UNSUPPORTED).  At most one MS_ABLATION_* flag, none with
 * MS_VARIANT_*. */
#define MS_VALIDATE        1u  /* flag precomputed ids >= m on the device; ms_plan_check reports it */
#define MS_VARIANT_3K      2u
#define MS_VARIANT_RANGED  4u
#define MS_VARIANT_ONE     8u
#define MS_ABLATION_DIRECT 16u
#define MS_ABLATION_NW2    32u
#define MS_ABLATION_NW4    64u
#define MS_ABLATION_BALLOT 128u
#define MS_ABLATION_WARP   256u

/* Create a plan for up to max_n elements (max_n < 2^32) on CUDA device
 * `device` (-1: the calling thread's current device; every later call of the
 * plan switches to that device for its duration).  with_values != 0 plans
 * key-value runs.  Host-only: validates the spec (m range, power-of-two m for
 * MS_LOWBITS, delta >= 1, sorted splitters, id_bytes) and the flags, and
 * precomputes the bucket-function constants.  Returns MS_ERR_INVALID_ARG on a
 * bad spec or flag combination, MS_ERR_UNSUPPORTED for a variant the spec
 * cannot use (m > 32 with MS_VARIANT_RANGED; MS_VARIANT_ONE with m > 64, or
 * with m > 32 and values or u32 ids). */
ms_status ms_plan_create(ms_plan_t *plan, const ms_bucket_spec *spec, uint64_t max_n,
                         int with_values, uint32_t flags, int device);

/* Device workspace bytes ms_run needs for n elements (n <= max_n). */
ms_status ms_plan_workspace_size(ms_plan_t plan, uint64_t n, size_t *bytes);

/* Tile geometry the plan uses for n elements: tile = T (keys per subproblem),
 * num_tiles = L = ceil(n / T), variant = 0 (tile, 3 launches), 1 (ranged, 2)
 * or 2 (ONE, 1) -- the variant a run of n elements (key-value if the plan has
 * values) takes.  T and L are those of the tile variant and the stage-wise
 * calls; a key-only ONE run with 17..32 computed-id buckets walks 8192-key
 * tiles internally. */
ms_status ms_plan_geometry(ms_plan_t plan, uint64_t n, uint32_t *tile, uint64_t *num_tiles,
                           int32_t *variant);

/* The whole multisplit.  keys_in[n] -> keys_out[n]; vals_in/vals_out NULL for
 * key-only (both non-NULL for key-value); ids[n] (id_bytes each) only for
 * MS_IDS, else NULL; offsets NULL or m+1 u32 entries (bucket j occupies
 * [offsets[j], offsets[j+1]), offsets[m] = n).  n = 0 only writes offsets. */
ms_status ms_run(ms_plan_t plan, const uint32_t *keys_in, const uint32_t *vals_in,
                 const void *ids, uint32_t *keys_out, uint32_t *vals_out, uint64_t n,
                 uint32_t *offsets, void *workspace, size_t workspace_bytes, void *stream);

/* ms_run over HOST buffers (pinned for full PCIe rate): copies the inputs to
 * device staging carved from `workspace`, runs, and copies keys/vals/offsets
 * back, all on `stream` (host outputs valid once it completes).  Workspace
 * size: ms_plan_workspace_size_host. */
ms_status ms_plan_workspace_size_host(ms_plan_t plan, uint64_t n, size_t *bytes);
ms_status ms_run_host(ms_plan_t plan, const uint32_t *keys_in_host, const uint32_t *vals_in_host,
                      const void *ids_host, uint32_t *keys_out_host, uint32_t *vals_out_host,
                      uint64_t n, uint32_t *offsets_host, void *workspace, size_t workspace_bytes,
                      void *stream);

/* The three stages of the 3-kernel path, individually (for intermediate
 * parity against Eq. (2); ms_run chains them).  L = ceil(n/T) from
 * ms_plan_geometry.  H and G are m*L u32, bucket-major (H[j*L + l] = h_{j,l}).
 *   ms_prescan : H[j][l]  = count of bucket j in tile l         (Alg. 1)
 *   ms_scan    : G        = exclusive scan of row-vectorised H, in place (H -> G),
 *                offsets (NULL or m+1) = G[:,0], n              (Alg. 1)
 *   ms_postscan: keys/vals to G[j][l] + stable local offset     (Alg. 1, §5.2)
 * `workspace` as for ms_run (ms_plan_workspace_size). */
ms_status ms_prescan(ms_plan_t plan, const uint32_t *keys_in, const void *ids, uint64_t n,
                     uint32_t *H, void *workspace, size_t workspace_bytes, void *stream);
ms_status ms_scan(ms_plan_t plan, uint32_t *HG, uint64_t n, uint32_t *offsets, void *workspace,
                  size_t workspace_bytes, void *stream);
ms_status ms_postscan(ms_plan_t plan, const uint32_t *keys_in, const uint32_t *vals_in,
                      const void *ids, const uint32_t *G, uint32_t *keys_out, uint32_t *vals_out,
                      uint64_t n, void *workspace, size_t workspace_bytes, void *stream);

/* Device-side whatBucket() only: out_ids[i] = id of keys_in[i] (u32), for
 * checking the bucket functors (e.g. exhaustively over all 2^32 keys). */
ms_status ms_bucket_ids(ms_plan_t plan, const uint32_t *keys_in, uint64_t n, uint32_t *out_ids,
                        void *stream);

/* Synchronises `stream`, then reports MS_ERR_BUCKET_RANGE if a run on this
 * workspace since the last check saw an id >= m (plans with MS_VALIDATE), or
 * MS_ERR_INVALID_ARG if an ms_postscan_scatter on it met a run beyond its
 * target's last window (inconsistent win_start / delta: the overflowing part
 * was not stored), clearing the flag; MS_OK otherwise. */
ms_status ms_plan_check(ms_plan_t plan, void *workspace, void *stream);

ms_status ms_plan_destroy(ms_plan_t plan);
const char *ms_status_string(ms_status s);

/* The plan's bucket spec (splitters reported as NULL) and whether it plans
 * key-value runs (host only). */
ms_status ms_plan_spec(ms_plan_t plan, ms_bucket_spec *spec, int32_t *with_values);

/* Number of kernel launches the last ms_run / ms_run_host on this plan
 * enqueued (for the bench's gpu_launches claim). */
int32_t ms_plan_last_launches(ms_plan_t plan);

/* Per-stage tracing (CUDA events, Table 4's pre-scan / scan /
 * post-scan split).  ms_plan_trace(plan, 1) clears the record
 * and makes every following ms_run record an event before its first kernel
 * and after each kernel on its stream (plan-owned events, created on first
 * use); ms_plan_trace(plan, 2) records only the first and the last event
 * of every run (no events between the kernels, so K2 and K3 keep their
 * programmatic dependent launch; stage durations then read 0);
 * ms_plan_trace(plan, 0) stops recording.  ms_plan_trace_read waits
 * for the recorded events and writes, for up to max_runs runs in order,
 * stage_ms[r * 4 + s] = duration of stage s of run r in milliseconds
 * (s = 0 K1 pre-scan, 1 K2 scan, 2 K3 post-scan, in either variant),
 * and stage_ms[r * 4 + 3] = the run's total; *runs and
 * *stages (3) report what was written.  Tracing is host-side bookkeeping
 * only; it adds no kernel launches.  With per-stage events (mode 1) the
 * kernels are launched without programmatic dependent launch. */
ms_status ms_plan_trace(ms_plan_t plan, int enable);
ms_status ms_plan_trace_read(ms_plan_t plan, float *stage_ms, int32_t max_runs, int32_t *runs,
                             int32_t *stages);

/* ---------------------------------------------------------------------------
 * Sharded multisplit over P ranks: Eq. (2) with the
 * GPUs as the outermost subproblem level.  Rank g multisplits its shard locally
 * (ms_run), the m-vectors of per-rank bucket counts h[g][b] are all-gathered,
 * and every element of rank g's local bucket b at local position i goes to
 * global position B[b] + sum_{g'<g} h[g'][b] + (i - off_g[b]), where
 * B[b] = sum_{b'<b} sum_g h[g][b'].  The global output is cut into P balanced
 * windows (rank r owns [r*q + min(r, rem), ...), q = N/P, rem = N%P), so the
 * concatenation of the windows is the single-GPU stable multisplit of the
 * concatenated shards.  Because rank g's local output is monotone in global
 * position, it leaves in at most m+P-1 contiguous pieces.
 *
 * ms_dist_pieces (HOST function, no device access): from the all-gathered
 * counts (host, P*m u64, row g = rank g), compute for rank `rank`:
 *   send[k] = {src_off (local output offset), len, peer (dst rank), dst_off (offset in the peer's window)}
 *   recv[k] = {src_off (offset in the sender's local output), len, peer (src rank), dst_off (offset in my window)}
 * in the order both sides must issue them (buckets ascending per peer), plus
 * the global bucket starts offsets_global[m+1] (u64) and this rank's window
 * [*win_start, *win_start + *win_len).  The arrays hold at most m+P-1 (send)
 * and m*P (recv) entries; *n_send / *n_recv report the counts.  Pieces with
 * peer == rank are local copies.  Returns MS_ERR_INVALID_ARG on bad sizes or if
 * a capacity is too small.
 * ------------------------------------------------------------------------- */
typedef struct {
  uint64_t src_off;
  uint64_t len;
  int32_t peer;
  int32_t pad_;
  uint64_t dst_off;
} ms_piece;

ms_status ms_dist_pieces(int32_t nranks, int32_t rank, uint32_t m, const uint64_t *counts,
                         ms_piece *send, int32_t send_cap, int32_t *n_send, ms_piece *recv,
                         int32_t recv_cap, int32_t *n_recv, uint64_t *offsets_global,
                         uint64_t *win_start, uint64_t *win_len);

/* ---------------------------------------------------------------------------
 * Fused sharded scatter: instead of a local output plus an
 * exchange, the post-scan kernel stores every bucket run straight into the
 * windows of the ranks that own it -- over NVLink / NVSwitch when the window
 * pointers are peer mappings (CUDA IPC / symmetric memory), so the transfer
 * overlaps the local reorder tile by tile and the local output is never
 * written.  Same windows and the same global result as ms_dist_pieces.
 *
 * ms_dist_targets (HOST function): from the all-gathered counts (P*m u64, row
 * g = rank g) compute for rank `rank`:
 *   delta[b]     = global position - local position of its local bucket b
 *                  (B[b] + sum_{g'<g} h[g'][b] - off_g[b]), b < m (u64[m]);
 *   win_start[r] = first global position of rank r's window, r <= P
 *                  (win_start[P] = N; u64[P+1]).
 * MS_ERR_INVALID_ARG on bad sizes.
 *
 * ms_postscan_scatter: the post-scan (K3) of the 3-kernel path with the
 * stores redirected: keys_in / vals_in (NULL = key-only) are this rank's shard
 * (n local keys), G the output of ms_scan on it (m*L u32, workspace as for
 * ms_run); every key goes to keys_dst[r][x - win_start[r]] (and the value to
 * vals_dst[r][...]) where x = local position + delta[bucket] and r owns x.
 * The window pointers must be dereferenceable from the calling GPU (its own
 * memory or peer-mapped memory) and 16-byte aligned; the call is
 * stream-ordered and the stores are complete when the kernel completes on
 * `stream` (the CALLER synchronises the ranks before reading the windows).
 * Supported for plans with m <= 32 and a computed bucket kind (not MS_IDS);
 * else MS_ERR_UNSUPPORTED. nranks in 1..MS_MAX_PEERS.
 * ------------------------------------------------------------------------- */
#define MS_MAX_PEERS 8
typedef struct {
  int32_t nranks;
  int32_t pad_;
  uint32_t *keys_dst[MS_MAX_PEERS];
  uint32_t *vals_dst[MS_MAX_PEERS];
  uint64_t win_start[MS_MAX_PEERS + 1];
  uint64_t delta[32];
} ms_scatter_target;

ms_status ms_dist_targets(int32_t nranks, int32_t rank, uint32_t m, const uint64_t *counts, uint64_t *delta,
                          uint64_t *win_start);

/* ---------------------------------------------------------------------------
 * ms_dist_run -- the sharded stable multisplit as ONE collective call per rank
 * over an NCCL communicator (Eq. (2), with the
 * ranks as the outermost subproblems, the hierarchical split of P:667-674):
 *   1. local stable multisplit of this rank's shard (ms_run) into staging
 *      buffers inside `workspace`;
 *   2. NCCL all-gather of the P x m per-rank bucket counts (u64), computed on
 *      the device from the local offsets; the count matrix is copied to the
 *      host -- the ONE point where the call synchronises `stream` (the piece
 *      sizes are host arguments of the NCCL point-to-point calls);
 *   3. ms_dist_pieces (above): global bucket starts, this rank's balanced
 *      window [win_start, win_start + win_len) and its <= m+P-1 pieces;
 *   4. one NCCL group of send/recv over NVLink/NVSwitch (pieces to self by
 *      device copies) landing every piece at its final offset in the owner's
 *      window -- no receive-side permutation.
 * Every rank calls it with the same plan spec; rank and P come from `comm`
 * (an ncclComm_t, e.g. from ms_nccl_comm_init), whose device the call runs on.
 * keys_in/vals_in/ids: this rank's shard (n_local elements, device); keys_out
 * / vals_out: this rank's window buffers of out_capacity elements (device; the
 * window length is at most ceil(N/P) for N = total elements), written in
 * [0, win_len).  offsets_global (HOST, m+1 u64, or NULL): global bucket
 * starts; win_start / win_len (HOST, or NULL).  The output is complete when
 * `stream` completes; the concatenation of the windows over ranks is the
 * single-GPU stable multisplit of the concatenated shards (rank order).
 * Workspace: ms_dist_workspace_size.  Errors: argument errors as ms_run, plus
 * MS_ERR_INVALID_ARG if the window exceeds out_capacity (checked after the
 * count exchange, before any data moves) and MS_ERR_NCCL if NCCL cannot be
 * loaded (libnccl.so.2, dlopen'ed at first use) or a call fails.
 * ------------------------------------------------------------------------- */
ms_status ms_dist_workspace_size(ms_plan_t plan, uint64_t n_local, int32_t nranks, size_t *bytes);
ms_status ms_dist_run(ms_plan_t plan, void *nccl_comm, const uint32_t *keys_in, const uint32_t *vals_in,
                      const void *ids, uint64_t n_local, uint32_t *keys_out, uint32_t *vals_out,
                      uint64_t out_capacity, uint64_t *offsets_global, uint64_t *win_start, uint64_t *win_len,
                      void *workspace, size_t workspace_bytes, void *stream);

/* ---------------------------------------------------------------------------
 * ms_dist_run_fused -- the same collective with the exchange fused into the
 * post-scan: local K1 + K2 (ms_prescan / ms_scan), the NCCL
 * all-gather of the counts (the one host synchronisation), ms_dist_targets,
 * then ONE post-scan kernel (ms_postscan_scatter) that stores every bucket run
 * straight into the owning rank's window -- over NVLink / NVSwitch when
 * keys_windows[r] / vals_windows[r] are peer mappings of rank r's window
 * buffers (e.g. torch symmetric memory); finally a one-word NCCL all-reduce on
 * `stream` as the barrier after which every window is complete.  No local
 * output and no staging copy: 12 / 20 B per key of HBM + NVLink traffic.
 * keys_windows / vals_windows: HOST arrays of P device pointers valid on this
 * GPU, each window holding window_capacity elements (MS_ERR_INVALID_ARG if a
 * window is too small for its balanced share, checked before any store).
 * m <= 32 and a computed bucket kind (else MS_ERR_UNSUPPORTED); P <=
 * MS_MAX_PEERS.  Workspace: ms_dist_workspace_size_fused.  Other arguments and
 * errors as ms_dist_run.
 * ------------------------------------------------------------------------- */
ms_status ms_dist_workspace_size_fused(ms_plan_t plan, uint64_t n_local, int32_t nranks, size_t *bytes);
ms_status ms_dist_run_fused(ms_plan_t plan, void *nccl_comm, const uint32_t *keys_in, const uint32_t *vals_in,
                            uint64_t n_local, uint32_t *const *keys_windows, uint32_t *const *vals_windows,
                            uint64_t window_capacity, uint64_t *offsets_global, uint64_t *win_start,
                            uint64_t *win_len, void *workspace, size_t workspace_bytes, void *stream);

/* NCCL bootstrap for ms_dist_run (the 128-byte unique id travels between the
 * processes by any means, e.g. a torch.distributed broadcast):
 * ms_nccl_get_unique_id writes NCCL_UNIQUE_ID_BYTES (128) bytes to `id` (rank 0);
 * ms_nccl_comm_init makes `device` current and creates rank `rank` of an
 * nranks-rank communicator (*comm = the ncclComm_t); ms_nccl_comm_destroy
 * frees it.  MS_ERR_NCCL if NCCL cannot be loaded or fails. */
ms_status ms_nccl_get_unique_id(void *id);
ms_status ms_nccl_comm_init(void **comm, int32_t nranks, int32_t rank, const void *id, int device);
ms_status ms_nccl_comm_destroy(void *comm);
ms_status ms_postscan_scatter(ms_plan_t plan, const uint32_t *keys_in, const uint32_t *vals_in,
                              const uint32_t *G, uint64_t n, const ms_scatter_target *target, void *workspace,
                              size_t workspace_bytes, void *stream);

#ifdef __cplusplus
}
#endif
#endif /* MS_H */
