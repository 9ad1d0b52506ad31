/*
 * tid.h — C ABI of the B200-native texture-identification hot path.
 *
 * Method: Wang, Zhang, Li, Lin, "Exploring HW/SW Co-Optimizations for
 * Accelerating Large-scale Texture Identification on Distributed GPUs",
 * ICPP'21.  Citations are PAPER.md line numbers (P:a-b).
 *
 * What the library computes (exact integer arithmetic, bit-identical to the
 * definition):
 *   d(q_j, r_i)  = sum_t (q_jt - r_it)^2 over d = 128 u8 dims     (Eq. 1)
 *   2-NN of every QUERY keypoint over ONE reference image           (Alg. 1 step 5 P:377)
 *   ratio test   den^2 * d1 < num^2 * d2  (strict)
 *   count(q, r)  = number of query keypoints passing the ratio test
 *   search       = count against every reference, rank by (count desc, global id asc),
 *                  return the first k
 * Ties in the 2-NN go to the lowest reference-keypoint index; a reference with
 * fewer than 2 keypoints never matches.  Readings are listed in DESIGN.md.
 *
 * Conventions (every entry point):
 *   - Status codes only; nothing throws across the ABI.  On failure the
 *     thread-local message is available from tid_last_error().
 *   - The caller owns every input and output buffer.  Buffers may be HOST
 *     (pageable or pinned) or DEVICE memory of the index's device; the library
 *     classifies each pointer (cudaPointerGetAttributes) and copies as needed.
 *   - `stream` is a cudaStream_t passed as void* (NULL = legacy default stream).
 *     Device outputs are valid once `stream` completes; host outputs are valid
 *     when the call returns (the call synchronises the stream).
 *   - One index per host thread; an index is not thread-safe.  Successive calls on one index
 *     may pass different streams: each call's work is ordered after the previous call's
 *     (the index records an event at the end of every call and the next call waits on it).
 *   - The library requires an sm_100a device (B200): TID_EUNSUPPORTED otherwise.
 *     There is no CPU fallback.
 */
#ifndef TID_H_
#define TID_H_

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct tid_index tid_index; /* opaque; owns all device + pinned memory it allocates */

typedef enum {
  TID_OK = 0,
  TID_EINVAL = -1,        /* bad argument (message says which)                       */
  TID_ENOMEM = -2,        /* device / pinned allocation failed or capacity exceeded  */
  TID_ECUDA = -3,         /* CUDA runtime / driver error                             */
  TID_ENCCL = -4,         /* NCCL error                                              */
  TID_EUNSUPPORTED = -5,  /* device is not sm_100 (tcgen05 kind::i8 needs sm_100a)   */
  TID_ESTATE = -6         /* call not valid in the index's current state            */
} tid_status;

typedef struct {
  int32_t  device;             /* CUDA device ordinal                                             */
  int32_t  dim;                /* descriptor length d; must be 128 (SIFT)              */
  int32_t  ref_kp;             /* m: stored keypoints per reference, 2..1024 (asymmetric budgets,
                                  §7); rows beyond a reference's own count are padding */
  int32_t  query_kp_max;       /* largest n a search/verify call may pass, 1..8192                */
  uint32_t ratio_num;          /* ratio threshold num/den, each 1..65535 (0.8 = 4/5)   */
  uint32_t ratio_den;
  uint64_t hbm_budget_bytes;   /* reference descriptor bytes kept resident in HBM (level-1 cache,
                                  §6.1); 0 = auto (free HBM minus 8 GiB workspace).
                                  Each resident reference additionally holds ceil(ref_kp/256) KiB
                                  of column terms (W = 256 sum r - N_R per keypoint).             */
  uint64_t host_budget_bytes;  /* pinned host tier capacity in bytes (level-2 cache); 0 = none    */
  int64_t  id_base;            /* global id of this rank's first reference (shard offset)         */
  int32_t  rank;               /* this process's rank; 0 when world_size == 1                     */
  int32_t  world_size;         /* number of shards (GPUs); 1 = single GPU                         */
  const void* nccl_unique_id;  /* 128-byte ncclUniqueId (same on all ranks); required when
                                  world_size > 1.  Given with world_size == 1, a one-rank NCCL
                                  communicator runs the same all-gather + merge path (tests).   */
  int32_t  cache_policy;       /* 0 = fill: HBM first, then the host tier (ids in insertion order);
                                  1 = FIFO (§6.1): every new batch enters HBM and the
                                  oldest batches are swapped out to the host tier when HBM is full */
  int32_t  descriptor;         /* 0 = u8 SIFT, exact integer path (default);
                                  1 = the paper's float path (SURVEY row f1, §4.2, §5.1
                                  P:555-576): u8 SIFT given to add/search is converted on the GPU
                                  to [RootSIFT] x f16_scale in fp16 and stored that way (2 B per
                                  value + 8 KiB of norm terms per 256 keypoints); matching on
                                  tcgen05.mma.kind::f16 (see tid_f16_search_counts for the
                                  arithmetic and the +-1 count acceptance).  ref_kp <= 512;
                                  save / load and tid_verify stay on the u8 path.              */
  float    f16_scale;          /* descriptor 1: scale factor before the fp16 conversion (0 = 1)  */
  int32_t  f16_rootsift;       /* descriptor 1: 1 = RootSIFT (L1-normalise, sqrt) first          */
} tid_config;

/* Create an index on cfg->device.  Allocates the HBM arena lazily (on first add).
 * With world_size > 1 this is collective: every rank must call it (NCCL init). */
tid_status tid_index_create(const tid_config* cfg, tid_index** out);

/* Release every device / pinned buffer and the NCCL communicator.  NULL is a no-op. */
tid_status tid_index_destroy(tid_index* idx);

/*
 * Append `count` references (offline ingest, Alg. 1 step 1 P:372).
 *   desc       : u8 [count][ref_kp][128], host or device.  Row i of reference r is
 *                keypoint i; rows >= kp_counts[r] are ignored (zeroed in the arena).
 *   kp_counts  : int32 [count] keypoints per reference (0..ref_kp), host or device;
 *                NULL = every reference has ref_kp keypoints.  A reference with < 2
 *                keypoints is stored but can never match (count 0).
 *   first_local_id (out, nullable): local index of the first appended reference;
 *                its global id is cfg.id_base + local index.
 * References go to HBM until hbm_budget_bytes, then to the pinned host tier until
 * host_budget_bytes (FIFO order preserved).  All-or-nothing: on any error (TID_ENOMEM,
 * TID_ECUDA, ...) no reference is added and ids are unchanged (under cache_policy FIFO, batches
 * already swapped out to the host tier to make room stay there: tier placement only, never
 * results).
 * The squared norms N_R are computed here and kept in HBM.
 */
tid_status tid_add_references(tid_index* idx, const uint8_t* desc, const int32_t* kp_counts,
                              int64_t count, int64_t* first_local_id);

/*
 * Zero-copy fill of the pinned host tier (level-2 of the hybrid cache, §6.1; pinned
 * rather than pageable host memory, Table 5): appends `count` references that live in
 * the host tier and returns, in *desc_out, a pointer to their pinned storage
 * u8 [count][ref_kp][128] (initialised to zeros = references that match nothing), which the
 * caller fills in place — no staging copy (descriptor 1: fp16 [count][ref_kp][128] values,
 * already RootSIFT / scaled).  Every reference has ref_kp keypoints.  Contents are
 * read when a search streams the tier, so they must be written before the next search; the
 * pointer stays valid until tid_index_destroy.  first_local_id as in tid_add_references.
 * Errors: TID_EINVAL (count < 1, null desc_out), TID_ENOMEM (host budget exceeded),
 * TID_ESTATE (cache_policy FIFO: its host tier holds evicted batches only).
 */
tid_status tid_host_tier_map(tid_index* idx, int64_t count, uint8_t** desc_out, int64_t* first_local_id);

/*
 * Index lifecycle (the service's delete / update calls; persistence).
 *   tid_delete_references: the given local ids score 0 and are never ranked again.
 *   tid_update_references: replace the descriptors (u8 [count][ref_kp][128], host or device)
 *                          and keypoint counts (nullable = ref_kp) of existing local ids in
 *                          place (un-deletes them).
 *   tid_index_save / tid_index_load: binary file of every reference (descriptors with padding
 *                          rows zeroed, keypoint counts, deleted flags) in local-id order; load
 *                          appends to an index with the same ref_kp (its own budgets / policy).
 */
tid_status tid_delete_references(tid_index* idx, const int64_t* local_ids, int64_t count);
tid_status tid_update_references(tid_index* idx, const int64_t* local_ids, const uint8_t* desc,
                                 const int32_t* kp_counts, int64_t count);
tid_status tid_index_save(const tid_index* idx, const char* path);
tid_status tid_index_load(tid_index* idx, const char* path, int64_t* first_local_id);

/*
 * One-to-many search, batched over B queries.
 *   queries          : u8 [B][n][128], host or device; n <= query_kp_max.
 *   n_q              : int32 [B] valid keypoints per query (<= n), host or device; NULL = all n.
 *   k                : 1..64 and k <= total references over all ranks, else TID_EINVAL on every
 *                      rank (with world_size > 1 the total is all-reduced first, so all ranks
 *                      decide alike).  Deleted references are never ranked: if fewer than k
 *                      live references exist, the tail is id -1, count 0.
 *                      A rank whose shard is empty still takes part (it contributes no
 *                      candidates); TID_ESTATE only when no rank holds a reference.
 *   ref_ids_out      : int64 [B][k]  global reference ids, rank order (count desc, id asc).
 *   match_counts_out : int32 [B][k]  their good-match counts.
 * With world_size > 1 the call is collective: every rank passes the same queries
 * and receives the same merged result (one NCCL all-gather of B*k candidates).
 * Repeated calls with the same device buffers and shape (world_size 1, references in HBM, no
 * profiling) replay a CUDA graph captured on the second such call; any change of the index
 * invalidates it.  Results are identical either way.
 */
tid_status tid_search(tid_index* idx, const uint8_t* queries, const int32_t* n_q, int32_t n,
                      int64_t B, int32_t k, int64_t* ref_ids_out, int32_t* match_counts_out,
                      void* stream);

/*
 * Parity/debug entry: the full local count matrix of a search (this rank's references only).
 *   counts_out : uint32 [B][num_local_references], host or device.
 */
tid_status tid_search_counts(tid_index* idx, const uint8_t* queries, const int32_t* n_q, int32_t n,
                             int64_t B, uint32_t* counts_out, void* stream);

/*
 * One-to-one verification of P independent pairs.
 * Does not touch the index's references (uses its ratio, device and workspace).
 *   q      : u8 [P][n][128], r : u8 [P][m][128] (host or device); n <= query_kp_max, 2 <= m <= 1024.
 *   n_q    : int32 [P] valid query rows per pair (nullable = n);
 *   m_r    : int32 [P] valid reference rows per pair (nullable = m).
 *   counts_out : uint32 [P] good-match counts.
 *   nn_out : nullable int32 [P][n][4] = (d1, i1, d2, i2) per query row, the exact
 *            squared distances and reference-keypoint indices of the two nearest
 *            neighbours (Alg. 1 step 8's 2 x n output); a missing
 *            neighbour (m_r < 2) is (-1, -1).  Rows >= n_q[p] are written as (-1, -1, -1, -1).
 * Without nn_out the counts come from the search path's folded arithmetic (s8 x u8 + norm K-step) run
 * on the pairs (same exact results).  For n > 256 the pairs stream through one persistent kernel that
 * also computes N_Q and the reference norms on chip (no preparation pass).
 * Errors: TID_EINVAL for null pointers or sizes out of range (nothing launched); TID_ECUDA / TID_ENOMEM
 * from the device.
 */
tid_status tid_verify(tid_index* idx, const uint8_t* q, int32_t n, const uint8_t* r, int32_t m,
                      int64_t P, const int32_t* n_q, const int32_t* m_r,
                      uint32_t* counts_out, int32_t* nn_out, void* stream);

/*
 * Post-match verification: one-to-one verification followed by the
 * paper's outlier removal, "the geometric verification is performed to remove the outliers that
 * may be mismatched" (§3.1) and "edge feature removing" (§4.1).  The paper
 * defines neither step; the readings (R14-R16) are:
 *   edge-feature removal: a good match (ratio test passed) is dropped when its query keypoint or
 *     its nearest reference keypoint lies within `border` px of its image's edge (x < border,
 *     y < border, x >= width - border or y >= height - border);
 *   geometric verification: a 2-D similarity X = a x - b y + tx, Y = b x + a y + ty from query to
 *     reference coordinates, fitted exactly to 2 matches per hypothesis; a match is an inlier
 *     when its squared reprojection error is < inlier_px^2; RANSAC over `iterations` hypotheses
 *     drawn with a counter-based generator (splitmix64 of seed, pair index and hypothesis
 *     index), or every pair of matches when iterations == 0; the best hypothesis has the most
 *     inliers, ties to the earliest.  Matches are taken in query-keypoint order.  Geometry is
 *     IEEE fp64 with every operation rounded separately, so results are deterministic.
 * Arguments as tid_verify, plus:
 *   q_xy : float [P][n][2] query keypoint (x, y) in pixels; r_xy : float [P][m][2] (host or device).
 *   counts_out  (nullable) uint32 [P]: ratio-test matches (= tid_verify's counts);
 *   good_out    uint32 [P]: matches left after edge-feature removal;
 *   inliers_out uint32 [P]: inliers of the best hypothesis (0 when fewer than 2 matches remain);
 *   model_out   (nullable) double [P][4]: (a, b, tx, ty) of the best hypothesis (zeros if none).
 * Errors: TID_EINVAL (null pointers, inlier_px <= 0, border < 0, iterations < 0, as tid_verify).
 */
typedef struct {
  float border;                      /* edge margin in pixels (0 = only points outside the image)   */
  float query_width, query_height;   /* query image extent in pixels                                  */
  float ref_width, ref_height;       /* reference image extent in pixels                              */
  float inlier_px;                   /* inlier threshold on the reprojection distance, pixels (> 0)  */
  int32_t iterations;                /* RANSAC hypotheses; 0 = exhaustive over all match pairs        */
  uint64_t seed;                     /* generator seed                                                */
} tid_geom_params;

tid_status tid_verify_geometric(tid_index* idx, const uint8_t* q, int32_t n, const uint8_t* r, int32_t m,
                                int64_t P, const int32_t* n_q, const int32_t* m_r, const float* q_xy,
                                const float* r_xy, const tid_geom_params* params, uint32_t* counts_out,
                                uint32_t* good_out, uint32_t* inliers_out, double* model_out, void* stream);

/*
 * Shard merge: merge G ranked lists per query into one.
 *   ids_in/counts_in : [G][B][k] (int64 / int32), host or device, each list in rank order.
 *   ids_out/counts_out : [B][k] in (count desc, id asc) order.
 * Used internally after the NCCL all-gather; exported so a single GPU can run G
 * virtual shards and prove merge == single-GPU.
 */
tid_status tid_merge_topk(tid_index* idx, const int64_t* ids_in, const int32_t* counts_in,
                          int32_t G, int64_t B, int32_t k, int64_t* ids_out, int32_t* counts_out,
                          void* stream);

/*
 * Float-descriptor path (the paper's RootSIFT + FP16 configuration,
 * §4.2, §5.1, Algorithm 2).  Uses the index only for its
 * device, ratio and workspace; references are passed per call (not stored).
 *
 * tid_f16_prepare: u8 SIFT [rows][128] (host or device) -> fp16 bits [rows][128] (host or device):
 *   rootsift != 0: x / sum(x), element-wise sqrt (RootSIFT; all-zero rows stay 0);
 *   then multiply by `scale` (> 0; the paper's fp16 scale factor, 2^-7 in practice, P:504-507,
 *   P:527-530) and round to nearest even.  Computed in fp32 on the GPU.
 *
 * tid_f16_search_counts: good-match counts of B fp16 queries [B][n][128] against R fp16 references
 *   [R][m][128] (host or device; n <= query_kp_max, 2 <= m <= 512) -> counts_out uint32 [B][R].
 *   The product q.r runs on tcgen05.mma.kind::f16 with fp32 accumulation; a ninth K-step adds
 *   C - N_R / 2 (N_R in fp32 from the fp16 values, split into three fp16 terms; C = power of two
 *   >= max N_R / 2), so d = N_Q + 2C - 2 X with X = C + q.r - N_R / 2 >= 0 read straight from the
 *   accumulator; 2-NN per query row; ratio test den^2 * d1 < num^2 * d2 with d computed and
 *   compared in fp64 from the fp32 X.  Counts equal the exact float64 definition
 *   on the same fp16 values except where fp32 rounding moves a ratio across the threshold
 *   (acceptance: within +-1 for >= 99.9% of pairs; exact for u8 SIFT x 2^-k).
 */
tid_status tid_f16_prepare(tid_index* idx, const uint8_t* sift, int64_t rows, int32_t rootsift, float scale,
                           uint16_t* out, void* stream);
tid_status tid_f16_search_counts(tid_index* idx, const uint16_t* q, int32_t n, int64_t B, const uint16_t* r,
                                 int32_t m, int64_t R, uint32_t* counts_out, void* stream);

/* 128-byte ncclUniqueId for rank 0 to broadcast before tid_index_create. */
tid_status tid_nccl_unique_id(void* out128);

typedef struct {
  int64_t num_references;      /* local references (HBM + host tier)                 */
  int64_t hbm_references;      /* resident in the HBM arena                          */
  int64_t host_references;     /* in the pinned host tier (streamed per search)      */
  int64_t hbm_bytes;           /* device bytes allocated by the index                */
  int64_t host_bytes;          /* pinned host bytes allocated by the index           */
  int32_t num_sms;
  int32_t world_size;          /* shards; with an NCCL communicator, ncclCommCount's rank count */
  int64_t hbm_capacity_references;  /* references the HBM budget holds (resident tier capacity) */
  int64_t host_capacity_references; /* references the pinned host budget holds                  */
  int64_t hbm_bytes_per_reference;  /* HBM bytes one resident reference occupies (descriptors +
                                       per-keypoint norm terms + column terms)                   */
} tid_info;

tid_status tid_get_info(const tid_index* idx, tid_info* out);

/*
 * Kernel timing (CUDA events recorded on the stream each kernel is launched on).
 * enable != 0 starts recording and clears the accumulators.
 */
typedef struct {
  int64_t match_launches;      /* fused TMA->tcgen05->top-2->ratio->count kernel launches */
  double  match_ms;            /* summed device time of those launches                    */
  int64_t kernel_launches;     /* all kernels of this library launched while enabled      */
  int64_t h2d_bytes;           /* host->device bytes copied by the library                */
  int64_t d2h_bytes;           /* device->host bytes copied by the library                */
} tid_stats;

tid_status tid_profile(tid_index* idx, int32_t enable);
tid_status tid_get_stats(tid_index* idx, tid_stats* out); /* synchronises recorded events */

/* Tuning knobs (0 = automatic).  refs_per_job: references resident per CTA job (1..4);
 * grid: persistent CTAs for the match kernel; host_chunk_refs: references per
 * host-tier staging buffer; window_refs: references per count window of tid_search
 * (automatic: the whole local set while its B x R u32 count matrix fits 512 MiB, else
 * 512 MiB / (4 B) references; each window's counts are reduced into a running top-k, so the
 * search workspace does not grow with R).  Results never depend on these knobs. */
typedef struct {
  int32_t refs_per_job;
  int32_t grid;
  int64_t host_chunk_refs;
  int64_t window_refs;
} tid_tuning;

tid_status tid_set_tuning(tid_index* idx, const tid_tuning* t);

/* Thread-local message describing the last non-OK status of this thread ("" if none). */
const char* tid_last_error(void);

#ifdef __cplusplus
}
#endif

#endif /* TID_H_ */
