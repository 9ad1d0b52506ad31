// tid_kernels.cuh — sm_100a device code for the texture-identification hot path.
//
// Kernels:
//   ref_prep_kernel    a1: zero padded reference rows, squared norms N_R -> packed column keys
//   query_prep_kernel  a2: squared norms N_Q per query row
//   match_kernel       a3+a4+a5: TMA -> tcgen05.mma.kind::i8 (u8 x u8 -> s32, TMEM) ->
//                      exact two-partition top-2 epilogue in registers -> integer ratio
//                      test -> count
//   topk_kernel        a6: per-(query, segment) top-k of the count matrix
//   merge_kernel       a6/a9: merge ranked candidate lists (segments or shards)
//
// Everything is integer.  No distance matrix is ever written to HBM (P:374-386
// materialised A in HBM; here the s32 accumulator lives only in TMEM).
#pragma once
#include <cstdint>
#include <cuda_runtime.h>
#include <cuda.h>

namespace tid {

constexpr int kDim = 128;          // SIFT descriptor length, bytes per keypoint row
constexpr int kBM = 128;           // query keypoints per MMA tile (TMEM lanes)
constexpr int kBN = 256;           // reference keypoints per chunk (MMA N, TMEM columns)
constexpr int kQStages = 3;        // query-tile ring
constexpr int kMaxSlots = 4;       // resident reference chunks per CTA
#ifndef TID_NG
#define TID_NG 3
#endif
#ifndef TID_NB
#define TID_NB 2
#endif
#ifndef TID_PIECE
#define TID_PIECE 64
#endif
constexpr int kNG = TID_NG;                    // epilogue groups of 4 warps (one per TMEM lane quarter)
constexpr int kPiece = TID_PIECE;              // accumulator columns per MMA piece (MMA N)
constexpr int kNB = TID_NB;                    // TMEM buffers per group
constexpr int kTmemBufs = kNG * kNB;           // 6 buffers of 64 columns (384 of the 512 allocated)
static_assert(kTmemBufs * kPiece <= 512, "TMEM has 512 columns");
constexpr int kPiecesPerChunk = kBN / kPiece;  // 4 pieces per 256-column reference chunk
constexpr int kEpiWarps = 4 * kNG;             // 12 epilogue warps, 3 per SMSP
constexpr int kNumThreads = 32 * (1 + kNG + kEpiWarps);  // w0 TMA, w1..w3 MMA (one per group), w4.. epilogue
constexpr uint32_t kQTileBytes = kBM * kDim;   // 16 KiB
constexpr uint32_t kRTileBytes = kBN * kDim;   // 32 KiB
constexpr int kColInts = kBN;                  // per chunk: 256 packed column keys
constexpr uint32_t kColBytes = kColInts * 4;   // 1 KiB per chunk
constexpr int32_t kSentinelNorm = (1 << 23) - 1;  // > 128*255^2: padded columns never win
constexpr int kXDim = 32;                      // bytes of the per-column norm-term operand (one MMA K-step)
constexpr uint32_t kXTileBytes = kBN * kXDim;  // 8 KiB per 256-column chunk

// Search path ("folded" norms).  With q' = q - 128 (s8) and r (u8),
//   S3 = sum_t q'_t r_t = S - 128 sum_t r_t,  W = sum_t r_t (256 - r_t) = 256 sum r - N_R >= 0,
//   d(q, r) = N_Q + N_R - 2S = N_Q - (2 S3 + W).
// A fifth MMA K-step adds E = floor(W / 2) (u8 digits of E against a constant u8 operand), so
// TMEM holds X = S3 + E and  d = N_Q - 2X - p,  p = W mod 2 in {0, 1}: the two LARGEST X of a
// row are its two nearest columns (ties broken by p), and d1, d2 are known to within 1.  Rows
// whose ratio decision the +-1 can flip are recomputed exactly (rare).  Column term array for
// search: W (>= 0) for real columns, -1 - kp(chunk) for padded ones.
//
// Packed column key (verify path), per 256-column chunk (global layout [ref][chunk][256] int32):
//   colkey[i] = N_R[i] * 256 + i   (i = index within the chunk).
// The epilogue forms key = colkey - 512 * S = 256 * (N_R - 2 q.r) + i with one IMAD, which
// orders exactly like (d_ji, i) for a fixed query row (Alg. 1 step 4 + lowest-index
// tie-break); keys are unique within a chunk, so the two smallest keys give (d1, i1, d2, i2).

enum : int { kModeSearch = 0, kModeVerify = 1 };

struct MatchParams {
  int32_t mode;
  int32_t n_jobs;
  int32_t refs_per_job;      // G: references resident per job (search); 1 (verify)
  int32_t cpr;               // 256-column chunks per reference (1..4)
  int32_t tiles_per_q;       // ceil(n / 128)
  int32_t num_q;             // queries in the launch (search: B; verify: P)
  int32_t q_per_job;         // search: queries per job (splits B across jobs); verify: 1
  int32_t n_qchunks;         // search: ceil(num_q / q_per_job)
  int64_t n_refs;            // references in this launch
  int64_t ref_map_base;      // index of the launch's first reference in the R tensor map
  const int32_t* colkey;     // [n_refs][cpr*256] packed column keys (launch-relative)
  const int32_t* nq;         // [num_q][tiles_per_q*128] squared query norms
  const int32_t* n_valid;    // [num_q] valid query rows (nullable = n_rows)
  const int32_t* m_valid;    // verify: [P] valid reference rows per pair (nullable = m)
  int32_t n_rows;            // stored rows per query (n)
  uint32_t* counts;          // search: [num_q][ldc] (+ col0); verify: [num_q]
  int64_t ldc;
  int64_t col0;
  int32_t* nn_out;           // verify: [num_q][n_rows][4] or null
  uint32_t num2, den2;       // ratio^2 = num2/den2
  // search (folded norms): exact fallback operands in global memory
  const uint8_t* qs;         // [num_q][n_rows][128] shifted queries q' = q ^ 0x80
  const uint8_t* rdesc;      // reference descriptors of the tensor map, [*][m][128] raw u8
  int32_t m;                 // stored rows per reference
  int32_t slot_banks;        // 2: jobs alternate between slots {0, 1} and {2, 3} (small batches: the next
                             //    job's references load while this one runs); else 1
};

struct RefPrepParams {
  uint8_t* desc;             // [count][m][128] destination (null = read-only, keys only)
  const uint8_t* src;        // optional source to copy from (null = in place)
  const int32_t* kp;         // [count] or null (= m)
  int32_t* colkey;           // [count][cpr][256]: packed keys (verify) or column terms (search)
  int32_t search;            // 1: search column terms W (the norm-term digits are expanded on chip
                             //    by the match kernel); 0: verify packed keys
  int64_t count;
  int32_t m;
  int32_t cpr;
};

void launch_ref_prep(const RefPrepParams& p, cudaStream_t s);
void launch_query_prep(const uint8_t* q, int64_t B, int32_t n, int32_t tiles_per_q, int32_t* nq,
                       uint8_t* qs, cudaStream_t s);
// fold = search path (s8 x u8 + on-chip norm-term K-step, counts); otherwise verify (exact 2-NN)
cudaError_t launch_match(const MatchParams& p, const CUtensorMap& qmap, const CUtensorMap& rmap, bool fold, int grid,
                         cudaStream_t s);
// one-to-one verification with pairs streamed through per-chunk reference slots (p.mode == kModeVerify,
// p.colkey == nullptr; fold = counts only through the folded norms)
cudaError_t launch_verify_stream(const MatchParams& p, const CUtensorMap& qmap, const CUtensorMap& rmap, bool fold,
                                 int grid, cudaStream_t s);
// ids_out / counts_out (optional): with segs == 1 the final ranking is written directly
// Candidate lists: cand_out holds lists_per_b lists of k keys per query; the launch's segments
// fill lists list0 .. list0 + segs - 1.
void launch_topk(const uint32_t* counts, int64_t B, int64_t R, int64_t ldc, int64_t id_base, int32_t k,
                 int32_t segs, const uint8_t* dead, uint64_t* cand_out, int32_t lists_per_b, int32_t list0,
                 cudaStream_t s, int64_t* ids_out = nullptr, int32_t* counts_out = nullptr);
// keys_out (optional) row stride keys_stride (0 = k); may alias list 0 of cand (in-place running merge:
// every block reads all its lists before writing).
void launch_merge(const uint64_t* cand, int32_t L, int64_t B, int32_t k, int64_t list_stride_b,
                  int64_t list_stride_l, uint64_t* keys_out, int64_t* ids_out, int32_t* counts_out,
                  cudaStream_t s, int64_t keys_stride = 0);
void launch_pack_lists(const int64_t* ids, const int32_t* counts, int64_t n, uint64_t* keys, cudaStream_t s);
size_t match_smem_bytes();

// f4 post-match verification (tid_geom.cu): edge-feature removal + 2-point similarity RANSAC
struct GeomParams {
  float border, qw, qh, rw, rh;  // edge margin (px) and the query / reference image extents
  float thr;                     // inlier threshold on the reprojection distance (px)
  int32_t iters;                 // hypotheses; <= 0: every pair (exhaustive)
  uint64_t seed;
  uint32_t num2, den2;           // ratio test den2 * d1 < num2 * d2
};
// nn [P][n][4] int32 (d1, i1, d2, i2) from the verify kernel; coordinates [P][n][2] / [P][m][2] float.
cudaError_t launch_geometric(const int32_t* nn, int32_t n, int32_t m, int64_t P, const int32_t* n_q,
                             const int32_t* m_r, const float* q_xy, const float* r_xy, const GeomParams& g,
                             uint32_t* good, uint32_t* inl, double* model, cudaStream_t s);

// f1 float path (tid_f16.cu)
size_t f16_smem_bytes();
cudaError_t launch_f16_prepare(const uint8_t* sift, int64_t rows, int32_t rootsift, float scale, void* out,
                               cudaStream_t s);
cudaError_t launch_f16_norms(const void* x, int64_t items, int32_t rows, int32_t rows_pad, float pad, float* out,
                             cudaStream_t s);
// norm-term operand [R][256 * ceil(m / 256)][16] fp16 of fp16 references [R][m][128] (m <= 512) and its
// constant C (device scalar)
cudaError_t launch_f16_xop(const void* r, int64_t R, int32_t m, uint32_t* scratch, float* nr, void* xop,
                           float* cterm, cudaStream_t s);
// counts[qi * ldc + col0 + r] for references rbase + r of the maps (ldc 0 = R)
cudaError_t launch_f16_match(const CUtensorMap& qmap, const CUtensorMap& rmap, const CUtensorMap& xmap,
                             const float* cterm, const float* nq, int32_t B, int32_t n, int32_t T, int64_t R,
                             uint32_t num2, uint32_t den2, uint32_t* counts, int num_sms, cudaStream_t s,
                             int64_t ldc = 0, int64_t col0 = 0, int64_t rbase = 0, const int32_t* n_valid = nullptr,
                             int32_t cpr = 1, int32_t m = 0);  // m: stored rows per reference (0 = cpr * 256)
// index path: norm-term rows with the index's fixed constant C and per-reference keypoint counts
cudaError_t launch_f16_xop_fixed(const void* r, int64_t R, int32_t m, const int32_t* kp, float C, float* nr, void* xop,
                                 cudaStream_t s);

}  // namespace tid
