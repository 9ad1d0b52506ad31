// tid_f16.cu — SURVEY §8 row f1: the paper's float-descriptor path on sm_100a.
//
//   prepare : SIFT u8 -> [RootSIFT (L1-normalise, element-wise sqrt; §5.1)] -> x * scale
//             (the fp16 scale factor, 2^-7 in practice; §4.2) -> fp16 (RNE).
//   match   : TMA -> tcgen05.mma.kind::f16 (fp16 x fp16 -> fp32 in TMEM; the paper's HGEMM, Alg. 2
//             step 1 P:648) -> epilogue d = N_Q + N_R - 2 q.r in fp32 (Alg. 1 / Eq. 1; for RootSIFT
//             N = 1 and this is Alg. 2's sqrt(2 + A) ordering) -> exact two-partition top-2
//             of d (non-negative fp32 orders like its bit pattern) -> ratio test den^2 d1 < num^2 d2
//             (compared in fp64) -> count per (query, reference).
//
// Folded norms (as in the integer path): a ninth K = 16 step adds, per reference keypoint, the
// constant C - N_R / 2 (three fp16 terms h1 + h2 + h3 against a constant A operand of ones), so
// TMEM holds X = C + q.r - N_R / 2 >= 0 and d = N_Q + 2C - 2X.  C is the smallest power of two
// >= max N_R / 2 of the launch, so X >= 0 and its fp32 bit pattern orders like its value: the
// epilogue scans raw TMEM words (two largest X = two nearest columns), with no per-element
// arithmetic.  Padded columns get h1 = -inf.  For u8 SIFT x 2^-k every term is exact.
//
// One CTA per job = (reference r, range of queries); warp 0 TMA producer, warp 1 MMA issuer,
// warps 2..9 epilogue: two warps per TMEM lane quarter, 16 lanes each (16x64b loads; a row's
// columns are split over a thread pair as even / odd columns).  The reference tile (256 keypoints
// x 128 fp16 = 64 KiB, two SWIZZLE_128B K-halves) and its 8 KiB norm-term tile stay in shared
// memory for the job; query tiles (128 x 128 fp16) stream through a 2-stage ring; the
// accumulator (128 x 256 fp32) is double-buffered in TMEM.
#include "tid_kernels.cuh"

#include <cuda_fp16.h>

#include <climits>

// Timing-experiment switches that skip work and give WRONG results (skeleton timings in DESIGN.md):
// refused unless the build says it is an experiment.
#if (defined(TID_NOSCAN) || defined(TID_NOMMA) || defined(TID_NOLOAD)) && !defined(TID_EXPERIMENT)
#error "TID_NOSCAN / TID_NOMMA / TID_NOLOAD skip work (wrong results): timing experiments only, add -DTID_EXPERIMENT"
#endif

namespace tid {
namespace f16 {

constexpr int kEpi = 8;                             // epilogue warps (2 per TMEM lane quarter)
constexpr int kThreads = 32 * (2 + kEpi);
constexpr int kHalfBytes = 128;                     // one SWIZZLE_128B row = 64 fp16
constexpr uint32_t kRHalf = kBN * kHalfBytes;       // 32 KiB: 256 reference rows x 64 fp16
constexpr uint32_t kQHalf = kBM * kHalfBytes;       // 16 KiB: 128 query rows x 64 fp16
constexpr int kXH = 16;                             // fp16 per norm-term row (one K = 16 step, 32 B)
constexpr uint32_t kXTile = kBN * kXH * 2;          // 8 KiB: 256 reference rows x 16 fp16
// MMA pieces of kFN = 128 columns through kFNB = 4 TMEM buffers (512 columns): a reference chunk
// of 256 keypoints is 2 pieces; global piece gp of the CTA uses buffer gp % 4 with phase
// (gp / 4) & 1, so with one chunk per reference the MMA runs up to 1.5 units ahead of the epilogue.
#ifndef TID_F16_N
#define TID_F16_N 128
#endif
constexpr int kFN = TID_F16_N;  // 256: one MMA per chunk through 2 buffers (B / A operand bytes per
                                // tensor cycle 96 instead of 128, the shared-memory port's width)
static_assert(kFN == 128 || kFN == 256, "MMA N");
constexpr int kFPieces = kBN / kFN;                 // pieces per 256-column chunk
constexpr int kFNB = 512 / kFN;                     // TMEM buffers

// Shared-memory plan for references of kCpr 256-row chunks (m <= 256 kCpr): the resident reference
// (kCpr x 64 KiB) and its norm-term tiles, a ring of query tiles (4 stages for one chunk, 2 for two:
// 227 KiB in all), the constant operand, barriers.
template <int kCpr>
struct Plan {
  static constexpr int kStages = kCpr == 1 ? 4 : 2;
  static constexpr uint32_t kR = 0;                                   // kCpr chunks x 2 K-halves
  static constexpr uint32_t kQ = kR + kCpr * 2 * kRHalf;              // kStages x 2 halves
  static constexpr uint32_t kX = kQ + kStages * 2 * kQHalf;           // kCpr norm-term tiles (SWIZZLE_32B)
  static constexpr uint32_t kAx = kX + kCpr * kXTile;                 // constant A operand (ones)
  static constexpr uint32_t kBar = kAx + kBM * kXH * 2;
  static constexpr uint32_t kQFull = kBar, kQEmpty = kBar + 8 * kStages;
  static constexpr uint32_t kRFull = kQEmpty + 8 * kStages, kREmpty = kRFull + 8;
  static constexpr uint32_t kTFull = kREmpty + 8, kTEmpty = kTFull + 8 * kFNB;
  static constexpr uint32_t kTmemPtr = kTEmpty + 8 * kFNB;
  static constexpr uint32_t kAlloc = kTmemPtr + 16 + 1024;
  static_assert(kAlloc <= 227 * 1024, "shared memory");
};

__device__ __forceinline__ uint32_t su32(const void* p) { return static_cast<uint32_t>(__cvta_generic_to_shared(p)); }
__device__ __forceinline__ void bar_init(uint32_t b, uint32_t c) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(b), "r"(c) : "memory");
}
__device__ __forceinline__ void bar_expect(uint32_t b, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(b), "r"(bytes) : "memory");
}
__device__ __forceinline__ void bar_arrive(uint32_t b) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(b) : "memory");
}
__device__ __forceinline__ void bar_wait(uint32_t b, uint32_t par) {
  asm volatile(
      "{\n\t.reg .pred P1;\n\tW:\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n\t"
      "@P1 bra D;\n\tbra W;\n\tD:\n\t}" ::"r"(b), "r"(par) : "memory");
}
__device__ __forceinline__ void tma3(uint32_t dst, const CUtensorMap* m, uint32_t bar, int c0, int c1, int c2) {
  asm volatile(
      "cp.async.bulk.tensor.3d.shared::cluster.global.tile.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4, %5}], [%2];"
      ::"r"(dst), "l"(reinterpret_cast<uint64_t>(m)), "r"(bar), "r"(c0), "r"(c1), "r"(c2) : "memory");
}
__device__ __forceinline__ void bulk(uint32_t dst, const void* src, uint32_t bytes, uint32_t bar) {
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
               ::"r"(dst), "l"(src), "r"(bytes), "r"(bar) : "memory");
}
__device__ __forceinline__ uint64_t desc128(uint32_t addr) {
  return static_cast<uint64_t>((addr & 0x3FFFF) >> 4) | (uint64_t(1) << 16) | (uint64_t(1024 >> 4) << 32) |
         (uint64_t(1) << 46) | (uint64_t(2) << 61);
}
// K-major SWIZZLE_32B (32-byte rows, 8-row groups 256 B apart): the norm-term operands.
__device__ __forceinline__ uint64_t desc32(uint32_t addr) {
  return static_cast<uint64_t>((addr & 0x3FFFF) >> 4) | (uint64_t(1) << 16) | (uint64_t(256 >> 4) << 32) |
         (uint64_t(1) << 46) | (uint64_t(6) << 61);
}
// kind::f16: D = F32 (bits 4-5 = 1), A = B = F16 (0), K-major, N = 256, M = 128.
constexpr uint32_t kIdesc = (1u << 4) | (uint32_t(kFN >> 3) << 17) | (uint32_t(kBM >> 4) << 24);

// D = Q . R^T over K = 128 fp16 (per K-half, one SWIZZLE_128B tile, four K = 16 steps of 32 B),
// then D += ones . (h1, h2, h3) (the norm-term step).
__device__ __forceinline__ void mma_unit(uint32_t d, uint64_t a0, uint64_t a1, uint64_t b0, uint64_t b1, uint64_t ax,
                                         uint64_t bx, uint32_t bar) {
  asm volatile(
      "{\n\t.reg .pred e, f, t;\n\t"
      "setp.ne.b32 f, 0, 0;\n\tsetp.eq.b32 t, 0, 0;\n\t"
      "elect.sync _|e, 0xffffffff;\n\t"
      "@e tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %3, %5, f;\n\t"
      "@e tcgen05.mma.cta_group::1.kind::f16 [%0], %7, %8, %5, t;\n\t"
      "@e tcgen05.mma.cta_group::1.kind::f16 [%0], %9, %10, %5, t;\n\t"
      "@e tcgen05.mma.cta_group::1.kind::f16 [%0], %11, %12, %5, t;\n\t"
      "@e tcgen05.mma.cta_group::1.kind::f16 [%0], %2, %4, %5, t;\n\t"
      "@e tcgen05.mma.cta_group::1.kind::f16 [%0], %13, %14, %5, t;\n\t"
      "@e tcgen05.mma.cta_group::1.kind::f16 [%0], %15, %16, %5, t;\n\t"
      "@e tcgen05.mma.cta_group::1.kind::f16 [%0], %17, %18, %5, t;\n\t"
      "@e tcgen05.mma.cta_group::1.kind::f16 [%0], %19, %20, %5, t;\n\t"
      "@e tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%6];\n\t}"
      ::"r"(d), "l"(a0), "l"(a1), "l"(b0), "l"(b1), "r"(kIdesc), "r"(bar),
        "l"(a0 + 2), "l"(b0 + 2), "l"(a0 + 4), "l"(b0 + 4), "l"(a0 + 6), "l"(b0 + 6),
        "l"(a1 + 2), "l"(b1 + 2), "l"(a1 + 4), "l"(b1 + 4), "l"(a1 + 6), "l"(b1 + 6), "l"(ax), "l"(bx)
      : "memory");
}
__device__ __forceinline__ void commit(uint32_t bar) {
  asm volatile("{\n\t.reg .pred e;\n\telect.sync _|e, 0xffffffff;\n\t"
               "@e tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];\n\t}" ::"r"(bar)
               : "memory");
}
#define F16_OUT32(v)                                                                                           \
  "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]), "=r"(v[7]), "=r"(v[8]),    \
      "=r"(v[9]), "=r"(v[10]), "=r"(v[11]), "=r"(v[12]), "=r"(v[13]), "=r"(v[14]), "=r"(v[15]), "=r"(v[16]),    \
      "=r"(v[17]), "=r"(v[18]), "=r"(v[19]), "=r"(v[20]), "=r"(v[21]), "=r"(v[22]), "=r"(v[23]), "=r"(v[24]),   \
      "=r"(v[25]), "=r"(v[26]), "=r"(v[27]), "=r"(v[28]), "=r"(v[29]), "=r"(v[30]), "=r"(v[31])
// 16 lanes x 128 columns (16x64b.x64): thread t holds lane (t >> 2) + 8 (t & 1) of the 16 and
// columns 2 i + ((t >> 1) & 1), i = 0..63 (tools/ld_shape_probe.cu).
__device__ __forceinline__ void ld16x64(uint32_t taddr, uint32_t (&v)[64]) {
  asm volatile(
      "tcgen05.ld.sync.aligned.16x64b.x64.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,%16,%17,%18,"
      "%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31,%32,%33,%34,%35,%36,%37,%38,%39,%40,%41,%42,%43,%44,"
      "%45,%46,%47,%48,%49,%50,%51,%52,%53,%54,%55,%56,%57,%58,%59,%60,%61,%62,%63}, [%64];"
      : F16_OUT32(v), F16_OUT32((v + 32)) : "r"(taddr));
  asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
#pragma unroll
  for (int i = 0; i < 64; ++i) asm volatile("" : "+r"(v[i]));
}

// Two-partition top-2 of the largest values (see tid_kernels.cu): P = 16-register halves of a
// 32-register block, P' = position mod 16; R[b] = P' maxima, T1 >= T2 = two largest P maxima.
__device__ __forceinline__ int mx3(int a, int b, int c) { return __vimax3_s32(a, b, c); }
__device__ __forceinline__ int mx16(const uint32_t* k) {
  const int a = mx3(k[0], k[1], k[2]), b = mx3(k[3], k[4], k[5]), c = mx3(k[6], k[7], k[8]);
  const int d = mx3(k[9], k[10], k[11]), e = mx3(k[12], k[13], k[14]);
  return max(mx3(a, b, c), mx3(d, e, static_cast<int>(k[15])));
}
__device__ __forceinline__ void scan32(const uint32_t* k, int (&R)[16], int& T1, int& T2) {
  const int x = mx16(k), y = mx16(k + 16);
#pragma unroll
  for (int b = 0; b < 16; ++b) R[b] = mx3(R[b], k[b], k[b + 16]);
  const int hi = max(x, y), lo = min(x, y);
  T2 = mx3(T2, min(T1, hi), lo);
  T1 = max(T1, hi);
}
__device__ __forceinline__ void finish(const int (&R)[16], int T1, int T2, int& x1, int& x2) {
  int rm[4], cm[4];
#pragma unroll
  for (int a = 0; a < 4; ++a) {
    rm[a] = max(mx3(R[4 * a], R[4 * a + 1], R[4 * a + 2]), R[4 * a + 3]);
    cm[a] = max(mx3(R[a], R[a + 4], R[a + 8]), R[a + 12]);
  }
  const int sr = mx3(min(max(rm[0], rm[1]), max(rm[2], rm[3])), min(rm[0], rm[1]), min(rm[2], rm[3]));
  const int sc = mx3(min(max(cm[0], cm[1]), max(cm[2], cm[3])), min(cm[0], cm[1]), min(cm[2], cm[3]));
  x1 = T1;
  x2 = mx3(T2, sr, sc);
}

// kSkip: the stored m leaves all-padding 128-column pieces (m = 384: the fourth), which are neither computed
// nor scanned; without it every loop keeps its static trip count (a run-time break cost 3 % at m = 256).
template <int kCpr, bool kSkip>
__global__ void __launch_bounds__(kThreads, 1)
    match_f16_kernel(const __grid_constant__ CUtensorMap qmap, const __grid_constant__ CUtensorMap rmap,
                     const __grid_constant__ CUtensorMap xmap, const float* __restrict__ cterm,
                     const float* __restrict__ nq_all, int32_t B, int32_t n, int32_t T, int64_t R, int32_t q_per_job,
                     uint32_t num2, uint32_t den2, uint32_t* __restrict__ counts, int64_t ldc, int64_t col0,
                     int64_t rbase, const int32_t* __restrict__ n_valid, int32_t m_rows) {
  using P = Plan<kCpr>;
  // pieces of kFN columns that can hold reference keypoints (rows >= m_rows are padding for every
  // reference: m = 384, the paper's operating point, computes 3 of the 4 pieces of its two chunks)
  const int np_ref = kSkip ? min(kCpr * kFPieces, (m_rows + kFN - 1) / kFN) : kCpr * kFPieces;
  constexpr int kStages = P::kStages;
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  const uint32_t sb = su32(smem);
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  auto qfull = [&](int i) { return sb + P::kQFull + 8 * i; };
  auto qempty = [&](int i) { return sb + P::kQEmpty + 8 * i; };
  const uint32_t rfull = sb + P::kRFull, rempty = sb + P::kREmpty;
  auto tfull = [&](int i) { return sb + P::kTFull + 8 * i; };
  auto tempty = [&](int i) { return sb + P::kTEmpty + 8 * i; };
  uint32_t* tptr = reinterpret_cast<uint32_t*>(smem + P::kTmemPtr);
  {  // constant A operand of the norm-term step: every row (1, 1, 1, 0 x 5) in both 16-B halves,
     // so the SWIZZLE_32B layout does not matter
    uint32_t* ax = reinterpret_cast<uint32_t*>(smem + P::kAx);
    const uint32_t one2 = 0x3C003C00u, one0 = 0x00003C00u;  // fp16 pairs (1, 1), (1, 0)
    for (int i = threadIdx.x; i < kBM * kXH / 2; i += blockDim.x) {
      const int w = i & 3;  // 32-bit word within a 16-B half
      ax[i] = w == 0 ? one2 : (w == 1 ? one0 : 0u);
    }
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  }
  if (threadIdx.x == 0) {
    for (int i = 0; i < kStages; ++i) { bar_init(qfull(i), 1); bar_init(qempty(i), 1); }
    bar_init(rfull, 1);
    bar_init(rempty, 1 + kEpi);
    for (int i = 0; i < kFNB; ++i) { bar_init(tfull(i), 1); bar_init(tempty(i), kEpi); }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (warp == 1) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 512;" ::"r"(su32(tptr)) : "memory");
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
  }
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
  const uint32_t tmem = *tptr;
  const int64_t qchunks = (B + q_per_job - 1) / q_per_job;
  const int64_t n_jobs = R * qchunks;

  if (warp == 0) {
    if (lane == 0) {
      uint32_t qc = 0, rc = 0;
      for (int64_t j = blockIdx.x; j < n_jobs; j += gridDim.x, ++rc) {
        const int64_t r = j / qchunks;
        const int q0 = static_cast<int>(j % qchunks) * q_per_job, nq = min(q_per_job, B - q0);
        bar_wait(rempty, (rc & 1) ^ 1);
        bar_expect(rfull, kCpr * (2 * kRHalf + kXTile));
#pragma unroll
        for (int c = 0; c < kCpr; ++c) {  // chunk c: reference rows 256 c .. (both K-halves) + norm terms
          tma3(sb + P::kR + c * 2 * kRHalf, &rmap, rfull, 0, c * kBN, static_cast<int>(rbase + r));
          tma3(sb + P::kR + c * 2 * kRHalf + kRHalf, &rmap, rfull, 64, c * kBN, static_cast<int>(rbase + r));
          tma3(sb + P::kX + c * kXTile, &xmap, rfull, 0, c * kBN, static_cast<int>(rbase + r));
        }
        for (int t = 0; t < nq * T; ++t, ++qc) {
          const int st = qc % kStages;
          bar_wait(qempty(st), ((qc / kStages) & 1) ^ 1);
          bar_expect(qfull(st), 2 * kQHalf);
          const uint32_t dst = sb + P::kQ + st * 2 * kQHalf;
          tma3(dst, &qmap, qfull(st), 0, (t % T) * kBM, q0 + t / T);
          tma3(dst + kQHalf, &qmap, qfull(st), 64, (t % T) * kBM, q0 + t / T);
        }
      }
    }
  } else if (warp == 1) {
    uint32_t qc = 0, rc = 0, gp = 0;  // gp: global piece counter (buffer gp % 4, phase (gp / 4) & 1)
    const uint64_t ax = desc32(sb + P::kAx);
    for (int64_t j = blockIdx.x; j < n_jobs; j += gridDim.x, ++rc) {
      const int q0 = static_cast<int>(j % qchunks) * q_per_job, nq = min(q_per_job, B - q0);
      bar_wait(rfull, rc & 1);
      for (int t = 0; t < nq * T; ++t, ++qc) {
        const int st = qc % kStages;
        bar_wait(qfull(st), (qc / kStages) & 1);
        const uint32_t qa = sb + P::kQ + st * 2 * kQHalf;
#pragma unroll
        for (int c = 0; c < kCpr; ++c) {
          const uint64_t b0 = desc128(sb + P::kR + c * 2 * kRHalf), b1 = desc128(sb + P::kR + c * 2 * kRHalf + kRHalf);
          const uint64_t bx = desc32(sb + P::kX + c * kXTile);
#pragma unroll
          for (int h = 0; h < kFPieces; ++h) {
            if (kSkip && c * kFPieces + h >= np_ref) break;  // all-padding piece: neither computed nor scanned
            const int buf = gp % kFNB;
            bar_wait(tempty(buf), ((gp / kFNB) & 1) ^ 1);
            asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
#ifdef TID_NOMMA  // timing experiment only
            commit(tfull(buf));
#else
            // reference rows kFN * h.. : SWIZZLE_128B 8-row groups of 1 KiB / SWIZZLE_32B groups of 256 B
            mma_unit(tmem + buf * kFN, desc128(qa), desc128(qa + kQHalf), b0 + h * (kFN * 128 >> 4),
                     b1 + h * (kFN * 128 >> 4), ax, bx + h * (kFN * 32 >> 4), tfull(buf));
#endif
            ++gp;
          }
        }
        commit(qempty(st));
      }
      commit(rempty);
    }
  } else {
    // warps 2..9: lane quarter warp % 4, 16-lane half (warp - 2) / 4
    const int quarter = warp & 3, half = (warp - 2) >> 2;
    const uint32_t tq = tmem + (static_cast<uint32_t>(quarter * 32 + 16 * half) << 16);
    const int row_in_tile = quarter * 32 + 16 * half + (lane >> 2) + 8 * (lane & 1);
    const double c2 = 2.0 * static_cast<double>(*cterm);
    const float c2f = static_cast<float>(c2);  // 2C: a power of two, exact in fp32
    const float den2f = static_cast<float>(den2), num2f = static_cast<float>(num2);  // small integers, exact
    uint32_t rc = 0, gp = 0;
    uint32_t v[64];
    for (int64_t j = blockIdx.x; j < n_jobs; j += gridDim.x, ++rc) {
      const int64_t r = j / qchunks;
      const int q0 = static_cast<int>(j % qchunks) * q_per_job, nq = min(q_per_job, B - q0);
      bar_wait(rfull, rc & 1);
      uint32_t cnt = 0;
      int qi = q0, tt = 0;  // query and tile of unit t (no divisions per unit)
      int nv = n_valid ? min(n_valid[qi], n) : n;
      for (int t = 0; t < nq * T; ++t) {
        const int row = tt * kBM + row_in_tile;
        const bool valid = row < nv;
        const float nqv = nq_all[static_cast<int64_t>(qi) * T * kBM + row];
        int Rm[16];
#pragma unroll
        for (int b = 0; b < 16; ++b) Rm[b] = INT_MIN;
        int T1 = INT_MIN, T2 = INT_MIN;
        // every chunk's pieces into one two-partition state: two columns of different loads are in
        // different P groups, two of one load differ in position mod 16, so the top-2 stays exact
#pragma unroll
        for (int pc = 0; pc < kCpr * kFPieces; ++pc, ++gp) {  // one x64 load per 128 columns of a piece
          if (kSkip && pc >= np_ref) break;  // all-padding piece (not computed)
          const int buf = gp % kFNB;
          bar_wait(tfull(buf), (gp / kFNB) & 1);
          asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
#pragma unroll
          for (int l = 0; l < kFN / 128; ++l) {
            ld16x64(tq + buf * kFN + l * 128, v);
            if (l == kFN / 128 - 1) {  // the piece is in registers: buffer free
              asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
              __syncwarp();
              if (lane == 0) bar_arrive(tempty(buf));
            }
#ifndef TID_NOSCAN  // timing experiment only
            scan32(v, Rm, T1, T2);
            scan32(v + 32, Rm, T1, T2);
#endif
          }
        }
        int x1, x2;
        finish(Rm, T1, T2, x1, x2);
        {  // merge with the partner thread holding the row's other columns
          const int o1 = __shfl_xor_sync(0xffffffffu, x1, 2), o2 = __shfl_xor_sync(0xffffffffu, x2, 2);
          x2 = mx3(min(x1, o1), x2, o2);
          x1 = max(x1, o1);
        }
        // d = N_Q + 2C - 2X (clamped at 0; padded columns have X < 0) and the ratio test
        // den^2 d1 < num^2 d2, decided exactly as in fp64 from these fp32 values (R10).
        // B200's fp64 pipe is narrow (fp64 here was ~30 % of the kernel's stall samples), so the sign of
        // den^2 d1 - num^2 d2 is first taken in fp32: its error is below 2^-20 (den^2 + num^2)(N_Q + 2C)
        // (d <= N_Q + 2C, a few roundings), so outside 8x that band the fp32 sign is the fp64 sign;
        // inside it (rare) the fp64 computation decides.
        bool pass = false;
        if (valid && x2 >= 0) {
          const float f1 = __int_as_float(x1), f2 = __int_as_float(x2);
          const float base = nqv + c2f;
          const float e1 = fmaxf(base - 2.0f * f1, 0.0f), e2 = fmaxf(base - 2.0f * f2, 0.0f);
          const float diff = fmaf(den2f, e1, -(num2f * e2));
          const float tol = 0x1p-17f * base * (den2f + num2f);
          if (diff < -tol) {
            pass = true;
          } else if (diff <= tol) {
            const double d1 = fmax(double(nqv) + c2 - 2.0 * double(f1), 0.0);
            const double d2 = fmax(double(nqv) + c2 - 2.0 * double(f2), 0.0);
            pass = double(den2) * d1 < double(num2) * d2;
          }
        }
        cnt += __popc(__ballot_sync(0xffffffffu, pass) & 0x33333333u);  // one thread per row
        if (++tt == T) {
          if (lane == 0 && cnt) atomicAdd(counts + static_cast<int64_t>(qi) * ldc + col0 + r, cnt);
          cnt = 0;
          tt = 0;
          ++qi;
          if (t + 1 < nq * T) nv = n_valid ? min(n_valid[qi], n) : n;
        }
      }
      __syncwarp();
      if (lane == 0) bar_arrive(rempty);
    }
  }
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  if (warp == 1) {
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 512;" ::"r"(tmem) : "memory");
  }
}

// Squared norm N_R (fp32) of every reference row, 8 lanes per row (each 32 contiguous bytes: the
// row's 256 bytes are read by one coalesced 8-lane group), plus the launch's largest N_R (fp32
// bits, non-negative: integer max).
__global__ void nr_rows_kernel(const __half* __restrict__ x, int64_t rows, float* __restrict__ nr,
                               uint32_t* __restrict__ max_bits) {
  const int64_t g = static_cast<int64_t>(blockIdx.x) * blockDim.x + threadIdx.x;
  const int64_t row = g >> 3;
  const int l8 = static_cast<int>(g & 7);
  float acc = 0.0f;
  if (row < rows) {
    const uint4* p = reinterpret_cast<const uint4*>(x + row * kDim) + 2 * l8;
#pragma unroll
    for (int w = 0; w < 2; ++w) {
      const uint4 u = p[w];
      const uint32_t words[4] = {u.x, u.y, u.z, u.w};
#pragma unroll
      for (int i = 0; i < 4; ++i) {
        const float2 f = __half22float2(*reinterpret_cast<const __half2*>(&words[i]));
        acc = fmaf(f.x, f.x, acc);
        acc = fmaf(f.y, f.y, acc);
      }
    }
  }
#pragma unroll
  for (int o = 1; o < 8; o <<= 1) acc += __shfl_xor_sync(0xffffffffu, acc, o);
  if (row < rows && l8 == 0) nr[row] = acc;
  float mx = row < rows ? acc : 0.0f;
#pragma unroll
  for (int o = 8; o < 32; o <<= 1) mx = fmaxf(mx, __shfl_xor_sync(0xffffffffu, mx, o));
  if ((threadIdx.x & 31) == 0 && max_bits) atomicMax(max_bits, __float_as_uint(mx));
}

// Norm-term rows [R][256][16] fp16: (h1, h2, h3, 0 ...) with h1 + h2 + h3 = C - N_R / 2 (three
// fp16 terms of the fp32 value, 33 significant bits), C = smallest power of two >= max N_R / 2;
// rows >= m: h1 = -inf.  Also writes C.  One thread per row (32 contiguous bytes out).
// fixed_c > 0: the index's constant (a bound on every N_R / 2 it can hold) instead of
// the launch's maximum; kp (nullable): rows >= kp[ref] are padding (h1 = -inf) like rows >= m.
__global__ void xop_kernel(const float* __restrict__ nr, int64_t R, int32_t m, const uint32_t* __restrict__ max_bits,
                           __half* __restrict__ xop, float* __restrict__ cterm, float fixed_c,
                           const int32_t* __restrict__ kp, int32_t rows_per_ref) {
  const int64_t g = static_cast<int64_t>(blockIdx.x) * blockDim.x + threadIdx.x;
  if (g >= R * rows_per_ref) return;
  float C = fixed_c;
  if (!(C > 0.0f)) {
    int e;
    frexpf(0.5f * __uint_as_float(*max_bits), &e);
    C = ldexpf(1.0f, e);  // > max N_R / 2 (or 1 if all norms are 0)
  }
  if (g == 0 && cterm) *cterm = C;
  const int64_t ref = g / rows_per_ref;
  const int row0 = static_cast<int>(g % rows_per_ref);
  const int row = (kp && row0 >= kp[ref]) ? rows_per_ref : row0;  // padding rows of a ragged reference
  __half h[kXH];
#pragma unroll
  for (int i = 0; i < kXH; ++i) h[i] = __float2half_rn(0.0f);
  if (row < m) {
    const float val = C - 0.5f * nr[ref * m + row0];
    h[0] = __float2half_rn(val);
    const float r1 = val - __half2float(h[0]);
    h[1] = __float2half_rn(r1);
    h[2] = __float2half_rn(r1 - __half2float(h[1]));
  } else {
    h[0] = __ushort_as_half(0xFC00u);  // -inf
  }
  uint4* dst = reinterpret_cast<uint4*>(xop + g * kXH);  // (ref, row0)
  const uint4* src = reinterpret_cast<const uint4*>(h);
  dst[0] = src[0];
  dst[1] = src[1];
}

// Squared norms in fp32 of fp16 rows: out[item][row] for rows < valid, `pad` beyond (items of
// `rows` rows, padded to `rows_pad`).
__global__ void norms_kernel(const __half* __restrict__ x, int64_t items, int32_t rows, int32_t rows_pad,
                             float pad, float* __restrict__ out) {
  const int64_t g = static_cast<int64_t>(blockIdx.x) * blockDim.x + threadIdx.x;
  if (g >= items * rows_pad) return;
  const int64_t it = g / rows_pad;
  const int row = static_cast<int>(g % rows_pad);
  float acc = pad;
  if (row < rows) {
    const __half2* p = reinterpret_cast<const __half2*>(x + (it * rows + row) * kDim);
    acc = 0.0f;
#pragma unroll 8
    for (int i = 0; i < kDim / 2; ++i) {
      const float2 f = __half22float2(p[i]);
      acc = fmaf(f.x, f.x, acc);
      acc = fmaf(f.y, f.y, acc);
    }
  }
  out[g] = acc;
}

// SIFT u8 -> [RootSIFT] -> * scale -> fp16 (round to nearest even).  8 lanes per row, 16 bytes in
// and 32 bytes out each (coalesced); the row's L1 sum is an exact integer in fp32 (<= 32,640).
__global__ void prepare_kernel(const uint8_t* __restrict__ sift, int64_t rows, int32_t rootsift, float scale,
                               __half* __restrict__ out) {
  const int64_t g = static_cast<int64_t>(blockIdx.x) * blockDim.x + threadIdx.x;
  const int64_t r = g >> 3;
  const int l8 = static_cast<int>(g & 7);
  uint4 in = make_uint4(0, 0, 0, 0);
  if (r < rows) in = reinterpret_cast<const uint4*>(sift + r * kDim)[l8];
  const uint8_t* b = reinterpret_cast<const uint8_t*>(&in);
  float sum = 0.0f;
#pragma unroll
  for (int i = 0; i < 16; ++i) sum += static_cast<float>(b[i]);
#pragma unroll
  for (int o = 1; o < 8; o <<= 1) sum += __shfl_xor_sync(0xffffffffu, sum, o);
  if (r >= rows) return;
  __align__(16) __half h[16];
#pragma unroll
  for (int i = 0; i < 16; ++i) {
    float v = static_cast<float>(b[i]);
    if (rootsift) v = sum > 0.0f ? sqrtf(v / sum) : 0.0f;
    h[i] = __float2half_rn(v * scale);
  }
  uint4* dst = reinterpret_cast<uint4*>(out + r * kDim) + 2 * l8;
  dst[0] = reinterpret_cast<const uint4*>(h)[0];
  dst[1] = reinterpret_cast<const uint4*>(h)[1];
}

}  // namespace f16

size_t f16_smem_bytes() { return f16::Plan<1>::kAlloc; }

cudaError_t launch_f16_prepare(const uint8_t* sift, int64_t rows, int32_t rootsift, float scale, void* out,
                               cudaStream_t s) {
  if (rows <= 0) return cudaSuccess;
  f16::prepare_kernel<<<static_cast<unsigned>((rows * 8 + 255) / 256), 256, 0, s>>>(sift, rows, rootsift, scale,
                                                                                      static_cast<__half*>(out));
  return cudaGetLastError();
}

cudaError_t launch_f16_norms(const void* x, int64_t items, int32_t rows, int32_t rows_pad, float pad, float* out,
                             cudaStream_t s) {
  const int64_t total = items * rows_pad;
  if (total <= 0) return cudaSuccess;
  f16::norms_kernel<<<static_cast<unsigned>((total + 255) / 256), 256, 0, s>>>(static_cast<const __half*>(x), items,
                                                                               rows, rows_pad, pad, out);
  return cudaGetLastError();
}

cudaError_t launch_f16_xop(const void* r, int64_t R, int32_t m, uint32_t* scratch, float* nr, void* xop,
                           float* cterm, cudaStream_t s) {
  cudaError_t e = cudaMemsetAsync(scratch, 0, 4, s);
  if (e != cudaSuccess) return e;
  const int64_t rows = R * m;
  f16::nr_rows_kernel<<<static_cast<unsigned>((rows * 8 + 255) / 256), 256, 0, s>>>(static_cast<const __half*>(r),
                                                                                   rows, nr, scratch);
  const int32_t rows_per_ref = ((m + kBN - 1) / kBN) * kBN;
  f16::xop_kernel<<<static_cast<unsigned>((R * rows_per_ref + 255) / 256), 256, 0, s>>>(
      nr, R, m, scratch, static_cast<__half*>(xop), cterm, 0.0f, nullptr, rows_per_ref);
  return cudaGetLastError();
}

cudaError_t launch_f16_xop_fixed(const void* r, int64_t R, int32_t m, const int32_t* kp, float C, float* nr, void* xop,
                                 cudaStream_t s) {
  if (R <= 0) return cudaSuccess;
  const int64_t rows = R * m;
  f16::nr_rows_kernel<<<static_cast<unsigned>((rows * 8 + 255) / 256), 256, 0, s>>>(static_cast<const __half*>(r),
                                                                                   rows, nr, nullptr);
  const int32_t rows_per_ref = ((m + kBN - 1) / kBN) * kBN;
  f16::xop_kernel<<<static_cast<unsigned>((R * rows_per_ref + 255) / 256), 256, 0, s>>>(
      nr, R, m, nullptr, static_cast<__half*>(xop), nullptr, C, kp, rows_per_ref);
  return cudaGetLastError();
}

cudaError_t launch_f16_match(const CUtensorMap& qmap, const CUtensorMap& rmap, const CUtensorMap& xmap,
                             const float* cterm, const float* nq, int32_t B, int32_t n, int32_t T, int64_t R,
                             uint32_t num2, uint32_t den2, uint32_t* counts, int num_sms, cudaStream_t s, int64_t ldc,
                             int64_t col0, int64_t rbase, const int32_t* n_valid, int32_t cpr, int32_t m) {
  if (cpr < 1 || cpr > 2) return cudaErrorInvalidValue;
  if (m <= 0 || m > cpr * kBN) m = cpr * kBN;
  const bool skip = (m + f16::kFN - 1) / f16::kFN < cpr * f16::kFPieces;
  auto kern = cpr == 1 ? (skip ? f16::match_f16_kernel<1, true> : f16::match_f16_kernel<1, false>)
                       : (skip ? f16::match_f16_kernel<2, true> : f16::match_f16_kernel<2, false>);
  const size_t smem = cpr == 1 ? f16::Plan<1>::kAlloc : f16::Plan<2>::kAlloc;
  cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, static_cast<int>(smem));
  if (e != cudaSuccess) return e;
  // queries per job: enough jobs to fill the SMs, otherwise all queries reuse the resident reference
  int32_t qpj = B;
  while (R * ((B + qpj - 1) / qpj) < 2LL * num_sms && qpj > 1) qpj = (qpj + 1) / 2;
  const int64_t jobs = R * ((B + qpj - 1) / qpj);
  const int grid = static_cast<int>(jobs < num_sms ? jobs : num_sms);
  kern<<<grid, f16::kThreads, smem, s>>>(qmap, rmap, xmap, cterm, nq, B, n, T, R, qpj, num2, den2, counts,
                                       ldc > 0 ? ldc : R, col0, rbase, n_valid, m);
  return cudaGetLastError();
}

}  // namespace tid
