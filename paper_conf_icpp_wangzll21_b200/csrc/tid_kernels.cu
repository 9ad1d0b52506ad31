// tid_kernels.cu — sm_100a kernels of the texture-identification hot path.
// See tid_kernels.cuh for the list and DESIGN.md for the rooflines.
#include "tid_kernels.cuh"

#include <climits>

namespace tid {

// ------------------------------------------------------------------ PTX helpers (sm_100a)
__device__ __forceinline__ uint32_t smem_u32(const void* p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}
__device__ __forceinline__ void mbar_init(uint32_t bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(bar), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint32_t bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint32_t bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(bar) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint32_t bar, uint32_t parity) {
  asm volatile(
      "{\n\t.reg .pred P1;\n\t"
      "TID_WAIT:\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n\t"
      "@P1 bra TID_DONE;\n\t"
      "bra TID_WAIT;\n\t"
      "TID_DONE:\n\t}" ::"r"(bar),
      "r"(parity)
      : "memory");
}
__device__ __forceinline__ void fence_barrier_init() {
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}
__device__ __forceinline__ void tma_load_3d(uint32_t dst, const CUtensorMap* map, uint32_t bar, int c0, int c1,
                                            int c2) {
  asm volatile(
      "cp.async.bulk.tensor.3d.shared::cluster.global.tile.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4, %5}], "
      "[%2];" ::"r"(dst),
      "l"(reinterpret_cast<uint64_t>(map)), "r"(bar), "r"(c0), "r"(c1), "r"(c2)
      : "memory");
}
__device__ __forceinline__ void bulk_load(uint32_t dst, const void* src, uint32_t bytes, uint32_t bar) {
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(dst),
               "l"(src), "r"(bytes), "r"(bar)
               : "memory");
}
__device__ __forceinline__ void prefetch_tmap(const CUtensorMap* map) {
  asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(map)) : "memory");
}
__device__ __forceinline__ void tc_fence_before() { asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory"); }
__device__ __forceinline__ void tc_fence_after() { asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory"); }

// K-major, SWIZZLE_128B shared-memory matrix descriptor (tile base 1024-B aligned,
// 128-B rows, 8-row core groups 1024 B apart).
__device__ __forceinline__ uint64_t smem_desc_sw128(uint32_t addr) {
  uint64_t d = 0;
  d |= static_cast<uint64_t>((addr & 0x3FFFF) >> 4);   // start address   [0,14)
  d |= static_cast<uint64_t>(1) << 16;                 // LBO (unused for SW128 K-major)
  d |= static_cast<uint64_t>(1024 >> 4) << 32;         // SBO = 1024 B    [32,46)
  d |= static_cast<uint64_t>(1) << 46;                 // descriptor version (sm_100)
  d |= static_cast<uint64_t>(2) << 61;                 // layout: SWIZZLE_128B
  return d;
}

// Instruction descriptor: kind::i8, A = u8, B = u8, D = s32, K-major A/B, M = 128, N = 256.
constexpr uint32_t kIdescI8 = (2u << 4)                       // D format S32
                              | (0u << 7) | (0u << 10)        // A, B unsigned 8-bit
                              | (0u << 15) | (0u << 16)       // A, B K-major
                              | (uint32_t(kBN >> 3) << 17)    // N >> 3
                              | (uint32_t(kBM >> 4) << 24);   // M >> 4

__device__ __forceinline__ void mma_i8(uint32_t tmem_d, uint64_t adesc, uint64_t bdesc, uint32_t accum) {
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "setp.ne.b32 p, %4, 0;\n\t"
      "tcgen05.mma.cta_group::1.kind::i8 [%0], %1, %2, %3, p;\n\t}" ::"r"(tmem_d),
      "l"(adesc), "l"(bdesc), "r"(kIdescI8), "r"(accum)
      : "memory");
}
__device__ __forceinline__ void mma_commit(uint32_t bar) {
  asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(bar) : "memory");
}

#define TID_LD32_OUT(v)                                                                                           \
  "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]), "=r"(v[7]), "=r"(v[8]),     \
      "=r"(v[9]), "=r"(v[10]), "=r"(v[11]), "=r"(v[12]), "=r"(v[13]), "=r"(v[14]), "=r"(v[15]), "=r"(v[16]),     \
      "=r"(v[17]), "=r"(v[18]), "=r"(v[19]), "=r"(v[20]), "=r"(v[21]), "=r"(v[22]), "=r"(v[23]), "=r"(v[24]),    \
      "=r"(v[25]), "=r"(v[26]), "=r"(v[27]), "=r"(v[28]), "=r"(v[29]), "=r"(v[30]), "=r"(v[31])

// 32 consecutive TMEM columns of this thread's lane (32x32b shape, .x32).
__device__ __forceinline__ void tmem_ld32(uint32_t taddr, uint32_t (&v)[32]) {
  asm volatile(
      "tcgen05.ld.sync.aligned.32x32b.x32.b32 {%0, %1, %2, %3, %4, %5, %6, %7, %8, %9, %10, %11, %12, %13, %14, "
      "%15, %16, %17, %18, %19, %20, %21, %22, %23, %24, %25, %26, %27, %28, %29, %30, %31}, [%32];"
      : TID_LD32_OUT(v)
      : "r"(taddr));
}
__device__ __forceinline__ int4 lds128(uint32_t addr) {
  int4 r;
  asm volatile("ld.shared.v4.s32 {%0, %1, %2, %3}, [%4];" : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w) : "r"(addr));
  return r;
}
__device__ __forceinline__ void tmem_wait_ld() { asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory"); }
// Registers written by an in-flight tcgen05.ld may only be read after wait::ld; the empty
// asm makes every later use depend on a point after the wait.
__device__ __forceinline__ void reg_fence(uint32_t (&v)[32]) {
#pragma unroll
  for (int i = 0; i < 32; ++i) asm volatile("" : "+r"(v[i]));
}

// ------------------------------------------------------------------ shared memory plan
struct SmemPlan {
  static constexpr uint32_t kR = 0;                                        // kMaxSlots x 32 KiB
  static constexpr uint32_t kQ = kR + kMaxSlots * kRTileBytes;             // kQStages x 16 KiB
  static constexpr uint32_t kCol = kQ + kQStages * kQTileBytes;            // kMaxSlots x 1 KiB
  static constexpr uint32_t kBar = kCol + kMaxSlots * kColBytes;           // mbarriers
  static constexpr uint32_t kQFull = kBar;
  static constexpr uint32_t kQEmpty = kQFull + 8 * kQStages;
  static constexpr uint32_t kRFull = kQEmpty + 8 * kQStages;
  static constexpr uint32_t kREmpty = kRFull + 8 * kMaxSlots;
  static constexpr uint32_t kTFull = kREmpty + 8 * kMaxSlots;
  static constexpr uint32_t kTEmpty = kTFull + 8 * 2;
  static constexpr uint32_t kTmemPtr = kTEmpty + 8 * 2;
  static constexpr uint32_t kCnt = kTmemPtr + 16;                          // [8 warps][kMaxSlots] u32
  static constexpr uint32_t kEnd = kCnt + 8 * kMaxSlots * 4;
  static constexpr uint32_t kAlloc = kEnd + 1024;                          // + alignment slack
};

size_t match_smem_bytes() { return SmemPlan::kAlloc; }

struct Job {
  int32_t q_first, nq;
  int64_t ref_first;
  int32_t nr;
};

__device__ __forceinline__ Job decode_job(const MatchParams& p, int32_t j) {
  Job J;
  if (p.mode == kModeVerify) {
    J.q_first = j; J.nq = 1; J.ref_first = j; J.nr = 1;
  } else {
    const int32_t g = j / p.n_qchunks, qc = j % p.n_qchunks;
    J.q_first = qc * p.q_per_job;
    J.nq = min(p.q_per_job, p.num_q - J.q_first);
    J.ref_first = static_cast<int64_t>(g) * p.refs_per_job;
    J.nr = static_cast<int32_t>(min(static_cast<int64_t>(p.refs_per_job), p.n_refs - J.ref_first));
  }
  return J;
}

// ------------------------------------------------------------------ fused match kernel
// One persistent CTA per SM.  A job = (reference group resident in SMEM) x (range of
// query tiles streamed through a 4-stage ring).  Unit u = (query tile t, reference s);
// unit u uses TMEM accumulator buffer u&1 and is drained by epilogue group u&1.
__global__ void __launch_bounds__(kNumThreads, 1)
    match_kernel(const __grid_constant__ CUtensorMap qmap, const __grid_constant__ CUtensorMap rmap,
                 const MatchParams p) {
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  const uint32_t sbase = smem_u32(smem);
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int T = p.tiles_per_q, cpr = p.cpr;

  auto qfull = [&](int i) { return sbase + SmemPlan::kQFull + 8 * i; };
  auto qempty = [&](int i) { return sbase + SmemPlan::kQEmpty + 8 * i; };
  auto rfull = [&](int i) { return sbase + SmemPlan::kRFull + 8 * i; };
  auto rempty = [&](int i) { return sbase + SmemPlan::kREmpty + 8 * i; };
  auto tfull = [&](int i) { return sbase + SmemPlan::kTFull + 8 * i; };
  auto tempty = [&](int i) { return sbase + SmemPlan::kTEmpty + 8 * i; };
  uint32_t* tmem_ptr_smem = reinterpret_cast<uint32_t*>(smem + SmemPlan::kTmemPtr);
  uint32_t* cnt_smem = reinterpret_cast<uint32_t*>(smem + SmemPlan::kCnt);

  if (threadIdx.x == 0) {
    prefetch_tmap(&qmap);
    prefetch_tmap(&rmap);
    for (int i = 0; i < kQStages; ++i) { mbar_init(qfull(i), 1); mbar_init(qempty(i), 1); }
    for (int i = 0; i < kMaxSlots; ++i) { mbar_init(rfull(i), 1); mbar_init(rempty(i), 1 + 8); }
    for (int i = 0; i < 2; ++i) { mbar_init(tfull(i), 1); mbar_init(tempty(i), 4); }
    fence_barrier_init();
  }
  if (threadIdx.x < 8 * kMaxSlots) cnt_smem[threadIdx.x] = 0;
  if (warp == 1) {  // TMEM: 2 accumulator buffers x 256 columns (all 512)
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 512;" ::"r"(
                     smem_u32(tmem_ptr_smem))
                 : "memory");
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
  }
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem_base = *tmem_ptr_smem;

  if (warp == 0) {
    // ===================== TMA producer =====================
    if (lane == 0) {
      uint32_t qctr = 0;
      uint32_t slot_use[kMaxSlots] = {0, 0, 0, 0};
      for (int32_t j = blockIdx.x; j < p.n_jobs; j += gridDim.x) {
        const Job J = decode_job(p, j);
        const int nslots = J.nr * cpr;
        for (int sl = 0; sl < nslots; ++sl) {
          mbar_wait(rempty(sl), (slot_use[sl] & 1) ^ 1);
          mbar_expect_tx(rfull(sl), kRTileBytes + kColBytes);
          const int s = sl / cpr, c = sl % cpr;
          const int64_t ref = J.ref_first + s;
          tma_load_3d(sbase + SmemPlan::kR + sl * kRTileBytes, &rmap, rfull(sl), 0, c * kBN,
                      static_cast<int>(p.ref_map_base + ref));
          bulk_load(sbase + SmemPlan::kCol + sl * kColBytes, p.colkey + (ref * cpr + c) * kBN, kColBytes, rfull(sl));
          ++slot_use[sl];
        }
        const int ntiles = J.nq * T;
        for (int t = 0; t < ntiles; ++t, ++qctr) {
          const int st = qctr % kQStages;
          mbar_wait(qempty(st), ((qctr / kQStages) & 1) ^ 1);
          mbar_expect_tx(qfull(st), kQTileBytes);
          tma_load_3d(sbase + SmemPlan::kQ + st * kQTileBytes, &qmap, qfull(st), 0, (t % T) * kBM, J.q_first + t / T);
        }
      }
    }
  } else if (warp == 1) {
    // ===================== MMA issuer (one thread) =====================
    if (lane == 0) {
      uint32_t qctr = 0;
      uint32_t slot_use[kMaxSlots] = {0, 0, 0, 0};
      uint32_t buf_use[2] = {0, 0};
      for (int32_t j = blockIdx.x; j < p.n_jobs; j += gridDim.x) {
        const Job J = decode_job(p, j);
        const int nslots = J.nr * cpr;
        const int U = J.nq * T * J.nr;
        bool slot_ready[kMaxSlots] = {false, false, false, false};
        int waited = 0;
        for (int u0 = 0; u0 < U; u0 += 2) {
          for (int c = 0; c < cpr; ++c) {
            for (int b = 0; b < 2; ++b) {
              const int u = u0 + b;
              if (u >= U) break;
              const int t = u / J.nr, s = u % J.nr, sl = s * cpr + c;
              while (waited <= t) {
                const uint32_t g = qctr + waited;
                mbar_wait(qfull(g % kQStages), (g / kQStages) & 1);
                ++waited;
              }
              if (!slot_ready[sl]) { mbar_wait(rfull(sl), slot_use[sl] & 1); slot_ready[sl] = true; }
              mbar_wait(tempty(b), (buf_use[b] & 1) ^ 1);
              tc_fence_after();
              const uint32_t st = (qctr + t) % kQStages;
              const uint64_t ad = smem_desc_sw128(sbase + SmemPlan::kQ + st * kQTileBytes);
              const uint64_t bd = smem_desc_sw128(sbase + SmemPlan::kR + sl * kRTileBytes);
              const uint32_t dt = tmem_base + b * kBN;
#pragma unroll
              for (int k = 0; k < kDim / 32; ++k)  // K = 32 bytes per tcgen05.mma.kind::i8
                mma_i8(dt, ad + 2 * k, bd + 2 * k, k > 0 ? 1u : 0u);
              mma_commit(tfull(b));
              ++buf_use[b];
              if (c == cpr - 1 && s == J.nr - 1) mma_commit(qempty(st));  // last reader of tile t
            }
          }
        }
        for (int sl = 0; sl < nslots; ++sl) { mma_commit(rempty(sl)); ++slot_use[sl]; }
        qctr += J.nq * T;
      }
    }
  } else {
    // ===================== epilogue: TMEM -> registers -> top-2 -> ratio -> count =====================
    const int e = (warp - 2) >> 2;          // group 0: warps 2..5, group 1: warps 6..9
    const int quarter = warp & 3;           // TMEM lanes 32*quarter .. +31 (hardware restriction)
    const int wslot = warp - 2;             // 0..7 for the count accumulators
    const uint32_t taddr_base = tmem_base + (static_cast<uint32_t>(quarter * 32) << 16) + e * kBN;
    uint32_t buf_use = 0;
    uint32_t slot_use[kMaxSlots] = {0, 0, 0, 0};
    const int row_in_tile = quarter * 32 + lane;
    const int nq_ld = T * kBM;

    for (int32_t j = blockIdx.x; j < p.n_jobs; j += gridDim.x) {
      const Job J = decode_job(p, j);
      const int nslots = J.nr * cpr;
      const int U = J.nq * T * J.nr;
      const int ustep = (J.nr % 2 == 0) ? J.nr : 2 * J.nr;  // next unit of this group with the same s
      for (int u = e; u < U; u += 2) {
        const int t = u / J.nr, s = u % J.nr;
        const int qi = J.q_first + t / T;
        const int row = (t % T) * kBM + row_in_tile;
        const int nvalid = p.n_valid ? p.n_valid[qi] : p.n_rows;
        const bool valid = row < nvalid && row < p.n_rows;
        const int32_t nqv = p.nq[static_cast<int64_t>(qi) * nq_ld + row];

        int g1d = INT_MAX, g1i = -1, g2d = INT_MAX, g2i = -1;  // running 2-NN over chunks
        for (int c = 0; c < cpr; ++c) {
          const int sl = s * cpr + c;
          mbar_wait(rfull(sl), slot_use[sl] & 1);  // column keys of this chunk have landed
          mbar_wait(tfull(e), buf_use & 1);
          tc_fence_after();
          const uint32_t ck_addr = sbase + SmemPlan::kCol + sl * kColBytes;
          int a1 = INT_MAX, a2 = INT_MAX, b1 = INT_MAX, b2 = INT_MAX;
#pragma unroll
          for (int jj = 0; jj < kBN / 32; ++jj) {
            uint32_t v[32];
            tmem_ld32(taddr_base + jj * 32, v);
            tmem_wait_ld();
            reg_fence(v);
#pragma unroll
            for (int i = 0; i < 32; i += 4) {
              const int4 c4 = lds128(ck_addr + (jj * 32 + i) * 4);
              const int x0 = c4.x - 512 * static_cast<int>(v[i]);
              const int x1 = c4.y - 512 * static_cast<int>(v[i + 1]);
              const int x2 = c4.z - 512 * static_cast<int>(v[i + 2]);
              const int x3 = c4.w - 512 * static_cast<int>(v[i + 3]);
              int lo = min(x0, x1), hi = max(x0, x1);
              int tt = max(a1, lo);
              a2 = min(min(a2, tt), hi);
              a1 = min(a1, lo);
              lo = min(x2, x3); hi = max(x2, x3);
              tt = max(b1, lo);
              b2 = min(min(b2, tt), hi);
              b1 = min(b1, lo);
            }
            // keep the scan streaming: the state must be final before the next TMEM load
            asm volatile("" : "+r"(a1), "+r"(a2), "+r"(b1), "+r"(b2));
          }
          tc_fence_before();
          __syncwarp();
          if (lane == 0) mbar_arrive(tempty(e));
          ++buf_use;
          // top-2 of the chunk from the two interleaved states (keys are unique: index bits)
          const int k1 = min(a1, b1);
          const int k2 = min(max(a1, b1), min(a2, b2));
          const int c1d = k1 >> 8, c1i = (k1 & 255) + c * kBN;
          const int c2d = k2 >> 8, c2i = (k2 & 255) + c * kBN;
          // merge into the running 2-NN; earlier chunks win ties (lower index)
          if (c1d < g1d) {
            if (c2d < g1d) { g2d = c2d; g2i = c2i; } else { g2d = g1d; g2i = g1i; }
            g1d = c1d; g1i = c1i;
          } else if (c1d < g2d) {
            g2d = c1d; g2i = c1i;
          }
        }
        // ratio test in exact integers: den^2 * d1 < num^2 * d2
        const bool real1 = g1d < kSentinelNorm, real2 = g2d < kSentinelNorm;
        const int64_t d1 = static_cast<int64_t>(nqv) + g1d;
        const int64_t d2 = static_cast<int64_t>(nqv) + g2d;
        const bool pass = valid && real2 &&
                          static_cast<uint64_t>(p.den2) * static_cast<uint64_t>(d1) <
                              static_cast<uint64_t>(p.num2) * static_cast<uint64_t>(d2);
        if (p.nn_out != nullptr && row < p.n_rows) {
          int4 o;
          o.x = (valid && real1) ? static_cast<int>(d1) : -1; o.y = (valid && real1) ? g1i : -1;
          o.z = (valid && real2) ? static_cast<int>(d2) : -1; o.w = (valid && real2) ? g2i : -1;
          reinterpret_cast<int4*>(p.nn_out)[static_cast<int64_t>(qi) * p.n_rows + row] = o;
        }
        const uint32_t bal = __ballot_sync(0xffffffffu, pass);
        if (lane == 0) {
          uint32_t& acc = cnt_smem[wslot * kMaxSlots + s];
          acc += __popc(bal);
          const int un = u + ustep;
          const bool flush = (un >= U) || ((un / J.nr) / T != t / T);
          if (flush) {
            if (acc) {
              const int64_t ci = (p.mode == kModeVerify) ? qi
                                                         : static_cast<int64_t>(qi) * p.ldc + p.col0 + J.ref_first + s;
              atomicAdd(p.counts + ci, acc);
            }
            acc = 0;
          }
        }
      }
      __syncwarp();
      if (lane == 0)
        for (int sl = 0; sl < nslots; ++sl) mbar_arrive(rempty(sl));
      for (int sl = 0; sl < nslots; ++sl) ++slot_use[sl];
    }
  }

  tc_fence_before();
  __syncthreads();
  if (warp == 1) {
    tc_fence_after();
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 512;" ::"r"(tmem_base) : "memory");
  }
}

cudaError_t launch_match(const MatchParams& p, const CUtensorMap& qmap, const CUtensorMap& rmap, int grid,
                         cudaStream_t s) {
  cudaError_t e = cudaFuncSetAttribute(match_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                       static_cast<int>(SmemPlan::kAlloc));
  if (e != cudaSuccess) return e;
  match_kernel<<<grid, kNumThreads, SmemPlan::kAlloc, s>>>(qmap, rmap, p);
  return cudaGetLastError();
}

// ------------------------------------------------------------------ a1: reference prep
// One thread per (reference, column) row: N_R = sum r^2 (dp4a) -> packed column key.
// Modes: desc != null && src == null : in place (rows >= kp zeroed);
//        desc != null && src != null : copy src -> desc (rows >= kp zeroed);
//        desc == null                : read-only (src), keys only (rows >= kp get the sentinel).
__global__ void ref_prep_kernel(RefPrepParams p) {
  const int cols = p.cpr * kBN;
  const int64_t gid = static_cast<int64_t>(blockIdx.x) * blockDim.x + threadIdx.x;
  if (gid >= p.count * cols) return;
  const int64_t r = gid / cols;
  const int i = static_cast<int>(gid % cols);
  int kp = p.kp ? p.kp[r] : p.m;
  kp = max(0, min(kp, p.m));
  int32_t norm = kSentinelNorm;
  if (i < p.m) {
    uint4* dst = p.desc ? reinterpret_cast<uint4*>(p.desc + (r * p.m + i) * kDim) : nullptr;
    if (i < kp) {
      const uint4* src = p.src ? reinterpret_cast<const uint4*>(p.src + (r * p.m + i) * kDim) : dst;
      uint32_t acc = 0;
#pragma unroll
      for (int w = 0; w < kDim / 16; ++w) {
        const uint4 x = src[w];
        acc = __dp4a(x.x, x.x, acc); acc = __dp4a(x.y, x.y, acc);
        acc = __dp4a(x.z, x.z, acc); acc = __dp4a(x.w, x.w, acc);
        if (p.src && dst) dst[w] = x;
      }
      norm = static_cast<int32_t>(acc);
    } else if (dst) {
#pragma unroll
      for (int w = 0; w < kDim / 16; ++w) dst[w] = make_uint4(0, 0, 0, 0);
    }
  }
  p.colkey[r * cols + i] = norm * 256 + (i & (kBN - 1));
}

void launch_ref_prep(const RefPrepParams& p, cudaStream_t s) {
  const int64_t total = p.count * p.cpr * kBN;
  if (total == 0) return;
  ref_prep_kernel<<<static_cast<unsigned>((total + 255) / 256), 256, 0, s>>>(p);
}

// ------------------------------------------------------------------ a2: query prep
__global__ void query_prep_kernel(const uint8_t* __restrict__ q, int64_t B, int32_t n, int32_t rows_pad,
                                  int32_t* __restrict__ nq) {
  const int64_t gid = static_cast<int64_t>(blockIdx.x) * blockDim.x + threadIdx.x;
  if (gid >= B * rows_pad) return;
  const int64_t b = gid / rows_pad;
  const int row = static_cast<int>(gid % rows_pad);
  uint32_t acc = 0;
  if (row < n) {
    const uint4* src = reinterpret_cast<const uint4*>(q + (b * n + row) * kDim);
#pragma unroll
    for (int w = 0; w < kDim / 16; ++w) {
      const uint4 x = src[w];
      acc = __dp4a(x.x, x.x, acc); acc = __dp4a(x.y, x.y, acc);
      acc = __dp4a(x.z, x.z, acc); acc = __dp4a(x.w, x.w, acc);
    }
  }
  nq[gid] = static_cast<int32_t>(acc);
}

void launch_query_prep(const uint8_t* q, int64_t B, int32_t n, int32_t tiles_per_q, int32_t* nq, cudaStream_t s) {
  const int32_t rows_pad = tiles_per_q * kBM;
  const int64_t total = B * rows_pad;
  if (total == 0) return;
  query_prep_kernel<<<static_cast<unsigned>((total + 255) / 256), 256, 0, s>>>(q, B, n, rows_pad, nq);
}

// ------------------------------------------------------------------ a6: top-k of the count matrix
// Candidate key = count << 40 | (2^40 - 1 - global id): larger key <=> (count desc, id asc).
constexpr uint64_t kIdMask = (uint64_t(1) << 40) - 1;
__device__ __forceinline__ uint64_t make_key(uint32_t count, int64_t id) {
  return (static_cast<uint64_t>(count) << 40) | (kIdMask - static_cast<uint64_t>(id));
}

__device__ __forceinline__ uint64_t warp_max_u64(uint64_t v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) {
    const uint64_t w = __shfl_xor_sync(0xffffffffu, v, o);
    v = w > v ? w : v;
  }
  return v;
}

// Block-wide k rounds of "take the largest remaining head".  Each thread owns a sorted
// (descending) list lists[tid*k .. +k) with cursor; returns winners in out[0..k).
__device__ void block_select(const uint64_t* lists, int k, uint64_t* out, uint64_t* red) {
  const int tid = threadIdx.x, nw = blockDim.x >> 5;
  int cur = 0;
  for (int r = 0; r < k; ++r) {
    const uint64_t head = cur < k ? lists[tid * k + cur] : 0;
    uint64_t m = warp_max_u64(head);
    if ((tid & 31) == 0) red[tid >> 5] = m;
    __syncthreads();
    if (tid < 32) {
      uint64_t x = tid < nw ? red[tid] : 0;
      x = warp_max_u64(x);
      if (tid == 0) red[32] = x;
    }
    __syncthreads();
    const uint64_t best = red[32];
    if (head == best && best != 0) ++cur;  // keys are unique; 0 = empty
    if (tid == 0) out[r] = best;
    __syncthreads();
  }
}

// grid (B, segs), 256 threads, dyn smem = 256*k*8 + 33*8.
__global__ void topk_kernel(const uint32_t* __restrict__ counts, int64_t R, int64_t ldc, int64_t id_base, int32_t k,
                            uint64_t* __restrict__ cand_out) {
  extern __shared__ uint64_t tk_smem[];
  uint64_t* lists = tk_smem;
  uint64_t* red = tk_smem + blockDim.x * k;
  const int b = blockIdx.x, seg = blockIdx.y, segs = gridDim.y;
  const int64_t len = (R + segs - 1) / segs;
  const int64_t r0 = seg * len, r1 = min(R, r0 + len);
  uint64_t* my = lists + threadIdx.x * k;
  for (int i = 0; i < k; ++i) my[i] = 0;
  uint64_t kth = 0;
  const uint32_t* row = counts + static_cast<int64_t>(b) * ldc;
  for (int64_t r = r0 + threadIdx.x; r < r1; r += blockDim.x) {
    const uint64_t key = make_key(row[r], id_base + r);
    if (key > kth) {  // insertion into the thread's descending list
      int pos = k - 1;
      while (pos > 0 && my[pos - 1] < key) { my[pos] = my[pos - 1]; --pos; }
      my[pos] = key;
      kth = my[k - 1];
    }
  }
  __syncthreads();
  block_select(lists, k, cand_out + (static_cast<int64_t>(b) * segs + seg) * k, red);
}

void launch_topk(const uint32_t* counts, int64_t B, int64_t R, int64_t ldc, int64_t id_base, int32_t k, int32_t segs,
                 uint64_t* cand_out, cudaStream_t s) {
  const size_t smem = (256 * static_cast<size_t>(k) + 33) * 8;
  static size_t attr = 0;
  if (smem > 48 * 1024 && smem > attr) {
    cudaFuncSetAttribute(topk_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, static_cast<int>(smem));
    attr = smem;
  }
  topk_kernel<<<dim3(static_cast<unsigned>(B), static_cast<unsigned>(segs)), 256, smem, s>>>(counts, R, ldc, id_base,
                                                                                              k, cand_out);
}

// ------------------------------------------------------------------ a6/a9: merge ranked lists
// L candidate lists of k keys per query (list l of query b at cand[b*sb + l*sl]).  One block
// of 128 threads per query: each thread gathers its share, sorts it, then block_select.
__global__ void merge_kernel(const uint64_t* __restrict__ cand, int32_t L, int32_t k, int64_t sb, int64_t sl,
                             uint64_t* __restrict__ keys_out, int64_t* __restrict__ ids_out,
                             int32_t* __restrict__ counts_out) {
  extern __shared__ uint64_t mg_smem[];
  uint64_t* lists = mg_smem;  // blockDim.x * k
  uint64_t* red = mg_smem + blockDim.x * k;
  uint64_t* win = red + 33;   // k
  const int b = blockIdx.x;
  uint64_t* my = lists + threadIdx.x * k;
  for (int i = 0; i < k; ++i) my[i] = 0;
  uint64_t kth = 0;
  const int64_t total = static_cast<int64_t>(L) * k;
  for (int64_t x = threadIdx.x; x < total; x += blockDim.x) {
    const int l = static_cast<int>(x / k), i = static_cast<int>(x % k);
    const uint64_t key = cand[b * sb + l * sl + i];
    if (key > kth) {
      int pos = k - 1;
      while (pos > 0 && my[pos - 1] < key) { my[pos] = my[pos - 1]; --pos; }
      my[pos] = key;
      kth = my[k - 1];
    }
  }
  __syncthreads();
  block_select(lists, k, win, red);
  for (int i = threadIdx.x; i < k; i += blockDim.x) {
    const uint64_t key = win[i];
    if (keys_out) keys_out[static_cast<int64_t>(b) * k + i] = key;
    if (ids_out) ids_out[static_cast<int64_t>(b) * k + i] = key ? static_cast<int64_t>(kIdMask - (key & kIdMask)) : -1;
    if (counts_out) counts_out[static_cast<int64_t>(b) * k + i] = static_cast<int32_t>(key >> 40);
  }
}

void launch_merge(const uint64_t* cand, int32_t L, int64_t B, int32_t k, int64_t sb, int64_t sl, uint64_t* keys_out,
                  int64_t* ids_out, int32_t* counts_out, cudaStream_t s) {
  const int threads = 128;
  const size_t smem = (threads * static_cast<size_t>(k) + 33 + k) * 8;
  static size_t attr = 0;
  if (smem > 48 * 1024 && smem > attr) {
    cudaFuncSetAttribute(merge_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, static_cast<int>(smem));
    attr = smem;
  }
  merge_kernel<<<static_cast<unsigned>(B), threads, smem, s>>>(cand, L, k, sb, sl, keys_out, ids_out, counts_out);
}

__global__ void pack_kernel(const int64_t* ids, const int32_t* counts, int64_t n, uint64_t* keys) {
  const int64_t i = static_cast<int64_t>(blockIdx.x) * blockDim.x + threadIdx.x;
  if (i < n) keys[i] = (ids[i] < 0) ? 0 : make_key(static_cast<uint32_t>(counts[i]), ids[i]);
}

void launch_pack_lists(const int64_t* ids, const int32_t* counts, int64_t n, uint64_t* keys, cudaStream_t s) {
  if (n == 0) return;
  pack_kernel<<<static_cast<unsigned>((n + 255) / 256), 256, 0, s>>>(ids, counts, n, keys);
}

}  // namespace tid
