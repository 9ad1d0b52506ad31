// tid_kernels.cu — sm_100a kernels of the texture-identification hot path.
// See tid_kernels.cuh for the list and DESIGN.md for the rooflines.
#include "tid_kernels.cuh"

#include <climits>

// Timing-experiment switches that skip work and give WRONG results (skeleton timings in DESIGN.md):
// refused unless the build says it is an experiment.
#if (defined(TID_NOSCAN) || defined(TID_NOMMA) || defined(TID_NOLOAD)) && !defined(TID_EXPERIMENT)
#error "TID_NOSCAN / TID_NOMMA / TID_NOLOAD skip work (wrong results): timing experiments only, add -DTID_EXPERIMENT"
#endif

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
      "mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1, 1000000;\n\t"
      "@P1 bra TID_DONE;\n\t"
      "bra TID_WAIT;\n\t"
      "TID_DONE:\n\t}" ::"r"(bar),
      "r"(parity)
      : "memory");
}
// Polling wait with exponential nanosleep back-off: used by the control warps (TMA producer,
// MMA issuers), which share SMSPs with the epilogue and must not steal its issue slots.
__device__ __forceinline__ void mbar_wait_sleep(uint32_t bar, uint32_t parity) {
  uint32_t ns = 32;
  while (true) {
    uint32_t done;
    asm volatile(
        "{\n\t.reg .pred P1;\n\t"
        "mbarrier.test_wait.parity.shared::cta.b64 P1, [%1], %2;\n\t"
        "selp.u32 %0, 1, 0, P1;\n\t}"
        : "=r"(done)
        : "r"(bar), "r"(parity)
        : "memory");
    if (done) return;
    __nanosleep(ns);
    ns = ns < 512 ? ns * 2 : 512;
  }
}
__device__ __forceinline__ void named_bar(uint32_t id, uint32_t count) {
  asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(count) : "memory");
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

// K-major, SWIZZLE_32B descriptor (32-byte rows, 8-row groups 256 B apart): the norm-term tiles.
__device__ __forceinline__ uint64_t smem_desc_sw32(uint32_t addr) {
  uint64_t d = 0;
  d |= static_cast<uint64_t>((addr & 0x3FFFF) >> 4);
  d |= static_cast<uint64_t>(1) << 16;
  d |= static_cast<uint64_t>(256 >> 4) << 32;           // SBO = 256 B
  d |= static_cast<uint64_t>(1) << 46;
  d |= static_cast<uint64_t>(6) << 61;                  // layout: SWIZZLE_32B
  return d;
}

// Instruction descriptor: kind::i8, D = s32, K-major A/B, M = 128, N = kPiece; A/B signedness.
constexpr uint32_t idesc_i8(bool a_signed, bool b_signed) {
  return (2u << 4)                                      // D format S32
         | (uint32_t(a_signed) << 7) | (uint32_t(b_signed) << 10)
         | (0u << 15) | (0u << 16)                      // A, B K-major
         | (uint32_t(kPiece >> 3) << 17)                // N >> 3
         | (uint32_t(kBM >> 4) << 24);                  // M >> 4
}
constexpr uint32_t kIdescI8 = idesc_i8(false, false);   // verify: u8 x u8
constexpr uint32_t kIdescFold = idesc_i8(true, false);  // search: q' (s8) x r (u8)

// Issued by the whole (converged) MMA warp: elect.sync picks one lane, so the descriptors stay in
// uniform registers and ptxas emits a bare UTCIMMA (no per-lane broadcast loop).
__device__ __forceinline__ void mma_i8(uint32_t tmem_d, uint64_t adesc, uint64_t bdesc, uint32_t accum) {
  asm volatile(
      "{\n\t.reg .pred p, e;\n\t"
      "setp.ne.b32 p, %4, 0;\n\t"
      "elect.sync _|e, 0xffffffff;\n\t"
      "@e tcgen05.mma.cta_group::1.kind::i8 [%0], %1, %2, %3, p;\n\t}" ::"r"(tmem_d),
      "l"(adesc), "l"(bdesc), "r"(kIdescI8), "r"(accum)
      : "memory");
}
// One accumulator piece: D = A * B over K = 128 bytes as four K = 32 MMAs (advancing both
// SWIZZLE_128B descriptors by 32 B = 2 units) + commit to `bar`, from a single elected lane.
template <uint32_t kIdesc>
__device__ __forceinline__ void mma_piece(uint32_t tmem_d, uint64_t adesc, uint64_t bdesc, uint32_t bar) {
  asm volatile(
      "{\n\t.reg .pred e, f, t;\n\t.reg .b64 a1, a2, a3, b1, b2, b3;\n\t"
      "setp.ne.b32 f, 0, 0;\n\t"
      "setp.eq.b32 t, 0, 0;\n\t"
      "add.s64 a1, %1, 2;\n\tadd.s64 a2, %1, 4;\n\tadd.s64 a3, %1, 6;\n\t"
      "add.s64 b1, %2, 2;\n\tadd.s64 b2, %2, 4;\n\tadd.s64 b3, %2, 6;\n\t"
      "elect.sync _|e, 0xffffffff;\n\t"
      "@e tcgen05.mma.cta_group::1.kind::i8 [%0], %1, %2, %3, f;\n\t"
      "@e tcgen05.mma.cta_group::1.kind::i8 [%0], a1, b1, %3, t;\n\t"
      "@e tcgen05.mma.cta_group::1.kind::i8 [%0], a2, b2, %3, t;\n\t"
      "@e tcgen05.mma.cta_group::1.kind::i8 [%0], a3, b3, %3, t;\n\t"
      "@e tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%4];\n\t}" ::"r"(tmem_d),
      "l"(adesc), "l"(bdesc), "r"(kIdesc), "r"(bar)
      : "memory");
}
// Search piece: the four q'.r K-steps, then the norm-term K-step (u8 x u8: D += a . digits(E)).
__device__ __forceinline__ void mma_piece_fold(uint32_t tmem_d, uint64_t adesc, uint64_t bdesc, uint64_t axdesc,
                                               uint64_t bxdesc, uint32_t bar) {
  asm volatile(
      "{\n\t.reg .pred e, f, t;\n\t.reg .b64 a1, a2, a3, b1, b2, b3;\n\t"
      "setp.ne.b32 f, 0, 0;\n\t"
      "setp.eq.b32 t, 0, 0;\n\t"
      "add.s64 a1, %1, 2;\n\tadd.s64 a2, %1, 4;\n\tadd.s64 a3, %1, 6;\n\t"
      "add.s64 b1, %2, 2;\n\tadd.s64 b2, %2, 4;\n\tadd.s64 b3, %2, 6;\n\t"
      "elect.sync _|e, 0xffffffff;\n\t"
      "@e tcgen05.mma.cta_group::1.kind::i8 [%0], %1, %2, %5, f;\n\t"
      "@e tcgen05.mma.cta_group::1.kind::i8 [%0], a1, b1, %5, t;\n\t"
      "@e tcgen05.mma.cta_group::1.kind::i8 [%0], a2, b2, %5, t;\n\t"
      "@e tcgen05.mma.cta_group::1.kind::i8 [%0], a3, b3, %5, t;\n\t"
      "@e tcgen05.mma.cta_group::1.kind::i8 [%0], %3, %4, %6, t;\n\t"
      "@e tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%7];\n\t}" ::"r"(tmem_d),
      "l"(adesc), "l"(bdesc), "l"(axdesc), "l"(bxdesc), "r"(kIdescFold), "r"(kIdescI8), "r"(bar)
      : "memory");
}

// SMEM (matrix descriptor) -> TMEM: 128 rows x 32 B into 128 lanes x 8 columns (single thread).
__device__ __forceinline__ void tmem_cp_128x256b(uint32_t taddr, uint64_t sdesc) {
  asm volatile("tcgen05.cp.cta_group::1.128x256b [%0], %1;" ::"r"(taddr), "l"(sdesc) : "memory");
}
__device__ __forceinline__ void commit_one(uint32_t bar) {  // single-thread form
  asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(bar) : "memory");
}
// Search piece with A in TMEM: four q'.r K-steps (A = 8 TMEM columns per K-step), then the norm-term
// K-step (A = constant operand in TMEM).  Only B is read from shared memory.
__device__ __forceinline__ void mma_piece_fold_ts(uint32_t tmem_d, uint32_t a_tmem, uint64_t bdesc, uint32_t ax_tmem,
                                                  uint64_t bxdesc, uint32_t bar) {
  asm volatile(
      "{\n\t.reg .pred e, f, t;\n\t.reg .b32 a1, a2, a3;\n\t.reg .b64 b1, b2, b3;\n\t"
      "setp.ne.b32 f, 0, 0;\n\t"
      "setp.eq.b32 t, 0, 0;\n\t"
      "add.u32 a1, %1, 8;\n\tadd.u32 a2, %1, 16;\n\tadd.u32 a3, %1, 24;\n\t"
      "add.s64 b1, %2, 2;\n\tadd.s64 b2, %2, 4;\n\tadd.s64 b3, %2, 6;\n\t"
      "elect.sync _|e, 0xffffffff;\n\t"
      "@e tcgen05.mma.cta_group::1.kind::i8 [%0], [%1], %2, %5, f;\n\t"
      "@e tcgen05.mma.cta_group::1.kind::i8 [%0], [a1], b1, %5, t;\n\t"
      "@e tcgen05.mma.cta_group::1.kind::i8 [%0], [a2], b2, %5, t;\n\t"
      "@e tcgen05.mma.cta_group::1.kind::i8 [%0], [a3], b3, %5, t;\n\t"
      "@e tcgen05.mma.cta_group::1.kind::i8 [%0], [%3], %4, %6, t;\n\t"
      "@e tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%7];\n\t}" ::"r"(tmem_d),
      "r"(a_tmem), "l"(bdesc), "r"(ax_tmem), "l"(bxdesc), "r"(kIdescFold), "r"(kIdescI8), "r"(bar)
      : "memory");
}

// Verify piece with A in TMEM: the four u8 x u8 K-steps (A = 8 TMEM columns per K-step), B from SMEM.
__device__ __forceinline__ void mma_piece_ts(uint32_t tmem_d, uint32_t a_tmem, uint64_t bdesc, uint32_t bar) {
  asm volatile(
      "{\n\t.reg .pred e, f, t;\n\t.reg .b32 a1, a2, a3;\n\t.reg .b64 b1, b2, b3;\n\t"
      "setp.ne.b32 f, 0, 0;\n\t"
      "setp.eq.b32 t, 0, 0;\n\t"
      "add.u32 a1, %1, 8;\n\tadd.u32 a2, %1, 16;\n\tadd.u32 a3, %1, 24;\n\t"
      "add.s64 b1, %2, 2;\n\tadd.s64 b2, %2, 4;\n\tadd.s64 b3, %2, 6;\n\t"
      "elect.sync _|e, 0xffffffff;\n\t"
      "@e tcgen05.mma.cta_group::1.kind::i8 [%0], [%1], %2, %3, f;\n\t"
      "@e tcgen05.mma.cta_group::1.kind::i8 [%0], [a1], b1, %3, t;\n\t"
      "@e tcgen05.mma.cta_group::1.kind::i8 [%0], [a2], b2, %3, t;\n\t"
      "@e tcgen05.mma.cta_group::1.kind::i8 [%0], [a3], b3, %3, t;\n\t"
      "@e tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%4];\n\t}" ::"r"(tmem_d),
      "r"(a_tmem), "l"(bdesc), "r"(kIdescI8), "r"(bar)
      : "memory");
}

// Search piece variant for the streamed verification: the four q'.r K-steps read A from TMEM, the norm-term
// K-step reads the constant operand from shared memory (its TMEM columns hold a fourth query-tile slot).
__device__ __forceinline__ void mma_piece_fold_ts_sx(uint32_t tmem_d, uint32_t a_tmem, uint64_t bdesc, uint64_t axdesc,
                                                     uint64_t bxdesc, uint32_t bar) {
  asm volatile(
      "{\n\t.reg .pred e, f, t;\n\t.reg .b32 a1, a2, a3;\n\t.reg .b64 b1, b2, b3;\n\t"
      "setp.ne.b32 f, 0, 0;\n\t"
      "setp.eq.b32 t, 0, 0;\n\t"
      "add.u32 a1, %1, 8;\n\tadd.u32 a2, %1, 16;\n\tadd.u32 a3, %1, 24;\n\t"
      "add.s64 b1, %2, 2;\n\tadd.s64 b2, %2, 4;\n\tadd.s64 b3, %2, 6;\n\t"
      "elect.sync _|e, 0xffffffff;\n\t"
      "@e tcgen05.mma.cta_group::1.kind::i8 [%0], [%1], %2, %5, f;\n\t"
      "@e tcgen05.mma.cta_group::1.kind::i8 [%0], [a1], b1, %5, t;\n\t"
      "@e tcgen05.mma.cta_group::1.kind::i8 [%0], [a2], b2, %5, t;\n\t"
      "@e tcgen05.mma.cta_group::1.kind::i8 [%0], [a3], b3, %5, t;\n\t"
      "@e tcgen05.mma.cta_group::1.kind::i8 [%0], %3, %4, %6, t;\n\t"
      "@e tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%7];\n\t}" ::"r"(tmem_d),
      "r"(a_tmem), "l"(bdesc), "l"(axdesc), "l"(bxdesc), "r"(kIdescFold), "r"(kIdescI8), "r"(bar)
      : "memory");
}

__device__ __forceinline__ void mma_commit(uint32_t bar) {
  asm volatile(
      "{\n\t.reg .pred e;\n\t"
      "elect.sync _|e, 0xffffffff;\n\t"
      "@e tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];\n\t}" ::"r"(bar)
      : "memory");
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

// 64 consecutive TMEM columns of this thread's lane (32x32b shape, .x64).
__device__ __forceinline__ void tmem_ld64(uint32_t taddr, uint32_t (&v)[64]) {
  asm volatile(
      "tcgen05.ld.sync.aligned.32x32b.x64.b32 {"
      "%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,%16,%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,"
      "%30,%31,%32,%33,%34,%35,%36,%37,%38,%39,%40,%41,%42,%43,%44,%45,%46,%47,%48,%49,%50,%51,%52,%53,%54,%55,%56,%57,"
      "%58,%59,%60,%61,%62,%63}, [%64];"
      : TID_LD32_OUT(v), TID_LD32_OUT((v + 32))
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

__device__ __forceinline__ void reg_fence64(uint32_t (&v)[64]) {
#pragma unroll
  for (int i = 0; i < 64; ++i) asm volatile("" : "+r"(v[i]));
}

// ------------------------------------------------------------------ optional cycle accounting
// Built only with -DTID_PROF (experiments): per-warp clock64 buckets, read back with
// tid_debug_read_prof().  Buckets: epilogue 0 wait-accumulator 1 scan 2 finalise 3 TMEM load + release
// (search) 4 wait-keys 5 unit tail: ratio test, count, next unit (search);
// MMA 0 wait-free-accumulator 1 wait-query 2 wait-ref; producer 0 wait-ref-slot 1 wait-query-stage;
// 7 = whole loop.
#ifdef TID_PROF
__device__ unsigned long long g_prof[148 * 32 * 8];
#define PROF_DECL unsigned long long prof_acc[8] = {0, 0, 0, 0, 0, 0, 0, 0}; long long prof_t0 = 0, prof_all = clock64();
#define PROF_B() prof_t0 = clock64();
#define PROF_E(k) prof_acc[k] += clock64() - prof_t0;
#define PROF_FLUSH()                                                                          \
  do {                                                                                        \
    prof_acc[7] = clock64() - prof_all;                                                       \
    if (lane == 0 && blockIdx.x < 148)                                                        \
      for (int k_ = 0; k_ < 8; ++k_) g_prof[(blockIdx.x * 32 + warp) * 8 + k_] = prof_acc[k_]; \
  } while (0)
#else
#define PROF_DECL
#define PROF_B()
#define PROF_E(k)
#define PROF_FLUSH()
#endif

// TMEM columns: accumulators [0, 384); search-path A operands: kTQ query tiles of 32 columns
// (128 rows x 128 B, K packed 4 bytes per column) and the constant norm-term operand (8 columns).
constexpr int kTQ = 3;
constexpr int kQCols = kDim / 4;
constexpr int kTQBase = kTmemBufs * kPiece;
constexpr int kAxCol = kTQBase + kTQ * kQCols;
static_assert(kAxCol + kXDim / 4 <= 512, "TMEM budget");

constexpr int kProducerWarp = 0;               // warp 0: TMA producer
constexpr int kFirstMmaWarp = 1;               // warps 1..kNG: MMA issuer of group mw
constexpr int kFirstEpiWarp = 1 + kNG;         // then 4 warps per group; lane quarter w % 4
// (any 4 consecutive warps cover the 4 TMEM lane quarters w % 4)
static_assert(kNumThreads <= 512, "at most 16 warps: >= 128 registers per thread");

// ------------------------------------------------------------------ shared memory plan
struct SmemPlan {
  static constexpr uint32_t kR = 0;                                        // kMaxSlots x 32 KiB
  static constexpr uint32_t kQ = kR + kMaxSlots * kRTileBytes;             // kQStages x 16 KiB
  static constexpr uint32_t kX = kQ + kQStages * kQTileBytes;              // kMaxSlots x 8 KiB norm-term tiles
  static constexpr uint32_t kAx = kX + kMaxSlots * kXTileBytes;            // 4 KiB constant norm-term operand
  static constexpr uint32_t kCol = kAx + kBM * kXDim;                      // kMaxSlots x 1 KiB
  static constexpr uint32_t kBar = kCol + kMaxSlots * kColBytes;           // mbarriers
  static constexpr uint32_t kQFull = kBar;
  static constexpr uint32_t kQEmpty = kQFull + 8 * kQStages;
  static constexpr uint32_t kRFull = kQEmpty + 8 * kQStages;
  static constexpr uint32_t kREmpty = kRFull + 8 * kMaxSlots;
  static constexpr uint32_t kTFull = kREmpty + 8 * kMaxSlots;
  static constexpr uint32_t kTEmpty = kTFull + 8 * kTmemBufs;
  static constexpr uint32_t kTQFull = kTEmpty + 8 * kTmemBufs;           // query tiles staged in TMEM (search)
  static constexpr uint32_t kTQEmpty = kTQFull + 8 * kTQ;
  static constexpr uint32_t kXReady = kTQEmpty + 8 * kTQ;                // norm digits expanded on chip (search)
  static constexpr uint32_t kAxFull = kXReady + 8 * kMaxSlots;
  static constexpr uint32_t kTmemPtr = kAxFull + 8;
  static constexpr uint32_t kEnd = kTmemPtr + 16;
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

// ------------------------------------------------------------------ epilogue: two-partition top-2
// Each epilogue thread owns one TMEM lane = one query row j, and needs the two smallest packed
// keys 256 * (N_R - 2 q_j.r_i) + i over the 256 columns i of a reference chunk (Alg. 1 steps
// 4-7 P:375-382; "keep two registers" P:420-425).  Instead of a running top-2 (min + max + min
// per element), the columns are covered by two partitions that separate every pair:
//   P : (x32 load c, half h)        -> 16 groups of 16 columns      (c = 0..7, h = j >= 16)
//   P': column position b = j % 16  -> 16 groups of 16 columns      (j = position in the load)
// Two columns in the same P group differ in b, so no pair shares both groups.  Then
//   min(all) = min(P minima)  and  second(all) = min(second(P minima), second(P' minima)):
// if the two smallest columns fall in different P groups, both are P minima; otherwise they
// are in different P' groups and both are P' minima; and neither side can undercut the true
// second.  Both partitions are pure 3-input minima (VIMNMX3, one per two new elements), so the
// scan costs ~1.3 ALU ops per element instead of 2.5, and it is exact (keys carry the index).
__device__ __forceinline__ int min3i(int a, int b, int c) { return __vimin3_s32(a, b, c); }
__device__ __forceinline__ int min16(const int* k) {
  const int a = min3i(k[0], k[1], k[2]), b = min3i(k[3], k[4], k[5]), c = min3i(k[6], k[7], k[8]);
  const int d = min3i(k[9], k[10], k[11]), e = min3i(k[12], k[13], k[14]);
  return min(min3i(a, b, c), min3i(d, e, k[15]));
}

// 32 consecutive columns of this lane (one x32 TMEM load, already landed in v) folded into the
// partition state: R[b] = P' minima, (T1 <= T2) = the two smallest P minima so far.
__device__ __forceinline__ void scan32_regs(const uint32_t* v, uint32_t ck_addr, int (&R)[16], int& T1, int& T2) {
  int k[32];
#pragma unroll
  for (int i = 0; i < 32; i += 4) {
    const int4 c4 = lds128(ck_addr + i * 4);
    k[i] = c4.x - 512 * static_cast<int>(v[i]);
    k[i + 1] = c4.y - 512 * static_cast<int>(v[i + 1]);
    k[i + 2] = c4.z - 512 * static_cast<int>(v[i + 2]);
    k[i + 3] = c4.w - 512 * static_cast<int>(v[i + 3]);
  }
  const int x = min16(k), y = min16(k + 16);
#pragma unroll
  for (int b = 0; b < 16; ++b) R[b] = min3i(R[b], k[b], k[b + 16]);
  const int lo = min(x, y), hi = max(x, y);
  T2 = min3i(T2, max(T1, lo), hi);
  T1 = min(T1, lo);
}

// Two smallest keys (k1 < k2) of a 256-column chunk from the partition state.  The 16 P'
// minima are themselves split by a 4 x 4 grid (rows R[4a..4a+3], columns R[b], R[b+4], ...),
// which again separates every pair, so second(R) = min(second(row minima), second(col minima)).
__device__ __forceinline__ void finish_partition(const int (&R)[16], int T1, int T2, int& k1, int& k2) {
  int rm[4], cm[4];
#pragma unroll
  for (int a = 0; a < 4; ++a) {
    rm[a] = min(min3i(R[4 * a], R[4 * a + 1], R[4 * a + 2]), R[4 * a + 3]);
    cm[a] = min(min3i(R[a], R[a + 4], R[a + 8]), R[a + 12]);
  }
  const int sr = min3i(max(min(rm[0], rm[1]), min(rm[2], rm[3])), max(rm[0], rm[1]), max(rm[2], rm[3]));
  const int sc = min3i(max(min(cm[0], cm[1]), min(cm[2], cm[3])), max(cm[0], cm[1]), max(cm[2], cm[3]));
  k1 = T1;  // the P minima cover every column
  k2 = min3i(T2, sr, sc);
}

// Search path: the same two-partition scan on the folded values X (TMEM, no column keys), for
// the two LARGEST X.  `lim` = real columns among these 32 (padding is masked to INT_MIN).
__device__ __forceinline__ int max3i(int a, int b, int c) { return __vimax3_s32(a, b, c); }
__device__ __forceinline__ int max16(const int* k) {
  const int a = max3i(k[0], k[1], k[2]), b = max3i(k[3], k[4], k[5]), c = max3i(k[6], k[7], k[8]);
  const int d = max3i(k[9], k[10], k[11]), e = max3i(k[12], k[13], k[14]);
  return max(max3i(a, b, c), max3i(d, e, k[15]));
}
template <bool kMask>
__device__ __forceinline__ void scan32_fold(const uint32_t* v, int lim, int (&R)[16], int& T1, int& T2) {
  int k[32];
#pragma unroll
  for (int i = 0; i < 32; ++i) k[i] = (!kMask || i < lim) ? static_cast<int>(v[i]) : INT_MIN;
  const int x = max16(k), y = max16(k + 16);
#pragma unroll
  for (int b = 0; b < 16; ++b) R[b] = max3i(R[b], k[b], k[b + 16]);
  const int hi = max(x, y), lo = min(x, y);
  T2 = max3i(T2, min(T1, hi), lo);
  T1 = max(T1, hi);
}
__device__ __forceinline__ void finish_fold(const int (&R)[16], int T1, int T2, int& x1, int& x2) {
  int rm[4], cm[4];
#pragma unroll
  for (int a = 0; a < 4; ++a) {
    rm[a] = max(max3i(R[4 * a], R[4 * a + 1], R[4 * a + 2]), R[4 * a + 3]);
    cm[a] = max(max3i(R[a], R[a + 4], R[a + 8]), R[a + 12]);
  }
  const int sr = max3i(min(max(rm[0], rm[1]), max(rm[2], rm[3])), min(rm[0], rm[1]), min(rm[2], rm[3]));
  const int sc = max3i(min(max(cm[0], cm[1]), max(cm[2], cm[3])), min(cm[0], cm[1]), min(cm[2], cm[3]));
  x1 = T1;
  x2 = max3i(T2, sr, sc);
}

__device__ __forceinline__ uint32_t dp4a_su(uint32_t a_s8, uint32_t b_u8, uint32_t c) {
  uint32_t d;
  asm("dp4a.s32.u32 %0, %1, %2, %3;" : "=r"(d) : "r"(a_s8), "r"(b_u8), "r"(c));
  return d;
}

// Exact 2-NN distances (d1 <= d2) of one query row against one reference, straight from global
// memory (the rare rows whose ratio decision the folded +-1 leaves open).  Whole warp; the
// result is valid in every lane.  d = N_Q - 2 q'.r - W (column term W, < 0 marks padding).
// W comes from the reference's column terms in shared memory (ck0 = its first chunk's 1 KiB; the
// chunks of one reference occupy consecutive slots): the copy of the stored W (search) or the terms
// the kernel computed from the tile (folded verification).
// kQRaw: p.qs holds the raw u8 queries (streamed verification shifts them on chip), shifted here.
template <bool kQRaw = false>
__device__ __forceinline__ void exact_row_global(const MatchParams& p, int qi, int row, int64_t ref, int32_t nqv,
                                                 int lane, int cpr, uint32_t ck0, int& d1, int& d2) {
  const uint4* qrow = reinterpret_cast<const uint4*>(p.qs + (static_cast<int64_t>(qi) * p.n_rows + row) * kDim);
  uint4 q[8];
#pragma unroll
  for (int w = 0; w < 8; ++w) {
    q[w] = qrow[w];
    if (kQRaw) q[w] = make_uint4(q[w].x ^ 0x80808080u, q[w].y ^ 0x80808080u, q[w].z ^ 0x80808080u, q[w].w ^ 0x80808080u);
  }
  int a1 = INT_MAX, a2 = INT_MAX;
  for (int col = lane; col < cpr * kBN; col += 32) {
    int32_t W;
    asm volatile("ld.shared.s32 %0, [%1];" : "=r"(W) : "r"(ck0 + col * 4));
    if (col >= p.m || W < 0) continue;
    const uint4* rr = reinterpret_cast<const uint4*>(p.rdesc + ((p.ref_map_base + ref) * p.m + col) * kDim);
    uint32_t dot = 0;
#pragma unroll
    for (int w = 0; w < 8; ++w) {
      const uint4 x = rr[w];
      dot = dp4a_su(q[w].x, x.x, dot); dot = dp4a_su(q[w].y, x.y, dot);
      dot = dp4a_su(q[w].z, x.z, dot); dot = dp4a_su(q[w].w, x.w, dot);
    }
    const int d = nqv - 2 * static_cast<int>(dot) - W;
    a2 = min(a2, max(a1, d));
    a1 = min(a1, d);
  }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) {
    const int b1 = __shfl_xor_sync(0xffffffffu, a1, o), b2 = __shfl_xor_sync(0xffffffffu, a2, o);
    const int m2 = min(max(a1, b1), min(a2, b2));
    a1 = min(a1, b1);
    a2 = m2;
  }
  d1 = a1;
  d2 = a2;
}

// Pieces of kPiece columns in a reference's last 256-column chunk that can hold real keypoints:
// columns >= m are padding for every reference (m = 384: the second chunk is half padding), so
// those pieces are neither computed nor scanned (a chunk with fewer than 4 pieces leaves the
// static buffer / phase schedule with odd use counts: use_parity() tracks the flips).
__host__ __device__ __forceinline__ int piece_count_last(int m, int cpr) {
  return (m - (cpr - 1) * kBN + kPiece - 1) / kPiece;
}
// Phase flips of the two TMEM buffers after a chunk of np pieces (buffer pp & 1): buffer 0 is used
// ceil(np / 2) times, buffer 1 floor(np / 2) times; bit b set when that count is odd.
__device__ __forceinline__ uint32_t use_parity(int np) {
  return (((np + 1) >> 1) & 1u) | (((np >> 1) & 1u) << 1);
}

// The fifth MMA K-step's B operand for one reference column: 32 u8 digits of E = floor(W / 2)
// against the constant operand a = (255 x 15, 1, 255 x 15, 1), i.e. E = 255 * (sum of the 30
// "255"-weighted digits) + d15 + d31.  The 30 weighted digits (positions 0..14, 16..30, ranks
// 0..29) are filled greedily: rank k holds clamp(hi - 255 k, 0, 255) with hi = E / 255 <= 4,112,
// so ranks < q = hi / 255 are 255, rank q holds hi mod 255 and the rest 0; d15 = E mod 255,
// d31 = 0 (capacity 7,650 * 255 + 254 > max E = 1,048,576).  Padding columns (W < 0): zeros.
// Built as 8 rank words, then moved into position order with byte permutes.
__device__ __forceinline__ void norm_digits(int32_t W, uint32_t (&w8)[8]) {
  const uint32_t E = W > 0 ? static_cast<uint32_t>(W) >> 1 : 0u;
  const uint32_t hi = E / 255u, lo = E - 255u * hi;
  const uint32_t q = hi / 255u, rem = hi - 255u * q;
  // Rank word i (ranks 4i .. 4i+3) has t = q - 4i full bytes, then rem, then zeros: one byte permute of
  // {0, b = rem | 0xFFFFFF00} whose selector (nibble 5 = 0xFF, 4 = rem, 0 = 0x00) is a 16-bit window
  // of the nibble string 0x4_5555_5555 at 4 (8 - clamp(t, -1, 5)) bits (tools/digits_check.py checks
  // every W against the greedy encoding).
  const uint32_t b = 0xFFFFFF00u | rem;
  const int s0 = 32 - 4 * static_cast<int>(q);
  uint32_t rk[8];  // rank words: byte b of rk[i] = digit of rank 4 i + b
#pragma unroll
  for (int i = 0; i < 8; ++i) {
    const int sh = min(max(s0 + 16 * i, 12), 36);
    const uint32_t sel = static_cast<uint32_t>(0x0000000455555555ull >> sh);
    rk[i] = __byte_perm(0u, b, sel);
  }
  w8[0] = rk[0];
  w8[1] = rk[1];
  w8[2] = rk[2];
  w8[3] = (rk[3] & 0x00FFFFFFu) | (lo << 24);              // ranks 12..14, then position 15 = lo
  w8[4] = __byte_perm(rk[3], rk[4], 0x6543);                // ranks 15..18
  w8[5] = __byte_perm(rk[4], rk[5], 0x6543);                // ranks 19..22
  w8[6] = __byte_perm(rk[5], rk[6], 0x6543);                // ranks 23..26
  w8[7] = __byte_perm(rk[6], rk[7], 0x6543) & 0x00FFFFFFu;  // ranks 27..29, position 31 = 0
}

// Per job: the fifth MMA K-step's digits of every slot column (see norm_digits) — and, for the folded
// verification (no stored column terms, p.colkey == nullptr), first the column terms themselves,
// W = 256 sum r - N_R from the tile row in shared memory (the order of its 16-byte chunks is
// irrelevant under SWIZZLE_128B), -1 - (real columns of the chunk) for padding.  Columns x = first,
// first + stride, ... of the job's nslots slots starting at slot b0.
__device__ __forceinline__ void expand_slot_terms(const MatchParams& p, uint32_t sbase, int b0, int nslots, int cpr,
                                                  int mcap, int first, int stride) {
  for (int x = first; x < nslots * kBN; x += stride) {
    const int sl = x / kBN, col = x % kBN;
    int W;
    const uint32_t wa = sbase + SmemPlan::kCol + (b0 + sl) * kColBytes + col * 4;
    if (p.colkey) {
      asm volatile("ld.shared.s32 %0, [%1];" : "=r"(W) : "r"(wa));
    } else {
      // folded verification: W = 256 sum r - N_R of the tile row (order of its 16-byte chunks
      // irrelevant under SWIZZLE_128B), -1 - (real columns of the chunk) for padding
      const int gcol = (sl % cpr) * kBN + col;
      if (gcol < mcap) {
        const uint32_t row = sbase + SmemPlan::kR + (b0 + sl) * kRTileBytes + col * kDim;
        uint32_t nr = 0, sr = 0;
#pragma unroll
        for (int w = 0; w < kDim / 16; ++w) {
          const int4 x4 = lds128(row + 16 * w);
          nr = __dp4a(static_cast<uint32_t>(x4.x), static_cast<uint32_t>(x4.x), nr);
          nr = __dp4a(static_cast<uint32_t>(x4.y), static_cast<uint32_t>(x4.y), nr);
          nr = __dp4a(static_cast<uint32_t>(x4.z), static_cast<uint32_t>(x4.z), nr);
          nr = __dp4a(static_cast<uint32_t>(x4.w), static_cast<uint32_t>(x4.w), nr);
          sr = __dp4a(static_cast<uint32_t>(x4.x), 0x01010101u, sr);
          sr = __dp4a(static_cast<uint32_t>(x4.y), 0x01010101u, sr);
          sr = __dp4a(static_cast<uint32_t>(x4.z), 0x01010101u, sr);
          sr = __dp4a(static_cast<uint32_t>(x4.w), 0x01010101u, sr);
        }
        W = 256 * static_cast<int>(sr) - static_cast<int>(nr);
      } else {
        W = -1 - max(0, min(mcap - (sl % cpr) * kBN, kBN));
      }
      asm volatile("st.shared.s32 [%0], %1;" ::"r"(wa), "r"(W) : "memory");
    }
    uint32_t w8[8];
    norm_digits(W, w8);
    const uint32_t dst = sbase + SmemPlan::kX + (b0 + sl) * kXTileBytes + col * kXDim;
    asm volatile("st.shared.v4.b32 [%0], {%1, %2, %3, %4};" ::"r"(dst), "r"(w8[0]), "r"(w8[1]), "r"(w8[2]),
                 "r"(w8[3]) : "memory");
    asm volatile("st.shared.v4.b32 [%0], {%1, %2, %3, %4};" ::"r"(dst + 16), "r"(w8[4]), "r"(w8[5]), "r"(w8[6]),
                 "r"(w8[7]) : "memory");
  }
}

// ------------------------------------------------------------------ fused match kernel
// One persistent CTA per SM.  A job = (up to kNG = 3 references resident in SMEM, fewer chunks'
// worth for m > 256) x (range of query tiles streamed through a kQStages ring; search: copied
// once per tile into TMEM).  Unit u = (query tile t, reference s), s fastest, belongs to epilogue
// group u % kNG (group g <-> reference g, so its counts accumulate in a register over the query's
// tiles).  Each 256-column reference chunk of a unit is 4 MMA pieces of 64 columns through the
// group's 2 TMEM buffers (buffer pp & 1, phase pp >> 1: compile-time, fully unrolled); group g has
// its own MMA warp, so the MMA of the next piece overlaps the scan of the current one, and the 3
// groups (3 epilogue warps per SMSP) hide each other's TMEM-load and barrier latency.
// kFold: the search path (folded norms, no column keys in the scan, counts only);
// otherwise the verify path (packed column keys, exact (d1, i1, d2, i2)).
// kSkip: the last chunk of every reference has fewer than 4 pieces that can hold keypoints
// (m mod 256 in 1..192): those pieces are skipped, with the buffer phases tracked at run time;
// otherwise every chunk is 4 pieces and the schedule is fully static.
template <bool kFold, bool kSkip>
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
  auto tqfull = [&](int i) { return sbase + SmemPlan::kTQFull + 8 * i; };
  auto tqempty = [&](int i) { return sbase + SmemPlan::kTQEmpty + 8 * i; };
  auto xready = [&](int i) { return sbase + SmemPlan::kXReady + 8 * i; };
  const uint32_t axfull = sbase + SmemPlan::kAxFull;
  uint32_t* tmem_ptr_smem = reinterpret_cast<uint32_t*>(smem + SmemPlan::kTmemPtr);

  if (kFold) {  // constant norm-term operand: every row (255 x 15, 1, 255 x 15, 1); both 16-B halves equal
    uint32_t* ax = reinterpret_cast<uint32_t*>(smem + SmemPlan::kAx);
    for (int i = threadIdx.x; i < kBM * kXDim / 4; i += blockDim.x) ax[i] = (i & 3) == 3 ? 0x01FFFFFFu : 0xFFFFFFFFu;
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");  // generic writes -> tensor-core reads
  }
  if (threadIdx.x == 0) {
    prefetch_tmap(&qmap);
    prefetch_tmap(&rmap);
    // query stages: each tile is copied SMEM -> TMEM once (freed by that copy); the MMAs read A from TMEM
    for (int i = 0; i < kQStages; ++i) { mbar_init(qfull(i), 1); mbar_init(qempty(i), 1); }
    for (int i = 0; i < kTQ; ++i) { mbar_init(tqfull(i), 1); mbar_init(tqempty(i), kNG); }
    mbar_init(axfull, 1);
    // reference slots: MMA operands + column keys read by every epilogue warp
    for (int i = 0; i < kMaxSlots; ++i) {
      mbar_init(rfull(i), 1);
      mbar_init(rempty(i), kNG + kEpiWarps);
      // search: the kNG MMA warps expanded the slot's norm digits; verify: the epilogue computed the
      // keys and masked rows beyond m_r (one arrival)
      mbar_init(xready(i), kFold ? (p.colkey ? kNG : kNG + kEpiWarps) : 1);
    }
    for (int i = 0; i < kTmemBufs; ++i) { mbar_init(tfull(i), 1); mbar_init(tempty(i), 4); }
    fence_barrier_init();
  }
  if (warp == kFirstMmaWarp) {  // TMEM: 8 accumulator buffers x 64 columns (all 512)
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 512;" ::"r"(
                     smem_u32(tmem_ptr_smem))
                 : "memory");
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
  }
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem_base = *tmem_ptr_smem;

  PROF_DECL
  if (warp == kProducerWarp) {
    // ===================== TMA producer (lane 0) + norm-digit expansion (whole warp) =====================
    if (kFold && lane == 0) {  // constant norm-term operand -> TMEM, once
      tc_fence_after();
      tmem_cp_128x256b(tmem_base + kAxCol, smem_desc_sw32(sbase + SmemPlan::kAx));
      commit_one(axfull);
    }
    {
      uint32_t qctr = 0;
      uint32_t slot_par = 0;  // bit sl = phase parity of reference slot sl
      uint32_t jc = 0;        // this CTA's job count: slot bank (jc & 1) when p.slot_banks == 2
      for (int32_t j = blockIdx.x; j < p.n_jobs; j += gridDim.x, ++jc) {
        const Job J = decode_job(p, j);
        const int nslots = J.nr * cpr;
        const int b0 = p.slot_banks == 2 ? static_cast<int>(jc & 1u) * (kMaxSlots / 2) : 0;
        if (lane == 0) {
          for (int sl = 0; sl < nslots; ++sl) {
            PROF_B(); mbar_wait_sleep(rempty(b0 + sl), (slot_par >> (b0 + sl) & 1u) ^ 1); PROF_E(0);
            const bool ck_global = kFold && p.colkey != nullptr;  // else computed on chip (folded verify)
            mbar_expect_tx(rfull(b0 + sl), kRTileBytes + (ck_global ? kColBytes : 0u));
            const int s = sl / cpr, c = sl % cpr;
            const int64_t ref = J.ref_first + s;
            tma_load_3d(sbase + SmemPlan::kR + (b0 + sl) * kRTileBytes, &rmap, rfull(b0 + sl), 0, c * kBN,
                        static_cast<int>(p.ref_map_base + ref));
            if (ck_global)  // search: the stored column terms W (verify computes them on chip)
              bulk_load(sbase + SmemPlan::kCol + (b0 + sl) * kColBytes, p.colkey + (ref * cpr + c) * kColInts, kColBytes,
                        rfull(b0 + sl));
          }
        }
        __syncwarp();
        slot_par ^= ((1u << nslots) - 1u) << b0;
        const int ntiles = J.nq * T;
        if (lane == 0) {
          // TMA tile t+1 into shared memory while tile t is copied to its TMEM slot (the MMAs read A
          // from TMEM, so each query tile crosses the shared-memory port once, not once per piece)
          auto issue = [&](int t) {
            const uint32_t gq = qctr + t, st = gq % kQStages;
            PROF_B(); mbar_wait_sleep(qempty(st), ((gq / kQStages) & 1) ^ 1); PROF_E(1);
            mbar_expect_tx(qfull(st), kQTileBytes);
            tma_load_3d(sbase + SmemPlan::kQ + st * kQTileBytes, &qmap, qfull(st), 0, (t % T) * kBM, J.q_first + t / T);
          };
          if (ntiles > 0) issue(0);
          for (int t = 0; t < ntiles; ++t) {
            if (t + 1 < ntiles) issue(t + 1);
            const uint32_t gq = qctr + t, st = gq % kQStages, sl = gq % kTQ;
            mbar_wait(qfull(st), (gq / kQStages) & 1);
            mbar_wait_sleep(tqempty(sl), ((gq / kTQ) & 1) ^ 1);
            tc_fence_after();
            const uint64_t sd = smem_desc_sw128(sbase + SmemPlan::kQ + st * kQTileBytes);
#pragma unroll
            for (int k = 0; k < kDim / kXDim; ++k) tmem_cp_128x256b(tmem_base + kTQBase + sl * kQCols + 8 * k, sd + 2 * k);
            commit_one(tqfull(sl));
            commit_one(qempty(st));
          }
          qctr += ntiles;
        }
      }
    }
  } else if (warp < kFirstEpiWarp) {
    // ===================== MMA issuers: warp mw serves epilogue group mw =====================
    // Issuing tcgen05.mma costs the issuing SMSP throughput, so the kNG issuers sit on SMSPs 1-3.
    // Warp mw issues the pieces of the units u with u % kNG == mw, in order, into its group's two
    // 64-column buffers (whole warp, one elected lane).  Every warp commits the release of every
    // query tile (waiting for tiles it never used, so the stage phases stay in order).
    const int mw = warp - kFirstMmaWarp;
    const int np_last = kSkip ? piece_count_last(p.m, cpr) : kPiecesPerChunk;
    uint32_t ph_t = 0;  // bit b: phase flip of this group's TMEM buffer b (chunks with an odd use count)
    uint32_t qctr = 0;
    if (kFold) mbar_wait(axfull, 0);  // constant norm-term operand in TMEM
    uint32_t slot_par = 0;  // bit sl = phase parity of reference slot sl
    uint32_t jc = 0;
    for (int32_t j = blockIdx.x; j < p.n_jobs; j += gridDim.x, ++jc) {
      const Job J = decode_job(p, j);
      const int nslots = J.nr * cpr;
      const int b0 = p.slot_banks == 2 ? static_cast<int>(jc & 1u) * (kMaxSlots / 2) : 0;
      const int U = J.nq * T * J.nr;
      if constexpr (kFold) {
        // the norm digits of the job's slots, expanded by the kNG MMA warps (HBM keeps only the column
        // terms W: 4 B per keypoint instead of 32 B of digits); both 16-byte halves of the constant
        // operand are equal, so the SWIZZLE_32B placement of a row's halves does not matter and rows
        // are written plainly, 32 B each
        for (int sl = 0; sl < nslots; ++sl) mbar_wait(rfull(b0 + sl), slot_par >> (b0 + sl) & 1u);
        const int mcap = p.colkey ? p.m : (p.m_valid ? min(p.m_valid[J.ref_first], p.m) : p.m);
        // folded verification: the 3 MMA warps and the 12 epilogue warps share the work (job start)
        if (p.colkey) expand_slot_terms(p, sbase, b0, nslots, cpr, mcap, mw * 32 + lane, kNG * 32);
        else expand_slot_terms(p, sbase, b0, nslots, cpr, mcap, mw * 32 + lane, (kNG + kEpiWarps) * 32);
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");  // generic writes -> tensor-core reads
        __syncwarp();
        if (lane == 0)
          for (int sl = 0; sl < nslots; ++sl) mbar_arrive(xready(b0 + sl));
      }
      uint32_t ready_mask = 0;
      int waited = 0, t = 0, s = 0, g = 0;
      for (int u = 0; u < U; ++u) {
        if (g == mw) {
          while (waited <= t) {
            const uint32_t gq = qctr + waited;
            PROF_B();
            mbar_wait(tqfull(gq % kTQ), (gq / kTQ) & 1);
            PROF_E(1);
            ++waited;
          }
          const uint32_t at = tmem_base + kTQBase + ((qctr + t) % kTQ) * kQCols;  // A (query tile) in TMEM
          for (int c = 0; c < cpr; ++c) {
            const int sl = b0 + s * cpr + c;
            if (!(ready_mask >> sl & 1u)) {
              PROF_B(); mbar_wait(rfull(sl), (slot_par >> sl & 1u));
              // search: norm digits expanded; verify with m_r: rows beyond m_r zeroed
              if (kFold || p.m_valid) mbar_wait(xready(sl), (slot_par >> sl & 1u));
              PROF_E(2);
              ready_mask |= 1u << sl;
            }
            const uint64_t bd0 = smem_desc_sw128(sbase + SmemPlan::kR + sl * kRTileBytes);
            const int np = c == cpr - 1 ? np_last : kPiecesPerChunk;
#pragma unroll
            for (int pp = 0; pp < kPiecesPerChunk; ++pp) {  // static buffer / phase (see the epilogue)
              if (kSkip && pp >= np) break;  // all-padding pieces of the last chunk are never computed
              const uint32_t buf = mw * kNB + (pp & 1);
              PROF_B(); mbar_wait(tempty(buf), (((pp >> 1) ^ (ph_t >> (pp & 1))) & 1) ^ 1); PROF_E(0);
              tc_fence_after();
              // rows kPiece*pp.. of the chunk: SWIZZLE_128B core groups of 8 rows x 128 B
              const uint64_t bd = bd0 + pp * (kPiece * kDim >> 4);
#ifdef TID_NOMMA  // timing experiment only: no MMAs (the commit still signals the buffer)
              if (kFold) mma_commit(tfull(buf)); else
#endif
              if (kFold)  // + norm-term K-step: rows kPiece*pp.. of the 32-B-wide tile
                mma_piece_fold_ts(tmem_base + buf * kPiece, at, bd, tmem_base + kAxCol,
                                  smem_desc_sw32(sbase + SmemPlan::kX + sl * kXTileBytes) + pp * (kPiece * kXDim >> 4),
                                  tfull(buf));
              else
                mma_piece_ts(tmem_base + buf * kPiece, at, bd, tfull(buf));
            }
            if (kSkip) ph_t ^= use_parity(np);
          }
        }
        if (s == J.nr - 1) {  // this warp's release of query tile t (covers all its prior MMAs)
          const uint32_t gq = qctr + t;
          if (waited <= t) {  // never touched tile t: still wait for it so the phase order holds
            mbar_wait(tqfull(gq % kTQ), (gq / kTQ) & 1);
            waited = t + 1;
          }
          mma_commit(tqempty(gq % kTQ));
        }
        if (++g == kNG) g = 0;
        if (++s == J.nr) { s = 0; ++t; }
      }
      for (int sl = b0; sl < b0 + nslots; ++sl) {
        if (!(ready_mask >> sl & 1u)) {  // keep rempty / xready phases ordered
          mbar_wait(rfull(sl), (slot_par >> sl & 1u));
          if (kFold || p.m_valid) mbar_wait(xready(sl), (slot_par >> sl & 1u));
        }
        mma_commit(rempty(sl));
        slot_par ^= 1u << sl;
      }
      qctr += J.nq * T;
    }
  } else {
    // ===================== epilogue: TMEM -> registers -> top-2 -> ratio -> count =====================
    // Each piece (64 columns) is fetched with one x64 TMEM load and its buffer released as soon
    // as the load has landed, so the MMA of the group's next-but-one piece overlaps the scan; the
    // 3 groups (3 epilogue warps per SMSP) hide each other's load latency.
    const int ew = warp - kFirstEpiWarp;  // 0 .. 4*kNG-1
    const int g = ew >> 2;                // group: units u with u % kNG == g
    const int quarter = warp & 3;         // TMEM lanes 32*quarter .. +31 (hardware restriction)
    const uint32_t taddr_q = tmem_base + (static_cast<uint32_t>(quarter * 32) << 16);
    const int row_in_tile = quarter * 32 + lane;
    const int nq_ld = T * kBM;
    const bool ratio32 = p.num2 <= 511u && p.den2 <= 511u;  // den^2 * d fits 32 bits (d <= 8,323,200)
    uint32_t slot_par = 0;                // bit sl = phase parity of reference slot sl
    const int np_last = kSkip ? piece_count_last(p.m, cpr) : kPiecesPerChunk;
    uint32_t ph_t = 0;                    // bit b: phase flip of TMEM buffer b (see the MMA warps)
    uint32_t v[64];

    uint32_t jc = 0;
    for (int32_t j = blockIdx.x; j < p.n_jobs; j += gridDim.x, ++jc) {
      const Job J = decode_job(p, j);
      const int nslots = J.nr * cpr;
      const int b0 = p.slot_banks == 2 ? static_cast<int>(jc & 1u) * (kMaxSlots / 2) : 0;
      const int U = J.nq * T * J.nr;
      // column keys of every slot of the job (also orders this warp's rempty arrivals)
      const int mcap = (!kFold && p.m_valid) ? min(p.m_valid[J.ref_first], p.m) : p.m;  // issued before the wait
      PROF_B();
      for (int sl = 0; sl < nslots; ++sl) mbar_wait(rfull(b0 + sl), slot_par >> (b0 + sl) & 1u);
      if (kFold && p.colkey == nullptr) {  // folded verification: column terms + digits, shared with the MMA warps
        const int mcap = p.m_valid ? min(p.m_valid[J.ref_first], p.m) : p.m;
        expand_slot_terms(p, sbase, b0, nslots, cpr, mcap, (kNG + ew) * 32 + lane, (kNG + kEpiWarps) * 32);
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
        __syncwarp();
        if (lane == 0)
          for (int sl = 0; sl < nslots; ++sl) mbar_arrive(xready(b0 + sl));
        for (int sl = 0; sl < nslots; ++sl) mbar_wait(xready(b0 + sl), slot_par >> (b0 + sl) & 1u);
      }
      if constexpr (!kFold) {
        // verify: the packed column keys N_R * 256 + i (Alg. 1 step 1) computed here from the
        // reference tile already in shared memory (no separate pass over the references in HBM).
        // A row's 128 bytes stay within its 128-byte line under SWIZZLE_128B, so the sum over its
        // eight 16-byte chunks does not depend on their order.  Rows >= min(m_r, m) get the sentinel.
        for (int x = ew * 32 + lane; x < nslots * kBN; x += kEpiWarps * 32) {
          const int sl = x / kBN, i = x % kBN;
          const int col = (sl % cpr) * kBN + i;
          uint32_t acc = 0;
          const uint32_t row = sbase + SmemPlan::kR + sl * kRTileBytes + i * kDim;
          if (col < mcap) {
#pragma unroll
            for (int w = 0; w < kDim / 16; ++w) {
              const int4 x4 = lds128(row + 16 * w);
              acc = __dp4a(static_cast<uint32_t>(x4.x), static_cast<uint32_t>(x4.x), acc);
              acc = __dp4a(static_cast<uint32_t>(x4.y), static_cast<uint32_t>(x4.y), acc);
              acc = __dp4a(static_cast<uint32_t>(x4.z), static_cast<uint32_t>(x4.z), acc);
              acc = __dp4a(static_cast<uint32_t>(x4.w), static_cast<uint32_t>(x4.w), acc);
            }
          } else if (col < p.m) {
            // a row beyond this pair's m_r holds the caller's bytes: zero it, so its product is 0 and
            // the sentinel key 256 * (2^23 - 1) + i never wins (rows >= m are zero-filled by TMA)
#pragma unroll
            for (int w = 0; w < kDim / 16; ++w)
              asm volatile("st.shared.v4.b32 [%0], {%1, %1, %1, %1};" ::"r"(row + 16 * w), "r"(0) : "memory");
          }
          const int32_t key = (col < mcap ? static_cast<int32_t>(acc) : kSentinelNorm) * 256 + i;
          asm volatile("st.shared.s32 [%0], %1;" ::"r"(sbase + SmemPlan::kCol + sl * kColBytes + i * 4), "r"(key)
                       : "memory");
        }
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");  // zeroed rows -> tensor-core reads
        named_bar(1, kEpiWarps * 32);  // every key of the job written before any warp scans
        if (p.m_valid && ew == 0 && lane == 0)  // the MMA warps may read the masked tiles
          for (int sl = 0; sl < nslots; ++sl) mbar_arrive(xready(sl));
      }
      PROF_E(4);
      // own units u = g, g + kNG, ...; unit u = (tile t = u / nr, reference s = u % nr), and
      // t = (query qi - q_first) * T + tq.  Tracked incrementally (no divisions per unit).
      int u = g, s = g % J.nr, tq = g / J.nr, qi = J.q_first;
      while (tq >= T) { tq -= T; ++qi; }
      int nvalid = u < U ? min(p.n_valid ? p.n_valid[qi] : p.n_rows, p.n_rows) : 0;
      const int32_t* nq_row = p.nq + static_cast<int64_t>(qi) * nq_ld + row_in_tile;
      uint32_t cnt = 0;
      while (u < U) {
        const int row = tq * kBM + row_in_tile;
        const bool valid = row < nvalid;
        const int32_t nqv = valid ? nq_row[tq * kBM] : 0;
        const bool has_next = u + kNG < U;
        bool pass = false;
        if constexpr (kFold) {
          int G1 = INT_MIN, G2 = INT_MIN;  // two largest folded values X over the reference
          for (int c = 0; c < cpr; ++c) {
            const uint32_t ck = sbase + SmemPlan::kCol + (b0 + s * cpr + c) * kColBytes;
            int kpc;  // real columns of this chunk: the last column term is -1 - kpc when padded
            asm volatile("ld.shared.s32 %0, [%1];" : "=r"(kpc) : "r"(ck + (kBN - 1) * 4));
            kpc = kpc < 0 ? -1 - kpc : kBN;
            int R[16];
#pragma unroll
            for (int b = 0; b < 16; ++b) R[b] = INT_MIN;
            int T1 = INT_MIN, T2 = INT_MIN;
            // 4 pieces per chunk through the group's 2 buffers: each buffer is used twice per chunk,
            // so buffer and phase are compile-time functions of pp (fully unrolled)
            static_assert(kNB == 2 && kPiecesPerChunk == 4, "static buffer / phase schedule");
            const int np = c == cpr - 1 ? np_last : kPiecesPerChunk;
#pragma unroll
            for (int pp = 0; pp < kPiecesPerChunk; ++pp) {
              if (kSkip && pp >= np) break;  // all-padding pieces (m not a multiple of 64 x 4) are not computed
              const uint32_t buf = g * kNB + (pp & 1);
              PROF_B(); mbar_wait(tfull(buf), ((pp >> 1) ^ (ph_t >> (pp & 1))) & 1); PROF_E(0);
              PROF_B();
              tc_fence_after();
#ifndef TID_NOLOAD  // timing experiment only: scan stale registers (wrong results)
              tmem_ld64(taddr_q + buf * kPiece, v);
#endif
              tmem_wait_ld();
              reg_fence64(v);
              tc_fence_before();  // the piece is in registers: buffer free
              __syncwarp();
              if (lane == 0) mbar_arrive(tempty(buf));
              PROF_E(3);
              PROF_B();
              if (kpc >= (pp + 1) * kPiece) {  // every column of the piece is real (the common case)
#ifndef TID_NOSCAN
                scan32_fold<false>(v, 32, R, T1, T2);
                scan32_fold<false>(v + 32, 32, R, T1, T2);
#endif
              } else {
                scan32_fold<true>(v, kpc - pp * kPiece, R, T1, T2);
                scan32_fold<true>(v + 32, kpc - pp * kPiece - 32, R, T1, T2);
              }
              PROF_E(1);
            }
            if (kSkip) ph_t ^= use_parity(np);
            PROF_B();
            int x1, x2;
            finish_fold(R, T1, T2, x1, x2);
            G2 = max3i(min(G1, x1), G2, x2);
            G1 = max(G1, x1);
            PROF_E(2);
          }
          PROF_B();
          // d = N_Q - 2X - p, p in {0, 1}: decide the ratio test from the bounds
          const bool real2 = G2 > INT_MIN;
          bool undecided = false;
          if (valid && real2) {
            const int hi1 = nqv - 2 * G1, hi2 = nqv - 2 * G2;
            const int lo1 = max(hi1 - 1, 0), lo2 = max(hi2 - 1, 0);
            bool pass_sure, fail_sure;
            if (ratio32) {
              pass_sure = p.den2 * static_cast<uint32_t>(hi1) < p.num2 * static_cast<uint32_t>(lo2);
              fail_sure = p.den2 * static_cast<uint32_t>(lo1) >= p.num2 * static_cast<uint32_t>(hi2);
            } else {
              pass_sure = uint64_t(p.den2) * uint64_t(hi1) < uint64_t(p.num2) * uint64_t(lo2);
              fail_sure = uint64_t(p.den2) * uint64_t(lo1) >= uint64_t(p.num2) * uint64_t(hi2);
            }
            pass = pass_sure;
            undecided = !pass_sure && !fail_sure;
          }
          uint32_t und = __ballot_sync(0xffffffffu, undecided);
#ifdef TID_PROF
          if (lane == 0) {  // g_prof[148 * 32 * 8 - 2 / -1]: undecided rows / warp-units with any
            atomicAdd(&g_prof[148 * 32 * 8 - 2], static_cast<unsigned long long>(__popc(und)));
            if (und) atomicAdd(&g_prof[148 * 32 * 8 - 1], 1ull);
          }
#endif
          while (und) {  // rare: recompute the row exactly
            const int l = __ffs(und) - 1;
            und &= und - 1;
            const int rl = __shfl_sync(0xffffffffu, row, l);
            const int nl = __shfl_sync(0xffffffffu, nqv, l);
            int d1, d2;
            exact_row_global(p, qi, rl, J.ref_first + s, nl, lane, cpr,
                             sbase + SmemPlan::kCol + (b0 + s * cpr) * kColBytes, d1, d2);
            if (lane == l)
              pass = d2 != INT_MAX && uint64_t(p.den2) * uint64_t(d1) < uint64_t(p.num2) * uint64_t(d2);
          }
        } else {
        int g1d = INT_MAX, g1i = -1, g2d = INT_MAX, g2i = -1;  // running exact 2-NN over chunks
        for (int c = 0; c < cpr; ++c) {
          const uint32_t ck = sbase + SmemPlan::kCol + (b0 + s * cpr + c) * kColBytes;
          int R[16];
#pragma unroll
          for (int b = 0; b < 16; ++b) R[b] = INT_MAX;
          int T1 = INT_MAX, T2 = INT_MAX;
          const int np = c == cpr - 1 ? np_last : kPiecesPerChunk;
#pragma unroll
          for (int pp = 0; pp < kPiecesPerChunk; ++pp) {
            if (kSkip && pp >= np) break;
            const uint32_t buf = g * kNB + (pp & 1);
            PROF_B(); mbar_wait(tfull(buf), ((pp >> 1) ^ (ph_t >> (pp & 1))) & 1); PROF_E(0);
            tc_fence_after();
            // x32 loads (32 registers live instead of 64: the verify epilogue also carries the running
            // 2-NN with indices); the buffer is released as soon as its last load has landed
            uint32_t (&h32)[32] = *reinterpret_cast<uint32_t(*)[32]>(v);
#pragma unroll
            for (int h = 0; h < kPiece / 32; ++h) {
              tmem_ld32(taddr_q + buf * kPiece + h * 32, h32);
              tmem_wait_ld();
              reg_fence(h32);
              if (h == kPiece / 32 - 1) {
                tc_fence_before();
                __syncwarp();
                if (lane == 0) mbar_arrive(tempty(buf));
              }
              PROF_B();
              scan32_regs(h32, ck + (pp * kPiece + h * 32) * 4, R, T1, T2);
              PROF_E(1);
            }
          }
          if (kSkip) ph_t ^= use_parity(np);
          PROF_B();
          int k1, k2;
          finish_partition(R, T1, T2, k1, k2);
          const int c1d = k1 >> 8, c1i = (k1 & 255) + c * kBN;
          const int c2d = k2 >> 8, c2i = (k2 & 255) + c * kBN;
          if (c == 0) {
            g1d = c1d; g1i = c1i; g2d = c2d; g2i = c2i;
          } else if (c1d < g1d) {  // merge into the running 2-NN; earlier chunks win ties (lower index)
            if (c2d < g1d) { g2d = c2d; g2i = c2i; } else { g2d = g1d; g2i = g1i; }
            g1d = c1d; g1i = c1i;
          } else if (c1d < g2d) {
            g2d = c1d; g2i = c1i;
          }
          PROF_E(2);
        }
        // ratio test in exact integers: den^2 * d1 < num^2 * d2
        const bool real1 = g1d < kSentinelNorm, real2 = g2d < kSentinelNorm;
        if (ratio32) {
          const uint32_t d1 = static_cast<uint32_t>(nqv + g1d), d2 = static_cast<uint32_t>(nqv + g2d);
          pass = p.den2 * d1 < p.num2 * d2;
        } else {
          const uint64_t d1 = static_cast<uint64_t>(static_cast<int64_t>(nqv) + g1d);
          const uint64_t d2 = static_cast<uint64_t>(static_cast<int64_t>(nqv) + g2d);
          pass = static_cast<uint64_t>(p.den2) * d1 < static_cast<uint64_t>(p.num2) * d2;
        }
        pass = pass && valid && real2;
        if (p.nn_out != nullptr && row < p.n_rows) {
          int4 o;
          o.x = (valid && real1) ? nqv + g1d : -1; o.y = (valid && real1) ? g1i : -1;
          o.z = (valid && real2) ? nqv + g2d : -1; o.w = (valid && real2) ? g2i : -1;
          reinterpret_cast<int4*>(p.nn_out)[static_cast<int64_t>(qi) * p.n_rows + row] = o;
        }
        }
        cnt += __popc(__ballot_sync(0xffffffffu, pass));
        // the unit after this one (same group): (ns, ntq, nqi)
        int ns = s + kNG, ntq = tq, nqi = qi;
        while (ns >= J.nr) {
          ns -= J.nr;
          if (++ntq == T) { ntq = 0; ++nqi; }
        }
        // flush the count when the group's next unit is another (query, reference) pair
        if (!has_next || ns != s || nqi != qi) {
          if (lane == 0 && cnt) {
            const int64_t ci = (p.mode == kModeVerify) ? qi : static_cast<int64_t>(qi) * p.ldc + p.col0 + J.ref_first + s;
            atomicAdd(p.counts + ci, cnt);
          }
          cnt = 0;
        }
        if constexpr (kFold) { PROF_E(5); }
        u += kNG; s = ns; tq = ntq;
        if (nqi != qi && has_next) {
          qi = nqi;
          nvalid = min(p.n_valid ? p.n_valid[qi] : p.n_rows, p.n_rows);
          nq_row = p.nq + static_cast<int64_t>(qi) * nq_ld + row_in_tile;
        }
      }
      __syncwarp();
      if (lane == 0)
        for (int sl = 0; sl < nslots; ++sl) mbar_arrive(rempty(b0 + sl));
      slot_par ^= ((1u << nslots) - 1u) << b0;
    }
  }

  PROF_FLUSH();
  tc_fence_before();
  __syncthreads();
  if (warp == kFirstMmaWarp) {
    tc_fence_after();
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 512;" ::"r"(tmem_base) : "memory");
  }
}

#ifdef TID_PROF
extern "C" int tid_debug_read_prof(void* host, size_t bytes) {
  return static_cast<int>(cudaMemcpyFromSymbol(host, g_prof, bytes));
}
#endif


cudaError_t launch_match(const MatchParams& p, const CUtensorMap& qmap, const CUtensorMap& rmap, bool fold, int grid,
                         cudaStream_t s) {
  // the shared-memory opt-in is per device: set once per device (host overhead matters for C1)
  static thread_local uint64_t attr_set = 0;  // bit d = device d configured
  int dev = 0;
  cudaGetDevice(&dev);
  if (dev >= 64 || !(attr_set >> dev & 1)) {
    for (auto k : {match_kernel<true, false>, match_kernel<true, true>, match_kernel<false, false>,
                   match_kernel<false, true>}) {
      cudaError_t e = cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                           static_cast<int>(SmemPlan::kAlloc));
      if (e != cudaSuccess) return e;
    }
    if (dev < 64) attr_set |= uint64_t(1) << dev;
  }
  const bool skip = piece_count_last(p.m, p.cpr) < kPiecesPerChunk;
  auto kern = fold ? (skip ? match_kernel<true, true> : match_kernel<true, false>)
                   : (skip ? match_kernel<false, true> : match_kernel<false, false>);
  kern<<<grid, kNumThreads, SmemPlan::kAlloc, s>>>(qmap, rmap, p);
  return cudaGetLastError();
}

// ------------------------------------------------------------------ one-to-one verification, streamed
// Pair-streaming verification (one query image against one reference image; counts, and for
// the packed-key variant (d1, i1, d2, i2), exactly as the job kernel above).  The job kernel loads a
// pair's whole reference (up to 4 chunks = all 4 slots), runs its T query tiles on the 3 groups
// (T = 8: 3 / 3 / 2) and only then releases the slots, so every pair boundary drains the pipeline on
// every group.  Here a CTA's pairs form one sequence of query tiles gt = lp * T + t (lp = the CTA's
// pair count), tile gt runs on group gt % 3 (SMEM stage gt % 3, TMEM query slot gt % 4: see kVTQ),
// and reference slot c is released as soon as all T tiles of pair lp have finished chunk c (one MMA
// commit per tile): the next pair's chunk c loads while the last tiles of this pair still run on
// chunks > c, and no group idles at a pair boundary unless the next pair's chunk is still in flight.
// The column terms (folded: W and the norm digits; packed-key: N_R * 256 + i and the zeroing of rows
// >= m_r) are computed on chip by the 4 warps of the group that runs the pair's first tile, chunk by
// chunk ahead of its MMAs, into a per-pair column buffer double-buffered by pair parity (released by
// the 4 * T epilogue warp-tiles that read it).
// Every wait below is a parity wait on a barrier whose phase advances once per pair (slots) or once per
// two pairs (column buffers); it is unambiguous because each group runs at least one tile of every pair,
// so no waiter can be two phases behind: the kernel requires T >= 3 (tid_verify routes n <= 256 to the
// job kernel).
// TMEM: the 6 x 64 accumulator columns and FOUR 32-column query-tile slots (tile gt in slot gt % 4): the
// producer fills a group's next tile into the spare slot while the group still runs its current one (the
// norm-term K-step's constant operand is read from shared memory instead of TMEM to make room).  A slot's
// parity wait cannot alias: group g reaches tile gt only after tile gt - 3, whose copy followed those of
// tiles gt - 4 and earlier (one thread, in order).
constexpr int kVTQ = 4;
static_assert(kTQBase + kVTQ * kQCols <= 512, "TMEM budget of the streamed verification");
constexpr int kVQStages = kNG;  // query stage g holds group g's next tile (TMA), prepared by the group, copied to TMEM
struct VSmem {
  static constexpr uint32_t kR = 0;                                        // 4 x 32 KiB reference chunks
  static constexpr uint32_t kQ = kR + kMaxSlots * kRTileBytes;             // 3 x 16 KiB query stages
  static constexpr uint32_t kX = kQ + kVQStages * kQTileBytes;             // 4 x 8 KiB norm digits (folded)
  static constexpr uint32_t kAx = kX + kMaxSlots * kXTileBytes;            // constant norm-term operand
  static constexpr uint32_t kCol = kAx + kBM * kXDim;                      // 2 pair buffers x 4 x 1 KiB
  static constexpr uint32_t kColPair = kMaxSlots * kColBytes;
  static constexpr uint32_t kBar = kCol + 2 * kColPair;
  static constexpr uint32_t kQFull = kBar;
  static constexpr uint32_t kQEmpty = kQFull + 8 * kVQStages;
  static constexpr uint32_t kRFull = kQEmpty + 8 * kVQStages;
  static constexpr uint32_t kREmpty = kRFull + 8 * kMaxSlots;
  static constexpr uint32_t kXReady = kREmpty + 8 * kMaxSlots;
  static constexpr uint32_t kTFull = kXReady + 8 * kMaxSlots;
  static constexpr uint32_t kTEmpty = kTFull + 8 * kTmemBufs;
  static constexpr uint32_t kTQFull = kTEmpty + 8 * kTmemBufs;
  static constexpr uint32_t kTQEmpty = kTQFull + 8 * kVTQ;
  static constexpr uint32_t kColEmpty = kTQEmpty + 8 * kVTQ;                // per pair buffer: all readers done
  static constexpr uint32_t kColReady = kColEmpty + 8 * 2;               // per (pair buffer, chunk): terms written
  static constexpr uint32_t kPrepped = kColReady + 8 * 2 * kMaxSlots;      // per stage: tile shifted + normed
  static constexpr uint32_t kTmemPtr = kPrepped + 8 * kVQStages;
  static constexpr uint32_t kEnd = kTmemPtr + 16;
  static constexpr uint32_t kAlloc = kEnd + 1024;
};
static_assert(VSmem::kAlloc <= 232448, "227 KiB of shared memory per CTA");
static_assert(kNG == 3, "tile gt -> group gt % 3");

// Column terms of chunk c of the current pair, columns col = tig, tig + 128 (the group's 128 threads):
// folded: W = 256 sum r - N_R (-1 - kpc for padding) into the pair's column buffer and the norm digits
// into X slot c; packed-key: N_R * 256 + i (sentinel for padding) and rows in [mcap, m) zeroed.
template <bool kFold>
__device__ __forceinline__ void vstream_terms(uint32_t sbase, uint32_t colbuf, int c, int mcap, int m, int tig) {
#pragma unroll 1
  for (int col = tig; col < kBN; col += 128) {
    const int gcol = c * kBN + col;
    const uint32_t row = sbase + VSmem::kR + c * kRTileBytes + col * kDim;
    uint32_t nr = 0, sr = 0;
    if (gcol < mcap) {
#pragma unroll
      for (int w = 0; w < kDim / 16; ++w) {
        const int4 x4 = lds128(row + 16 * w);
        nr = __dp4a(static_cast<uint32_t>(x4.x), static_cast<uint32_t>(x4.x), nr);
        nr = __dp4a(static_cast<uint32_t>(x4.y), static_cast<uint32_t>(x4.y), nr);
        nr = __dp4a(static_cast<uint32_t>(x4.z), static_cast<uint32_t>(x4.z), nr);
        nr = __dp4a(static_cast<uint32_t>(x4.w), static_cast<uint32_t>(x4.w), nr);
        if (kFold) {
          sr = __dp4a(static_cast<uint32_t>(x4.x), 0x01010101u, sr);
          sr = __dp4a(static_cast<uint32_t>(x4.y), 0x01010101u, sr);
          sr = __dp4a(static_cast<uint32_t>(x4.z), 0x01010101u, sr);
          sr = __dp4a(static_cast<uint32_t>(x4.w), 0x01010101u, sr);
        }
      }
    } else if (!kFold && gcol < m) {
      // a row beyond this pair's m_r holds the caller's bytes: zeroed, so its product is 0 and the
      // sentinel key never wins (rows >= m are zero-filled by TMA).  The folded path masks by W < 0.
#pragma unroll
      for (int w = 0; w < kDim / 16; ++w)
        asm volatile("st.shared.v4.b32 [%0], {%1, %1, %1, %1};" ::"r"(row + 16 * w), "r"(0) : "memory");
    }
    int32_t term;
    if (kFold) {
      term = gcol < mcap ? 256 * static_cast<int>(sr) - static_cast<int>(nr) : -1 - max(0, min(mcap - c * kBN, kBN));
      uint32_t w8[8];
      norm_digits(term, w8);
      const uint32_t dst = sbase + VSmem::kX + c * kXTileBytes + col * kXDim;
      asm volatile("st.shared.v4.b32 [%0], {%1, %2, %3, %4};" ::"r"(dst), "r"(w8[0]), "r"(w8[1]), "r"(w8[2]),
                   "r"(w8[3]) : "memory");
      asm volatile("st.shared.v4.b32 [%0], {%1, %2, %3, %4};" ::"r"(dst + 16), "r"(w8[4]), "r"(w8[5]), "r"(w8[6]),
                   "r"(w8[7]) : "memory");
    } else {
      term = (gcol < mcap ? static_cast<int32_t>(nr) : kSentinelNorm) * 256 + col;
    }
    asm volatile("st.shared.s32 [%0], %1;" ::"r"(colbuf + c * kColBytes + col * 4), "r"(term) : "memory");
  }
}

template <bool kFold, bool kSkip>
__global__ void __launch_bounds__(kNumThreads, 1)
    verify_stream_kernel(const __grid_constant__ CUtensorMap qmap, const __grid_constant__ CUtensorMap rmap,
                         const MatchParams p) {
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  const uint32_t sbase = smem_u32(smem);
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int T = p.tiles_per_q, cpr = p.cpr;
  const int npairs = static_cast<int>(blockIdx.x) < p.num_q
                         ? (p.num_q - static_cast<int>(blockIdx.x) + static_cast<int>(gridDim.x) - 1) /
                               static_cast<int>(gridDim.x)
                         : 0;
  const int ntiles = npairs * T;  // this CTA's tile sequence gt = lp * T + t, pair = blockIdx.x + lp * gridDim.x

  auto bar = [&](uint32_t base, int i) { return sbase + base + 8 * i; };
  uint32_t* tmem_ptr_smem = reinterpret_cast<uint32_t*>(smem + VSmem::kTmemPtr);

  if (kFold) {  // constant norm-term operand (see the job kernel)
    uint32_t* ax = reinterpret_cast<uint32_t*>(smem + VSmem::kAx);
    for (int i = threadIdx.x; i < kBM * kXDim / 4; i += blockDim.x) ax[i] = (i & 3) == 3 ? 0x01FFFFFFu : 0xFFFFFFFFu;
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  }
  if (threadIdx.x == 0) {
    prefetch_tmap(&qmap);
    prefetch_tmap(&rmap);
    for (int i = 0; i < kVQStages; ++i) {
      mbar_init(bar(VSmem::kQFull, i), 1);
      mbar_init(bar(VSmem::kQEmpty, i), 1);
      mbar_init(bar(VSmem::kPrepped, i), 4);  // the group's 4 epilogue warps
    }
    for (int i = 0; i < kVTQ; ++i) { mbar_init(bar(VSmem::kTQFull, i), 1); mbar_init(bar(VSmem::kTQEmpty, i), 1); }
    for (int c = 0; c < kMaxSlots; ++c) {
      mbar_init(bar(VSmem::kRFull, c), 1);
      mbar_init(bar(VSmem::kREmpty, c), T);   // one MMA commit per tile of the pair
      mbar_init(bar(VSmem::kXReady, c), 4);   // the 4 warps of the first tile's group
    }
    for (int i = 0; i < kTmemBufs; ++i) { mbar_init(bar(VSmem::kTFull, i), 1); mbar_init(bar(VSmem::kTEmpty, i), 4); }
    for (int b = 0; b < 2; ++b) mbar_init(bar(VSmem::kColEmpty, b), 4 * T);  // every warp-tile of the pair
    for (int i = 0; i < 2 * kMaxSlots; ++i) mbar_init(bar(VSmem::kColReady, i), 4);
    fence_barrier_init();
  }
  if (warp == kFirstMmaWarp) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 512;" ::"r"(smem_u32(tmem_ptr_smem))
                 : "memory");
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
  }
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem_base = *tmem_ptr_smem;

  // -DTID_PROF buckets: epilogue 0 wait-accumulator 1 scan + chunk finish 2 wait for a chunk (terms)
  // 3 TMEM load + release 4 column terms 5 wait column buffer 6 next tile's query prep + tile tail;
  // MMA 0 wait-free-accumulator 1 wait-query 2 wait-ref; producer 0 wait-stage 1 wait-prep 2 wait-TMEM-slot
  PROF_DECL
  if (warp == kProducerWarp) {
    // ---- lane 0: query tiles + reference chunks.  Tile gt (group g = gt % 3) lands raw in stage g by TMA;
    // the group's epilogue warps compute N_Q of its rows and, for the folded path, shift them in place
    // (during the group's previous tile, off its critical path); then SMEM -> TMEM slot gt % 4 here.
    // Reference chunk c of pair lp is loaded as soon as pair lp - 1 has finished with slot c (serviced
    // whenever lane 0 waits).
    if (lane == 0) {
      int r_lp = 0, r_c = 0;  // next reference chunk
      auto service_refs = [&]() {
        while (r_lp < npairs) {
          uint32_t free_;
          asm volatile(
              "{\n\t.reg .pred P1;\n\tmbarrier.test_wait.parity.shared::cta.b64 P1, [%1], %2;\n\t"
              "selp.u32 %0, 1, 0, P1;\n\t}"
              : "=r"(free_)
              : "r"(bar(VSmem::kREmpty, r_c)), "r"(static_cast<uint32_t>((r_lp & 1) ^ 1))
              : "memory");
          if (!free_) return;
          mbar_expect_tx(bar(VSmem::kRFull, r_c), kRTileBytes);
          tma_load_3d(sbase + VSmem::kR + r_c * kRTileBytes, &rmap, bar(VSmem::kRFull, r_c), 0, r_c * kBN,
                      static_cast<int>(blockIdx.x) + r_lp * static_cast<int>(gridDim.x));
          if (++r_c == cpr) { r_c = 0; ++r_lp; }
        }
      };
      auto wait_serving = [&](uint32_t b, uint32_t par) {  // poll, issuing reference loads meanwhile
        uint32_t ns = 32;
        while (true) {
          uint32_t done;
          asm volatile(
              "{\n\t.reg .pred P1;\n\tmbarrier.test_wait.parity.shared::cta.b64 P1, [%1], %2;\n\t"
              "selp.u32 %0, 1, 0, P1;\n\t}"
              : "=r"(done)
              : "r"(b), "r"(par)
              : "memory");
          if (done) return;
          service_refs();
          __nanosleep(ns);
          ns = ns < 256 ? ns * 2 : 256;
        }
      };
      auto issue = [&](int gt) {  // tile gt -> stage gt % 3 (its previous occupant, tile gt - 3, is in TMEM)
        const int st = gt % kVQStages, k = gt / kVQStages;
        PROF_B(); wait_serving(bar(VSmem::kQEmpty, st), (k & 1) ^ 1); PROF_E(0);
        mbar_expect_tx(bar(VSmem::kQFull, st), kQTileBytes);
        const int lp = gt / T, t = gt - lp * T;
        tma_load_3d(sbase + VSmem::kQ + st * kQTileBytes, &qmap, bar(VSmem::kQFull, st), 0, t * kBM,
                    static_cast<int>(blockIdx.x) + lp * static_cast<int>(gridDim.x));
      };
      service_refs();
      for (int gt = 0; gt < min(ntiles, kVQStages); ++gt) issue(gt);
      for (int gt = 0; gt < ntiles; ++gt) {
        const int st = gt % kVQStages, sl = gt % kVTQ;
        PROF_B(); wait_serving(bar(VSmem::kPrepped, st), (gt / kVQStages) & 1); PROF_E(1);
        // the slot's previous tile (gt - 4) has left TMEM
        PROF_B(); wait_serving(bar(VSmem::kTQEmpty, sl), ((gt / kVTQ) & 1) ^ 1); PROF_E(2);
        tc_fence_after();
        const uint64_t sd = smem_desc_sw128(sbase + VSmem::kQ + st * kQTileBytes);
#pragma unroll
        for (int kk = 0; kk < kDim / kXDim; ++kk)
          tmem_cp_128x256b(tmem_base + kTQBase + sl * kQCols + 8 * kk, sd + 2 * kk);
        commit_one(bar(VSmem::kTQFull, sl));
        commit_one(bar(VSmem::kQEmpty, st));
        if (gt + kVQStages < ntiles) issue(gt + kVQStages);
        service_refs();
      }
      while (r_lp < npairs) {  // the remaining reference chunks
        mbar_wait_sleep(bar(VSmem::kREmpty, r_c), (r_lp & 1) ^ 1);
        service_refs();
      }
    }
  } else if (warp < kFirstEpiWarp) {
    // ---- MMA issuer of group g: tiles gt = g, g + 3, ...
    const int g = warp - kFirstMmaWarp;
    const int np_last = kSkip ? piece_count_last(p.m, cpr) : kPiecesPerChunk;
    uint32_t ph_t = 0;
    for (int gt = g; gt < ntiles; gt += kNG) {
      const int lp = gt / T, sl = gt % kVTQ;
      const uint32_t at = tmem_base + kTQBase + sl * kQCols;
      PROF_B(); mbar_wait(bar(VSmem::kTQFull, sl), (gt / kVTQ) & 1); PROF_E(1);
      for (int c = 0; c < cpr; ++c) {
        PROF_B();
        mbar_wait(bar(VSmem::kRFull, c), lp & 1);
        mbar_wait(bar(VSmem::kXReady, c), lp & 1);
        PROF_E(2);
        const uint64_t bd0 = smem_desc_sw128(sbase + VSmem::kR + c * kRTileBytes);
        const int np = c == cpr - 1 ? np_last : kPiecesPerChunk;
#pragma unroll
        for (int pp = 0; pp < kPiecesPerChunk; ++pp) {
          if (kSkip && pp >= np) break;
          const uint32_t buf = g * kNB + (pp & 1);
          PROF_B(); mbar_wait(bar(VSmem::kTEmpty, buf), (((pp >> 1) ^ (ph_t >> (pp & 1))) & 1) ^ 1); PROF_E(0);
          tc_fence_after();
          const uint64_t bd = bd0 + pp * (kPiece * kDim >> 4);
          if (kFold)
            mma_piece_fold_ts_sx(tmem_base + buf * kPiece, at, bd, smem_desc_sw32(sbase + VSmem::kAx),
                                 smem_desc_sw32(sbase + VSmem::kX + c * kXTileBytes) + pp * (kPiece * kXDim >> 4),
                                 bar(VSmem::kTFull, buf));
          else
            mma_piece_ts(tmem_base + buf * kPiece, at, bd, bar(VSmem::kTFull, buf));
        }
        if (kSkip) ph_t ^= use_parity(np);
        mma_commit(bar(VSmem::kREmpty, c));  // this tile's MMAs on chunk c done: slot c may be refilled
      }
      mma_commit(bar(VSmem::kTQEmpty, sl));
    }
  } else {
    // ---- epilogue group g: TMEM -> registers -> top-2 -> ratio -> count (and (d1, i1, d2, i2))
    const int ew = warp - kFirstEpiWarp;
    const int g = ew >> 2;
    const int quarter = warp & 3;
    const int tig = (ew & 3) * 32 + lane;  // thread in group (column-term work)
    const uint32_t taddr_q = tmem_base + (static_cast<uint32_t>(quarter * 32) << 16);
    const int row_in_tile = quarter * 32 + lane;
    const bool ratio32 = p.num2 <= 511u && p.den2 <= 511u;
    const int np_last = kSkip ? piece_count_last(p.m, cpr) : kPiecesPerChunk;
    uint32_t ph_t = 0;
    uint32_t v[64];
    // Query prep of tile gt (in stage g): this thread's row N_Q (Alg. 1 step 2) and, folded, the
    // shifted row q' = q ^ 0x80 (= q - 128 as s8; rows beyond n stay zero).  A row's 16-byte chunks sit
    // permuted within its 128-byte line (SWIZZLE_128B): neither the sum nor the XOR depends on the order.
    auto prep_tile = [&](int gt) -> int32_t {
      const int lp = gt / T, t = gt - lp * T;
      mbar_wait(bar(VSmem::kQFull, g), (gt / kNG) & 1);
      const uint32_t ra = sbase + VSmem::kQ + g * kQTileBytes + row_in_tile * kDim;
      const bool shift = kFold && t * kBM + row_in_tile < p.n_rows;
      uint32_t acc = 0;
#pragma unroll
      for (int w = 0; w < kDim / 16; ++w) {
        const uint32_t ca = ra + 16 * (w ^ (row_in_tile & 7));  // 8 lanes of a phase on distinct banks
        const int4 x4 = lds128(ca);
        acc = __dp4a(static_cast<uint32_t>(x4.x), static_cast<uint32_t>(x4.x), acc);
        acc = __dp4a(static_cast<uint32_t>(x4.y), static_cast<uint32_t>(x4.y), acc);
        acc = __dp4a(static_cast<uint32_t>(x4.z), static_cast<uint32_t>(x4.z), acc);
        acc = __dp4a(static_cast<uint32_t>(x4.w), static_cast<uint32_t>(x4.w), acc);
        if (shift)
          asm volatile("st.shared.v4.b32 [%0], {%1, %2, %3, %4};" ::"r"(ca), "r"(x4.x ^ 0x80808080),
                       "r"(x4.y ^ 0x80808080), "r"(x4.z ^ 0x80808080), "r"(x4.w ^ 0x80808080)
                       : "memory");
      }
      if (kFold) asm volatile("fence.proxy.async.shared::cta;" ::: "memory");  // shifted rows -> TMEM copy
      __syncwarp();
      if (lane == 0) mbar_arrive(bar(VSmem::kPrepped, g));
      return static_cast<int32_t>(acc);
    };
    int32_t nq_next = 0;
    for (int gt = g; gt < ntiles; gt += kNG) {
      const int lp = gt / T, t = gt - lp * T;
      const int pair = static_cast<int>(blockIdx.x) + lp * static_cast<int>(gridDim.x);
      const uint32_t colbuf = sbase + VSmem::kCol + (lp & 1) * VSmem::kColPair;
      const int mcap = p.m_valid ? min(p.m_valid[pair], p.m) : p.m;
      const int nvalid = min(p.n_valid ? p.n_valid[pair] : p.n_rows, p.n_rows);
      const int row = t * kBM + row_in_tile;
      const bool valid = row < nvalid;
      if (gt == g) nq_next = prep_tile(gt);  // the group's first tile: nothing to overlap it with
      const int32_t nqv = valid ? nq_next : 0;
      int done_terms = cpr;  // chunks whose column terms this warp has written (first tile of a pair only)
      auto terms = [&](int c) {
        PROF_B(); mbar_wait(bar(VSmem::kRFull, c), lp & 1); PROF_E(2);
        PROF_B();
        vstream_terms<kFold>(sbase, colbuf, c, mcap, p.m, tig);
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");  // digits / zeroed rows -> tensor core
        __syncwarp();
        if (lane == 0) {
          mbar_arrive(bar(VSmem::kXReady, c));                    // for the MMA warps (slot phase = pair)
          mbar_arrive(bar(VSmem::kColReady, (lp & 1) * kMaxSlots + c));  // for the epilogue (buffer phase)
        }
        PROF_E(4);
      };
      if (t == 0) {  // this group computes the pair's column terms, one chunk ahead of its MMAs
        PROF_B(); mbar_wait(bar(VSmem::kColEmpty, lp & 1), ((lp >> 1) & 1) ^ 1); PROF_E(5);
        terms(0);
        done_terms = 1;
      }
      bool pass = false;
      int G1 = INT_MIN, G2 = INT_MIN;                                      // folded: two largest X
      int g1d = INT_MAX, g1i = -1, g2d = INT_MAX, g2i = -1;                // packed keys: running 2-NN
      for (int c = 0; c < cpr; ++c) {
        if (done_terms < cpr) {
          while (done_terms <= c) { terms(done_terms); ++done_terms; }
          // the next chunk's terms now if its tile has landed (the MMAs of chunk c run meanwhile)
          if (done_terms == c + 1 && done_terms < cpr) {
            uint32_t ready;
            asm volatile(
                "{\n\t.reg .pred P1;\n\tmbarrier.test_wait.parity.shared::cta.b64 P1, [%1], %2;\n\t"
                "selp.u32 %0, 1, 0, P1;\n\t}"
                : "=r"(ready)
                : "r"(bar(VSmem::kRFull, c + 1)), "r"(static_cast<uint32_t>(lp & 1))
                : "memory");
            if (__shfl_sync(0xffffffffu, ready, 0)) { terms(done_terms); ++done_terms; }
          }
        }
        // this chunk's column buffer is written (a per-pair-buffer barrier: the slot's xready may already
        // be in the next pair's phase once every tile's MMAs have left chunk c)
        PROF_B(); mbar_wait(bar(VSmem::kColReady, (lp & 1) * kMaxSlots + c), (lp >> 1) & 1); PROF_E(5);
        const uint32_t ck = colbuf + c * kColBytes;
        const int np = c == cpr - 1 ? np_last : kPiecesPerChunk;
        if constexpr (kFold) {
          int kpc;
          asm volatile("ld.shared.s32 %0, [%1];" : "=r"(kpc) : "r"(ck + (kBN - 1) * 4));
          kpc = kpc < 0 ? -1 - kpc : kBN;
          int R[16];
#pragma unroll
          for (int b = 0; b < 16; ++b) R[b] = INT_MIN;
          int T1 = INT_MIN, T2 = INT_MIN;
#pragma unroll
          for (int pp = 0; pp < kPiecesPerChunk; ++pp) {
            if (kSkip && pp >= np) break;
            const uint32_t buf = g * kNB + (pp & 1);
            PROF_B(); mbar_wait(bar(VSmem::kTFull, buf), ((pp >> 1) ^ (ph_t >> (pp & 1))) & 1); PROF_E(0);
            PROF_B();
            tc_fence_after();
            tmem_ld64(taddr_q + buf * kPiece, v);
            tmem_wait_ld();
            reg_fence64(v);
            tc_fence_before();
            __syncwarp();
            if (lane == 0) mbar_arrive(bar(VSmem::kTEmpty, buf));
            PROF_E(3);
            PROF_B();
            if (kpc >= (pp + 1) * kPiece) {
              scan32_fold<false>(v, 32, R, T1, T2);
              scan32_fold<false>(v + 32, 32, R, T1, T2);
            } else {
              scan32_fold<true>(v, kpc - pp * kPiece, R, T1, T2);
              scan32_fold<true>(v + 32, kpc - pp * kPiece - 32, R, T1, T2);
            }
            PROF_E(1);
          }
          PROF_B();
          int x1, x2;
          finish_fold(R, T1, T2, x1, x2);
          G2 = max3i(min(G1, x1), G2, x2);
          G1 = max(G1, x1);
          PROF_E(1);
        } else {
          int R[16];
#pragma unroll
          for (int b = 0; b < 16; ++b) R[b] = INT_MAX;
          int T1 = INT_MAX, T2 = INT_MAX;
#pragma unroll
          for (int pp = 0; pp < kPiecesPerChunk; ++pp) {
            if (kSkip && pp >= np) break;
            const uint32_t buf = g * kNB + (pp & 1);
            mbar_wait(bar(VSmem::kTFull, buf), ((pp >> 1) ^ (ph_t >> (pp & 1))) & 1);
            tc_fence_after();
            uint32_t (&h32)[32] = *reinterpret_cast<uint32_t(*)[32]>(v);
#pragma unroll
            for (int h = 0; h < kPiece / 32; ++h) {
              tmem_ld32(taddr_q + buf * kPiece + h * 32, h32);
              tmem_wait_ld();
              reg_fence(h32);
              if (h == kPiece / 32 - 1) {
                tc_fence_before();
                __syncwarp();
                if (lane == 0) mbar_arrive(bar(VSmem::kTEmpty, buf));
              }
              scan32_regs(h32, ck + (pp * kPiece + h * 32) * 4, R, T1, T2);
            }
          }
          int k1, k2;
          finish_partition(R, T1, T2, k1, k2);
          const int c1d = k1 >> 8, c1i = (k1 & 255) + c * kBN;
          const int c2d = k2 >> 8, c2i = (k2 & 255) + c * kBN;
          if (c == 0) {
            g1d = c1d; g1i = c1i; g2d = c2d; g2i = c2i;
          } else if (c1d < g1d) {  // earlier chunks win ties (lower index)
            if (c2d < g1d) { g2d = c2d; g2i = c2i; } else { g2d = g1d; g2i = g1i; }
            g1d = c1d; g1i = c1i;
          } else if (c1d < g2d) {
            g2d = c1d; g2i = c1i;
          }
        }
        if (kSkip) ph_t ^= use_parity(np);
        // the group's next tile (already in stage g): prepared here, off the MMA's critical path
        if (c == 0 && gt + kNG < ntiles) { PROF_B(); nq_next = prep_tile(gt + kNG); PROF_E(6); }
      }
      PROF_B();
      if constexpr (kFold) {
        // d = N_Q - 2X - p, p in {0, 1}: the ratio test from the bounds, exact recompute if open
        const bool real2 = G2 > INT_MIN;
        bool undecided = false;
        if (valid && real2) {
          const int hi1 = nqv - 2 * G1, hi2 = nqv - 2 * G2;
          const int lo1 = max(hi1 - 1, 0), lo2 = max(hi2 - 1, 0);
          bool pass_sure, fail_sure;
          if (ratio32) {
            pass_sure = p.den2 * static_cast<uint32_t>(hi1) < p.num2 * static_cast<uint32_t>(lo2);
            fail_sure = p.den2 * static_cast<uint32_t>(lo1) >= p.num2 * static_cast<uint32_t>(hi2);
          } else {
            pass_sure = uint64_t(p.den2) * uint64_t(hi1) < uint64_t(p.num2) * uint64_t(lo2);
            fail_sure = uint64_t(p.den2) * uint64_t(lo1) >= uint64_t(p.num2) * uint64_t(hi2);
          }
          pass = pass_sure;
          undecided = !pass_sure && !fail_sure;
        }
        uint32_t und = __ballot_sync(0xffffffffu, undecided);
        while (und) {
          const int l = __ffs(und) - 1;
          und &= und - 1;
          const int rl = __shfl_sync(0xffffffffu, row, l);
          const int nl = __shfl_sync(0xffffffffu, nqv, l);
          int d1, d2;
          exact_row_global<true>(p, pair, rl, pair, nl, lane, cpr, colbuf, d1, d2);
          if (lane == l) pass = d2 != INT_MAX && uint64_t(p.den2) * uint64_t(d1) < uint64_t(p.num2) * uint64_t(d2);
        }
      } else {
        const bool real1 = g1d < kSentinelNorm, real2 = g2d < kSentinelNorm;
        if (ratio32) {
          const uint32_t d1 = static_cast<uint32_t>(nqv + g1d), d2 = static_cast<uint32_t>(nqv + g2d);
          pass = p.den2 * d1 < p.num2 * d2;
        } else {
          const uint64_t d1 = static_cast<uint64_t>(static_cast<int64_t>(nqv) + g1d);
          const uint64_t d2 = static_cast<uint64_t>(static_cast<int64_t>(nqv) + g2d);
          pass = static_cast<uint64_t>(p.den2) * d1 < static_cast<uint64_t>(p.num2) * d2;
        }
        pass = pass && valid && real2;
        if (p.nn_out != nullptr && row < p.n_rows) {
          int4 o;
          o.x = (valid && real1) ? nqv + g1d : -1; o.y = (valid && real1) ? g1i : -1;
          o.z = (valid && real2) ? nqv + g2d : -1; o.w = (valid && real2) ? g2i : -1;
          reinterpret_cast<int4*>(p.nn_out)[static_cast<int64_t>(pair) * p.n_rows + row] = o;
        }
      }
      const uint32_t cnt = __popc(__ballot_sync(0xffffffffu, pass));
      if (lane == 0) {
        if (cnt) atomicAdd(p.counts + pair, cnt);
        mbar_arrive(bar(VSmem::kColEmpty, lp & 1));  // this warp-tile's last read of the pair's column buffer
      }
      __syncwarp();
      PROF_E(6);
    }
  }

  PROF_FLUSH();
  tc_fence_before();
  __syncthreads();
  if (warp == kFirstMmaWarp) {
    tc_fence_after();
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 512;" ::"r"(tmem_base) : "memory");
  }
}

cudaError_t launch_verify_stream(const MatchParams& p, const CUtensorMap& qmap, const CUtensorMap& rmap, bool fold,
                                 int grid, cudaStream_t s) {
  static thread_local uint64_t attr_set = 0;  // bit d = device d configured (the opt-in is per device)
  int dev = 0;
  cudaGetDevice(&dev);
  if (dev >= 64 || !(attr_set >> dev & 1)) {
    for (auto k : {verify_stream_kernel<true, false>, verify_stream_kernel<true, true>,
                   verify_stream_kernel<false, false>, verify_stream_kernel<false, true>}) {
      cudaError_t e = cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                           static_cast<int>(VSmem::kAlloc));
      if (e != cudaSuccess) return e;
    }
    if (dev < 64) attr_set |= uint64_t(1) << dev;
  }
  const bool skip = piece_count_last(p.m, p.cpr) < kPiecesPerChunk;
  auto kern = fold ? (skip ? verify_stream_kernel<true, true> : verify_stream_kernel<true, false>)
                   : (skip ? verify_stream_kernel<false, true> : verify_stream_kernel<false, false>);
  kern<<<grid, kNumThreads, VSmem::kAlloc, s>>>(qmap, rmap, p);
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
  const int c = i / kBN, ii = i & (kBN - 1);
  int32_t norm = kSentinelNorm;  // N_R = sum r^2 (Alg. 1 step 1)
  int32_t sum = 0;               // sum r (search column term W = 256 sum r - N_R)
  const bool real = i < kp;
  if (i < p.m) {
    uint4* dst = p.desc ? reinterpret_cast<uint4*>(p.desc + (r * p.m + i) * kDim) : nullptr;
    if (real) {
      const uint4* src = p.src ? reinterpret_cast<const uint4*>(p.src + (r * p.m + i) * kDim) : dst;
      uint32_t acc = 0, s1 = 0;
#pragma unroll
      for (int w = 0; w < kDim / 16; ++w) {
        const uint4 x = src[w];
        acc = __dp4a(x.x, x.x, acc); acc = __dp4a(x.y, x.y, acc);
        acc = __dp4a(x.z, x.z, acc); acc = __dp4a(x.w, x.w, acc);
        s1 = __dp4a(x.x, 0x01010101u, s1); s1 = __dp4a(x.y, 0x01010101u, s1);
        s1 = __dp4a(x.z, 0x01010101u, s1); s1 = __dp4a(x.w, 0x01010101u, s1);
        if (p.src && dst) dst[w] = x;
      }
      norm = static_cast<int32_t>(acc);
      sum = static_cast<int32_t>(s1);
    } else if (dst) {
#pragma unroll
      for (int w = 0; w < kDim / 16; ++w) dst[w] = make_uint4(0, 0, 0, 0);
    }
  }
  int32_t* ck = p.colkey + (r * p.cpr + c) * kColInts;
  if (p.search) {
    const int kpc = max(0, min(kp - c * kBN, kBN));  // real columns in this chunk
    ck[ii] = real ? 256 * sum - norm : -1 - kpc;
  } else {
    ck[ii] = norm * 256 + ii;
  }
}

void launch_ref_prep(const RefPrepParams& p, cudaStream_t s) {
  const int64_t total = p.count * p.cpr * kBN;
  if (total == 0) return;
  ref_prep_kernel<<<static_cast<unsigned>((total + 255) / 256), 256, 0, s>>>(p);
}

// ------------------------------------------------------------------ a2: query prep
// N_Q per row (Alg. 1 step 2) and, for the search path, the shifted copy q' = q ^ 0x80
// (= q - 128 as s8).  Eight lanes per 128-byte row, one 16-byte word each, so a warp reads and
// writes four whole rows (512 contiguous bytes) per instruction; the row sum by shuffles.
__global__ void query_prep_kernel(const uint8_t* __restrict__ q, int64_t B, int32_t n, int32_t rows_pad,
                                  int32_t* __restrict__ nq, uint8_t* __restrict__ qs) {
  constexpr int kRows = 4;  // rows per 8-lane group: four independent 16-byte loads in flight per lane
  const int64_t gid = static_cast<int64_t>(blockIdx.x) * blockDim.x + threadIdx.x;
  const int l8 = static_cast<int>(gid & 7);
  const int64_t g = gid >> 3;  // 8-lane group
  const int64_t total = B * rows_pad;
  uint4 x[kRows];
  bool have[kRows];
#pragma unroll
  for (int k = 0; k < kRows; ++k) {  // rows g + k * groups: consecutive groups read consecutive rows
    const int64_t r = g + k * (static_cast<int64_t>(gridDim.x) * blockDim.x >> 3);
    const int64_t b = r < total ? r / rows_pad : 0;
    const int row = r < total ? static_cast<int>(r - b * rows_pad) : 0;
    have[k] = r < total && row < n;
    x[k] = have[k] ? *reinterpret_cast<const uint4*>(q + (b * n + row) * kDim + l8 * 16) : make_uint4(0, 0, 0, 0);
  }
#pragma unroll
  for (int k = 0; k < kRows; ++k) {
    const int64_t r = g + k * (static_cast<int64_t>(gridDim.x) * blockDim.x >> 3);
    uint32_t acc = 0;
    acc = __dp4a(x[k].x, x[k].x, acc); acc = __dp4a(x[k].y, x[k].y, acc);
    acc = __dp4a(x[k].z, x[k].z, acc); acc = __dp4a(x[k].w, x[k].w, acc);
    if (qs && have[k]) {
      const int64_t b = r / rows_pad;
      const int row = static_cast<int>(r - b * rows_pad);
      *reinterpret_cast<uint4*>(qs + (b * n + row) * kDim + l8 * 16) = make_uint4(
          x[k].x ^ 0x80808080u, x[k].y ^ 0x80808080u, x[k].z ^ 0x80808080u, x[k].w ^ 0x80808080u);
    }
#pragma unroll
    for (int o = 1; o < 8; o <<= 1) acc += __shfl_xor_sync(0xffffffffu, acc, o);
    if (r < total && l8 == 0) nq[r] = static_cast<int32_t>(acc);
  }
}

void launch_query_prep(const uint8_t* q, int64_t B, int32_t n, int32_t tiles_per_q, int32_t* nq, uint8_t* qs,
                       cudaStream_t s) {
  const int32_t rows_pad = tiles_per_q * kBM;
  const int64_t groups = (B * rows_pad + 3) / 4;  // 4 rows per 8-lane group
  if (B * rows_pad == 0) return;
  query_prep_kernel<<<static_cast<unsigned>((groups * 8 + 255) / 256), 256, 0, s>>>(q, B, n, rows_pad, nq, qs);
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

// grid (B, segs), 256 threads, dyn smem = 256*k*8 + 33*8.  Block (b, seg) writes its k winners to
// list (list0 + seg) of query b, lists_per_b lists per query (a search over several reference
// windows keeps its running top-k in list 0 and the window's segments after it).  With one
// segment and ids_out set, the block's winners are the final ranking: written as (ids, counts)
// directly (no merge launch).
__global__ void topk_kernel(const uint32_t* __restrict__ counts, int64_t R, int64_t ldc, int64_t id_base, int32_t k,
                            const uint8_t* __restrict__ dead, uint64_t* __restrict__ cand_out, int32_t lists_per_b,
                            int32_t list0, int64_t* __restrict__ ids_out, int32_t* __restrict__ counts_out) {
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
    if (dead && dead[r]) continue;  // deleted references are never ranked
    const uint64_t key = make_key(row[r], id_base + r);
    if (key > kth) {  // insertion into the thread's descending list
      int pos = k - 1;
      while (pos > 0 && my[pos - 1] < key) { my[pos] = my[pos - 1]; --pos; }
      my[pos] = key;
      kth = my[k - 1];
    }
  }
  __syncthreads();
  uint64_t* out = cand_out + (static_cast<int64_t>(b) * lists_per_b + list0 + seg) * k;
  block_select(lists, k, out, red);
  if (ids_out) {  // segs == 1: final (count desc, id asc) ranking
    __syncthreads();
    for (int i = threadIdx.x; i < k; i += blockDim.x) {
      const uint64_t key = out[i];
      ids_out[static_cast<int64_t>(b) * k + i] = key ? static_cast<int64_t>(kIdMask - (key & kIdMask)) : -1;
      counts_out[static_cast<int64_t>(b) * k + i] = static_cast<int32_t>(key >> 40);
    }
  }
}

// Opt a kernel into > 48 KiB of dynamic shared memory once per (device, size): the attribute is
// per device, so one bit per device and size class (thread-local: no shared mutable state).
template <class F>
void ensure_smem_attr(F* fn, size_t smem, int which) {
  if (smem <= 48 * 1024) return;
  static thread_local size_t done[2][64] = {};
  int dev = 0;
  cudaGetDevice(&dev);
  if (dev < 64 && done[which][dev] >= smem) return;
  cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, static_cast<int>(smem));
  if (dev < 64) done[which][dev] = smem;
}

void launch_topk(const uint32_t* counts, int64_t B, int64_t R, int64_t ldc, int64_t id_base, int32_t k, int32_t segs,
                 const uint8_t* dead, uint64_t* cand_out, int32_t lists_per_b, int32_t list0, cudaStream_t s,
                 int64_t* ids_out, int32_t* counts_out) {
  const size_t smem = (256 * static_cast<size_t>(k) + 33) * 8;
  ensure_smem_attr(topk_kernel, smem, 0);
  topk_kernel<<<dim3(static_cast<unsigned>(B), static_cast<unsigned>(segs)), 256, smem, s>>>(
      counts, R, ldc, id_base, k, dead, cand_out, lists_per_b, list0, segs == 1 ? ids_out : nullptr,
      segs == 1 ? counts_out : nullptr);
}

// ------------------------------------------------------------------ a6/a9: merge ranked lists
// L candidate lists of k keys per query (list l of query b at cand[b*sb + l*sl]).  One block
// of 128 threads per query: each thread gathers its share, sorts it, then block_select.
__global__ void merge_kernel(const uint64_t* cand, int32_t L, int32_t k, int64_t sb, int64_t sl,
                             uint64_t* keys_out, int64_t keys_stride, int64_t* __restrict__ ids_out,
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
    if (keys_out) keys_out[static_cast<int64_t>(b) * keys_stride + i] = key;
    if (ids_out) ids_out[static_cast<int64_t>(b) * k + i] = key ? static_cast<int64_t>(kIdMask - (key & kIdMask)) : -1;
    if (counts_out) counts_out[static_cast<int64_t>(b) * k + i] = static_cast<int32_t>(key >> 40);
  }
}

void launch_merge(const uint64_t* cand, int32_t L, int64_t B, int32_t k, int64_t sb, int64_t sl, uint64_t* keys_out,
                  int64_t* ids_out, int32_t* counts_out, cudaStream_t s, int64_t keys_stride) {
  const int threads = 128;
  const size_t smem = (threads * static_cast<size_t>(k) + 33 + k) * 8;
  ensure_smem_attr(merge_kernel, smem, 1);
  merge_kernel<<<static_cast<unsigned>(B), threads, smem, s>>>(cand, L, k, sb, sl, keys_out,
                                                               keys_stride > 0 ? keys_stride : k, ids_out, counts_out);
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
