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

// Instruction descriptor: kind::i8, A = u8, B = u8, D = s32, K-major A/B, M = 128, N = 128.
constexpr uint32_t kIdescI8 = (2u << 4)                       // D format S32
                              | (0u << 7) | (0u << 10)        // A, B unsigned 8-bit
                              | (0u << 15) | (0u << 16)       // A, B K-major
                              | (uint32_t(kPiece >> 3) << 17) // N >> 3
                              | (uint32_t(kBM >> 4) << 24);   // M >> 4

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
      "l"(adesc), "l"(bdesc), "r"(kIdescI8), "r"(bar)
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

// 128 consecutive TMEM columns of this thread's lane in one load (32x32b shape, .x128).
__device__ __forceinline__ void tmem_ld128(uint32_t taddr, uint32_t (&v)[128]) {
  asm volatile(
      "tcgen05.ld.sync.aligned.32x32b.x128.b32 {"
      "%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,%16,%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,"
      "%30,%31,%32,%33,%34,%35,%36,%37,%38,%39,%40,%41,%42,%43,%44,%45,%46,%47,%48,%49,%50,%51,%52,%53,%54,%55,%56,%57,"
      "%58,%59,%60,%61,%62,%63,%64,%65,%66,%67,%68,%69,%70,%71,%72,%73,%74,%75,%76,%77,%78,%79,%80,%81,%82,%83,%84,%85,"
      "%86,%87,%88,%89,%90,%91,%92,%93,%94,%95,%96,%97,%98,%99,%100,%101,%102,%103,%104,%105,%106,%107,%108,%109,%110,"
      "%111,%112,%113,%114,%115,%116,%117,%118,%119,%120,%121,%122,%123,%124,%125,%126,%127}, [%128];"
      : TID_LD32_OUT(v), TID_LD32_OUT((v + 32)), TID_LD32_OUT((v + 64)), TID_LD32_OUT((v + 96))
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

// ------------------------------------------------------------------ optional cycle accounting
// Built only with -DTID_PROF (experiments): per-warp clock64 buckets, read back with
// tid_debug_read_prof().  Buckets: epilogue 0 wait-accumulator 1 scan 2 finalise 3 fallback
// 4 wait-keys; MMA 0 wait-free-accumulator 1 wait-query 2 wait-ref 3 issue; producer 0 wait-ref-slot
// 1 wait-query-stage; 7 = whole loop.
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

#ifndef TID_X128
#define TID_X128 0
#endif
constexpr int kProducerWarp = 0;               // warp 0: TMA producer
constexpr int kFirstMmaWarp = 1;               // warps 1..4: MMA issuers (SMSPs 1, 2, 3, 0)
constexpr int kFirstEpiWarp = 5;               // warps 5..: epilogue (4 per group)
static_assert(kNG == 2 || kNG == 4, "4 MMA warps own the 4 TMEM buffers (2 groups x 2 halves, or 4 groups)");

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
  static constexpr uint32_t kTEmpty = kTFull + 8 * kTmemBufs;
  static constexpr uint32_t kTmemPtr = kTEmpty + 8 * kTmemBufs;
  static constexpr uint32_t kCnt = kTmemPtr + 16;                          // [4*kNG finalisers][kMaxSlots] u32
  static constexpr uint32_t kXch = (kCnt + 4 * kNG * kMaxSlots * 4 + 15) & ~15u;  // split-warp state exchange
  static constexpr uint32_t kEnd = kXch + 4 * kNG * 2 * 32 * (kSplit - 1) * 16 + 16;
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

// ------------------------------------------------------------------ epilogue scans
// A "piece" = one 128-column accumulator buffer (MMA N = 128) of one (query tile, reference
// chunk half).  Each epilogue thread owns one TMEM lane = one query row.

// Exact top-2 over one piece, accumulated into running states (a1 <= a2, b1 <= b2) of packed keys
// 256 * (N_R - 2S) + i (unique per column within a 256-column chunk).  ~2.5 ALU ops / element.
template <int NCOL>
__device__ __forceinline__ void scan_exact(uint32_t taddr, uint32_t ck_addr, int& a1, int& a2, int& b1, int& b2) {
  uint32_t v[2][32];
  tmem_ld32(taddr, v[0]);
  tmem_wait_ld();
  reg_fence(v[0]);
#pragma unroll
  for (int jj = 0; jj < NCOL / 32; ++jj) {
    // software pipeline: the next 32 columns are in flight while these are scanned
    if (jj + 1 < NCOL / 32) tmem_ld32(taddr + (jj + 1) * 32, v[(jj + 1) & 1]);
    const uint32_t* w = v[jj & 1];
#pragma unroll
    for (int i = 0; i < 32; i += 4) {
      const int4 c4 = lds128(ck_addr + (jj * 32 + i) * 4);
      const int x0 = c4.x - 512 * static_cast<int>(w[i]);
      const int x1 = c4.y - 512 * static_cast<int>(w[i + 1]);
      const int x2 = c4.z - 512 * static_cast<int>(w[i + 2]);
      const int x3 = c4.w - 512 * static_cast<int>(w[i + 3]);
      int lo = min(x0, x1), hi = max(x0, x1);
      int tt = max(a1, lo);
      a2 = min(min(a2, tt), hi);
      a1 = min(a1, lo);
      lo = min(x2, x3); hi = max(x2, x3);
      tt = max(b1, lo);
      b2 = min(min(b2, tt), hi);
      b1 = min(b1, lo);
    }
    // the state must be final before waiting for the next TMEM load (keeps the scan streaming)
    asm volatile("" : "+r"(a1), "+r"(a2), "+r"(b1), "+r"(b2));
    if (jj + 1 < NCOL / 32) { tmem_wait_ld(); reg_fence(v[(jj + 1) & 1]); }
  }
}

__device__ __forceinline__ uint32_t prmt_top16x2(uint32_t a, uint32_t b) {  // a[31:16] | b[31:16] << 16
  uint32_t r;
  asm("prmt.b32 %0, %1, %2, 0x7632;" : "=r"(r) : "r"(a), "r"(b));
  return r;
}

// Coarse top-2 over one piece (search fast path): the exact key 256*(N_R - 2S) + i is formed by
// the same IMAD (FMA pipe); its top 16 bits floor((N_R - 2S)/256) are packed two columns per
// register (one PRMT) and the top-2 runs on s16x2 lanes (VIMNMX.S16x2 and 3-input forms):
// ~1.75 ALU ops per element instead of 2.5.  Accumulates into four sorted packed states; the two
// smallest coarse keys u1 <= u2 of their union bound N_R - 2S of the true 1st / 2nd neighbour
// to [256 u, 256 u + 255].
template <int NCOL>
__device__ __forceinline__ void scan_coarse(uint32_t taddr, uint32_t ck_addr, uint32_t& A1, uint32_t& A2,
                                            uint32_t& B1, uint32_t& B2) {
  uint32_t v[2][32];
  int4 ck[2][8];  // column keys, loaded one 32-column chunk ahead (hides the LDS latency)
  tmem_ld32(taddr, v[0]);
#pragma unroll
  for (int i = 0; i < 8; ++i) ck[0][i] = lds128(ck_addr + i * 16);
  tmem_wait_ld();
  reg_fence(v[0]);
#pragma unroll
  for (int jj = 0; jj < NCOL / 32; ++jj) {
    if (jj + 1 < NCOL / 32) {
      tmem_ld32(taddr + (jj + 1) * 32, v[(jj + 1) & 1]);
#pragma unroll
      for (int i = 0; i < 8; ++i) ck[(jj + 1) & 1][i] = lds128(ck_addr + ((jj + 1) * 32 + i * 4) * 4);
    }
    const uint32_t* w = v[jj & 1];
    const int4* c4 = ck[jj & 1];
#pragma unroll
    for (int i = 0; i < 32; i += 8) {
      const int4 c0 = c4[i / 4], c1 = c4[i / 4 + 1];
      const uint32_t k0 = static_cast<uint32_t>(c0.x - 512 * static_cast<int>(w[i]));
      const uint32_t k1 = static_cast<uint32_t>(c0.y - 512 * static_cast<int>(w[i + 1]));
      const uint32_t k2 = static_cast<uint32_t>(c0.z - 512 * static_cast<int>(w[i + 2]));
      const uint32_t k3 = static_cast<uint32_t>(c0.w - 512 * static_cast<int>(w[i + 3]));
      const uint32_t k4 = static_cast<uint32_t>(c1.x - 512 * static_cast<int>(w[i + 4]));
      const uint32_t k5 = static_cast<uint32_t>(c1.y - 512 * static_cast<int>(w[i + 5]));
      const uint32_t k6 = static_cast<uint32_t>(c1.z - 512 * static_cast<int>(w[i + 6]));
      const uint32_t k7 = static_cast<uint32_t>(c1.w - 512 * static_cast<int>(w[i + 7]));
      const uint32_t x = prmt_top16x2(k0, k1), y = prmt_top16x2(k2, k3);
      const uint32_t z = prmt_top16x2(k4, k5), ww = prmt_top16x2(k6, k7);
      uint32_t lo = __vmins2(x, y), hi = __vmaxs2(x, y);
      uint32_t tt = __vmaxs2(A1, lo);
      A2 = __vmins2(__vmins2(A2, tt), hi);
      A1 = __vmins2(A1, lo);
      lo = __vmins2(z, ww); hi = __vmaxs2(z, ww);
      tt = __vmaxs2(B1, lo);
      B2 = __vmins2(__vmins2(B2, tt), hi);
      B1 = __vmins2(B1, lo);
    }
    asm volatile("" : "+r"(A1), "+r"(A2), "+r"(B1), "+r"(B2));
    if (jj + 1 < NCOL / 32) { tmem_wait_ld(); reg_fence(v[(jj + 1) & 1]); }
  }
}

// Same scan, one .x128 TMEM load per piece and a single wait (latency exposed once per piece).
__device__ __forceinline__ void scan_coarse_x128(uint32_t taddr, uint32_t ck_addr, uint32_t& A1, uint32_t& A2,
                                                 uint32_t& B1, uint32_t& B2) {
  uint32_t v[128];
  tmem_ld128(taddr, v);
  tmem_wait_ld();
#pragma unroll
  for (int i = 0; i < 128; ++i) asm volatile("" : "+r"(v[i]));
#pragma unroll
  for (int i = 0; i < 128; i += 8) {
    const int4 c0 = lds128(ck_addr + i * 4), c1 = lds128(ck_addr + (i + 4) * 4);
    const uint32_t k0 = static_cast<uint32_t>(c0.x - 512 * static_cast<int>(v[i]));
    const uint32_t k1 = static_cast<uint32_t>(c0.y - 512 * static_cast<int>(v[i + 1]));
    const uint32_t k2 = static_cast<uint32_t>(c0.z - 512 * static_cast<int>(v[i + 2]));
    const uint32_t k3 = static_cast<uint32_t>(c0.w - 512 * static_cast<int>(v[i + 3]));
    const uint32_t k4 = static_cast<uint32_t>(c1.x - 512 * static_cast<int>(v[i + 4]));
    const uint32_t k5 = static_cast<uint32_t>(c1.y - 512 * static_cast<int>(v[i + 5]));
    const uint32_t k6 = static_cast<uint32_t>(c1.z - 512 * static_cast<int>(v[i + 6]));
    const uint32_t k7 = static_cast<uint32_t>(c1.w - 512 * static_cast<int>(v[i + 7]));
    const uint32_t x = prmt_top16x2(k0, k1), y = prmt_top16x2(k2, k3);
    const uint32_t z = prmt_top16x2(k4, k5), ww = prmt_top16x2(k6, k7);
    uint32_t lo = __vmins2(x, y), hi = __vmaxs2(x, y);
    uint32_t tt = __vmaxs2(A1, lo);
    A2 = __vmins2(__vmins2(A2, tt), hi);
    A1 = __vmins2(A1, lo);
    lo = __vmins2(z, ww); hi = __vmaxs2(z, ww);
    tt = __vmaxs2(B1, lo);
    B2 = __vmins2(__vmins2(B2, tt), hi);
    B1 = __vmins2(B1, lo);
    if ((i & 31) == 24) asm volatile("" : "+r"(A1), "+r"(A2), "+r"(B1), "+r"(B2));
  }
}

// Top-2 (per 16-bit lane) of the union of two sorted packed states: (X1 <= X2) U (Y1 <= Y2).
__device__ __forceinline__ void merge_top2_s16x2(uint32_t& X1, uint32_t& X2, uint32_t Y1, uint32_t Y2) {
  const uint32_t m2 = __vmins2(__vmaxs2(X1, Y1), __vmins2(X2, Y2));
  X1 = __vmins2(X1, Y1);
  X2 = m2;
}

// Two smallest coarse keys u1 <= u2 (multiset order statistics) of four packed states.
__device__ __forceinline__ void finish_coarse(uint32_t A1, uint32_t A2, uint32_t B1, uint32_t B2, int& u1, int& u2) {
  merge_top2_s16x2(A1, A2, B1, B2);
  const int l1 = static_cast<int16_t>(A1 & 0xFFFFu), h1 = static_cast<int16_t>(A1 >> 16);
  const int l2 = static_cast<int16_t>(A2 & 0xFFFFu), h2 = static_cast<int16_t>(A2 >> 16);
  u1 = min(l1, h1);
  u2 = min(max(l1, h1), min(l2, h2));
}

// Exact fallback for one undecided query row (rare): the warp recomputes the 256 dot products of
// that row against the resident reference chunk straight from shared memory (both tiles are
// SWIZZLE_128B: 16-byte chunk c of row r sits at chunk c ^ (r & 7)), 8 columns per lane with
// dp4a, and reduces the exact top-2 packed keys across the warp.
__device__ __forceinline__ void exact_row_from_smem(uint32_t q_tile, int qrow, uint32_t r_tile, uint32_t ck_addr,
                                                    int lane, int& k1, int& k2) {
  uint4 q[8];
#pragma unroll
  for (int c = 0; c < 8; ++c) {
    const int4 t = lds128(q_tile + qrow * 128 + ((c ^ (qrow & 7)) << 4));
    q[c] = make_uint4(t.x, t.y, t.z, t.w);
  }
  int a1 = INT_MAX, a2 = INT_MAX;
#pragma unroll 2
  for (int jj = 0; jj < kBN / 32; ++jj) {
    const int col = jj * 32 + lane;
    uint32_t dot = 0;
#pragma unroll
    for (int c = 0; c < 8; ++c) {
      const int4 r = lds128(r_tile + col * 128 + ((c ^ (col & 7)) << 4));
      dot = __dp4a(q[c].x, static_cast<uint32_t>(r.x), dot);
      dot = __dp4a(q[c].y, static_cast<uint32_t>(r.y), dot);
      dot = __dp4a(q[c].z, static_cast<uint32_t>(r.z), dot);
      dot = __dp4a(q[c].w, static_cast<uint32_t>(r.w), dot);
    }
    int ck;
    asm volatile("ld.shared.s32 %0, [%1];" : "=r"(ck) : "r"(ck_addr + col * 4));
    const int key = ck - 512 * static_cast<int>(dot);
    a2 = min(a2, max(a1, key));
    a1 = min(a1, key);
  }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) {
    const int b1 = __shfl_xor_sync(0xffffffffu, a1, o), b2 = __shfl_xor_sync(0xffffffffu, a2, o);
    const int m2 = min(max(a1, b1), min(a2, b2));
    a1 = min(a1, b1);
    a2 = m2;
  }
  k1 = a1;
  k2 = a2;
}

// ------------------------------------------------------------------ fused match kernel
// One persistent CTA per SM.  A job = (reference group resident in SMEM) x (range of query
// tiles streamed through a 4-stage ring).  Unit u = (query tile t, reference s) belongs to
// epilogue group u % kNG; each unit is 2*cpr pieces of 128 accumulator columns.  Group g owns
// kNB TMEM buffers and double-buffers its pieces, so the MMA of its next piece overlaps the
// scan of the current one.
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
  uint32_t* xch_smem = reinterpret_cast<uint32_t*>(smem + SmemPlan::kXch);
  const bool use_coarse = p.coarse && cpr == 1 && p.mode == kModeSearch && p.nn_out == nullptr;

  if (threadIdx.x == 0) {
    prefetch_tmap(&qmap);
    prefetch_tmap(&rmap);
    // query stages: freed by the MMA commit and by every epilogue warp (the exact fallback reads them)
    for (int i = 0; i < kQStages; ++i) { mbar_init(qfull(i), 1); mbar_init(qempty(i), 4 + kEpiWarps); }
    for (int i = 0; i < kMaxSlots; ++i) { mbar_init(rfull(i), 1); mbar_init(rempty(i), 4 + kEpiWarps); }
    for (int i = 0; i < kTmemBufs; ++i) { mbar_init(tfull(i), 1); mbar_init(tempty(i), 4 * kSplit); }
    fence_barrier_init();
  }
  if (threadIdx.x < 4 * kNG * kMaxSlots) cnt_smem[threadIdx.x] = 0;
  if (warp == kFirstMmaWarp) {  // TMEM: kTmemBufs accumulator buffers x 128 columns (all 512)
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
    // ===================== TMA producer =====================
    if (lane == 0) {
      uint32_t qctr = 0;
      uint32_t slot_use[kMaxSlots] = {0, 0, 0, 0};
      for (int32_t j = blockIdx.x; j < p.n_jobs; j += gridDim.x) {
        const Job J = decode_job(p, j);
        const int nslots = J.nr * cpr;
        for (int sl = 0; sl < nslots; ++sl) {
          PROF_B(); mbar_wait_sleep(rempty(sl), (slot_use[sl] & 1) ^ 1); PROF_E(0);
          mbar_expect_tx(rfull(sl), kRTileBytes + kColBytes);
          const int s = sl / cpr, c = sl % cpr;
          const int64_t ref = J.ref_first + s;
          tma_load_3d(sbase + SmemPlan::kR + sl * kRTileBytes, &rmap, rfull(sl), 0, c * kBN,
                      static_cast<int>(p.ref_map_base + ref));
          bulk_load(sbase + SmemPlan::kCol + sl * kColBytes, p.colkey + (ref * cpr + c) * kColInts, kColBytes,
                    rfull(sl));
          ++slot_use[sl];
        }
        const int ntiles = J.nq * T;
        for (int t = 0; t < ntiles; ++t, ++qctr) {
          const int st = qctr % kQStages;
          PROF_B(); mbar_wait_sleep(qempty(st), ((qctr / kQStages) & 1) ^ 1); PROF_E(1);
          mbar_expect_tx(qfull(st), kQTileBytes);
          tma_load_3d(sbase + SmemPlan::kQ + st * kQTileBytes, &qmap, qfull(st), 0, (t % T) * kBM, J.q_first + t / T);
        }
      }
    }
  } else if (warp >= kFirstMmaWarp && warp < kFirstMmaWarp + 4) {
    // ===================== MMA issuers: 4 warps, one per SMSP, one per TMEM buffer ==============
    // Issuing tcgen05.mma costs the issuing SMSP real throughput, and each SMSP's epilogue warps
    // own one TMEM lane quarter, so the issue load is spread evenly: MMA warp mw owns accumulator
    // buffer mw = (epilogue group g = mw / 2, column half h = mw % 2) and issues exactly the
    // pieces (unit u with u % 2 == g, chunk c, half h), in order.  Whole warp, one elected lane.
    {
      const int mw = warp - kFirstMmaWarp;
      // kNG == 2: buffer mw = (group mw/2, half mw%2); kNG == 4: buffer mw = group mw, both halves
      const int my_g = kNG == 2 ? (mw >> 1) : mw;
      const int h_lo = kNG == 2 ? (mw & 1) : 0, h_hi = kNG == 2 ? (mw & 1) : 1;
      uint32_t qctr = 0, pc = 0;
      uint32_t slot_use[kMaxSlots] = {0, 0, 0, 0};
      const uint32_t dt = tmem_base + mw * kPiece;
      for (int32_t j = blockIdx.x; j < p.n_jobs; j += gridDim.x) {
        const Job J = decode_job(p, j);
        const int nslots = J.nr * cpr;
        const int U = J.nq * T * J.nr;
        uint32_t ready_mask = 0;
        int waited = 0, t = 0, s = 0, g = 0;
        for (int u = 0; u < U; ++u) {
          if (g == my_g) {
            while (waited <= t) {
              const uint32_t gq = qctr + waited;
              PROF_B(); mbar_wait_sleep(qfull(gq % kQStages), (gq / kQStages) & 1); PROF_E(1);
              ++waited;
            }
            const uint32_t st = (qctr + t) % kQStages;
            const uint64_t ad = smem_desc_sw128(sbase + SmemPlan::kQ + st * kQTileBytes);
            for (int c = 0; c < cpr; ++c) {
              const int sl = s * cpr + c;
              if (!(ready_mask >> sl & 1u)) { PROF_B(); mbar_wait_sleep(rfull(sl), slot_use[sl] & 1); PROF_E(2); ready_mask |= 1u << sl; }
              for (int h = h_lo; h <= h_hi; ++h) {
                const uint64_t bd = smem_desc_sw128(sbase + SmemPlan::kR + sl * kRTileBytes) +
                                    h * (kPiece * kDim >> 4);  // rows 128h.. of the chunk
                PROF_B(); mbar_wait_sleep(tempty(mw), (pc & 1) ^ 1); PROF_E(0);
                tc_fence_after();
                mma_piece(dt, ad, bd, tfull(mw));
                ++pc;
              }
            }
          }
          if (s == J.nr - 1) {  // this warp's release of query tile t (covers all its prior MMAs)
            if (waited <= t) {  // never touched tile t: still wait for it so the phase order holds
              const uint32_t gq = qctr + t;
              mbar_wait_sleep(qfull(gq % kQStages), (gq / kQStages) & 1);
              waited = t + 1;
            }
            mma_commit(qempty((qctr + t) % kQStages));
          }
          if (++g == kNG) g = 0;
          if (++s == J.nr) { s = 0; ++t; }
        }
        for (int sl = 0; sl < nslots; ++sl) { mma_commit(rempty(sl)); ++slot_use[sl]; }
        qctr += J.nq * T;
      }
    }
  } else {
    // ===================== epilogue: TMEM -> registers -> top-2 -> ratio -> count =====================
    const int ew = warp - kFirstEpiWarp;     // 0 .. 4*kNG*kSplit-1
    const int g = ew / (4 * kSplit);         // epilogue group (units u with u % kNG == g)
    const int cq = (ew >> 2) % kSplit;       // column part of every piece this warp scans
    const int quarter = warp & 3;            // TMEM lanes 32*quarter .. +31 (hardware restriction)
    const int fin = g * 4 + quarter;         // finaliser slot (the cq == 0 warp of this lane quarter)
    const uint32_t pair_bar = 1 + fin;       // named barrier of the kSplit warps of (group, quarter)
    uint32_t xc = 0;                         // exchanges done (parity selects the exchange slot)
    const uint32_t taddr_q = tmem_base + (static_cast<uint32_t>(quarter * 32) << 16) + cq * kCPW;
    uint32_t mp = 0;                         // pieces consumed by this group
    uint32_t qctr = 0;
    uint32_t slot_use[kMaxSlots] = {0, 0, 0, 0};
    const int row_in_tile = quarter * 32 + lane;
    const int nq_ld = T * kBM;

    for (int32_t j = blockIdx.x; j < p.n_jobs; j += gridDim.x) {
      const Job J = decode_job(p, j);
      const int nslots = J.nr * cpr;
      const int U = J.nq * T * J.nr;
      int t = 0, s = 0, tq = 0, qi = J.q_first, ug = 0;
      bool touched = false;
      for (int u = 0; u < U; ++u) {
        if (ug == g) {
          touched = true;
          PROF_B();
          const int row = tq * kBM + row_in_tile;
          const int nvalid = p.n_valid ? p.n_valid[qi] : p.n_rows;
          const bool valid = row < nvalid && row < p.n_rows;
          const int32_t nqv = p.nq[static_cast<int64_t>(qi) * nq_ld + row];
          PROF_E(6);
          int g1d = INT_MAX, g1i = -1, g2d = INT_MAX, g2i = -1;  // running exact 2-NN over chunks
          bool pass = false;
          uint32_t A1 = 0x7FFF7FFFu, A2 = 0x7FFF7FFFu, B1 = 0x7FFF7FFFu, B2 = 0x7FFF7FFFu;
          if (use_coarse) {
            const int sl = s;
            PROF_B(); mbar_wait(rfull(sl), slot_use[sl] & 1); PROF_E(4);  // column keys have landed
#pragma unroll
            for (int h = 0; h < 2; ++h) {
              const uint32_t buf = g * kNB + mp % kNB;
              PROF_B(); mbar_wait(tfull(buf), (mp / kNB) & 1); PROF_E(0);
              tc_fence_after();
              PROF_B();
#if TID_X128
              scan_coarse_x128(taddr_q + buf * kPiece, sbase + SmemPlan::kCol + sl * kColBytes + h * kPiece * 4, A1,
                               A2, B1, B2);
#else
              scan_coarse<kCPW>(taddr_q + buf * kPiece,
                                sbase + SmemPlan::kCol + sl * kColBytes + (h * kPiece + cq * kCPW) * 4, A1, A2, B1, B2);
#endif
              PROF_E(1);
              PROF_B();
              tc_fence_before();
              __syncwarp();
              if (lane == 0) mbar_arrive(tempty(buf));  // accumulator free as soon as it is scanned
              PROF_E(5);
              ++mp;
            }
            if (kSplit > 1) {  // the kSplit warps of this lane quarter merge their states
              uint4* x = reinterpret_cast<uint4*>(xch_smem) + (fin * 2 + (xc & 1)) * 32 * (kSplit - 1);
              if (cq > 0) x[(cq - 1) * 32 + lane] = make_uint4(A1, A2, B1, B2);
              named_bar(pair_bar, 32 * kSplit);
              if (cq == 0) {
#pragma unroll
                for (int o = 0; o < kSplit - 1; ++o) {
                  const uint4 r = x[o * 32 + lane];
                  merge_top2_s16x2(A1, A2, r.x, r.y);
                  merge_top2_s16x2(B1, B2, r.z, r.w);
                }
              }
              ++xc;
            }
          }
          if (use_coarse && cq == 0) {
            const int sl = s;
            PROF_B();
            int u1, u2;
            finish_coarse(A1, A2, B1, B2, u1, u2);
            // bounds: N_R - 2S of the 1st / 2nd neighbour lies in [256 u, 256 u + 255]
            const int64_t d1lo = static_cast<int64_t>(nqv) + 256 * static_cast<int64_t>(u1);
            const int64_t d2lo = static_cast<int64_t>(nqv) + 256 * static_cast<int64_t>(u2);
            const int64_t den2 = p.den2, num2 = p.num2;
            // u == 0x7FFF only for padding columns (sentinel N_R); real keys are <= 32512
            const bool fail_sure = (u2 >= 0x7FFF) || den2 * d1lo >= num2 * (d2lo + 255);
            const bool pass_sure = !fail_sure && den2 * (d1lo + 255) < num2 * d2lo;
            pass = valid && pass_sure;
            uint32_t undecided = __ballot_sync(0xffffffffu, valid && !pass_sure && !fail_sure);
            PROF_E(2);
            if (undecided) {
              PROF_B();
              const uint32_t qt = sbase + SmemPlan::kQ + ((qctr + t) % kQStages) * kQTileBytes;
              const uint32_t rt = sbase + SmemPlan::kR + sl * kRTileBytes;
              const uint32_t ck = sbase + SmemPlan::kCol + sl * kColBytes;
              while (undecided) {
                const int l = __ffs(undecided) - 1;
                undecided &= undecided - 1;
                int k1, k2;
                exact_row_from_smem(qt, quarter * 32 + l, rt, ck, lane, k1, k2);
                if (lane == l) {
                  const int64_t d1 = static_cast<int64_t>(nqv) + (k1 >> 8);
                  const int64_t d2 = static_cast<int64_t>(nqv) + (k2 >> 8);
                  pass = (k2 >> 8) < kSentinelNorm && den2 * d1 < num2 * d2;
                }
              }
              PROF_E(3);
            }
          } else if (!use_coarse) {
            for (int c = 0; c < cpr; ++c) {
              const int sl = s * cpr + c;
              mbar_wait(rfull(sl), slot_use[sl] & 1);
              int a1 = INT_MAX, a2 = INT_MAX, b1 = INT_MAX, b2 = INT_MAX;
#pragma unroll
              for (int h = 0; h < 2; ++h) {
                const uint32_t buf = g * kNB + mp % kNB;
                mbar_wait(tfull(buf), (mp / kNB) & 1);
                tc_fence_after();
                scan_exact<kCPW>(taddr_q + buf * kPiece,
                                 sbase + SmemPlan::kCol + sl * kColBytes + (h * kPiece + cq * kCPW) * 4, a1, a2, b1, b2);
                tc_fence_before();
                __syncwarp();
                if (lane == 0) mbar_arrive(tempty(buf));
                ++mp;
              }
              int k1 = min(a1, b1);
              int k2 = min(max(a1, b1), min(a2, b2));
              if (kSplit > 1) {
                uint4* x = reinterpret_cast<uint4*>(xch_smem) + (fin * 2 + (xc & 1)) * 32 * (kSplit - 1);
                if (cq > 0) x[(cq - 1) * 32 + lane] = make_uint4(static_cast<uint32_t>(k1), static_cast<uint32_t>(k2), 0, 0);
                named_bar(pair_bar, 32 * kSplit);
                if (cq == 0) {
#pragma unroll
                  for (int o = 0; o < kSplit - 1; ++o) {
                    const uint4 r = x[o * 32 + lane];
                    const int p1 = static_cast<int>(r.x), p2 = static_cast<int>(r.y);
                    const int m2 = min(max(k1, p1), min(k2, p2));
                    k1 = min(k1, p1);
                    k2 = m2;
                  }
                }
                ++xc;
              }
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
            pass = valid && real2 &&
                   static_cast<uint64_t>(p.den2) * static_cast<uint64_t>(d1) <
                       static_cast<uint64_t>(p.num2) * static_cast<uint64_t>(d2);
            if (cq == 0 && p.nn_out != nullptr && row < p.n_rows) {
              int4 o;
              o.x = (valid && real1) ? static_cast<int>(d1) : -1; o.y = (valid && real1) ? g1i : -1;
              o.z = (valid && real2) ? static_cast<int>(d2) : -1; o.w = (valid && real2) ? g2i : -1;
              reinterpret_cast<int4*>(p.nn_out)[static_cast<int64_t>(qi) * p.n_rows + row] = o;
            }
          }
          const uint32_t bal = __ballot_sync(0xffffffffu, pass);
          if (lane == 0 && cq == 0) {
            uint32_t& acc = cnt_smem[fin * kMaxSlots + s];
            acc += __popc(bal);
            // flush when this group holds no further unit of this (query, reference) pair
            if (tq == T - 1 || u + J.nr >= U || J.nr % kNG != 0) {
              if (acc) {
                const int64_t ci = (p.mode == kModeVerify)
                                       ? qi : static_cast<int64_t>(qi) * p.ldc + p.col0 + J.ref_first + s;
                atomicAdd(p.counts + ci, acc);
              }
              acc = 0;
            }
          }
        }
        if (s == J.nr - 1) {  // this warp is done with query tile t (fallback reads it)
          const uint32_t gq = qctr + t;
          // a warp with no unit in tile t must not arrive before tile t has landed, or its
          // arrival would count towards the stage's previous phase
          if (!touched) mbar_wait(qfull(gq % kQStages), (gq / kQStages) & 1);
          touched = false;
          __syncwarp();
          if (lane == 0) mbar_arrive(qempty(gq % kQStages));
        }
        if (++ug == kNG) ug = 0;
        if (++s == J.nr) {
          s = 0; ++t;
          if (++tq == T) { tq = 0; ++qi; }
        }
      }
      __syncwarp();
      if (lane == 0)
        for (int sl = 0; sl < nslots; ++sl) mbar_arrive(rempty(sl));
      for (int sl = 0; sl < nslots; ++sl) ++slot_use[sl];
      qctr += J.nq * T;
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
  const int c = i / kBN, ii = i & (kBN - 1);
  int32_t* ck = p.colkey + (r * p.cpr + c) * kColInts;
  ck[ii] = norm * 256 + ii;
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
                            const uint8_t* __restrict__ dead, uint64_t* __restrict__ cand_out) {
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
  block_select(lists, k, cand_out + (static_cast<int64_t>(b) * segs + seg) * k, red);
}

void launch_topk(const uint32_t* counts, int64_t B, int64_t R, int64_t ldc, int64_t id_base, int32_t k, int32_t segs,
                 const uint8_t* dead, uint64_t* cand_out, cudaStream_t s) {
  const size_t smem = (256 * static_cast<size_t>(k) + 33) * 8;
  static size_t attr = 0;
  if (smem > 48 * 1024 && smem > attr) {
    cudaFuncSetAttribute(topk_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, static_cast<int>(smem));
    attr = smem;
  }
  topk_kernel<<<dim3(static_cast<unsigned>(B), static_cast<unsigned>(segs)), 256, smem, s>>>(counts, R, ldc, id_base,
                                                                                              k, dead, cand_out);
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
