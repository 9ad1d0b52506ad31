// tcgen05.mma throughput, one CTA per SM, one elected thread issuing back-to-back MMAs into one
// TMEM accumulator (no epilogue): cycles per MMA for kind::f16 / kind::i8, SS operands
// (A and B from shared memory, SWIZZLE_128B K-major, contents irrelevant), M = 128, N = 64/128/256.
#include <cstdint>
#include <cstdio>

__device__ __forceinline__ uint64_t desc128(uint32_t addr) {
  return static_cast<uint64_t>((addr & 0x3FFFF) >> 4) | (uint64_t(1) << 16) | (uint64_t(1024 >> 4) << 32) |
         (uint64_t(1) << 46) | (uint64_t(2) << 61);
}
template <int KIND>  // 0 = f16 (D f32), 1 = i8 (D s32); 2 / 3 = i8 / f16 with A from TMEM
__host__ __device__ constexpr uint32_t idesc(int n) {
  return (KIND == 0 || KIND == 3) ? ((1u << 4) | (uint32_t(n >> 3) << 17) | (uint32_t(128 >> 4) << 24))
                                  : ((2u << 4) | (uint32_t(n >> 3) << 17) | (uint32_t(128 >> 4) << 24));
}
template <int KIND, int N, int NACC>
__global__ void k(int iters, long long* cyc) {
  extern __shared__ __align__(1024) uint8_t sm[];
  __shared__ uint32_t tptr;
  __shared__ __align__(8) uint64_t bar;
  const int warp = threadIdx.x >> 5;
  const uint32_t sa = static_cast<uint32_t>(__cvta_generic_to_shared(sm));
  const uint32_t sb = sa + 16384;
  if (threadIdx.x == 0) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"((uint32_t)__cvta_generic_to_shared(&bar)));
    asm volatile("fence.mbarrier_init.release.cluster;");
  }
  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 512;" ::"r"((uint32_t)__cvta_generic_to_shared(&tptr)));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;");
  const uint32_t t = tptr;
  if (KIND == 5 && (threadIdx.x & 31) == 0 && warp < NACC) {
    const uint64_t b = desc128(sb);
    const uint32_t id = idesc<1>(N);
    const uint32_t d = t + warp * N;
    long long t0 = clock64();
    for (int i = 0; i < iters; ++i)
      asm volatile("{\n\t.reg .pred p;\n\tsetp.eq.b32 p, 0, 0;\n\t"
                   "tcgen05.mma.cta_group::1.kind::i8 [%0], [%1], %2, %3, p;\n\t"
                   "tcgen05.mma.cta_group::1.kind::i8 [%0], [%1], %2, %3, p;\n\t"
                   "tcgen05.mma.cta_group::1.kind::i8 [%0], [%1], %2, %3, p;\n\t"
                   "tcgen05.mma.cta_group::1.kind::i8 [%0], [%1], %2, %3, p;\n\t"
                   "tcgen05.mma.cta_group::1.kind::i8 [%0], [%1], %2, %3, p;\n\t"
                   "tcgen05.mma.cta_group::1.kind::i8 [%0], [%1], %2, %3, p;\n\t"
                   "tcgen05.mma.cta_group::1.kind::i8 [%0], [%1], %2, %3, p;\n\t"
                   "tcgen05.mma.cta_group::1.kind::i8 [%0], [%1], %2, %3, p;\n\t}" ::"r"(d), "r"(t + 448), "l"(b), "r"(id));
    if (warp == 0) {
      asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"((uint32_t)__cvta_generic_to_shared(&bar)));
      asm volatile("{\n\t.reg .pred P1;\n\tW:\n\tmbarrier.try_wait.parity.shared::cta.b64 P1, [%0], 0;\n\t@P1 bra D;\n\tbra W;\n\tD:\n\t}" ::"r"((uint32_t)__cvta_generic_to_shared(&bar)));
      cyc[blockIdx.x] = clock64() - t0;
    }
  }
  if (KIND != 5 && threadIdx.x == 0) {
    const uint64_t a = desc128(sa), b = desc128(sb);
    const uint32_t id = idesc<KIND>(N);
    long long t0 = clock64();
    for (int i = 0; i < iters; ++i) {
      const uint32_t t_ = t;
      const uint32_t t = t_ + (i % NACC) * N;  // NACC independent accumulators, interleaved
      if (KIND == 0)
        asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
                     "tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n\t}" ::"r"(t), "l"(a), "l"(b), "r"(id), "r"(i));
      else if (KIND == 1)
        asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
                     "tcgen05.mma.cta_group::1.kind::i8 [%0], %1, %2, %3, p;\n\t}" ::"r"(t), "l"(a), "l"(b), "r"(id), "r"(i));
      else if (KIND == 2)
        asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
                     "tcgen05.mma.cta_group::1.kind::i8 [%0], [%1], %2, %3, p;\n\t}" ::"r"(t), "r"(t + 256), "l"(b), "r"(id), "r"(i));
      else if (KIND == 3)
        asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
                     "tcgen05.mma.cta_group::1.kind::f16 [%0], [%1], %2, %3, p;\n\t}" ::"r"(t), "r"(t + 256), "l"(b), "r"(id), "r"(i));
      else {  // 8 back-to-back i8 TS MMAs per block, into NACC... accumulator t (dependent chain)
        asm volatile("{\n\t.reg .pred p;\n\tsetp.eq.b32 p, 0, 0;\n\t"
                     "tcgen05.mma.cta_group::1.kind::i8 [%0], [%1], %2, %3, p;\n\t"
                     "tcgen05.mma.cta_group::1.kind::i8 [%0], [%1], %2, %3, p;\n\t"
                     "tcgen05.mma.cta_group::1.kind::i8 [%0], [%1], %2, %3, p;\n\t"
                     "tcgen05.mma.cta_group::1.kind::i8 [%0], [%1], %2, %3, p;\n\t"
                     "tcgen05.mma.cta_group::1.kind::i8 [%0], [%1], %2, %3, p;\n\t"
                     "tcgen05.mma.cta_group::1.kind::i8 [%0], [%1], %2, %3, p;\n\t"
                     "tcgen05.mma.cta_group::1.kind::i8 [%0], [%1], %2, %3, p;\n\t"
                     "tcgen05.mma.cta_group::1.kind::i8 [%0], [%1], %2, %3, p;\n\t}" ::"r"(t), "r"(t_ + 448), "l"(b), "r"(id));
      }
    }
    asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"((uint32_t)__cvta_generic_to_shared(&bar)));
    asm volatile("{\n\t.reg .pred P1;\n\tW:\n\tmbarrier.try_wait.parity.shared::cta.b64 P1, [%0], 0;\n\t@P1 bra D;\n\tbra W;\n\tD:\n\t}" ::"r"((uint32_t)__cvta_generic_to_shared(&bar)));
    long long t1 = clock64();
    cyc[blockIdx.x] = t1 - t0;
  }
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  if (warp == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 512;" ::"r"(t));
}
template <int KIND, int N, int NACC = 1>
void run(const char* name) {
  long long* cyc;
  cudaMalloc(&cyc, 148 * 8);
  const int smem = 16384 + N * 128 + 2048;
  cudaFuncSetAttribute(k<KIND, N, NACC>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  const int iters = 20000;
  k<KIND, N, NACC><<<148, 128, smem>>>(100, cyc);
  k<KIND, N, NACC><<<148, 128, smem>>>(iters, cyc);
  cudaError_t e = cudaDeviceSynchronize();
  long long c[148];
  cudaMemcpy(c, cyc, sizeof(c), cudaMemcpyDeviceToHost);
  const double per = (double)c[0] / iters / (KIND == 4 ? 8 : KIND == 5 ? 8 * NACC : 1);
  const double floor = 128.0 * N / 256.0;
  printf("%-5s acc=%d N=%3d : %7.1f cycles/MMA  (floor %5.1f, %.0f%%)  %s\n", name, NACC, N, per, floor, 100 * floor / per,
         cudaGetErrorString(e));
  cudaFree(cyc);
}
int main() {
  run<0, 64>("f16");
  run<0, 128>("f16");
  run<0, 256>("f16");
  run<1, 64>("i8");
  run<1, 128>("i8");
  run<1, 256>("i8");
  run<2, 64>("i8TS");
  run<2, 128>("i8TS");
  run<3, 64>("f16TS");
  run<3, 128>("f16TS");
  run<2, 64, 2>("i8TS");
  run<2, 64, 3>("i8TS");
  run<1, 64, 2>("i8");
  run<1, 64, 3>("i8");
  run<0, 128, 2>("f16");
  run<4, 64, 1>("i8TSx8");
  run<4, 64, 2>("i8TSx8");
  run<4, 64, 3>("i8TSx8");
  run<5, 64, 1>("i8x8w");
  run<5, 64, 2>("i8x8w");
  run<5, 64, 3>("i8x8w");
  run<5, 128, 2>("i8x8w");
}
