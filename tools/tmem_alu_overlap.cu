// Does a TMEM -> register load stream on one warp slow down ALU work of the other warps on the
// same SMSP?  (the search epilogue's TMEM reads and its two-partition scan overlap
// only partly.)  One CTA per SM, 16 warps (4 per SMSP, like the match kernel).  Per SMSP:
//   S scanner warps: repeatedly run the epilogue's 64-column two-partition max scan (VIMNMX3)
//     on register values perturbed through the FMA pipe (IMAD), so nothing is loop-invariant;
//   L loader warps: repeatedly tcgen05.ld.32x32b.x<W> their lane quarter + wait::ld.
// Prints the scanners' ALU rate (VIMNMX3 warp-instructions / clk / SM) and the loaders' TMEM
// bytes / clk / SM for L = 0..3 loaders next to S scanners.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/tmem_alu_overlap tools/tmem_alu_overlap.cu
#include <climits>
#include <cstdint>
#include <cstdio>

#define R4(i) "=r"(v[i]), "=r"(v[i + 1]), "=r"(v[i + 2]), "=r"(v[i + 3])
__device__ __forceinline__ void ld64(uint32_t taddr, uint32_t* v) {
  asm volatile(
      "tcgen05.ld.sync.aligned.32x32b.x64.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,%16,%17,%18,%19,"
      "%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31,%32,%33,%34,%35,%36,%37,%38,%39,%40,%41,%42,%43,%44,%45,%46,%47,"
      "%48,%49,%50,%51,%52,%53,%54,%55,%56,%57,%58,%59,%60,%61,%62,%63}, [%64];"
      : R4(0), R4(4), R4(8), R4(12), R4(16), R4(20), R4(24), R4(28), R4(32), R4(36), R4(40), R4(44), R4(48), R4(52),
        R4(56), R4(60)
      : "r"(taddr));
  asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
}
__device__ __forceinline__ int mx3(int a, int b, int c) { return __vimax3_s32(a, b, c); }
__device__ __forceinline__ int mx16(const int* k) {
  const int a = mx3(k[0], k[1], k[2]), b = mx3(k[3], k[4], k[5]), c = mx3(k[6], k[7], k[8]);
  const int d = mx3(k[9], k[10], k[11]), e = mx3(k[12], k[13], k[14]);
  return max(mx3(a, b, c), mx3(d, e, k[15]));
}
__device__ __forceinline__ void scan32(const int* k, int (&R)[16], int& T1, int& T2) {
  const int x = mx16(k), y = mx16(k + 16);
#pragma unroll
  for (int b = 0; b < 16; ++b) R[b] = mx3(R[b], k[b], k[b + 16]);
  const int hi = max(x, y), lo = min(x, y);
  T2 = mx3(T2, min(T1, hi), lo);
  T1 = max(T1, hi);
}

__global__ void __launch_bounds__(512, 1) k(int loaders, int scanners, int iters, unsigned long long* cyc, uint32_t* sink) {
  __shared__ uint32_t tptr;
  const int warp = threadIdx.x >> 5;
  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 512;" ::"r"(
        (uint32_t)__cvta_generic_to_shared(&tptr)));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;");
  const int slot = warp >> 2;  // 0..3: position of this warp on its SMSP (warp % 4 = SMSP)
  const uint32_t taddr = tptr + ((uint32_t)((warp & 3) * 32) << 16) + slot * 64;
  uint32_t acc = 0;
  unsigned long long t0 = clock64();
  if (slot < loaders) {
    uint32_t v[64];
    for (int it = 0; it < iters; ++it) {
      ld64(taddr + (it & 1) * 256, v);
      acc ^= v[0] ^ v[63];
    }
  } else if (slot < loaders + scanners) {
    int kk[32];
#pragma unroll
    for (int i = 0; i < 32; ++i) kk[i] = (threadIdx.x * 7919 + i * 104729) & 0xFFFFF;
    int R[16], T1 = INT_MIN, T2 = INT_MIN;
#pragma unroll
    for (int b = 0; b < 16; ++b) R[b] = INT_MIN;
    for (int it = 0; it < iters; ++it) {
#pragma unroll
      for (int i = 0; i < 32; ++i) kk[i] = kk[i] * 3 + it;  // IMAD (FMA pipe): fresh values each pass
      scan32(kk, R, T1, T2);
#pragma unroll
      for (int i = 0; i < 32; ++i) kk[i] = kk[i] * 5 + it;
      scan32(kk, R, T1, T2);
    }
#pragma unroll
    for (int b = 0; b < 16; ++b) acc += R[b];
    acc += T1 + T2;
  }
  unsigned long long t1 = clock64();
  sink[blockIdx.x * blockDim.x + threadIdx.x] = acc;
  if ((threadIdx.x & 31) == 0) cyc[blockIdx.x * 16 + warp] = t1 - t0;
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  if (warp == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 512;" ::"r"(tptr));
}

int main() {
  unsigned long long* cyc;
  uint32_t* sink;
  cudaMalloc(&cyc, 148 * 16 * 8);
  cudaMalloc(&sink, 148 * 512 * 4);
  const int iters = 20000;
  printf("per SMSP: L loader warps (tcgen05.ld 32x32b.x64 + wait) next to S scanner warps (64-column two-partition scan)\n");
  for (int S = 0; S <= 3; ++S)
    for (int L = 0; L + S <= 4; ++L) {
      if (S == 0 && L == 0) continue;
      k<<<148, 512>>>(L, S, 100, cyc, sink);
      k<<<148, 512>>>(L, S, iters, cyc, sink);
      cudaError_t e = cudaGetLastError();
      if (e == cudaSuccess) e = cudaDeviceSynchronize();
      unsigned long long c[16];
      cudaError_t e2 = cudaMemcpy(c, cyc, sizeof(c), cudaMemcpyDeviceToHost);  // CTA 0
      if (S == 1 && L == 1) printf("raw cycles w0..3: %llu %llu %llu %llu w4..7 %llu %llu (%s)\n", c[0], c[1], c[2], c[3], c[4], c[5], cudaGetErrorString(e2));
      double lc = 0, sc = 0;
      for (int w = 0; w < 16; ++w) {
        if ((w >> 2) < L) lc = lc > c[w] ? lc : c[w];
        else if ((w >> 2) < L + S) sc = sc > c[w] ? sc : c[w];
      }
      // scan: 2 x 35 ALU-pipe instructions per pass per warp; 4 SMSPs
      const double alu = S ? 4.0 * S * 70.0 * iters / sc : 0.0;
      const double tm = L ? 4.0 * L * 8192.0 * iters / lc : 0.0;
      printf("S=%d L=%d : scan %6.3f ALU warp-inst/clk/SM   TMEM %6.1f B/clk/SM   (%s)\n", S, L, alu, tm,
             cudaGetErrorString(e));
    }
  return 0;
}
