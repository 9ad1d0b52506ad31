// TMEM -> register load throughput on sm_100a (tcgen05.ld), bytes / clk / SM.
// One CTA per SM allocates all 512 TMEM columns; W warps (W/4 per lane quarter) each load
// their lane quarter repeatedly with a given shape/width, waiting after each load (as an
// epilogue must before using the registers) or after every 2 loads.
#include <cstdint>
#include <cstdio>

__device__ __forceinline__ void fence_view() { asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory"); }

template <int NREG>
__device__ __forceinline__ void ld32x32b(uint32_t taddr, uint32_t* v);

#define R4(i) "=r"(v[i]), "=r"(v[i + 1]), "=r"(v[i + 2]), "=r"(v[i + 3])
template <>
__device__ __forceinline__ void ld32x32b<16>(uint32_t taddr, uint32_t* v) {
  asm volatile("tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%16];"
               : R4(0), R4(4), R4(8), R4(12) : "r"(taddr));
}
template <>
__device__ __forceinline__ void ld32x32b<32>(uint32_t taddr, uint32_t* v) {
  asm volatile(
      "tcgen05.ld.sync.aligned.32x32b.x32.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,%16,%17,%18,%19,"
      "%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31}, [%32];"
      : R4(0), R4(4), R4(8), R4(12), R4(16), R4(20), R4(24), R4(28) : "r"(taddr));
}
template <>
__device__ __forceinline__ void ld32x32b<64>(uint32_t taddr, uint32_t* v) {
  asm volatile(
      "tcgen05.ld.sync.aligned.32x32b.x64.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,%16,%17,%18,%19,"
      "%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31,%32,%33,%34,%35,%36,%37,%38,%39,%40,%41,%42,%43,%44,%45,%46,%47,"
      "%48,%49,%50,%51,%52,%53,%54,%55,%56,%57,%58,%59,%60,%61,%62,%63}, [%64];"
      : R4(0), R4(4), R4(8), R4(12), R4(16), R4(20), R4(24), R4(28), R4(32), R4(36), R4(40), R4(44), R4(48), R4(52),
        R4(56), R4(60)
      : "r"(taddr));
}


#define OUT64 R4(0), R4(4), R4(8), R4(12), R4(16), R4(20), R4(24), R4(28), R4(32), R4(36), R4(40), R4(44), R4(48), R4(52), R4(56), R4(60)
#define REGS64 "{%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,%16,%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31,%32,%33,%34,%35,%36,%37,%38,%39,%40,%41,%42,%43,%44,%45,%46,%47,%48,%49,%50,%51,%52,%53,%54,%55,%56,%57,%58,%59,%60,%61,%62,%63}"
template <int SHAPE>
__device__ __forceinline__ void ld_shape64(uint32_t taddr, uint32_t* v) {
  if (SHAPE == 1) asm volatile("tcgen05.ld.sync.aligned.16x256b.x16.b32 " REGS64 ", [%64];" : OUT64 : "r"(taddr));
  if (SHAPE == 2) asm volatile("tcgen05.ld.sync.aligned.16x128b.x32.b32 " REGS64 ", [%64];" : OUT64 : "r"(taddr));
  if (SHAPE == 3) asm volatile("tcgen05.ld.sync.aligned.16x64b.x64.b32 " REGS64 ", [%64];" : OUT64 : "r"(taddr));
}
// 16-lane shapes: a warp covers its 32 lanes with two loads (lane offset 0 and 16).
template <int SHAPE>
__global__ void k16(uint32_t* out, int iters, long long* cyc) {
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
  const uint32_t base = tptr + ((uint32_t)((warp & 3) * 32) << 16);
  const int cols_per_warp = 512 / (blockDim.x / 128);
  const uint32_t wbase = base + (warp >> 2) * cols_per_warp;
  // columns covered per load: 16x256b.x16 -> 128 cols (8 cols/rep); 16x128b.x32 -> 128; 16x64b.x64 -> 128
  uint32_t acc = 0;
  uint32_t v[64];
  long long t0 = clock64();
  for (int it = 0; it < iters; ++it) {
    for (int c = 0; c < cols_per_warp; c += 128) {
      for (int h = 0; h < 2; ++h) {
        ld_shape64<SHAPE>(wbase + c + ((uint32_t)(16 * h) << 16), v);
        fence_view();
#pragma unroll
        for (int i = 0; i < 64; ++i) acc ^= v[i];
      }
    }
  }
  long long t1 = clock64();
  out[blockIdx.x * blockDim.x + threadIdx.x] = acc;
  if (threadIdx.x == 0) cyc[blockIdx.x] = t1 - t0;
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  if (warp == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 512;" ::"r"(tptr));
}
template <int SHAPE>
void run16(int warps) {
  uint32_t* out; long long* cyc;
  cudaMalloc(&out, 148 * 1024 * 4); cudaMalloc(&cyc, 148 * 8);
  const int iters = 2000;
  k16<SHAPE><<<148, warps * 32>>>(out, 10, cyc);
  cudaDeviceSynchronize();
  k16<SHAPE><<<148, warps * 32>>>(out, iters, cyc);
  cudaError_t e = cudaDeviceSynchronize();
  long long c[148];
  cudaMemcpy(c, cyc, sizeof(c), cudaMemcpyDeviceToHost);
  double bytes = (double)iters * 128 * 512 * 4;
  const char* nm[] = {"", "16x256b.x16", "16x128b.x32", "16x64b.x64"};
  printf("%-12s warps=%2d : %7.1f B/clk/SM  (%s)\n", nm[SHAPE], warps, bytes / c[0], cudaGetErrorString(e));
  cudaFree(out); cudaFree(cyc);
}

template <int NREG, int PAIR>
__global__ void k(uint32_t* out, int iters, long long* cyc) {
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
  const uint32_t base = tptr + ((uint32_t)((warp & 3) * 32) << 16);
  const int cols_per_warp = 512 / (blockDim.x / 128);
  const uint32_t wbase = base + (warp >> 2) * cols_per_warp;
  uint32_t acc = 0;
  uint32_t v[NREG];
  long long t0 = clock64();
  for (int it = 0; it < iters; ++it) {
    for (int c = 0; c < cols_per_warp; c += NREG * PAIR) {
      ld32x32b<NREG>(wbase + c, v);
      if (PAIR == 2) {
        uint32_t w[NREG];
        ld32x32b<NREG>(wbase + c + NREG, w);
        fence_view();
#pragma unroll
        for (int i = 0; i < NREG; ++i) acc += w[i];
      } else {
        fence_view();
      }
#pragma unroll
      for (int i = 0; i < NREG; ++i) acc ^= v[i];
    }
  }
  long long t1 = clock64();
  out[blockIdx.x * blockDim.x + threadIdx.x] = acc;
  if (threadIdx.x == 0) cyc[blockIdx.x] = t1 - t0;
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  if (warp == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 512;" ::"r"(tptr));
}

template <int NREG, int PAIR>
void run(int warps) {
  uint32_t* out;
  long long* cyc;
  cudaMalloc(&out, 148 * 1024 * 4);
  cudaMalloc(&cyc, 148 * 8);
  const int iters = 2000;
  k<NREG, PAIR><<<148, warps * 32>>>(out, 10, cyc);
  cudaDeviceSynchronize();
  k<NREG, PAIR><<<148, warps * 32>>>(out, iters, cyc);
  cudaError_t e = cudaDeviceSynchronize();
  long long c[148];
  cudaMemcpy(c, cyc, sizeof(c), cudaMemcpyDeviceToHost);
  double bytes = (double)iters * 128 * 512 * 4;  // whole TMEM per iteration per SM
  printf("x%-3d pair=%d warps=%2d : %7.1f B/clk/SM  (%s)\n", NREG, PAIR, warps, bytes / c[0], cudaGetErrorString(e));
  cudaFree(out);
  cudaFree(cyc);
}

int main() {
  for (int w : {4, 8, 16}) {
    run<16, 1>(w);
    run<32, 1>(w);
    run<64, 1>(w);
    run<32, 2>(w);
    run16<1>(w);
    run16<2>(w);
    run16<3>(w);
  }
}
