// Epilogue scan in isolation: real TMEM loads (32x32b.x32) + the coarse top-2 code of
// tid_kernels.cu, W warps per SMSP.  Variants add concurrent tensor-core work:
//   v0: scanners only
//   v1: + one extra warp issuing back-to-back M=128 N=128 K=128 i8 MMA pieces from SMEM into
//       TMEM columns 256..511 (untouched by the scanners)
//   v2: + four MMA warps (one per SMSP) sharing the same MMA stream
// Reports cycles per 32-column chunk per SMSP (ALU bound = 2 x ALU instructions per chunk).
#include <climits>
#include <cstdint>
#include <cstdio>

#include "../paper_conf_icpp_wangzll21_b200/csrc/tid_kernels.cu"

using namespace tid;

template <int VARIANT, int X128>
__global__ void scan_k(int iters, uint32_t* out, long long* cyc) {
  extern __shared__ uint8_t sm[];
  __shared__ uint32_t tptr;
  __shared__ __align__(8) uint64_t bars[4];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  int32_t* keys = reinterpret_cast<int32_t*>(sm);
  for (int i = threadIdx.x; i < 512; i += blockDim.x) keys[i] = (i * 7919) * 256 + (i & 255);
  const int nmma = VARIANT == 0 ? 0 : (VARIANT == 1 ? 1 : 4);
  const int nscan = blockDim.x / 32 - nmma;
  if (threadIdx.x < 4) mbar_init((uint32_t)__cvta_generic_to_shared(&bars[threadIdx.x]), 1);
  fence_barrier_init();
  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 512;" ::"r"(
        (uint32_t)__cvta_generic_to_shared(&tptr)));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  uint32_t acc = 0;
  if (warp >= nscan) {
    const uint32_t base = ((uint32_t)__cvta_generic_to_shared(sm) + 4096 + 1023) & ~1023u;
    const uint64_t ad = smem_desc_sw128(base), bd = smem_desc_sw128(base + 16384);
    const int mw = warp - nscan;
    const uint32_t bar = (uint32_t)__cvta_generic_to_shared(&bars[mw]);
    const int n_pieces = iters * 8 / nmma;  // ~ the pieces a real kernel issues per scanned chunk set
    for (int it = 0; it < n_pieces; ++it) {
      mma_piece(tptr + 256 + (mw & 1) * 128, ad, bd, bar);
      mbar_wait(bar, it & 1);
    }
  } else {
    const uint32_t taddr = tptr + ((uint32_t)((warp & 3) * 32) << 16) + ((warp >> 2) & 1) * 128;
    const uint32_t ck = (uint32_t)__cvta_generic_to_shared(keys);
    long long t0 = clock64();
    for (int it = 0; it < iters; ++it) {
      uint32_t A1 = 0x7FFF7FFFu, A2 = 0x7FFF7FFFu, B1 = 0x7FFF7FFFu, B2 = 0x7FFF7FFFu;
      if (X128) scan_coarse_x128(taddr, ck + (it & 1) * 512, A1, A2, B1, B2);
      else scan_coarse(taddr, ck + (it & 1) * 512, A1, A2, B1, B2);
      acc ^= A1 ^ A2 ^ B1 ^ B2;
    }
    long long t1 = clock64();
    if (threadIdx.x == 0) cyc[blockIdx.x] = t1 - t0;
  }
  out[blockIdx.x * blockDim.x + threadIdx.x] = acc;
  tc_fence_before();
  __syncthreads();
  if (warp == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 512;" ::"r"(tptr));
}

int main() {
  uint32_t* out;
  long long* cyc;
  cudaMalloc(&out, 148 * 1024 * 4);
  cudaMalloc(&cyc, 148 * 8);
  const int iters = 4000;
  for (int x = 0; x < 2; ++x)
  for (int v = 0; v < 3; ++v) {
    for (int w : {2, 4}) {
      const int threads = 128 * w + 32 * (v == 0 ? 0 : (v == 1 ? 1 : 4));
      void (*kern)(int, uint32_t*, long long*) =
          x == 0 ? (v == 0 ? scan_k<0, 0> : (v == 1 ? scan_k<1, 0> : scan_k<2, 0>))
                 : (v == 0 ? scan_k<0, 1> : (v == 1 ? scan_k<1, 1> : scan_k<2, 1>));
      cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, 40960);
      kern<<<148, threads, 40960>>>(10, out, cyc);
      cudaDeviceSynchronize();
      kern<<<148, threads, 40960>>>(iters, out, cyc);
      cudaError_t e = cudaDeviceSynchronize();
      long long c[148];
      cudaMemcpy(c, cyc, sizeof(c), cudaMemcpyDeviceToHost);
      const double chunks = (double)iters * 4 * w;
      printf("x128=%d variant=%d warps/SMSP=%d  cycles per 32-col chunk per SMSP = %6.1f   (%s)\n", x, v, w, c[0] / chunks,
             cudaGetErrorString(e));
    }
  }
}
