// Clean issue-rate measurement of the epilogue's instructions on sm_100a.
// Each kernel runs 8 independent chains per thread; min/max alternate so ptxas cannot fuse
// two 2-input ops into one 3-input op (and 3-input kernels use explicit 3-input forms).
// Reports SASS instructions / clk / SM (warp-instructions x 32 = lane-ops).
#include <cstdint>
#include <cstdio>
#define IT 1024

__device__ __forceinline__ uint32_t vmin2(uint32_t a, uint32_t b) { uint32_t r; asm volatile("min.s16x2 %0, %1, %2;" : "=r"(r) : "r"(a), "r"(b)); return r; }
__device__ __forceinline__ uint32_t vmax2(uint32_t a, uint32_t b) { uint32_t r; asm volatile("max.s16x2 %0, %1, %2;" : "=r"(r) : "r"(a), "r"(b)); return r; }
__device__ __forceinline__ int smin(int a, int b) { int r; asm volatile("min.s32 %0, %1, %2;" : "=r"(r) : "r"(a), "r"(b)); return r; }
__device__ __forceinline__ int smax(int a, int b) { int r; asm volatile("max.s32 %0, %1, %2;" : "=r"(r) : "r"(a), "r"(b)); return r; }

template <int OP>
__global__ void __launch_bounds__(256) k(const uint32_t* __restrict__ in, uint32_t* out) {
  uint32_t a[8], b[8];
  const uint32_t* p = in + (blockIdx.x * blockDim.x + threadIdx.x) * 16;
#pragma unroll
  for (int i = 0; i < 8; ++i) { a[i] = p[i]; b[i] = p[8 + i]; }
  for (int it = 0; it < IT; ++it) {
#pragma unroll
    for (int i = 0; i < 8; ++i) {
      const uint32_t c = b[(i + 3) & 7];
      if (OP == 0) { a[i] = vmin2(a[i], b[i]); b[i] = vmax2(b[i], c); }                       // 2x VIMNMX.S16x2
      if (OP == 1) { a[i] = smin(a[i], b[i]); b[i] = smax(b[i], c); }                         // 2x VIMNMX (s32)
      if (OP == 2) { a[i] = vmin2(vmin2(a[i], b[i]), c); b[i] = vmax2(vmax2(b[i], a[i]), c); } // 2x VIMNMX3.S16x2
      if (OP == 3) { a[i] = smin(smin(a[i], b[i]), c); b[i] = smax(smax(b[i], a[i]), c); }     // 2x VIMNMX3 (s32)
      if (OP == 4) { asm volatile("prmt.b32 %0, %1, %2, 0x7632;" : "=r"(a[i]) : "r"(a[i]), "r"(b[i]));
                     asm volatile("prmt.b32 %0, %1, %2, 0x5410;" : "=r"(b[i]) : "r"(b[i]), "r"(c)); }  // 2x PRMT
      if (OP == 5) { a[i] = b[i] - 512u * a[i]; b[i] = c - 512u * b[i]; }                       // 2x IMAD imm
      if (OP == 6) { a[i] = vmin2(a[i], b[i]); b[i] = b[i] - 512u * c; }                        // VIMNMX.S16x2 + IMAD
      if (OP == 7) { a[i] = smin(a[i], b[i]); b[i] = b[i] - 512u * c; }                         // VIMNMX + IMAD
      if (OP == 8) { a[i] = a[i] ^ b[i]; b[i] = b[i] + c; }                                     // LOP3 + IADD3
      if (OP == 9) { asm volatile("min.f16x2 %0, %1, %2;" : "=r"(a[i]) : "r"(a[i]), "r"(b[i]));
                     asm volatile("max.f16x2 %0, %1, %2;" : "=r"(b[i]) : "r"(b[i]), "r"(c)); }          // 2x HMNMX2
      if (OP == 10) { asm volatile("min.f32 %0, %1, %2;" : "=r"(a[i]) : "r"(a[i]), "r"(b[i]));
                      asm volatile("max.f32 %0, %1, %2;" : "=r"(b[i]) : "r"(b[i]), "r"(c)); }           // 2x FMNMX
      if (OP == 11) { asm volatile("min.f16x2 %0, %1, %2;" : "=r"(a[i]) : "r"(a[i]), "r"(b[i]));
                      b[i] = vmax2(b[i], c); }                                                        // HMNMX2 + VIMNMX.S16x2
      if (OP == 12) { asm volatile("min.bf16x2 %0, %1, %2;" : "=r"(a[i]) : "r"(a[i]), "r"(b[i]));
                      asm volatile("max.bf16x2 %0, %1, %2;" : "=r"(b[i]) : "r"(b[i]), "r"(c)); }        // bf16x2
      if (OP == 14) { uint64_t wv = (uint64_t)a[i] * 65536ull + ((uint64_t)c << 16);               // IMAD.WIDE.U32
                      a[i] = (uint32_t)(wv >> 32) ^ b[i]; b[i] = (uint32_t)wv; }
      if (OP == 15) { long long wv; asm volatile("mad.wide.s32 %0, %1, %2, %3;" : "=l"(wv) : "r"(a[i]), "r"(-33554432), "l"(((long long)c) << 16));
                      a[i] = (uint32_t)(wv >> 32); b[i] = b[i] * 65536u + a[i]; }                     // IMAD.WIDE + IMAD(pack)
      if (OP == 16) { float f; asm volatile("cvt.rn.f32.s32 %0, %1;" : "=f"(f) : "r"(a[i])); a[i] = __float_as_uint(f) ^ b[i];
                      asm volatile("cvt.rn.f32.s32 %0, %1;" : "=f"(f) : "r"(b[i])); b[i] = __float_as_uint(f) + c; }   // I2FP
      if (OP == 17) { uint32_t h; asm volatile("cvt.rn.f16x2.f32 %0, %1, %2;" : "=r"(h) : "f"(__uint_as_float(a[i])), "f"(__uint_as_float(b[i]))); a[i] = h;
                      asm volatile("cvt.rn.f16x2.f32 %0, %1, %2;" : "=r"(h) : "f"(__uint_as_float(b[i])), "f"(__uint_as_float(c))); b[i] = h; } // F2FP pack
      if (OP == 18) { float x = __uint_as_float(a[i]), y = __uint_as_float(b[i]);
                      asm volatile("fma.rn.f32 %0, %1, %2, %3;" : "=f"(x) : "f"(x), "f"(-2.0f), "f"(y));
                      asm volatile("fma.rn.f32 %0, %1, %2, %3;" : "=f"(y) : "f"(y), "f"(-2.0f), "f"(__uint_as_float(c)));
                      a[i] = __float_as_uint(x); b[i] = __float_as_uint(y); }                              // FFMA
      if (OP == 19) { uint32_t h; asm volatile("fma.rn.f16x2 %0, %1, %2, %3;" : "=r"(h) : "r"(a[i]), "r"(b[i]), "r"(c)); a[i] = h;
                      asm volatile("fma.rn.f16x2 %0, %1, %2, %3;" : "=r"(h) : "r"(b[i]), "r"(c), "r"(a[i])); b[i] = h; } // HFMA2
      if (OP == 13) { asm volatile("min.f16x2 %0, %1, %2;" : "=r"(a[i]) : "r"(a[i]), "r"(b[i]));
                      b[i] = b[i] - 512u * c; }                                                       // HMNMX2 + IMAD
    }
  }
  uint32_t s = 0;
#pragma unroll
  for (int i = 0; i < 8; ++i) s ^= a[i] + b[i];
  out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}

template <int OP>
void run(const char* name, const uint32_t* in, uint32_t* out, int blocks, int thr, int clk) {
  k<OP><<<blocks, thr>>>(in, out);
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  cudaEventRecord(e0);
  k<OP><<<blocks, thr>>>(in, out);
  cudaEventRecord(e1);
  cudaEventSynchronize(e1);
  float ms;
  cudaEventElapsedTime(&ms, e0, e1);
  const double warp_inst = (double)blocks * (thr / 32) * IT * 8 * 2;  // 2 SASS instructions per chain step
  const double cyc = ms * 1e-3 * clk * 1e3;
  printf("%-26s thr/blk=%4d  %7.3f ms  warp-inst/clk/SM = %5.2f  (lane-ops %6.1f)\n", name, thr, ms,
         warp_inst / cyc / 148, 32 * warp_inst / cyc / 148);
}

int main() {
  int clk;
  cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);
  for (int thr : {256}) {
    int blocks = 148 * 8;
    uint32_t *in, *out;
    cudaMalloc(&in, (size_t)blocks * thr * 16 * 4);
    cudaMalloc(&out, (size_t)blocks * thr * 4);
    cudaMemset(in, 0x37, (size_t)blocks * thr * 16 * 4);
    run<0>("VIMNMX.S16x2", in, out, blocks, thr, clk);
    run<1>("VIMNMX.S32", in, out, blocks, thr, clk);
    run<2>("VIMNMX3.S16x2", in, out, blocks, thr, clk);
    run<3>("VIMNMX3.S32", in, out, blocks, thr, clk);
    run<4>("PRMT", in, out, blocks, thr, clk);
    run<5>("IMAD imm", in, out, blocks, thr, clk);
    run<6>("VIMNMX.S16x2 + IMAD", in, out, blocks, thr, clk);
    run<7>("VIMNMX + IMAD", in, out, blocks, thr, clk);
    run<8>("LOP3 + IADD3", in, out, blocks, thr, clk);
    run<9>("HMNMX2", in, out, blocks, thr, clk);
    run<10>("FMNMX", in, out, blocks, thr, clk);
    run<11>("HMNMX2 + VIMNMX.S16x2", in, out, blocks, thr, clk);
    run<12>("bf16x2 min/max", in, out, blocks, thr, clk);
    run<13>("HMNMX2 + IMAD", in, out, blocks, thr, clk);
    run<14>("IMAD.WIDE.U32 (+LOP)", in, out, blocks, thr, clk);
    run<15>("IMAD.WIDE + IMAD", in, out, blocks, thr, clk);
    run<16>("I2FP (+LOP/IADD)", in, out, blocks, thr, clk);
    run<17>("F2FP.PACK_AB", in, out, blocks, thr, clk);
    run<18>("FFMA", in, out, blocks, thr, clk);
    run<19>("HFMA2", in, out, blocks, thr, clk);
    cudaFree(in);
    cudaFree(out);
  }
  printf("clock %d kHz\n", clk);
}
