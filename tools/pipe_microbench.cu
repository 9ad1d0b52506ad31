// Per-pipe throughput on sm_100a for the epilogue's candidate instructions.
// Each thread runs 8 independent dependency chains over values loaded from global memory,
// so nothing constant-folds; results are stored.  Reports lane-ops / clk / SM.
#include <cstdint>
#include <cstdio>
#define IT 2048
template <int OP>
__global__ void __launch_bounds__(512) k(const uint32_t* __restrict__ in, uint32_t* out) {
  uint32_t a[8], b[8];
  const uint32_t* p = in + (blockIdx.x * blockDim.x + threadIdx.x) * 16;
#pragma unroll
  for (int i = 0; i < 8; ++i) { a[i] = p[i]; b[i] = p[8 + i]; }
  for (int it = 0; it < IT; ++it) {
#pragma unroll
    for (int i = 0; i < 8; ++i) {
      uint32_t x = a[i], y = b[i], z = b[(i + 1) & 7];
      if (OP == 0) asm volatile("mad.lo.u32 %0, %1, %2, %3;" : "=r"(x) : "r"(x), "r"(y), "r"(z));
      if (OP == 1) asm volatile("mad.hi.u32 %0, %1, %2, %3;" : "=r"(x) : "r"(x), "r"(y), "r"(z));
      if (OP == 2) asm volatile("prmt.b32 %0, %1, %2, 0x6521;" : "=r"(x) : "r"(x), "r"(y));
      if (OP == 3) asm volatile("min.u16x2 %0, %1, %2;" : "=r"(x) : "r"(x), "r"(y));
      if (OP == 4) asm volatile("min.s32 %0, %1, %2;" : "=r"(x) : "r"(x), "r"(y));
      if (OP == 5) {
        asm volatile("mad.hi.u32 %0, %1, %2, %3;" : "=r"(x) : "r"(x), "r"(y), "r"(z));
        asm volatile("min.u16x2 %0, %1, %2;" : "=r"(y) : "r"(y), "r"(z));
      }
      if (OP == 6) {
        asm volatile("mad.lo.u32 %0, %1, %2, %3;" : "=r"(x) : "r"(x), "r"(y), "r"(z));
        asm volatile("prmt.b32 %0, %1, %2, 0x6521;" : "=r"(y) : "r"(y), "r"(z));
      }
      if (OP == 7) asm volatile("max.f16x2 %0, %1, %2;" : "=r"(x) : "r"(x), "r"(y));
      if (OP == 8) {
        asm volatile("mad.lo.u32 %0, %1, %2, %3;" : "=r"(x) : "r"(x), "r"(y), "r"(z));
        asm volatile("mad.lo.u32 %0, %1, %2, %3;" : "=r"(y) : "r"(y), "r"(z), "r"(x));
      }
      if (OP == 9) asm volatile("mad.lo.u32 %0, %1, 65536, %2;" : "=r"(x) : "r"(x), "r"(y));
      if (OP == 10) {
        asm volatile("min.u16x2 %0, %1, %2;" : "=r"(x) : "r"(x), "r"(y));
        asm volatile("max.f16x2 %0, %1, %2;" : "=r"(y) : "r"(y), "r"(z));
      }
      if (OP == 11) {
        asm volatile("mad.hi.u32 %0, %1, %2, %3;" : "=r"(x) : "r"(x), "r"(y), "r"(z));
        asm volatile("mad.hi.u32 %0, %1, %2, %3;" : "=r"(y) : "r"(y), "r"(z), "r"(x));
        asm volatile("min.u16x2 %0, %1, %2;" : "=r"(z) : "r"(z), "r"(x));
      }
      a[i] = x; b[i] = y;
      if (OP == 11) b[(i + 1) & 7] = z;
    }
  }
  uint32_t s = 0;
#pragma unroll
  for (int i = 0; i < 8; ++i) s ^= a[i] + b[i];
  out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}
template <int OP>
float run(const uint32_t* in, uint32_t* out, int blocks, int thr) {
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
  return ms;
}
int main() {
  int blocks = 148 * 4, thr = 512;
  uint32_t *in, *out;
  cudaMalloc(&in, (size_t)blocks * thr * 16 * 4);
  cudaMalloc(&out, (size_t)blocks * thr * 4);
  cudaMemset(in, 0x37, (size_t)blocks * thr * 16 * 4);
  int clk;
  cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);
  const char* nm[] = {"IMAD", "IMAD.HI", "PRMT", "VIMNMX.U16x2", "VIMNMX.S32", "IMAD.HI+VIMNMX.U16x2",
                      "IMAD+PRMT", "HMNMX2", "IMAD x2 chains", "IMAD imm", "VIMNMX.U16x2+HMNMX2",
                      "2 IMAD.HI + 1 VIMNMX.U16x2"};
  int per[] = {1, 1, 1, 1, 1, 2, 2, 1, 2, 1, 2, 3};
  float ms[12];
  ms[0] = run<0>(in, out, blocks, thr); ms[1] = run<1>(in, out, blocks, thr);
  ms[2] = run<2>(in, out, blocks, thr); ms[3] = run<3>(in, out, blocks, thr);
  ms[4] = run<4>(in, out, blocks, thr); ms[5] = run<5>(in, out, blocks, thr);
  ms[6] = run<6>(in, out, blocks, thr); ms[7] = run<7>(in, out, blocks, thr);
  ms[8] = run<8>(in, out, blocks, thr); ms[9] = run<9>(in, out, blocks, thr);
  ms[10] = run<10>(in, out, blocks, thr); ms[11] = run<11>(in, out, blocks, thr);
  for (int o = 0; o < 12; ++o) {
    double ops = (double)blocks * thr * IT * 8 * per[o];
    double cyc = ms[o] * 1e-3 * clk * 1e3;
    printf("%-28s %8.3f ms  lane-ops/clk/SM = %6.1f\n", nm[o], ms[o], ops / cyc / 148);
  }
  printf("clock %d kHz\n", clk);
}
