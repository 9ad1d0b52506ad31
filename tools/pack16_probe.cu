// Probe: which 16 bits does tcgen05.ld ... .pack::16b take from 32-bit TMEM cells?
// Writes known 32-bit values with tcgen05.st (32x32b), reads back with 16x64b.x1 (plain) and
// 16x64b.x1.pack::16b, prints lane 0's registers.
#include <cstdint>
#include <cstdio>
__global__ void probe(uint32_t* out) {
  __shared__ uint32_t tptr;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 32;" ::"r"((uint32_t)__cvta_generic_to_shared(&tptr)) : "memory");
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
  }
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
  const uint32_t t = tptr;
  if (warp == 0) {
    // lane l, column c holds 0xAAAA0000 | (l << 8) | c  with high half 0x1000 + 16*l + c
    uint32_t v[8];
    for (int c = 0; c < 8; ++c) v[c] = ((0x1000u + 16u * lane + c) << 16) | (lane << 8) | c;
    asm volatile("tcgen05.st.sync.aligned.32x32b.x8.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8};" ::"r"(t), "r"(v[0]), "r"(v[1]), "r"(v[2]), "r"(v[3]),
                 "r"(v[4]), "r"(v[5]), "r"(v[6]), "r"(v[7]) : "memory");
    asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory");
    uint32_t a[8], b[4];
    asm volatile("tcgen05.ld.sync.aligned.32x32b.x8.b32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
                 : "=r"(a[0]), "=r"(a[1]), "=r"(a[2]), "=r"(a[3]), "=r"(a[4]), "=r"(a[5]), "=r"(a[6]), "=r"(a[7]) : "r"(t) : "memory");
    asm volatile("tcgen05.ld.sync.aligned.32x32b.x4.pack::16b.b32 {%0,%1,%2,%3}, [%4];"
                 : "=r"(b[0]), "=r"(b[1]), "=r"(b[2]), "=r"(b[3]) : "r"(t) : "memory");
    asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
    for (int i = 0; i < 8; ++i) out[lane * 16 + i] = a[i];
    for (int i = 0; i < 4; ++i) out[lane * 16 + 8 + i] = b[i];
  }
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  if (warp == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 32;" ::"r"(t) : "memory");
}
int main() {
  uint32_t* d; cudaMalloc(&d, 32 * 16 * 4); cudaMemset(d, 0, 32 * 16 * 4);
  probe<<<1, 128>>>(d);
  cudaError_t e = cudaDeviceSynchronize();
  uint32_t h[32 * 16]; cudaMemcpy(h, d, sizeof h, cudaMemcpyDeviceToHost);
  printf("err=%s\n", cudaGetErrorString(e));
  for (int l : {0, 1, 5}) {
    printf("lane %d plain:", l); for (int i = 0; i < 8; ++i) printf(" %08x", h[l * 16 + i]);
    printf("\nlane %d pack16:", l); for (int i = 0; i < 4; ++i) printf(" %08x", h[l * 16 + 8 + i]);
    printf("\n");
  }
}
