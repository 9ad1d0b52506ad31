// Probe: thread/register -> (TMEM lane, column) mapping of tcgen05.ld.16x64b.x4 and 16x32bx2.x4.
// Cell (lane l, column c) holds l * 1000 + c (written with 32x32b stores).
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
    uint32_t v[8];
    for (int c = 0; c < 8; ++c) v[c] = lane * 1000 + c;
    asm volatile("tcgen05.st.sync.aligned.32x32b.x8.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8};" ::"r"(t), "r"(v[0]), "r"(v[1]), "r"(v[2]), "r"(v[3]),
                 "r"(v[4]), "r"(v[5]), "r"(v[6]), "r"(v[7]) : "memory");
    asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory");
    uint32_t a[4], b[4];
    asm volatile("tcgen05.ld.sync.aligned.16x64b.x4.b32 {%0,%1,%2,%3}, [%4];"
                 : "=r"(a[0]), "=r"(a[1]), "=r"(a[2]), "=r"(a[3]) : "r"(t) : "memory");
    asm volatile("tcgen05.ld.sync.aligned.16x64b.x4.b32 {%0,%1,%2,%3}, [%4];"
                 : "=r"(b[0]), "=r"(b[1]), "=r"(b[2]), "=r"(b[3]) : "r"(t + (16u << 16)) : "memory");
    asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
    for (int i = 0; i < 4; ++i) { out[lane * 8 + i] = a[i]; out[lane * 8 + 4 + i] = b[i]; }
  }
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  if (warp == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 32;" ::"r"(t) : "memory");
}
int main() {
  uint32_t* d; cudaMalloc(&d, 32 * 8 * 4); cudaMemset(d, 0xff, 32 * 8 * 4);
  probe<<<1, 128>>>(d);
  cudaError_t e = cudaDeviceSynchronize();
  uint32_t h[32 * 8]; cudaMemcpy(h, d, sizeof h, cudaMemcpyDeviceToHost);
  printf("err=%s  (value = lane*1000 + column)\n", cudaGetErrorString(e));
  for (int l = 0; l < 32; ++l) {
    printf("thr %2d  16x64b@0:", l); for (int i = 0; i < 4; ++i) printf(" %5u", h[l * 8 + i]);
    printf("   @lane16:"); for (int i = 0; i < 4; ++i) printf(" %5u", h[l * 8 + 4 + i]);
    printf("\n");
  }
}
