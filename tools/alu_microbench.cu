#include <cstdio>
#include <cstdint>
#define N_ITERS 4096
// 8 independent chains per thread to avoid latency-bound
template<int OP>
__global__ void k(uint32_t* out, uint32_t seed, long long* cyc) {
  uint32_t a[8], b[8], c[8];
  #pragma unroll
  for (int i=0;i<8;i++){a[i]=seed*(threadIdx.x+i); b[i]=a[i]^0x12345; c[i]=a[i]+77;}
  long long t0 = clock64();
  for (int it=0; it<N_ITERS; it++) {
    #pragma unroll
    for (int i=0;i<8;i++){
      if (OP==0) { a[i] = min((int)a[i], (int)b[i]); b[i] = max((int)b[i],(int)c[i]); }             // 2 s32 minmax
      if (OP==1) { a[i] = __vminu2(a[i], b[i]); b[i] = __vmaxu2(b[i], c[i]); }                       // 2 u16x2
      if (OP==2) { a[i] = min(min((int)a[i],(int)b[i]),(int)c[i]); b[i]=min(min((int)b[i],(int)c[i]),(int)a[i]);} // 2 min3
      if (OP==3) { a[i] = a[i]*0xfffffe00u + b[i]; b[i] = b[i]*0xfffffe00u + c[i]; }                // 2 IMAD
      if (OP==4) { a[i] = __byte_perm(a[i], b[i], 0x6521); b[i] = __byte_perm(b[i], c[i], 0x6521);}  // 2 PRMT
      if (OP==5) { a[i] = a[i]*0xfffffe00u + b[i]; b[i] = min((int)b[i],(int)c[i]); }               // IMAD + IMNMX
      if (OP==6) { a[i] = __vminu2(__vminu2(a[i], b[i]),c[i]); b[i] = __vminu2(__vminu2(b[i], c[i]),a[i]); }  // u16x2 min3
      if (OP==7) { a[i] = a[i]+b[i]; b[i] = b[i]^c[i]; }  // IADD3 + LOP3
    }
  }
  long long t1 = clock64();
  uint32_t s=0;
  #pragma unroll
  for (int i=0;i<8;i++) s ^= a[i]^b[i];
  out[blockIdx.x*blockDim.x+threadIdx.x]=s;
  if (threadIdx.x==0) cyc[blockIdx.x]=t1-t0;
}
int main(){
  uint32_t* out; long long* cyc; cudaMalloc(&out, 148*1024*4*4); cudaMalloc(&cyc, 148*8*4);
  const char* names[]={"s32 min/max","u16x2 vmin/vmax","s32 min3","IMAD","PRMT","IMAD+IMNMX","u16x2 min3","IADD+LOP"};
  for (int op=0; op<8; op++) for (int thr : {128, 256, 512, 1024}) {
    void (*f)(uint32_t*,uint32_t,long long*);
    switch(op){case 0:f=k<0>;break;case 1:f=k<1>;break;case 2:f=k<2>;break;case 3:f=k<3>;break;case 4:f=k<4>;break;case 5:f=k<5>;break;case 6:f=k<6>;break;default:f=k<7>;}
    f<<<148,thr>>>(out,1,cyc); cudaDeviceSynchronize();
    cudaEvent_t e0,e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
    cudaEventRecord(e0); f<<<148,thr>>>(out,1,cyc); cudaEventRecord(e1); cudaEventSynchronize(e1);
    float ms; cudaEventElapsedTime(&ms,e0,e1);
    long long hc[148]; cudaMemcpy(hc,cyc,148*8,cudaMemcpyDeviceToHost);
    double ops = 148.0*thr*N_ITERS*8*2; // "source ops" (min3 counted as 1)
    printf("%-18s thr=%4d  %.3f ms  lane-ops/clk/SM(by cyc)=%.1f  Gops/s=%.0f\n", names[op], thr, ms, (double)thr*N_ITERS*16/hc[0], ops/ms/1e6);
  }
  int clk; cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0); printf("clock kHz %d\n", clk);
}
