// Micro-benchmark: issue/pipe rate of FFMA vs packed FFMA2 (fma.rn.f32x2) on sm_100a,
// mixed with integer LOP3 work, to decide whether pairing particles pays.
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>
__device__ __forceinline__ unsigned long long f2fma(unsigned long long a, unsigned long long b, unsigned long long c){
  unsigned long long d; asm volatile("fma.rn.f32x2 %0, %1, %2, %3;" : "=l"(d) : "l"(a), "l"(b), "l"(c)); return d; }
template<int MODE>
__global__ void k(float* out, int iters, float s){
  float a[8]; unsigned long long p[4]; uint32_t x[8];
  for(int i=0;i<8;++i){ a[i]=threadIdx.x*0.001f+i; x[i]=threadIdx.x*7+i; }
  for(int i=0;i<4;++i){ p[i]=(unsigned long long)__float_as_uint(a[2*i]) | ((unsigned long long)__float_as_uint(a[2*i+1])<<32); }
  unsigned long long ss = (unsigned long long)__float_as_uint(s) | ((unsigned long long)__float_as_uint(s)<<32);
  for(int it=0; it<iters; ++it){
    #pragma unroll
    for(int r=0;r<16;++r){
      if (MODE==0){  // 8 scalar FFMA
        #pragma unroll
        for(int i=0;i<8;++i) a[i]=__fmaf_rn(a[i], s, 0.5f*i+0.25f);
      } else if (MODE==1){ // 4 FFMA2 (= 8 fp32 fmas)
        #pragma unroll
        for(int i=0;i<4;++i) p[i]=f2fma(p[i], ss, p[i]);
      } else if (MODE==2){ // 8 FFMA + 8 LOP3
        #pragma unroll
        for(int i=0;i<8;++i){ a[i]=__fmaf_rn(a[i], s, a[(i+1)&7]); x[i]=x[i]^x[(i+1)&7]^(x[(i+3)&7]>>1); }
      } else { // 4 FFMA2 + 8 LOP3
        #pragma unroll
        for(int i=0;i<4;++i) p[i]=f2fma(p[i], ss, p[(i+1)&3]);
        #pragma unroll
        for(int i=0;i<8;++i) x[i]=x[i]^x[(i+1)&7]^(x[(i+3)&7]>>1);
      }
    }
  }
  float acc=0; for(int i=0;i<8;++i) acc+=a[i]+x[i]; for(int i=0;i<4;++i) acc+=__uint_as_float((uint32_t)p[i]);
  out[blockIdx.x*blockDim.x+threadIdx.x]=acc;
}
int main(){
  float* out; cudaMalloc(&out, 148*8*256*4*4);
  int iters=4096; cudaEvent_t e0,e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  const char* names[4]={"8 FFMA","4 FFMA2","8 FFMA+8 LOP3","4 FFMA2+8 LOP3"};
  for(int mode=0;mode<4;++mode){
    for(int rep=0;rep<2;++rep){
      cudaEventRecord(e0);
      if(mode==0) k<0><<<148*8,256>>>(out,iters,0.999f);
      if(mode==1) k<1><<<148*8,256>>>(out,iters,0.999f);
      if(mode==2) k<2><<<148*8,256>>>(out,iters,0.999f);
      if(mode==3) k<3><<<148*8,256>>>(out,iters,0.999f);
      cudaEventRecord(e1); cudaEventSynchronize(e1);
      float ms; cudaEventElapsedTime(&ms,e0,e1);
      double warp_iters = 148.0*8*8*iters*16;  // warps * iterations of the r-loop
      if(rep==1) printf("%-16s %.3f ms  -> %.3f SMSP-cycles per r-iteration per warp (at 1.965GHz)\n", names[mode], ms,
        ms*1e-3*1.965e9*148*4/warp_iters);
    }
  }
  return 0;
}
