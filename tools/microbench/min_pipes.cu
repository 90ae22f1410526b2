// which pipe do candidate min instructions run on? alone and paired 1:1 with VABSDIFF4
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>
#include <cuda_fp16.h>
__device__ __forceinline__ uint32_t vad4(uint32_t a, uint32_t b, uint32_t c){
  uint32_t d; asm volatile("vabsdiff4.u32.u32.u32.add %0,%1,%2,%3;" : "=r"(d) : "r"(a),"r"(b),"r"(c)); return d; }
constexpr int NACC=16, ITERS=4096;
template<int MODE, bool PAIR>
__global__ void __launch_bounds__(1024) kern(uint32_t seed, uint32_t* out, unsigned long long* cyc){
  uint32_t a[NACC], b[NACC];
#pragma unroll
  for(int i=0;i<NACC;i++){ a[i]=seed*(i+1)+threadIdx.x; b[i]=seed^(i*0x9e3779b9u); }
  uint32_t x = seed + threadIdx.x*3u, y = seed*7u + threadIdx.x;
  __syncthreads();
  unsigned long long t0 = clock64();
  for(int it=0; it<ITERS; ++it){
#pragma unroll
    for(int i=0;i<NACC;i++){
      uint32_t d;
      if (PAIR) a[i]=vad4(x,y,a[i]);
      if (MODE==0) { float f; asm volatile("min.f32 %0,%1,%2;" : "=f"(f):"f"(__uint_as_float(b[i])),"f"(__uint_as_float(x))); d=__float_as_uint(f);}
      if (MODE==1) { float f; asm volatile("min.f32 %0,%1,%2,%3;" : "=f"(f):"f"(__uint_as_float(b[i])),"f"(__uint_as_float(x)),"f"(__uint_as_float(y))); d=__float_as_uint(f);}
      if (MODE==2) asm volatile("min.f16x2 %0,%1,%2;" : "=r"(d):"r"(b[i]),"r"(x));
      if (MODE==3) asm volatile("min.u16x2 %0,%1,%2;" : "=r"(d):"r"(b[i]),"r"(x));
      if (MODE==4) asm volatile("{.reg .b32 t; min.u16x2 t,%1,%2; min.u16x2 %0,t,%3;}" : "=r"(d):"r"(b[i]),"r"(x),"r"(y));
      if (MODE==5) asm volatile("min.u32 %0,%1,%2;" : "=r"(d):"r"(b[i]),"r"(x));
      if (MODE==6) asm volatile("min.s32 %0,%1,%2;" : "=r"(d):"r"(b[i]),"r"(x));
      if (MODE==7) asm volatile("add.u32 %0,%1,%2;" : "=r"(d):"r"(b[i]),"r"(x));
      if (MODE==8) asm volatile("lop3.b32 %0,%1,%2,%3,0x96;" : "=r"(d):"r"(b[i]),"r"(x),"r"(y));
      if (MODE==9) asm volatile("prmt.b32 %0,%1,%2,0x5410;" : "=r"(d):"r"(b[i]),"r"(x));
      if (MODE==10) asm volatile("shf.l.wrap.b32 %0,%1,%2,%3;" : "=r"(d):"r"(b[i]),"r"(x),"r"(y));
      if (MODE==11) asm volatile("sad.u32 %0,%1,%2,%3;" : "=r"(d):"r"(b[i]),"r"(x),"r"(y));
      if (MODE==13) { float f; asm volatile("max.f32 %0,%1,%2;" : "=f"(f):"f"(__uint_as_float(b[i])),"f"(__uint_as_float(x))); d=__float_as_uint(f);}
      if (MODE==14) { float f; asm volatile("{.reg .f32 t; min.f32 t,%1,%2; min.f32 %0,t,%3;}" : "=f"(f):"f"(__uint_as_float(b[i])),"f"(__uint_as_float(x)),"f"(__uint_as_float(y))); d=__float_as_uint(f);}
      if (MODE==15) asm volatile("vabsdiff2.u32.u32.u32.add %0,%1,%2,%3;" : "=r"(d):"r"(b[i]),"r"(x),"r"(y));
      b[i]=d;
    }
  }
  unsigned long long t1 = clock64();
  uint32_t s=0;
#pragma unroll
  for(int i=0;i<NACC;i++) s+=a[i]^b[i];
  out[blockIdx.x*blockDim.x+threadIdx.x]=s;
  if(threadIdx.x==0) cyc[blockIdx.x]=t1-t0;
}
template<int M, bool P> void run(const char* name, int nsm){
  uint32_t* out; unsigned long long* cyc; const int thr=1024;
  cudaMalloc(&out, 4*nsm*thr); cudaMalloc(&cyc, 8*nsm);
  kern<M,P><<<nsm,thr>>>(1,out,cyc); cudaDeviceSynchronize();
  kern<M,P><<<nsm,thr>>>(2,out,cyc); cudaDeviceSynchronize();
  unsigned long long* h=new unsigned long long[nsm]; cudaMemcpy(h,cyc,8*nsm,cudaMemcpyDeviceToHost);
  double sum=0; for(int i=0;i<nsm;i++) sum+=h[i];
  double per_clk = (double)NACC*ITERS*thr/(sum/nsm);
  printf("%-28s %s: %.1f ops/clk/SM (x%d instr)\n", name, P?"paired":"alone ", per_clk, P?2:1);
  cudaFree(out); cudaFree(cyc);
}
#define R(M,n) run<M,false>(n,nsm); run<M,true>(n,nsm);
int main(){ int nsm; cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, 0);
  R(0,"min.f32") R(1,"min.f32 3-input") R(2,"min.f16x2") R(3,"min.u16x2") R(4,"2x min.u16x2 (vimnmx3 16x2?)")
  R(5,"min.u32") R(6,"min.s32") R(7,"add.u32") R(8,"lop3") R(9,"prmt") R(10,"shf") R(11,"sad.u32") R(13,"max.f32") R(14,"2x min.f32") R(15,"vabsdiff2.add")
  return 0; }
