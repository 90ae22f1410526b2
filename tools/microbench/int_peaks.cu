// Integer-pipe microbenchmarks for the FSBM roofline.
// Measures per-SM issue throughput of the instructions the ME/SME kernels are
// built from: VABSDIFF4.U8.ACC, VIMNMX3.U32, LEA, IADD3, IMAD, LDS.32/LDS.128.
// Output: one JSON object (ops per clock per SM, plus ops/s at the clock seen).
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

#define CK(x) do{cudaError_t e=(x); if(e!=cudaSuccess){fprintf(stderr,"%s:%d %s\n",__FILE__,__LINE__,cudaGetErrorString(e)); return 1;}}while(0)

__device__ __forceinline__ uint32_t vad4(uint32_t a, uint32_t b, uint32_t c){
  uint32_t d; asm volatile("vabsdiff4.u32.u32.u32.add %0,%1,%2,%3;" : "=r"(d) : "r"(a),"r"(b),"r"(c)); return d; }
__device__ __forceinline__ uint32_t min3(uint32_t a, uint32_t b, uint32_t c){
  uint32_t d; asm volatile("min.u32 %0,%1,%2;" : "=r"(d) : "r"(a),"r"(b)); asm volatile("min.u32 %0,%1,%2;" : "=r"(d) : "r"(d),"r"(c)); return d; }

constexpr int NACC = 16;   // independent chains per thread
constexpr int ITERS = 4096;

// mode 0: VABSDIFF4 only; 1: VIMNMX3 only; 2: LEA only; 3: IMAD only; 4: IADD3 only;
// 5: VABSDIFF4 + IMAD (1:1); 6: VABSDIFF4 + VIMNMX3 (1:1); 7: VABSDIFF4 + LEA (1:1)
template<int MODE>
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
      if (MODE==0) a[i]=vad4(x,b[i],a[i]);
      if (MODE==1) a[i]=min3(a[i],b[i],x);
      if (MODE==2) { uint32_t d; asm volatile("{.reg .u32 t; shl.b32 t,%1,16; add.u32 %0,t,%2;}" : "=r"(d):"r"(a[i]),"r"(x)); a[i]=d; }
      if (MODE==3) { uint32_t d; asm volatile("mad.lo.u32 %0,%1,%2,%3;" : "=r"(d):"r"(a[i]),"r"(y),"r"(x)); a[i]=d; }
      if (MODE==4) { uint32_t d; asm volatile("{.reg .u32 t; add.u32 t,%1,%2; sub.u32 %0,t,%3;}" : "=r"(d):"r"(a[i]),"r"(b[i]),"r"(x)); a[i]=d; }
      if (MODE==5) { a[i]=vad4(x,b[i],a[i]); uint32_t d; asm volatile("mad.lo.u32 %0,%1,%2,%3;" : "=r"(d):"r"(b[i]),"r"(y),"r"(x)); b[i]=d; }
      if (MODE==6) { a[i]=vad4(x,y,a[i]); b[i]=min3(b[i],a[i],x); }
      if (MODE==7) { a[i]=vad4(x,y,a[i]); uint32_t d; asm volatile("{.reg .u32 t; shl.b32 t,%1,16; add.u32 %0,t,%2;}" : "=r"(d):"r"(b[i]),"r"(x)); b[i]=d; }
    }
  }
  unsigned long long t1 = clock64();
  uint32_t s=0;
#pragma unroll
  for(int i=0;i<NACC;i++) s+=a[i]^b[i];
  out[blockIdx.x*blockDim.x+threadIdx.x]=s;
  if(threadIdx.x==0) cyc[blockIdx.x]=t1-t0;
}

// SMEM read throughput: LDS.32 and LDS.128, conflict-free, all lanes distinct words.
template<int W>
__global__ void __launch_bounds__(1024) lds_kern(uint32_t seed, uint32_t* out, unsigned long long* cyc){
  __shared__ uint4 sm[2048];
  for(int i=threadIdx.x;i<2048;i+=blockDim.x) sm[i]=make_uint4(i,seed,i^seed,i+seed);
  __syncthreads();
  uint32_t acc=0; int idx=threadIdx.x;
  unsigned long long t0=clock64();
  for(int it=0; it<ITERS; ++it){
#pragma unroll
    for(int i=0;i<8;i++){
      if(W==4){ const uint32_t* p=(const uint32_t*)sm; acc += p[((idx+i*32)&8191)]; }
      else    { uint4 v=sm[(idx+i*32)&2047]; acc += v.x^v.y^v.z^v.w; }
    }
    idx += acc&1;
  }
  unsigned long long t1=clock64();
  out[blockIdx.x*blockDim.x+threadIdx.x]=acc;
  if(threadIdx.x==0) cyc[blockIdx.x]=t1-t0;
}

int run(const char* name, void(*k)(uint32_t,uint32_t*,unsigned long long*), double ops_per_iter_thread, int nsm, bool last){
  uint32_t* out; unsigned long long* cyc;
  const int thr=1024;
  CK(cudaMalloc(&out, sizeof(uint32_t)*nsm*thr)); CK(cudaMalloc(&cyc, sizeof(unsigned long long)*nsm));
  k<<<nsm,thr>>>(1,out,cyc); CK(cudaDeviceSynchronize());
  cudaEvent_t e0,e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  cudaEventRecord(e0); k<<<nsm,thr>>>(2,out,cyc); cudaEventRecord(e1); CK(cudaEventSynchronize(e1));
  float ms; cudaEventElapsedTime(&ms,e0,e1);
  unsigned long long* h=new unsigned long long[nsm]; CK(cudaMemcpy(h,cyc,sizeof(unsigned long long)*nsm,cudaMemcpyDeviceToHost));
  double mx=0, sum=0; for(int i=0;i<nsm;i++){ if(h[i]>mx) mx=h[i]; sum+=h[i]; }
  double ops_cta = ops_per_iter_thread*ITERS*thr;
  double per_clk = ops_cta/(sum/nsm);
  double ops_s = ops_cta*nsm/(ms*1e-3);
  printf("  \"%s\": {\"ops_per_clk_per_sm\": %.2f, \"ops_per_s\": %.4e, \"ms\": %.3f, \"implied_mhz\": %.0f}%s\n",
         name, per_clk, ops_s, ms, ops_s/nsm/per_clk/1e6, last?"":",");
  delete[] h; cudaFree(out); cudaFree(cyc); return 0;
}

int main(){
  cudaDeviceProp p; CK(cudaGetDeviceProperties(&p,0));
  int nsm=p.multiProcessorCount;
  printf("{\n  \"device\": \"%s\", \"sms\": %d, \"l2_bytes\": %d, \"smem_per_block_optin\": %zu,\n", p.name, nsm, p.l2CacheSize, p.sharedMemPerBlockOptin);
  printf("  \"note\": \"ops = warp-lane instructions; per_clk from clock64 per CTA (1 CTA x 1024 thr per SM)\",\n");
  run("vabsdiff4_acc", kern<0>, NACC, nsm, false);
  run("vimnmx3",       kern<1>, NACC, nsm, false);
  run("lea_shl_add",   kern<2>, NACC, nsm, false);
  run("imad",          kern<3>, NACC, nsm, false);
  run("iadd3",         kern<4>, NACC, nsm, false);
  run("vabsdiff4+imad_pairs", kern<5>, NACC, nsm, false);
  run("vabsdiff4+vimnmx3_pairs", kern<6>, NACC, nsm, false);
  run("vabsdiff4+lea_pairs", kern<7>, NACC, nsm, false);
  run("lds32", lds_kern<4>, 8, nsm, false);
  run("lds128", lds_kern<16>, 8, nsm, true);
  printf("}\n");
  return 0;
}
