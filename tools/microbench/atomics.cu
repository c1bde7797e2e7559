// Microbenchmark: shared/global atomic throughput on sm_100a (design evidence for the
// hash/dense accumulators).
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>
#define CK(x) do{cudaError_t e=(x); if(e!=cudaSuccess){printf("err %s line %d\n",cudaGetErrorString(e),__LINE__);return 1;}}while(0)

__device__ __forceinline__ uint32_t hsh(uint32_t x){ x^=x>>16; x*=0x7feb352dU; x^=x>>15; x*=0x846ca68bU; x^=x>>16; return x; }

template<int OP>
__global__ void k_smem(int iters, uint32_t words, float* sink){
  extern __shared__ uint32_t sm[];
  for (uint32_t i=threadIdx.x;i<words;i+=blockDim.x) sm[i]=0;
  __syncthreads();
  uint32_t s = hsh(blockIdx.x*blockDim.x+threadIdx.x);
  uint32_t acc=0;
  for(int it=0;it<iters;++it){
    s = s*1664525u+1013904223u;
    uint32_t a = (s>>8) % words;
    if(OP==0) atomicAdd(&sm[a],1u);
    else if(OP==1) acc += atomicCAS(&sm[a], 0u, s);
    else if(OP==2) atomicAdd((float*)&sm[a], 1.0f);
    else if(OP==3) atomicAdd((double*)&sm[a & ~1u], 1.0);
    else if(OP==4) atomicOr(&sm[a], 1u<<(s&31));
    else if(OP==5) sm[a] = s;            // plain store
    else if(OP==6) acc += sm[a];         // plain load
    else if(OP==7) { uint32_t v = sm[a]; if (v==0) acc += atomicCAS(&sm[a],0u,s); else acc+=v; } // probe-then-CAS
  }
  __syncthreads();
  if(acc==0x12345 ) sink[0]=acc;
  if(threadIdx.x==0) sink[blockIdx.x+1]=sm[0];
}

template<int OP>
__global__ void k_gmem(int iters, uint32_t words, uint32_t* base){
  uint32_t* g = base + (size_t)blockIdx.x*words;
  uint32_t s = hsh(blockIdx.x*blockDim.x+threadIdx.x);
  for(int it=0;it<iters;++it){
    s = s*1664525u+1013904223u;
    uint32_t a = (s>>8) % words;
    if(OP==0) atomicAdd((float*)&g[a], 1.0f);
    else if(OP==1) atomicOr(&g[a], 1u<<(s&31));
  }
}

int main(){
  float* sink; CK(cudaMalloc(&sink, 1<<20));
  cudaEvent_t a,b; cudaEventCreate(&a); cudaEventCreate(&b);
  int iters=4096;
  const char* names[]={"ATOMS.ADD.u32","ATOMS.CAS","atomicAdd f32 smem","atomicAdd f64 smem","ATOMS.OR","STS","LDS","probe+CAS"};
  int threads[] = {256, 1024};
  for (int ti=0; ti<2; ++ti){
   int T = threads[ti];
   uint32_t words = (ti==0)? 6*1024 : 24*1024; // 24KB*8 CTAs or 96KB*2 CTAs per SM
   int blocks = 148*(2048/T);
   for(int op=0;op<8;++op){
    void(*kp)(int,uint32_t,float*);
    switch(op){case 0:kp=k_smem<0>;break;case 1:kp=k_smem<1>;break;case 2:kp=k_smem<2>;break;case 3:kp=k_smem<3>;break;case 4:kp=k_smem<4>;break;case 5:kp=k_smem<5>;break;case 6:kp=k_smem<6>;break;default:kp=k_smem<7>;}
    CK(cudaFuncSetAttribute(kp, cudaFuncAttributeMaxDynamicSharedMemorySize, words*4));
    kp<<<blocks,T,words*4>>>(64,words,sink);
    CK(cudaDeviceSynchronize());
    cudaEventRecord(a); kp<<<blocks,T,words*4>>>(iters,words,sink); cudaEventRecord(b); CK(cudaEventSynchronize(b));
    float ms; cudaEventElapsedTime(&ms,a,b);
    double ops=(double)blocks*T*iters;
    printf("T=%4d words=%6u %-22s %8.1f Gop/s  (%.2f op/clk/SM @1.9GHz)\n",T,words,names[op],ops/ms/1e6, ops/ms/1e6/148/1.9);
   }
  }
  // global atomics: per-CTA region of 1M words (4MB) -- 148 CTAs x 4MB = 592MB (not L2 resident) and 16K words (L2 resident)
  uint32_t* gbuf; size_t gwords=(size_t)148*2*(1<<20); CK(cudaMalloc(&gbuf, gwords*4)); cudaMemset(gbuf,0,gwords*4);
  uint32_t regs[]={1<<14, 1<<17, 1<<20};
  for(int r=0;r<3;++r) for(int op=0;op<2;++op){
    void(*kp)(int,uint32_t,uint32_t*) = op==0? k_gmem<0>:k_gmem<1>;
    int blocks=148*2, T=1024;
    kp<<<blocks,T>>>(16,regs[r],gbuf); CK(cudaDeviceSynchronize());
    cudaEventRecord(a); kp<<<blocks,T>>>(256,regs[r],gbuf); cudaEventRecord(b); CK(cudaEventSynchronize(b));
    float ms; cudaEventElapsedTime(&ms,a,b);
    double ops=(double)blocks*T*256;
    printf("global %s region=%u words/CTA: %8.1f Gop/s\n", op==0?"RED.ADD.F32":"RED.OR", regs[r], ops/ms/1e6);
  }
  // random 8B gather from HBM (B-row style: 4 consecutive lanes)
  return 0;
}
