// Microbenchmark: shared-memory histogram throughput, local tables vs a table distributed over a
// thread-block cluster (DSMEM remote atomics, red.shared::cluster). Random bins, 2^28 samples.
#include <cooperative_groups.h>
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>
namespace cg = cooperative_groups;
#define CK(x) do{cudaError_t e=(x); if(e!=cudaSuccess){printf("CUDA %s @%d\n",cudaGetErrorString(e),__LINE__); return 1;}}while(0)
__device__ __forceinline__ uint32_t mix(uint32_t x){ x^=x>>16; x*=0x7feb352d; x^=x>>15; x*=0x846ca68b; x^=x>>16; return x; }
__global__ void k_gen(uint32_t* s, uint64_t n, uint32_t nb){
  for(uint64_t i=blockIdx.x*(uint64_t)blockDim.x+threadIdx.x;i<n;i+=(uint64_t)gridDim.x*blockDim.x) s[i]=mix((uint32_t)i*2654435761u+7u)%nb; }
constexpr int WORDS = 56*1024 - 64;
// local: each CTA counts bins [0, WORDS) mod WORDS
__global__ void __launch_bounds__(1024,1) k_local(const uint4* __restrict__ s, uint64_t n4, uint32_t* out){
  extern __shared__ uint32_t t[];
  for(int i=threadIdx.x;i<WORDS;i+=blockDim.x) t[i]=0; __syncthreads();
  uint64_t per=(n4+gridDim.x-1)/gridDim.x, a=blockIdx.x*per, e=min(n4,a+per);
  for(uint64_t i=a+threadIdx.x;i<e;i+=blockDim.x){ uint4 v=__ldg(s+i);
    atomicAdd(t+v.x%WORDS,1u); atomicAdd(t+v.y%WORDS,1u); atomicAdd(t+v.z%WORDS,1u); atomicAdd(t+v.w%WORDS,1u);}
  __syncthreads(); if(threadIdx.x==0) out[blockIdx.x]=t[5];
}
// cluster: bins [0, CS*WORDS); bin b lives in CTA b / WORDS of the cluster
template<int CS>
__global__ void __launch_bounds__(1024,1) k_cluster(const uint4* __restrict__ s, uint64_t n4, uint32_t* out){
  extern __shared__ uint32_t t[];
  cg::cluster_group cl = cg::this_cluster();
  for(int i=threadIdx.x;i<WORDS;i+=blockDim.x) t[i]=0;
  cl.sync();
  uint32_t* remote[CS];
  for(int r=0;r<CS;r++) remote[r]=cl.map_shared_rank(t, r);
  uint64_t per=(n4+gridDim.x-1)/gridDim.x, a=blockIdx.x*per, e=min(n4,a+per);
  for(uint64_t i=a+threadIdx.x;i<e;i+=blockDim.x){ uint4 v=__ldg(s+i);
    uint32_t w[4]={v.x,v.y,v.z,v.w};
    #pragma unroll
    for(int q=0;q<4;q++){ uint32_t b=w[q]%(CS*WORDS); uint32_t r=b/WORDS, o=b%WORDS; atomicAdd(remote[r]+o,1u);} }
  cl.sync(); if(threadIdx.x==0) out[blockIdx.x]=t[5];
}
int main(){
  const uint64_t n=1ull<<28; uint32_t *s,*o; CK(cudaMalloc(&s,n*4)); CK(cudaMalloc(&o,4096*4));
  cudaEvent_t a,b; cudaEventCreate(&a); cudaEventCreate(&b);
  size_t sm=WORDS*4;
  CK(cudaFuncSetAttribute(k_local,cudaFuncAttributeMaxDynamicSharedMemorySize,(int)sm));
  CK(cudaFuncSetAttribute(k_cluster<2>,cudaFuncAttributeMaxDynamicSharedMemorySize,(int)sm));
  CK(cudaFuncSetAttribute(k_cluster<4>,cudaFuncAttributeMaxDynamicSharedMemorySize,(int)sm));
  auto timeit=[&](const char* nm, auto f){ for(int w=0;w<2;w++) f(); cudaEventRecord(a); for(int r=0;r<5;r++) f(); cudaEventRecord(b); cudaEventSynchronize(b);
     float ms; cudaEventElapsedTime(&ms,a,b); ms/=5; printf("%-28s %8.3f ms %8.1f Gsamp/s\n",nm,ms,n/ms/1e6); };
  for(uint32_t nb: {100000u, 200000u, 400000u}){
    k_gen<<<1184,512>>>(s,n,nb); CK(cudaDeviceSynchronize());
    printf("bins %u\n",nb);
    timeit("local (mod WORDS)",[&]{k_local<<<148,1024,sm>>>((uint4*)s,n/4,o);});
    { cudaLaunchConfig_t cfg={}; cfg.gridDim=148; cfg.blockDim=1024; cfg.dynamicSmemBytes=sm; cudaLaunchAttribute at[1]; at[0].id=cudaLaunchAttributeClusterDimension; at[0].val.clusterDim.x=2; at[0].val.clusterDim.y=1; at[0].val.clusterDim.z=1; cfg.attrs=at; cfg.numAttrs=1;
      timeit("cluster2 DSMEM",[&]{cudaLaunchKernelEx(&cfg,k_cluster<2>,(const uint4*)s,n/4,o);}); }
    { cudaLaunchConfig_t cfg={}; cfg.gridDim=148; cfg.blockDim=1024; cfg.dynamicSmemBytes=sm; cudaLaunchAttribute at[1]; at[0].id=cudaLaunchAttributeClusterDimension; at[0].val.clusterDim.x=4; at[0].val.clusterDim.y=1; at[0].val.clusterDim.z=1; cfg.attrs=at; cfg.numAttrs=1;
      timeit("cluster4 DSMEM",[&]{cudaLaunchKernelEx(&cfg,k_cluster<4>,(const uint4*)s,n/4,o);}); }
    CK(cudaGetLastError());
  }
  return 0;
}
