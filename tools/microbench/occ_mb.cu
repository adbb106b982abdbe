// Microbenchmark: shared-memory atomic histogram throughput vs occupancy and per-thread batching.
// Samples are pre-reduced to table offsets (no decode), uniform over the table.
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>
#define CK(x) do{cudaError_t e=(x); if(e!=cudaSuccess){printf("CUDA %s @%d\n",cudaGetErrorString(e),__LINE__); return 1;}}while(0)
__device__ __forceinline__ uint32_t mix(uint32_t x){ x^=x>>16; x*=0x7feb352d; x^=x>>15; x*=0x846ca68b; x^=x>>16; return x; }
__global__ void k_gen(uint32_t* s, uint64_t n, uint32_t nb){
  for(uint64_t i=blockIdx.x*(uint64_t)blockDim.x+threadIdx.x;i<n;i+=(uint64_t)gridDim.x*blockDim.x) s[i]=mix((uint32_t)i*2654435761u+7u)%nb; }
template<int VEC, int RET>
__global__ void k_h(const uint4* __restrict__ s, uint64_t n4, uint32_t words, uint32_t* out){
  extern __shared__ uint32_t t[];
  for(uint32_t i=threadIdx.x;i<words;i+=blockDim.x) t[i]=0; __syncthreads();
  uint64_t per=(n4+gridDim.x-1)/gridDim.x, a=blockIdx.x*per, e=min(n4,a+per);
  uint32_t acc=0;
  uint64_t i=a+threadIdx.x;
  for(;i+(VEC-1)*blockDim.x<e;i+=VEC*blockDim.x){
    uint4 v[VEC];
    #pragma unroll
    for(int u=0;u<VEC;u++) v[u]=__ldg(s+i+u*blockDim.x);
    #pragma unroll
    for(int u=0;u<VEC;u++){
      if(RET){ acc+=atomicAdd(t+v[u].x,1u); acc+=atomicAdd(t+v[u].y,1u); acc+=atomicAdd(t+v[u].z,1u); acc+=atomicAdd(t+v[u].w,1u);}
      else { atomicAdd(t+v[u].x,1u); atomicAdd(t+v[u].y,1u); atomicAdd(t+v[u].z,1u); atomicAdd(t+v[u].w,1u);} }
  }
  for(;i<e;i+=blockDim.x){ uint4 v=__ldg(s+i); atomicAdd(t+v.x,1u); atomicAdd(t+v.y,1u); atomicAdd(t+v.z,1u); atomicAdd(t+v.w,1u);}
  __syncthreads(); if(threadIdx.x==0) out[blockIdx.x]=t[5]+acc;
}
int main(){
  const uint64_t n=1ull<<28; uint32_t *s,*o; CK(cudaMalloc(&s,n*4)); CK(cudaMalloc(&o,4096*4));
  cudaEvent_t a,b; cudaEventCreate(&a); cudaEventCreate(&b);
  auto timeit=[&](const char* nm, auto f){ for(int w=0;w<2;w++) f(); CK(cudaGetLastError()); cudaEventRecord(a); for(int r=0;r<5;r++) f(); cudaEventRecord(b); cudaEventSynchronize(b);
     float ms; cudaEventElapsedTime(&ms,a,b); ms/=5; printf("%-44s %8.3f ms %8.1f Gsamp/s\n",nm,ms,n/ms/1e6); return 0; };
  struct C{int ctas_per_sm, threads; uint32_t words; const char* nm;};
  C cs[]={{1,1024,57000,"1x1024 57K"},{2,1024,28000,"2x1024 28K"},{4,512,14000,"4x512 14K"},{2,512,28000,"2x512 28K"},{1,1024,28000,"1x1024 28K"},{8,256,7000,"8x256 7K"}};
  for(auto c: cs){
    k_gen<<<1184,512>>>(s,n,c.words); CK(cudaDeviceSynchronize());
    size_t sm=c.words*4; int grid=148*c.ctas_per_sm;
    CK(cudaFuncSetAttribute(k_h<1,0>,cudaFuncAttributeMaxDynamicSharedMemorySize,(int)sm));
    CK(cudaFuncSetAttribute(k_h<4,0>,cudaFuncAttributeMaxDynamicSharedMemorySize,(int)sm));
    CK(cudaFuncSetAttribute(k_h<4,1>,cudaFuncAttributeMaxDynamicSharedMemorySize,(int)sm));
    char nm[96];
    snprintf(nm,96,"%s vec1",c.nm); timeit(nm,[&]{k_h<1,0><<<grid,c.threads,sm>>>((uint4*)s,n/4,c.words,o);});
    snprintf(nm,96,"%s vec4",c.nm); timeit(nm,[&]{k_h<4,0><<<grid,c.threads,sm>>>((uint4*)s,n/4,c.words,o);});
    snprintf(nm,96,"%s vec4 ret",c.nm); timeit(nm,[&]{k_h<4,1><<<grid,c.threads,sm>>>((uint4*)s,n/4,c.words,o);});
    int occ=0; cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ,k_h<4,0>,c.threads,sm); printf("   (occupancy %d CTAs/SM)\n",occ);
  }
  return 0;
}
