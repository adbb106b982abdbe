// The product's per-sample fast path (count16) over ONE fixed window, no items / flushes / stealing:
// the counting ceiling of the attribution pass on a real packed stream (offsets pre-reduced to the
// window). extern "C" launcher for ctypes (tools/microbench/gk_run.py).
#include <cstdint>
#include <cuda_runtime.h>
__global__ void __launch_bounds__(1024, 1) k_g(const uint4* __restrict__ s, uint64_t n4, uint32_t words, uint32_t wb,
                                                uint32_t lim, uint32_t one, uint32_t* out){
  extern __shared__ uint32_t t[];
  for(uint32_t i=threadIdx.x;i<words+32;i+=blockDim.x) t[i]=0; __syncthreads();
  const uint32_t spare = words + (threadIdx.x & 31);
  uint64_t per=(n4+gridDim.x-1)/gridDim.x, a=blockIdx.x*per, e=min(n4,a+per);
  uint32_t acc=0;
  for(uint64_t i=a+threadIdx.x;i+3*blockDim.x<e;i+=4*blockDim.x){
    uint32_t w[16];
    #pragma unroll
    for(int u=0;u<4;u++){ uint4 v=__ldg(s+i+u*blockDim.x); w[4*u]=v.x; w[4*u+1]=v.y; w[4*u+2]=v.z; w[4*u+3]=v.w; }
    uint32_t flag=0;
    #pragma unroll
    for(int q=0;q<16;q++){
      const uint32_t off = w[q] - wb;
      const bool in = off < lim;
      const uint32_t inc = one << ((off & 1u) << 4);
      flag |= atomicAdd(t + (in ? off >> 1 : spare), inc) & (in ? inc << 15 : 0xffffffffu);
    }
    if(__any_sync(0xffffffffu, flag)) acc += flag;
  }
  __syncthreads(); if(threadIdx.x==0) out[blockIdx.x]=t[5]+acc;
}
extern "C" float run_g(const uint32_t* d, uint64_t n, uint32_t nbins, int grid, int iters) {
  static uint32_t* o = nullptr; if (!o) cudaMalloc(&o, 4096 * 4);
  uint32_t words = (nbins + 1) / 2; size_t sm = (words + 32) * 4;
  cudaFuncSetAttribute(k_g, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
  cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
  for (int w = 0; w < 2; w++) k_g<<<grid, 1024, sm>>>((const uint4*)d, n / 4, words, 0, nbins, 1u, o);
  cudaEventRecord(a);
  for (int r = 0; r < iters; r++) k_g<<<grid, 1024, sm>>>((const uint4*)d, n / 4, words, 0, nbins, 1u, o);
  cudaEventRecord(b); cudaEventSynchronize(b);
  float ms; cudaEventElapsedTime(&ms, a, b); return ms / iters;
}
