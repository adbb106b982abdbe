#ifndef NLOG
#define NLOG 28
#endif
// Microbenchmark: shared-memory atomic counting rate on a C4-shaped stream (2^28 words, 1 GB >
// L2): 80% of samples on a hot 10% of a 77824-bin window, 20% uniform. Compares
//   A  1 CTA x 1024 thr / SM, 16-bit pairs (38912 words), returning atomics + flag vote, 16 samples/thread batch
//   B  same, non-returning (no overflow check) — the atomic-unit ceiling at 32 warps
//   C  2 CTAs x 1024 thr / SM, 8-bit quads (19456 words each), returning + flag vote, 4 samples/batch
//   D  same as C, non-returning
//   E  2 CTAs x 1024, 8-bit quads, returning, 8 samples/batch (2 uint4)
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o atoms_occ2 atoms_occ2.cu
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>
#define CK(x) do{cudaError_t e=(x); if(e!=cudaSuccess){printf("CUDA %s @%d\n",cudaGetErrorString(e),__LINE__); return 1;}}while(0)
__device__ __forceinline__ uint32_t mix(uint32_t x){ x^=x>>16; x*=0x7feb352d; x^=x>>15; x*=0x846ca68b; x^=x>>16; return x; }
__global__ void k_gen(uint32_t* s, uint64_t n, uint32_t nb){
  for(uint64_t i=blockIdx.x*(uint64_t)blockDim.x+threadIdx.x;i<n;i+=(uint64_t)gridDim.x*blockDim.x){
    uint32_t h=mix((uint32_t)i*2654435761u+7u), u=mix(h+0x9e37u);
    s[i] = (h%10<8) ? (nb/3 + u%(nb/10)) : u%nb; } }
// BITS = counter width (16 or 8), RET = use returned value for overflow detection, V = uint4 per batch
template<int BITS, int RET, int V>
__global__ void __launch_bounds__(1024, (BITS==8?2:1)) k_h(const uint4* __restrict__ s, uint64_t n4, uint32_t words, uint32_t* out){
  extern __shared__ uint32_t t[];
  for(uint32_t i=threadIdx.x;i<words+32;i+=blockDim.x) t[i]=0; __syncthreads();
  constexpr uint32_t PER = 32/BITS, SH = BITS==16?1:2, HB = 1u<<(BITS-1);
  uint64_t per=(n4+gridDim.x-1)/gridDim.x, a=blockIdx.x*per, e=min(n4,a+per);
  uint32_t acc=0;
  for(uint64_t i=a+threadIdx.x;i+(V-1)*blockDim.x<e;i+=V*blockDim.x){
    uint32_t w[4*V];
    #pragma unroll
    for(int u=0;u<V;u++){ uint4 v=__ldg(s+i+u*blockDim.x); w[4*u]=v.x; w[4*u+1]=v.y; w[4*u+2]=v.z; w[4*u+3]=v.w; }
    uint32_t flag=0;
    #pragma unroll
    for(int q=0;q<4*V;q++){
      const uint32_t off=w[q]; const uint32_t inc=1u<<((off&(PER-1))*BITS);
      if(RET) flag |= atomicAdd(t+(off>>SH), inc) & (inc*HB);
      else atomicAdd(t+(off>>SH), inc);
    }
    if(RET && __any_sync(0xffffffffu, flag)) acc += flag;   // rare path stand-in
  }
  __syncthreads(); if(threadIdx.x==0) out[blockIdx.x]=t[5]+acc;
}
// G: the product's per-sample fast path (count16): window offset, bounds check, per-lane spare
// word for out-of-window lanes, returning atomic, mask of the flag bit, one vote per batch
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
// H: trimmed fast path: inc and flag mask from one predicate, byte address straight from off
__global__ void __launch_bounds__(1024, 1) k_h2(const uint4* __restrict__ s, uint64_t n4, uint32_t words, uint32_t wb,
                                                uint32_t lim, uint32_t* out){
  extern __shared__ uint32_t t[];
  for(uint32_t i=threadIdx.x;i<words+32;i+=blockDim.x) t[i]=0; __syncthreads();
  const uint32_t spare_b = (words + (threadIdx.x & 31)) * 4;
  const uint32_t tb = (uint32_t)__cvta_generic_to_shared(t);
  uint64_t per=(n4+gridDim.x-1)/gridDim.x, a=blockIdx.x*per, e=min(n4,a+per);
  uint32_t acc=0;
  for(uint64_t i=a+threadIdx.x;i+3*blockDim.x<e;i+=4*blockDim.x){
    uint32_t w[16];
    #pragma unroll
    for(int u=0;u<4;u++){ uint4 v=__ldg(s+i+u*blockDim.x); w[4*u]=v.x; w[4*u+1]=v.y; w[4*u+2]=v.z; w[4*u+3]=v.w; }
    uint32_t flag=0, outm=0;
    #pragma unroll
    for(int q=0;q<16;q++){
      const uint32_t off = w[q] - wb;
      const bool in = off < lim;
      const bool hi = off & 1u;
      const uint32_t inc = hi ? 0x10000u : 1u;
      const uint32_t addr = tb + (in ? ((off << 1) & ~3u) : spare_b);
      uint32_t old;
      asm volatile("atom.shared.add.u32 %0, [%1], %2;" : "=r"(old) : "r"(addr), "r"(inc) : "memory");
      flag |= old & (hi ? 0x80000000u : 0x8000u);
      outm |= in ? 0u : 1u;
    }
    if(__any_sync(0xffffffffu, flag | outm)) acc += flag;
  }
  __syncthreads(); if(threadIdx.x==0) out[blockIdx.x]=t[5]+acc;
}
int main(){ setvbuf(stdout, NULL, _IONBF, 0); printf("start\n");
  const uint64_t n=1ull<<NLOG; uint32_t *s,*o; CK(cudaMalloc(&s,n*4)); CK(cudaMalloc(&o,4096*4));
  k_gen<<<1184,512>>>(s,n,77824); CK(cudaDeviceSynchronize()); printf("gen done\n");
  cudaEvent_t a,b; cudaEventCreate(&a); cudaEventCreate(&b);
  auto timeit=[&](const char* nm, auto f){ for(int w=0;w<2;w++) f(); CK(cudaGetLastError()); cudaEventRecord(a); for(int r=0;r<10;r++) f(); cudaEventRecord(b); cudaEventSynchronize(b);
     float ms; cudaEventElapsedTime(&ms,a,b); ms/=10; printf("%-58s %8.3f ms %8.1f Gsamp/s  (x%d = %.3f ms for 2^30)\n",nm,ms,n/ms/1e6, (int)((1ull<<30)/n), ((1ull<<30)/n)*ms); return 0; };
  #define RUN(NM, BITS, RET, V, CPS) { auto k=k_h<BITS,RET,V>; size_t sm=(77824/(32/BITS)+32)*4; \
    CK(cudaFuncSetAttribute(k,cudaFuncAttributeMaxDynamicSharedMemorySize,(int)sm)); int occ=0; \
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ,k,1024,sm); cudaFuncAttributes fa; cudaFuncGetAttributes(&fa,k); \
    char nm[128]; snprintf(nm,128,"%s occ=%d regs=%d",NM,occ,fa.numRegs); \
    timeit(nm,[&]{k<<<148*CPS,1024,sm>>>((const uint4*)s,n/4,77824/(32/BITS),o);}); }
  RUN("A 1x1024 16b ret V4", 16, 1, 4, 1)
  RUN("B 1x1024 16b noret V4", 16, 0, 4, 1)
  RUN("A2 1x1024 16b ret V2", 16, 1, 2, 1)
  RUN("C 2x1024 8b ret V1", 8, 1, 1, 2)
  RUN("D 2x1024 8b noret V1", 8, 0, 1, 2)
  RUN("E 2x1024 8b ret V2", 8, 1, 2, 2)
  RUN("F 2x1024 8b ret V4", 8, 1, 4, 2)
  { size_t sm=(38912+32)*4; CK(cudaFuncSetAttribute(k_g,cudaFuncAttributeMaxDynamicSharedMemorySize,(int)sm));
    cudaFuncAttributes fa; cudaFuncGetAttributes(&fa,k_g); char nm[128]; snprintf(nm,128,"G product fast path 1x1024 regs=%d",fa.numRegs);
    timeit(nm,[&]{k_g<<<148,1024,sm>>>((const uint4*)s,n/4,38912,0,77824,1u,o);}); }
  { size_t sm=(38912+32)*4; CK(cudaFuncSetAttribute(k_h2,cudaFuncAttributeMaxDynamicSharedMemorySize,(int)sm));
    cudaFuncAttributes fa; cudaFuncGetAttributes(&fa,k_h2); char nm[128]; snprintf(nm,128,"H trimmed fast path 1x1024 regs=%d",fa.numRegs);
    timeit(nm,[&]{k_h2<<<148,1024,sm>>>((const uint4*)s,n/4,38912,0,77824,o);}); }
  return 0;
}
