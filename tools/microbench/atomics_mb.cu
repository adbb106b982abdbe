// Microbenchmark: what bounds a per-sample histogram on B200 (sm_100a)?
// Measures streaming read BW, global RED throughput (uniform / skewed bins),
// shared-memory ATOMS throughput, and warp-aggregation variants.
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>
#define CK(x) do{cudaError_t e=(x); if(e!=cudaSuccess){printf("CUDA %s @%d\n",cudaGetErrorString(e),__LINE__); return 1;}}while(0)

__device__ __forceinline__ uint32_t mix(uint32_t x){ x^=x>>16; x*=0x7feb352d; x^=x>>15; x*=0x846ca68b; x^=x>>16; return x; }

__global__ void k_gen(uint32_t* s, uint64_t n, uint32_t nbins, int mode){
  for(uint64_t i=blockIdx.x*(uint64_t)blockDim.x+threadIdx.x;i<n;i+=(uint64_t)gridDim.x*blockDim.x){
    uint32_t h=mix((uint32_t)i*2654435761u+12345u);
    uint32_t b;
    if(mode==0) b=h%nbins;                       // uniform
    else if(mode==1) b=(h%10u)*997u%nbins;       // 10 hot bins only
    else { // locality: blocks of 1M samples confined to a 64K-bin window
      uint32_t win=(uint32_t)(i>>20); b=(win*65536u + (h&65535u))%nbins; }
    s[i]=b;
  }
}
__global__ void k_read(const uint4* __restrict__ s, uint64_t n4, uint32_t* out){
  uint32_t acc=0;
  for(uint64_t i=blockIdx.x*(uint64_t)blockDim.x+threadIdx.x;i<n4;i+=(uint64_t)gridDim.x*blockDim.x){
    uint4 v=__ldg(s+i); acc^=v.x^v.y^v.z^v.w; }
  if(acc==0x12345678u) out[0]=acc;
}
__global__ void k_red(const uint4* __restrict__ s, uint64_t n4, uint32_t* h){
  for(uint64_t i=blockIdx.x*(uint64_t)blockDim.x+threadIdx.x;i<n4;i+=(uint64_t)gridDim.x*blockDim.x){
    uint4 v=__ldg(s+i); atomicAdd(h+v.x,1u); atomicAdd(h+v.y,1u); atomicAdd(h+v.z,1u); atomicAdd(h+v.w,1u); }
}
__device__ __forceinline__ void agg_add(uint32_t* h, uint32_t b){
  uint32_t m=__match_any_sync(0xffffffffu,b); int lane=threadIdx.x&31;
  if((__ffs(m)-1)==lane) atomicAdd(h+b,(uint32_t)__popc(m));
}
__global__ void k_red_match(const uint4* __restrict__ s, uint64_t n4, uint32_t* h){
  for(uint64_t i=blockIdx.x*(uint64_t)blockDim.x+threadIdx.x;i<n4;i+=(uint64_t)gridDim.x*blockDim.x){
    uint4 v=__ldg(s+i); agg_add(h,v.x); agg_add(h,v.y); agg_add(h,v.z); agg_add(h,v.w); }
}
// smem atomics into a private table of `nb` words (bins folded mod nb), flush at end
__global__ void k_atoms(const uint4* __restrict__ s, uint64_t n4, uint32_t* h, uint32_t nb){
  extern __shared__ uint32_t t[];
  for(uint32_t i=threadIdx.x;i<nb;i+=blockDim.x) t[i]=0; __syncthreads();
  for(uint64_t i=blockIdx.x*(uint64_t)blockDim.x+threadIdx.x;i<n4;i+=(uint64_t)gridDim.x*blockDim.x){
    uint4 v=__ldg(s+i); atomicAdd(t+(v.x%nb),1u); atomicAdd(t+(v.y%nb),1u); atomicAdd(t+(v.z%nb),1u); atomicAdd(t+(v.w%nb),1u); }
  __syncthreads();
  for(uint32_t i=threadIdx.x;i<nb;i+=blockDim.x) if(t[i]) atomicAdd(h+i,t[i]);
}
// smem non-atomic per-warp RMW with match_any dedup (per-warp sub-table)
__global__ void k_lds_match(const uint4* __restrict__ s, uint64_t n4, uint32_t* h, uint32_t nb){
  extern __shared__ uint32_t t[];
  for(uint32_t i=threadIdx.x;i<nb;i+=blockDim.x) t[i]=0; __syncthreads();
  for(uint64_t i=blockIdx.x*(uint64_t)blockDim.x+threadIdx.x;i<n4;i+=(uint64_t)gridDim.x*blockDim.x){
    uint4 v=__ldg(s+i);
    uint32_t b[4]={v.x%nb,v.y%nb,v.z%nb,v.w%nb};
    #pragma unroll
    for(int k=0;k<4;k++){ uint32_t m=__match_any_sync(0xffffffffu,b[k]); if((__ffs(m)-1)==(int)(threadIdx.x&31)) atomicAdd(t+b[k],(uint32_t)__popc(m)); }
  }
  __syncthreads();
  for(uint32_t i=threadIdx.x;i<nb;i+=blockDim.x) if(t[i]) atomicAdd(h+i,t[i]);
}

int main(){
  int dev=0; cudaDeviceProp p; CK(cudaGetDeviceProperties(&p,dev));
  printf("dev %s SMs %d smemOptin %zu L2 %d\n",p.name,p.multiProcessorCount,p.sharedMemPerBlockOptin,p.l2CacheSize);
  const uint64_t n=1ull<<28; // 268M samples = 1 GiB
  uint32_t *s,*h,*o; CK(cudaMalloc(&s,n*4)); CK(cudaMalloc(&h,(1u<<25)*4)); CK(cudaMalloc(&o,64));
  cudaEvent_t a,b; cudaEventCreate(&a); cudaEventCreate(&b);
  int SM=p.multiProcessorCount;
  uint32_t nbins_list[3]={1u<<25,1u<<20,19u*4096u};
  for(int mode=0;mode<3;mode++) for(int nbi=0;nbi<3;nbi++){
    if(mode!=0 && nbi!=0) continue;
    uint32_t nbins=nbins_list[nbi];
    k_gen<<<SM*8,512>>>(s,n,nbins,mode); CK(cudaDeviceSynchronize());
    auto run=[&](const char* name,auto launch){
      for(int w=0;w<2;w++) launch();
      cudaEventRecord(a); for(int r=0;r<3;r++) launch(); cudaEventRecord(b); cudaEventSynchronize(b);
      float ms; cudaEventElapsedTime(&ms,a,b); ms/=3;
      printf("mode %d nbins %8u %-22s %8.3f ms  %8.1f Gsamp/s  %7.1f GB/s\n",mode,nbins,name,ms,n/ms/1e6,n*4.0/ms/1e6);
    };
    uint64_t n4=n/4;
    for(int bs: {256,512}) for(int occ: {4,8,16}){
      char nm[64]; snprintf(nm,64,"read b%d g%dx",bs,occ);
      if(mode==0&&nbi==0) run(nm,[&]{k_read<<<SM*occ,bs>>>((uint4*)s,n4,o);});
    }
    cudaMemset(h,0,(1u<<25)*4);
    run("red",[&]{k_red<<<SM*8,512>>>((uint4*)s,n4,h);});
    run("red_match",[&]{k_red_match<<<SM*8,512>>>((uint4*)s,n4,h);});
    for(uint32_t nb: {12288u, 49152u}){
      size_t sm=nb*4; cudaFuncSetAttribute(k_atoms,cudaFuncAttributeMaxDynamicSharedMemorySize,(int)sm);
      cudaFuncSetAttribute(k_lds_match,cudaFuncAttributeMaxDynamicSharedMemorySize,(int)sm);
      int occ=(nb==12288u)?4:1;
      char nm[64]; snprintf(nm,64,"atoms nb%u",nb);
      run(nm,[&]{k_atoms<<<SM*occ,512,sm>>>((uint4*)s,n4,h,nb);});
      snprintf(nm,64,"atoms_match nb%u",nb);
      run(nm,[&]{k_lds_match<<<SM*occ,512,sm>>>((uint4*)s,n4,h,nb);});
    }
  }
  CK(cudaGetLastError());
  return 0;
}
