// Microbenchmark: the shared-memory atomic ceiling of the attribution pass's counting pattern on
// B200, with the sample words generated in registers (no HBM traffic): random bins of a window of
// `bins` compact bins, 16-bit counters packed two per word (the WINDOW kernel's table) or 32-bit.
// Reports samples/clk/SM for returning atomics (the kernel's flag test), non-returning ones, and
// different CTA shapes. Usage: atoms_ceiling  (prints one line per variant)
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t mix(uint32_t x) {
  x ^= x >> 16; x *= 0x7feb352du; x ^= x >> 15; x *= 0x846ca68bu; x ^= x >> 16;
  return x;
}

// MODE 0: 16-bit returning + flag; 1: 16-bit non-returning; 2: 32-bit non-returning; 3: 32-bit returning
// HOT: 80% of the bins fall in the first 10% of the window (C4's hot span)
template <int MODE, bool HOT>
__global__ void k(uint32_t bins, uint32_t iters, uint32_t* out) {
  extern __shared__ uint32_t tab[];
  const uint32_t words = (MODE <= 1) ? (bins + 1) / 2 : bins;
  for (uint32_t i = threadIdx.x; i < words; i += blockDim.x) tab[i] = 0;
  __syncthreads();
  uint32_t flag = 0, x = mix(blockIdx.x * 4096u + threadIdx.x);
  const uint32_t hot = bins / 10;
  for (uint32_t it = 0; it < iters; it++) {
#pragma unroll
    for (int q = 0; q < 32; q++) {
      x = x * 1664525u + 1013904223u;
      const uint32_t h = mix(x);
      uint32_t off;
      if (HOT) off = (h & 1023u) < 819u ? (h >> 10) % hot : (h >> 10) % bins;
      else off = h % bins;
      if (MODE == 0) {
        const uint32_t inc = 1u << ((off & 1u) << 4);
        flag |= atomicAdd(tab + (off >> 1), inc) & (inc << 15);
      } else if (MODE == 1) {
        atomicAdd(tab + (off >> 1), 1u << ((off & 1u) << 4));
      } else if (MODE == 2) {
        atomicAdd(tab + off, 1u);
      } else {
        flag |= atomicAdd(tab + off, 1u) & 0x80000000u;
      }
    }
  }
  __syncthreads();
  uint32_t s = flag;
  for (uint32_t i = threadIdx.x; i < words; i += blockDim.x) s += tab[i];
  if (s == 0x12345u) out[0] = s;
}

template <int MODE, bool HOT>
void run(const char* name, uint32_t bins, int threads, int ctas_per_sm, int sms, int clk_khz) {
  const uint32_t words = (MODE <= 1) ? (bins + 1) / 2 : bins;
  const size_t smem = words * 4;
  cudaFuncSetAttribute(k<MODE, HOT>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  uint32_t* out;
  cudaMalloc(&out, 64);
  const uint32_t iters = 512;
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  k<MODE, HOT><<<sms * ctas_per_sm, threads, smem>>>(bins, 8, out);
  cudaEventRecord(a);
  k<MODE, HOT><<<sms * ctas_per_sm, threads, smem>>>(bins, iters, out);
  cudaEventRecord(b);
  cudaEventSynchronize(b);
  float ms;
  cudaEventElapsedTime(&ms, a, b);
  const double samples = (double)sms * ctas_per_sm * threads * iters * 32;
  const double clk = ms * 1e-3 * clk_khz * 1e3;
  printf("%-34s bins %6u threads %4d x %d CTA/SM  %7.3f ms  %6.1f G samp/s  %5.2f samp/clk/SM  (%s)\n", name, bins,
         threads, ctas_per_sm, ms, samples / ms / 1e6, samples / clk / sms, cudaGetErrorString(cudaGetLastError()));
  cudaFree(out);
}

int main() {
  int sms = 0, clk = 0;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);
  printf("SMs %d clock %d kHz\n", sms, clk);
  const uint32_t c4 = 4097 * 19;  // a C4 kernel (+1 slot) in compact bins
  run<0, false>("16b ret+flag random", c4, 1024, 1, sms, clk);
  run<0, true>("16b ret+flag hot-span", c4, 1024, 1, sms, clk);
  run<1, false>("16b no-ret random", c4, 1024, 1, sms, clk);
  run<1, true>("16b no-ret hot-span", c4, 1024, 1, sms, clk);
  run<0, false>("16b ret+flag random 512t", c4, 512, 1, sms, clk);
  run<0, false>("16b ret+flag random 2x512", 2048 * 19, 512, 2, sms, clk);
  run<0, false>("16b ret+flag random 2x1024", 2048 * 19, 1024, 2, sms, clk);
  run<1, false>("16b no-ret random 2x1024", 2048 * 19, 1024, 2, sms, clk);
  run<3, false>("32b ret random 1024", 2600 * 19, 1024, 1, sms, clk);
  run<2, false>("32b no-ret random 1024", 2600 * 19, 1024, 1, sms, clk);
  run<2, false>("32b no-ret random 2x1024", 1300 * 19, 1024, 2, sms, clk);
  run<0, false>("16b ret+flag small 4096 bins", 4096, 1024, 1, sms, clk);
  return 0;
}
