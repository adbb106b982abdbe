// Microbenchmark: sorting ~90K (key u64 of ~38 significant bits, value u32) pairs, as the rank
// step does: CUB onesweep radix sort over 40 bits vs CUB stable merge sort.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o sort_mb sort_mb.cu
#include <cub/device/device_merge_sort.cuh>
#include <cub/device/device_radix_sort.cuh>
#include <cstdio>
#include <cstdint>
#include <vector>
#include <random>
struct Less { __device__ bool operator()(unsigned long long a, unsigned long long b) const { return a < b; } };
int main() {
  for (int n : {90000, 300000, 1000000}) {
    std::vector<unsigned long long> hk(n); std::vector<uint32_t> hv(n);
    std::mt19937_64 rng(1);
    for (int i = 0; i < n; i++) { hk[i] = rng() & ((1ull << 38) - 1); hv[i] = i; }
    unsigned long long *k0, *k1; uint32_t *v0, *v1;
    cudaMalloc(&k0, n * 8); cudaMalloc(&k1, n * 8); cudaMalloc(&v0, n * 4); cudaMalloc(&v1, n * 4);
    cudaStream_t st; cudaStreamCreateWithFlags(&st, cudaStreamNonBlocking);
    size_t tb = 0, tm = 0;
    cub::DeviceRadixSort::SortPairs(nullptr, tb, k0, k1, v0, v1, n, 0, 40, st);
    cub::DeviceMergeSort::StableSortPairs(nullptr, tm, k0, v0, n, Less(), st);
    void* tmp; cudaMalloc(&tmp, tb > tm ? tb : tm);
    cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
    auto run = [&](int which) {
      cudaMemcpyAsync(k0, hk.data(), n * 8, cudaMemcpyHostToDevice, st);
      cudaMemcpyAsync(v0, hv.data(), n * 4, cudaMemcpyHostToDevice, st);
      cudaEventRecord(a, st);
      size_t t1 = tb, t2 = tm;
      if (which == 0) cub::DeviceRadixSort::SortPairs(tmp, t1, k0, k1, v0, v1, n, 0, 40, st);
      else cub::DeviceMergeSort::StableSortPairs(tmp, t2, k0, v0, n, Less(), st);
      cudaEventRecord(b, st);
      cudaStreamSynchronize(st);
      float ms; cudaEventElapsedTime(&ms, a, b); return ms;
    };
    for (int w = 0; w < 2; w++) { float t[2] = {0, 0}; for (int r = 0; r < 20; r++) { t[0] += run(0); t[1] += run(1); }
      if (w) printf("n=%d radix(40 bits) %.1f us  merge %.1f us\n", n, t[0] / 20 * 1e3, t[1] / 20 * 1e3); }
    cudaFree(k0); cudaFree(k1); cudaFree(v0); cudaFree(v1); cudaFree(tmp);
  }
  return 0;
}
