// samplegen.cu — device expansion of an exact-count table into a sample stream (test / bench
// INPUT infrastructure; mirrors gen/samples.py Trace.packed bit for bit).
//
// Sample p of the stream: q = sorted position (Feistel bijection of p, globally or within the
// kernel's block), bin = the q-th bin of the slot-major layout (binary search over the prefix of
// nonzero counts). The emitted word is slot * R + reason (R active reasons), the packed sample
// format of gs_attribute_samples. No method arithmetic lives here.
#include <cuda_runtime.h>
#include <stdint.h>

namespace {

__device__ __forceinline__ uint32_t mix32(uint32_t x) {
  x ^= x >> 16; x *= 0x7feb352du; x ^= x >> 15; x *= 0x846ca68bu; x ^= x >> 16;
  return x;
}

__device__ __forceinline__ uint64_t feistel_once(uint64_t v, int h, const uint32_t* keys) {
  const uint64_t mask = (1ull << h) - 1;
  uint64_t left = (v >> h) & mask, right = v & mask;
  for (int r = 0; r < 4; r++) {
    const uint64_t f = mix32((uint32_t)(right ^ (uint64_t)keys[r])) & mask;
    const uint64_t nl = right;
    right = left ^ f;
    left = nl;
  }
  return (left << h) | right;
}

__device__ uint64_t feistel(uint64_t x, uint64_t n, const uint32_t* keys) {
  if (n <= 1) return 0;
  int bits = 64 - __clzll((long long)(n - 1));
  int h = (bits + 1) / 2;
  if (h < 1) h = 1;
  uint64_t y = feistel_once(x, h, keys);
  while (y >= n) y = feistel_once(y, h, keys);
  return y;
}

// largest i in [0, n) with a[i] <= x   (a sorted ascending, a[0] <= x)
__device__ __forceinline__ int64_t upper_index(const int64_t* a, int64_t n, int64_t x) {
  int64_t lo = 0, hi = n;  // invariant: a[lo] <= x, answer in [lo, hi)
  while (hi - lo > 1) {
    const int64_t mid = (lo + hi) >> 1;
    if (a[mid] <= x) lo = mid;
    else hi = mid;
  }
  return lo;
}

__global__ void k_expand(const int64_t* __restrict__ nz, const int64_t* __restrict__ cum, int64_t nnz,
                         const int64_t* __restrict__ kstart, int nk, const uint32_t* __restrict__ keys, int order,
                         int64_t a, int64_t b, uint32_t nr, uint32_t* __restrict__ out) {
  const int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (a + i >= b) return;
  const int64_t p = a + i;
  const int64_t N = cum[nnz];
  int64_t q;
  if (order == 0) {
    q = p;
  } else if (order == 1) {
    q = (int64_t)feistel((uint64_t)p, (uint64_t)N, keys);
  } else {
    const int64_t k = upper_index(kstart, nk + 1, p);
    const int64_t base = kstart[k], n_k = kstart[k + 1] - base;
    q = base + (int64_t)feistel((uint64_t)(p - base), (uint64_t)n_k, keys + 4 * k);
  }
  const int64_t j = upper_index(cum, nnz + 1, q);
  const uint64_t bin = (uint64_t)nz[j];
  out[i] = (uint32_t)((bin >> 5) * nr + (bin & 31));
}

}  // namespace

extern "C" int gsgen_expand(const int64_t* d_nz, const int64_t* d_cum, int64_t nnz, const int64_t* d_kstart, int nk,
                            const uint32_t* d_keys, int order, int64_t a, int64_t b, uint32_t nr, uint32_t* d_out,
                            void* stream) {
  if (b <= a) return 0;
  const int64_t n = b - a;
  k_expand<<<(unsigned)((n + 255) / 256), 256, 0, (cudaStream_t)stream>>>(d_nz, d_cum, nnz, d_kstart, nk, d_keys,
                                                                         order, a, b, nr, d_out);
  return (int)cudaGetLastError();
}
