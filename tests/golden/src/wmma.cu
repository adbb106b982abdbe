// wmma 16x16x16 half -> f32 (HMMA.16816.F32, LDSM.16.M88.4, CS2R pairs): register-fragment widths (R38b/c)
#include <mma.h>
#include <cuda_fp16.h>
using namespace nvcuda;
__global__ void wmma_gemm(const half* __restrict__ A, const half* __restrict__ B, float* C, int K) {
  wmma::fragment<wmma::matrix_a, 16, 16, 16, half, wmma::row_major> a;
  wmma::fragment<wmma::matrix_b, 16, 16, 16, half, wmma::col_major> b;
  wmma::fragment<wmma::accumulator, 16, 16, 16, float> c;
  wmma::fill_fragment(c, 0.0f);
  __shared__ half sa[16 * 16], sb[16 * 16];
  for (int k = 0; k < K; k += 16) {
    for (int i = threadIdx.x; i < 256; i += 32) { sa[i] = A[k * 16 + i]; sb[i] = B[k * 16 + i]; }
    __syncthreads();
    wmma::load_matrix_sync(a, sa, 16);
    wmma::load_matrix_sync(b, sb, 16);
    wmma::mma_sync(c, a, b, c);
    __syncthreads();
  }
  wmma::store_matrix_sync(C + blockIdx.x * 256, c, 16, wmma::mem_row_major);
}
