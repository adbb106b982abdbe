// Atomics probe (paper 4.4): a shared-memory atomic and a global
// atomic inside a loop, and one more global atomic after it.
__global__ void atomics(const int* __restrict__ keys, int* gcount, int* gtotal, int n) {
  __shared__ int scount[256];
  scount[threadIdx.x] = 0;
  __syncthreads();
  int local = 0;
  for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x) {
    int k = keys[i];
    atomicAdd(&scount[k & 255], 1);
    atomicAdd(&gcount[k & 1023], 1);
    local += k;
  }
  __syncthreads();
  atomicAdd(gtotal, local + scount[threadIdx.x]);
}
