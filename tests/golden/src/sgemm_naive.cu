// Naive SGEMM, the starting point of the paper's case study 5.3:
// one thread computes one element of C <- alpha*A*B + beta*C.
// Params (sm_100 param base 0x380): M 0x380, N 0x384, K 0x388, alpha 0x38c,
// A 0x390, B 0x398, beta 0x3a0, C 0x3a8.
__global__ void sgemm_naive(int M, int N, int K, float alpha, const float* A,
                            const float* B, float beta, float* C) {
  int x = blockIdx.x * blockDim.x + threadIdx.x;
  int y = blockIdx.y * blockDim.y + threadIdx.y;
  if (x < M && y < N) {
    float tmp = 0.0f;
    for (int i = 0; i < K; ++i) tmp += A[x * K + i] * B[i * N + y];
    C[x * N + y] = alpha * tmp + beta * C[x * N + y];
  }
}
