// Register-spill probe (SURVEY [probe 5]): 48 live values that a register cap
// forces into local memory. Compiled at -maxrregcount 24/32/40/64; ptxas -v
// reports "N bytes spill stores, M bytes spill loads" for each cap.
__global__ void spill48(const float* __restrict__ in, float* out, int n) {
  int t = blockIdx.x * blockDim.x + threadIdx.x;
  float v[48];
#pragma unroll
  for (int k = 0; k < 48; k++) v[k] = in[t + k * n];
  for (int it = 0; it < n; it++) {
#pragma unroll
    for (int k = 0; k < 48; k++) v[k] = v[k] * v[(k + 7) % 48] + v[(k + 13) % 48];
  }
  float s = 0.f;
#pragma unroll
  for (int k = 0; k < 48; k++) s += v[k] * (float)(k + 1);
  out[t] = s;
}
