// Conversion probe (paper 4.7): one int->float and one
// double->float conversion.
__global__ void conv(const int* __restrict__ a, const double* __restrict__ d, float* out) {
  int t = threadIdx.x;
  out[t] = (float)a[t] + (float)d[t];
}
