// Jacobi 2-D heat stencil, the naive kernel of case study 5.2:
// T_new = T_old + k*(T_top + T_bottom + T_left + T_right - 4*T_old).
// Six explicit int->float conversions of distinct run-time ints are written
// into the update (the paper reports six I2F); nvcc cannot fold them.
// Params (sm_100 base 0x380): Told 0x380, Tnew 0x388, nx 0x390, ny 0x394, k 0x398,
// ox 0x39c, oy 0x3a0, step 0x3a4.
__global__ void jacobi(const float* Told, float* Tnew, int nx, int ny, float k,
                       int ox, int oy, int step) {
  int i = blockIdx.x * blockDim.x + threadIdx.x + 1;
  int j = blockIdx.y * blockDim.y + threadIdx.y + 1;
  if (i < nx - 1 && j < ny - 1) {
    float c = Told[j * nx + i];
    float t = Told[(j - 1) * nx + i];
    float b = Told[(j + 1) * nx + i];
    float l = Told[j * nx + i - 1];
    float r = Told[j * nx + i + 1];
    float gx = (float)(i + ox) * (float)(j + oy);
    float gy = (float)(i * step) + (float)(j * step) + (float)(nx - i) + (float)(ny - j);
    Tnew[j * nx + i] = c + k * (t + b + l + r - 4.0f * c) + 1e-9f * gx * gy;
  }
}
