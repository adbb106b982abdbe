// tcgen05 tensor-memory round trip: LDTM / STTM register quads on sm_100a
#include <cstdint>
__global__ void tmem_roundtrip(const float* __restrict__ in, float* out) {
  __shared__ uint32_t taddr_s;
  const uint32_t sa = (uint32_t)__cvta_generic_to_shared(&taddr_s);
  if (threadIdx.x < 32) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 32;" :: "r"(sa));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  __syncthreads();
  const uint32_t t = taddr_s;
  if (threadIdx.x < 32) {
    uint32_t v[8];
    for (int i = 0; i < 8; i++) v[i] = __float_as_uint(in[threadIdx.x * 8 + i] * 2.0f);
    asm volatile("tcgen05.st.sync.aligned.32x32b.x8.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8};"
                 :: "r"(t), "r"(v[0]), "r"(v[1]), "r"(v[2]), "r"(v[3]), "r"(v[4]), "r"(v[5]), "r"(v[6]), "r"(v[7]));
    asm volatile("tcgen05.wait::st.sync.aligned;");
    uint32_t a[16];
    asm volatile("tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%16];"
                 : "=r"(a[0]), "=r"(a[1]), "=r"(a[2]), "=r"(a[3]), "=r"(a[4]), "=r"(a[5]), "=r"(a[6]), "=r"(a[7]),
                   "=r"(a[8]), "=r"(a[9]), "=r"(a[10]), "=r"(a[11]), "=r"(a[12]), "=r"(a[13]), "=r"(a[14]), "=r"(a[15])
                 : "r"(t));
    uint32_t b[8];
    asm volatile("tcgen05.ld.sync.aligned.16x256b.x2.b32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
                 : "=r"(b[0]), "=r"(b[1]), "=r"(b[2]), "=r"(b[3]), "=r"(b[4]), "=r"(b[5]), "=r"(b[6]), "=r"(b[7]) : "r"(t));
    asm volatile("tcgen05.wait::ld.sync.aligned;");
    float s = 0.f;
    for (int i = 0; i < 16; i++) s += __uint_as_float(a[i]) * (float)(i + 1);
    for (int i = 0; i < 8; i++) s += __uint_as_float(b[i]);
    out[threadIdx.x] = s;
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 32;" :: "r"(t));
  }
}
