// Accuracy of sqrt.approx.f32 (MUFU.SQRT) on sm_100a: exhaustive over all positive
// normal floats, max error in ulps of the correctly rounded result.
#include <cstdio>
#include <cstdint>
#include <cmath>
#include <cuda_runtime.h>
__global__ void k(unsigned *maxulp, unsigned long long *n_ne, uint32_t lo, uint32_t hi) {
  uint32_t b = lo + blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
  if (b >= hi) return;
  float x = __uint_as_float(b), a, r = __fsqrt_rn(x);
  asm("sqrt.approx.f32 %0, %1;" : "=f"(a) : "f"(x));
  int d = (int)__float_as_uint(a) - (int)__float_as_uint(r);
  unsigned ad = d < 0 ? -d : d;
  if (ad) { atomicMax(maxulp, ad); atomicAdd(n_ne, 1ull); }
}
int main() {
  unsigned *m; unsigned long long *n; cudaMalloc(&m, 4); cudaMalloc(&n, 8);
  cudaMemset(m, 0, 4); cudaMemset(n, 0, 8);
  uint32_t lo = 0x00800000u, hi = 0x7f800000u;
  k<<<(hi - lo + 255) / 256, 256>>>(m, n, lo, hi);
  unsigned hm; unsigned long long hn; cudaMemcpy(&hm, m, 4, cudaMemcpyDeviceToHost); cudaMemcpy(&hn, n, 8, cudaMemcpyDeviceToHost);
  printf("sqrt.approx.f32 vs correctly rounded over %u normal floats: max %u ulp, %llu differ\n", hi - lo, hm, hn);
  return 0;
}
