// Checks that Markstein's correction  y = RN(1/d), q0 = RN(a*y), r = fma(-q0, d, a),
// q = fma(r, y, q0)  reproduces the IEEE quotient RN(a/d) bit for bit on random
// operands (the TRSM/POTRF solves use it to take the division off the serial chain).
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>
__device__ uint64_t mix(uint64_t x) {
  x += 0x9E3779B97F4A7C15ull; uint64_t z = (x ^ (x >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull; return z ^ (z >> 31);
}
__global__ void k(unsigned long long* bad, unsigned long long n, int mode) {
  for (unsigned long long i = blockIdx.x * (unsigned long long)blockDim.x + threadIdx.x; i < n;
       i += (unsigned long long)gridDim.x * blockDim.x) {
    uint64_t h1 = mix(2 * i), h2 = mix(2 * i + 1);
    double a, d;
    if (mode == 0) {  // uniform mantissas, exponents in [-20, 20]
      a = __longlong_as_double((long long)((h1 & 0x000FFFFFFFFFFFFFull) | ((uint64_t)(1023 + (int)(h1 >> 58) - 20 + (int)((h1 >> 52) & 7)) << 52)));
      d = __longlong_as_double((long long)((h2 & 0x000FFFFFFFFFFFFFull) | ((uint64_t)(1023 + (int)(h2 >> 58) - 20) << 52)));
      if (h1 & (1ull << 57)) a = -a;
    } else {  // values like the solves see: a in (-2, 2), d in [0.5, 200]
      a = 4.0 * ((h1 >> 11) * 0x1.0p-53) - 2.0;
      d = 0.5 + 199.5 * ((h2 >> 11) * 0x1.0p-53);
    }
    double y = 1.0 / d;
    double q0 = a * y;
    double r = fma(-q0, d, a);
    double q = fma(r, y, q0);
    double ref = a / d;
    if (__double_as_longlong(q) != __double_as_longlong(ref)) atomicAdd(bad, 1ull);
  }
}
int main() {
  unsigned long long* bad; cudaMallocManaged(&bad, 8);
  for (int mode = 0; mode < 2; ++mode) {
    *bad = 0;
    unsigned long long n = 1ull << 32;
    k<<<148 * 16, 256>>>(bad, n, mode);
    cudaDeviceSynchronize();
    printf("mode %d: %llu mismatches of %llu\n", mode, *bad, n);
  }
  return 0;
}
