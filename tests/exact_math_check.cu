// Exhaustive check of csrc/exact_math.cuh against the CUDA library's
// correctly rounded __frcp_rn(__fsqrt_rn(x)): every float in [1, 2^26) and
// 2^28 pseudo-random floats in [2^26, 3.4e38).  Prints the mismatch count.
#include <cstdio>
#include <cstdint>
#include "../paper_conf_sc_tanlta25_b200/csrc/exact_math.cuh"

__global__ void check(uint32_t lo, uint32_t n, int random, unsigned long long *bad) {
  for (uint32_t k = blockIdx.x * blockDim.x + threadIdx.x; k < n; k += gridDim.x * blockDim.x) {
    uint32_t bits;
    if (random) {
      uint64_t h = (uint64_t)k * 0x9E3779B97F4A7C15ull;
      h ^= h >> 29; h *= 0xBF58476D1CE4E5B9ull; h ^= h >> 32;
      bits = 0x4c800000u + (uint32_t)(h % (0x7f7fffffu - 0x4c800000u));   // [2^26, FLT_MAX]
    } else {
      bits = lo + k;
    }
    const float x = __uint_as_float(bits);
    const float a = vpic::rsqrt_rn2(x), b = __frcp_rn(__fsqrt_rn(x));
    const float s1 = vpic::sqrt_rn_normal(x), s2 = __fsqrt_rn(x);
    if (__float_as_uint(a) != __float_as_uint(b) || __float_as_uint(s1) != __float_as_uint(s2))
      atomicAdd(bad, 1ull);
  }
}

int main() {
  unsigned long long *bad, h = 0;
  cudaMalloc(&bad, 8);
  cudaMemset(bad, 0, 8);
  const uint32_t lo = 0x3f800000u, hi = 0x4c800000u;   // [1, 2^26)
  check<<<148 * 8, 256>>>(lo, hi - lo, 0, bad);
  check<<<148 * 8, 256>>>(0, 1u << 28, 1, bad);
  cudaMemcpy(&h, bad, 8, cudaMemcpyDeviceToHost);
  cudaError_t e = cudaDeviceSynchronize();
  printf("checked %u + %u floats, mismatches %llu, %s\n", hi - lo, 1u << 28, h, cudaGetErrorString(e));
  return (h == 0 && e == cudaSuccess) ? 0 : 1;
}
