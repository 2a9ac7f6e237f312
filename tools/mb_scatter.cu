// Dev microbenchmark: move 32-B records by gather (out[j] = in[perm[j]]) or
// scatter (out[inv[i]] = in[i]), and invert a permutation; two lanes per
// record like the product's k_gather.  Built by tools/gather_vs_scatter.py.
#include <cstdint>
#include <cuda_runtime.h>

__global__ void k_gather(const float4 *in, float4 *out, const int64_t *perm, int64_t n) {
  for (int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; t < 2 * n; t += (int64_t)gridDim.x * blockDim.x)
    __stcs(out + t, __ldg(in + 2 * perm[t >> 1] + (t & 1)));
}
__global__ void k_scatter(const float4 *in, float4 *out, const int64_t *inv, int64_t n) {
  for (int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; t < 2 * n; t += (int64_t)gridDim.x * blockDim.x)
    out[2 * __ldcs(inv + (t >> 1)) + (t & 1)] = __ldcs(in + t);
}
__global__ void k_invert(const int64_t *perm, int64_t *inv, int64_t n) {
  for (int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; t < n; t += (int64_t)gridDim.x * blockDim.x)
    inv[__ldcs(perm + t)] = t;
}
extern "C" void mb_gather(const void *in, void *out, const int64_t *perm, int64_t n) {
  k_gather<<<148 * 8, 256>>>((const float4 *)in, (float4 *)out, perm, n);
}
extern "C" void mb_scatter(const void *in, void *out, const int64_t *inv, int64_t n) {
  k_scatter<<<148 * 8, 256>>>((const float4 *)in, (float4 *)out, inv, n);
}
extern "C" void mb_invert(const int64_t *perm, int64_t *inv, int64_t n) {
  k_invert<<<148 * 8, 256>>>(perm, inv, n);
}
