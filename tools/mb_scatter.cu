// Dev microbenchmark: move 32-B records by gather (out[j] = in[perm[j]]) or
// scatter (out[inv[i]] = in[i]), and invert a permutation; two lanes per
// record like the product's k_gather.  Built by tools/gather_vs_scatter.py.
#include <cstdint>
#include <cuda_runtime.h>

__global__ void k_gather(const float4 *in, float4 *out, const int64_t *perm, int64_t n) {
  for (int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; t < 2 * n; t += (int64_t)gridDim.x * blockDim.x)
    __stcs(out + t, __ldg(in + 2 * perm[t >> 1] + (t & 1)));
}
template <int V>
__device__ __forceinline__ float4 ldv(const float4 *p) {
  float4 r;
  if (V == 1)
    asm volatile("ld.global.nc.L2::64B.v4.f32 {%0,%1,%2,%3}, [%4];" : "=f"(r.x), "=f"(r.y), "=f"(r.z), "=f"(r.w) : "l"(p));
  else if (V == 2)
    asm volatile("ld.global.nc.L1::no_allocate.v4.f32 {%0,%1,%2,%3}, [%4];" : "=f"(r.x), "=f"(r.y), "=f"(r.z), "=f"(r.w) : "l"(p));
  else if (V == 3)
    asm volatile("ld.global.nc.L2::128B.v4.f32 {%0,%1,%2,%3}, [%4];" : "=f"(r.x), "=f"(r.y), "=f"(r.z), "=f"(r.w) : "l"(p));
  else if (V == 4)
    asm volatile("ld.global.cg.v4.f32 {%0,%1,%2,%3}, [%4];" : "=f"(r.x), "=f"(r.y), "=f"(r.z), "=f"(r.w) : "l"(p));
  else
    r = __ldg(p);
  return r;
}
template <int V>
__global__ void k_gatherv(const float4 *in, float4 *out, const int64_t *perm, int64_t n) {
  for (int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; t < 2 * n; t += (int64_t)gridDim.x * blockDim.x)
    __stcs(out + t, ldv<V>(in + 2 * perm[t >> 1] + (t & 1)));
}
extern "C" void mb_gatherv(int v, const void *in, void *out, const int64_t *perm, int64_t n) {
  const float4 *i = (const float4 *)in;
  float4 *o = (float4 *)out;
  if (v == 1) k_gatherv<1><<<148 * 8, 256>>>(i, o, perm, n);
  else if (v == 2) k_gatherv<2><<<148 * 8, 256>>>(i, o, perm, n);
  else if (v == 3) k_gatherv<3><<<148 * 8, 256>>>(i, o, perm, n);
  else if (v == 4) k_gatherv<4><<<148 * 8, 256>>>(i, o, perm, n);
  else k_gatherv<0><<<148 * 8, 256>>>(i, o, perm, n);
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
