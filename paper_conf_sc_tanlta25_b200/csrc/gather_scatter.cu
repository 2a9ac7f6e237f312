// Gather-scatter microbenchmark of the paper's sorting study (PAPER.md:236-242,
// Figs. 5-6, reading F2): for each element i with key
// k = keys[i], gather table[] over the access set ({k}, or the 5-point stencil
// {k, k-1, k+1, k-nx, k+nx} mod nkeys) into out[i] and scatter-add x[i] into
// acc[] over the same set.  FP64.  Two scatter strategies: per-lane
// red.global.add.f64 (the paper's atomic scatter) or warp-aggregated (lanes
// holding the same key summed with shuffles, one atomic per distinct key).
#include "vpic_internal.cuh"

namespace vpic {
namespace {

constexpr unsigned FULL = 0xffffffffu;

__device__ __forceinline__ void red_add_f64(double *a, double v) {
  asm volatile("red.global.add.f64 [%0], %1;" ::"l"(a), "d"(v) : "memory");
}

__device__ __forceinline__ int64_t wrap(int64_t k, int64_t n) {
  return k < 0 ? k + n : (k >= n ? k - n : k);
}

template <bool AGG, bool STENCIL>
__global__ void __launch_bounds__(256)
k_gather_scatter(const int32_t *__restrict__ keys, const double *__restrict__ x, int64_t n,
                 const double *__restrict__ table, double *__restrict__ out,
                 double *__restrict__ acc, int64_t nkeys, int64_t nx) {
  const int lane = threadIdx.x & 31;
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  constexpr int NP = STENCIL ? 5 : 1;
  for (int64_t base = (int64_t)blockIdx.x * blockDim.x + (threadIdx.x & ~31); base < n;
       base += stride) {
    const int64_t i = base + lane;
    const bool valid = i < n;
    const int64_t k = valid ? (int64_t)__ldcs(keys + i) : 0;
    const double xv = valid ? __ldcs(x + i) : 0.0;
    int64_t set[NP];
    set[0] = k;
    if (STENCIL) {
      set[1] = wrap(k - 1, nkeys);
      set[2] = wrap(k + 1, nkeys);
      set[3] = wrap(k - nx % nkeys, nkeys);
      set[4] = wrap(k + nx % nkeys, nkeys);
    }
    double s = 0.0;
#pragma unroll
    for (int j = 0; j < NP; ++j) s += __ldg(table + set[j]);
    if (valid) __stcs(out + i, s);
#pragma unroll
    for (int j = 0; j < NP; ++j) {
      if (!AGG) {
        if (valid) red_add_f64(acc + set[j], xv);
      } else {
        const long long key = valid ? (long long)set[j] : -1 - lane;
        const unsigned peers = __match_any_sync(FULL, key);
        double sum = 0.0;
#pragma unroll 4
        for (int src = 0; src < 32; ++src) {
          const double v = __shfl_sync(FULL, xv, src);
          if ((peers >> src) & 1u) sum += v;
        }
        if (valid && (__ffs(peers) - 1) == lane) red_add_f64(acc + set[j], sum);
      }
    }
  }
}

}  // namespace

cudaError_t launch_gather_scatter(const vpic_ctx *c, const int32_t *keys, const double *x,
                                  int64_t n, const double *table, double *out, double *acc,
                                  int64_t nkeys, int64_t nx, int aggregate, cudaStream_t s) {
  if (n <= 0) return cudaSuccess;
  int64_t blocks = (n + 255) / 256;
  const int64_t cap = (int64_t)c->num_sms * 8;
  if (blocks > cap) blocks = cap;
  const unsigned b = (unsigned)blocks;
  if (nx > 0) {
    if (aggregate) k_gather_scatter<true, true><<<b, 256, 0, s>>>(keys, x, n, table, out, acc, nkeys, nx);
    else k_gather_scatter<false, true><<<b, 256, 0, s>>>(keys, x, n, table, out, acc, nkeys, nx);
  } else {
    if (aggregate) k_gather_scatter<true, false><<<b, 256, 0, s>>>(keys, x, n, table, out, acc, nkeys, nx);
    else k_gather_scatter<false, false><<<b, 256, 0, s>>>(keys, x, n, table, out, acc, nkeys, nx);
  }
  note_launch();
  return cudaGetLastError();
}

}  // namespace vpic
