// Dev microbenchmark: per-particle 48-B row reduction into scattered rows --
// 3 x red.global.add.v4.f32 per lane vs one cp.reduce.async.bulk .add.f32 of
// 48 B per lane (smem-staged, TMA unit) vs a warp-transposed variant.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/mb_bulkred tools/mb_bulkred.cu
#include <cstdio>
#include <cuda_runtime.h>
__device__ __forceinline__ void red4(float *a, float x) {
  asm volatile("red.global.add.v4.f32 [%0], {%1,%1,%1,%1};" ::"l"(a), "f"(x) : "memory");
}
__device__ __forceinline__ unsigned sptr(const void *p) { return (unsigned)__cvta_generic_to_shared(p); }
__device__ __forceinline__ unsigned hash(unsigned x) {
  x ^= x >> 16; x *= 0x7feb352d; x ^= x >> 15; x *= 0x846ca68b; x ^= x >> 16; return x;
}
// mode 0: 3 red.v4 per lane; mode 1: bulk reduce 48 B per lane; mode 2: mode 1 with
// wait_group.read 0 each iteration (staging slot reuse)
__global__ void k(float *acc, unsigned nrows, int mode, int iters, unsigned spread) {
  __shared__ __align__(16) float stage[256 * 12 * 2];
  const unsigned t = blockIdx.x * blockDim.x + threadIdx.x;
  for (int i = 0; i < iters; ++i) {
    const unsigned r = hash(t * 7919u + i * 104729u) % spread % nrows;
    float *row = acc + 12ull * r;
    if (mode == 0) {
      red4(row, 1.0f); red4(row + 4, 1.0f); red4(row + 8, 1.0f);
    } else {
      float *s = stage + (threadIdx.x * 2 + (i & 1)) * 12;
      if (mode == 2) asm volatile("cp.async.bulk.wait_group.read 1;" ::: "memory");
      else asm volatile("cp.async.bulk.wait_group.read 1;" ::: "memory");
      *reinterpret_cast<float4 *>(s) = make_float4(1.f, 1.f, 1.f, 1.f);
      *reinterpret_cast<float4 *>(s + 4) = make_float4(1.f, 1.f, 1.f, 1.f);
      *reinterpret_cast<float4 *>(s + 8) = make_float4(1.f, 1.f, 1.f, 1.f);
      asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
      asm volatile("cp.reduce.async.bulk.global.shared::cta.bulk_group.add.f32 [%0], [%1], 48;"
                   ::"l"(row), "r"(sptr(s)) : "memory");
      asm volatile("cp.async.bulk.commit_group;" ::: "memory");
    }
  }
  if (mode) asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
}
int main() {
  int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  const unsigned nrows = 2197000;   // C2 voxels: 105 MB accumulator
  float *acc; cudaMalloc(&acc, 12ull * nrows * 4); cudaMemset(acc, 0, 12ull * nrows * 4);
  const int blocks = sms * 4, threads = 256, iters = 400;
  cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
  const char *names[] = {"3x red.v4 / lane", "bulk reduce 48B / lane", "bulk reduce (wait.read 1)"};
  for (unsigned spread : {4096u, 2197000u}) {
    for (int mode = 0; mode < 3; ++mode) {
      k<<<blocks, threads>>>(acc, nrows, mode, 20, spread);
      cudaEventRecord(a);
      k<<<blocks, threads>>>(acc, nrows, mode, iters, spread);
      cudaEventRecord(b); cudaEventSynchronize(b);
      float ms; cudaEventElapsedTime(&ms, a, b);
      const double rows = (double)blocks * threads * iters;
      printf("rows<=%8u %-28s %7.3f ms  %6.2f G rows/s  (%s)\n", spread, names[mode], ms, rows / ms / 1e6,
             cudaGetErrorString(cudaGetLastError()));
    }
  }
  return 0;
}
