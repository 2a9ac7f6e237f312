// Dev microbenchmark: L1/L2 cost of red.global.add patterns on B200.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/mb_red tools/mb_red.cu && /tmp/mb_red
#include <cstdio>
#include <cuda_runtime.h>
__device__ __forceinline__ void red4(float *a, float x) {
  asm volatile("red.global.add.v4.f32 [%0], {%1,%1,%1,%1};" ::"l"(a), "f"(x) : "memory");
}
__device__ __forceinline__ void red1(float *a, float x) {
  asm volatile("red.global.add.f32 [%0], %1;" ::"l"(a), "f"(x) : "memory");
}
// byte offset of lane's target inside the warp's 1 KB window, per pattern
__device__ __forceinline__ int off(int pat, int lane) {
  switch (pat) {
    case 0: return lane * 32;                         // v4, one lane per sector
    case 1: return (lane >> 1) * 32 + (lane & 1) * 16; // v4, two lanes per sector (full sector)
    case 2: return lane * 16;                         // v4, fully coalesced (512 B)
    case 3: return 0;                                 // v4, all lanes one address
    case 4: return lane * 32;                         // f32, one lane per sector
    case 5: return lane * 4;                          // f32, coalesced (128 B)
    case 6: return (lane >> 1) * 32 * 2 + (lane & 1) * 16; // v4, pairs but every other sector
    case 7: return (lane & 15) * 32;                  // v4, two lanes per sector, same 16 B
    case 8: return lane * 1024 * 37;                  // v4, one lane per line, scattered
    case 9: return (lane >> 1) * 1024 * 37 + (lane & 1) * 16;  // v4, lane pairs fill a sector, scattered
    case 10: return (lane >> 1) * 1024 * 37 + (lane & 1) * 32; // v4, lane pairs in one line, 2 sectors
    default: return (lane >> 2) * 1024 * 37 + (lane & 3) * 16; // v4, 4 lanes fill 2 sectors of a line
  }
}
__global__ void k(float *buf, size_t nwin, int pat, int iters) {
  const int lane = threadIdx.x & 31;
  const size_t gw = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const size_t GW = (gridDim.x * blockDim.x) >> 5;
  const int o = off(pat, lane);
  size_t w = gw;
  for (int i = 0; i < iters; ++i) {
    char *p = (char *)buf + ((w % nwin) * 1024 + o) % (nwin * 1024);
    if (pat >= 4 && pat <= 5) red1((float *)p, 1.0f); else red4((float *)p, 1.0f);
    w += GW;
  }
}
int main() {
  int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  const size_t bytes = 32ull << 20;
  float *buf; cudaMalloc(&buf, bytes); cudaMemset(buf, 0, bytes);
  const size_t nwin = bytes / 1024;
  const int iters = 2000, blocks = sms * 4, threads = 512;
  const char *names[] = {"v4 1lane/sector", "v4 2lanes/sector", "v4 coalesced", "v4 same addr",
                         "f32 1lane/sector", "f32 coalesced", "v4 pairs sparse", "v4 2lanes same16B",
                         "v4 scattered 1/line", "v4 scat pairs/sector", "v4 scat pairs/line", "v4 scat 4/line"};
  cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
  for (int pat = 0; pat < 12; ++pat) {
    k<<<blocks, threads>>>(buf, nwin, pat, 50);
    cudaEventRecord(a);
    k<<<blocks, threads>>>(buf, nwin, pat, iters);
    cudaEventRecord(b); cudaEventSynchronize(b);
    float ms; cudaEventElapsedTime(&ms, a, b);
    const double winst = (double)blocks * threads / 32 * iters;
    const double per_sm = winst / sms;
    printf("%-22s %8.3f ms  %6.2f ns/warp-instr/SM  %6.2f cyc@1.9GHz/warp-instr/SM\n", names[pat], ms,
           ms * 1e6 / per_sm, ms * 1e6 / per_sm * 1.9);
  }
  return 0;
}
