// Dev experiment: the sort's record gather out[j] = in[perm[j]]
// done in an L2-friendly traversal: output rows (y, z) visited y-block by
// y-block, z inside, so that the sources of the rows in flight (their 3x3
// neighbour rows of the pre-sort order) stay within ~3 (YB + 2) rows of L2;
// work items are C-record chunks of rows, taken in traversal order from an
// atomic ticket by persistent CTAs (a small in-flight window).
#include <cstdint>
#include <cuda_runtime.h>

__global__ void k_row_chunks(const int32_t *counts, int sx, int sy, int sz, int YB, int C,
                             int64_t *row_off, int32_t *row_order, int32_t *nchunk) {
  // one thread: traversal order of rows + output offsets + chunk prefix
  if (blockIdx.x || threadIdx.x) return;
  // output offset of each row in voxel order
  int64_t o = 0;
  for (int r = 0; r < sy * sz; ++r) {
    row_off[r] = o;
    const int64_t v0 = (int64_t)r * sx;
    for (int x = 0; x < sx; ++x) o += counts[v0 + x];
  }
  row_off[sy * sz] = o;
  int k = 0;
  int64_t ch = 0;
  for (int yb = 0; yb < sy; yb += YB)
    for (int z = 0; z < sz; ++z)
      for (int y = yb; y < yb + YB && y < sy; ++y) {
        const int r = y + sy * z;
        row_order[k] = r;
        nchunk[k] = (int32_t)ch;
        ch += (row_off[r + 1] - row_off[r] + C - 1) / C;
        ++k;
      }
  nchunk[k] = (int32_t)ch;
}

__global__ void __launch_bounds__(256) k_gather_ordered(const float4 *__restrict__ src, float4 *__restrict__ dst,
                                                         const int64_t *__restrict__ perm,
                                                         const int64_t *__restrict__ row_off,
                                                         const int32_t *__restrict__ row_order,
                                                         const int32_t *__restrict__ nchunk, int nrows, int C,
                                                         unsigned *ticket) {
  __shared__ unsigned t;
  const int total = nchunk[nrows];
  while (true) {
    if (threadIdx.x == 0) t = atomicAdd(ticket, 1u);
    __syncthreads();
    const int tk = (int)t;
    __syncthreads();
    if (tk >= total) return;
    // row k with nchunk[k] <= tk < nchunk[k+1]
    int lo = 0, hi = nrows;
    while (hi - lo > 1) {
      const int mid = (lo + hi) >> 1;
      if (nchunk[mid] <= tk) lo = mid; else hi = mid;
    }
    const int r = row_order[lo];
    const int64_t b = row_off[r] + (int64_t)(tk - nchunk[lo]) * C;
    const int64_t e = min(b + C, row_off[r + 1]);
    for (int64_t h = 2 * b + threadIdx.x; h < 2 * e; h += blockDim.x) {
      const int64_t j = h >> 1;
      const float4 *a = src + 2 * perm[j] + (h & 1);
      float4 v;
      asm volatile("ld.global.nc.L2::64B.v4.f32 {%0,%1,%2,%3}, [%4];" : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w) : "l"(a));
      __stcs(dst + h, v);
    }
  }
}

extern "C" int gather_prep(const int32_t *counts, int sx, int sy, int sz, int YB, int C, void *scratch,
                           cudaStream_t s) {
  char *w = static_cast<char *>(scratch);
  int64_t *row_off = reinterpret_cast<int64_t *>(w);
  int32_t *row_order = reinterpret_cast<int32_t *>(w + 8 * (size_t)(sy * sz + 1));
  int32_t *nchunk = row_order + (sy * sz + 1);
  k_row_chunks<<<1, 1, 0, s>>>(counts, sx, sy, sz, YB, C, row_off, row_order, nchunk);
  return (int)cudaGetLastError();
}

extern "C" int gather_run(const void *src, void *dst, const int64_t *perm, int sx, int sy, int sz, int C,
                          void *scratch, int blocks, cudaStream_t s) {
  char *w = static_cast<char *>(scratch);
  int64_t *row_off = reinterpret_cast<int64_t *>(w);
  int32_t *row_order = reinterpret_cast<int32_t *>(w + 8 * (size_t)(sy * sz + 1));
  int32_t *nchunk = row_order + (sy * sz + 1);
  unsigned *ticket = reinterpret_cast<unsigned *>(nchunk + (sy * sz + 1));
  cudaMemsetAsync(ticket, 0, 4, s);
  k_gather_ordered<<<blocks, 256, 0, s>>>(static_cast<const float4 *>(src), static_cast<float4 *>(dst), perm,
                                          row_off, row_order, nchunk, sy * sz, C, ticket);
  return (int)cudaGetLastError();
}
