// On-line charge-conservation diagnostics (second half):
// cloud-in-cell charge on the nodes (VPIC accumulate_rho_p, ref. [3]) and the
// discrete continuity residual  drho/dt + div J  that the charge-conserving
// deposit of P:238 makes zero to round-off (BASELINE.json north_star: "the
// discrete continuity invariant").  Compiled without FMA contraction.
#include "vpic_internal.cuh"

namespace vpic {
namespace {

constexpr unsigned FULL = 0xffffffffu;

struct Per {
  int px, py, pz;
};

__device__ __forceinline__ void red_f32(float *a, float x) {
  asm volatile("red.global.add.f32 [%0], %1;" ::"l"(a), "f"(x) : "memory");
}

// Node of corner k (bit 0: +x, bit 1: +y, bit 2: +z) of voxel (x, y, z); the
// n+1 node of a locally periodic axis is node 1 (reading D1).
__device__ __forceinline__ int64_t corner_node(const GridK &g, const Per &per, int x, int y, int z,
                                               int k) {
  int cx = x + (k & 1), cy = y + ((k >> 1) & 1), cz = z + ((k >> 2) & 1);
  if (per.px && cx == g.nx + 1) cx = 1;
  if (per.py && cy == g.ny + 1) cy = 1;
  if (per.pz && cz == g.nz + 1) cz = 1;
  return cx + (int64_t)g.sx * (cy + (int64_t)g.sy * cz);
}

// rho[node] += q w (1 +- dx)(1 +- dy)(1 +- dz) / 8 over the 8 nodes of the
// particle's voxel.  One particle per thread; lanes sharing a voxel (sorted
// particles) are summed with a transposing butterfly first (lanes 4k..4k+3
// end with corner k), other lanes issue 8 red.global.add.f32.
__global__ void __launch_bounds__(256)
k_accumulate_rho(const __grid_constant__ GridK g, const Per per, const float q,
                 const float4 *__restrict__ p, const int64_t np, float *__restrict__ rho) {
  const int lane = threadIdx.x & 31;
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  const int64_t nround = (np + 31) / 32 * 32;
  for (int64_t n = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; n < nround; n += stride) {
    const bool valid = n < np;
    float4 a = make_float4(0.f, 0.f, 0.f, 0.f), b = a;
    if (valid) {
      a = __ldg(p + 2 * n);
      b = __ldg(p + 2 * n + 1);
    }
    const int v = valid ? __float_as_int(a.w) : -1 - lane;
    const float qw8 = (q * b.w) * 0.125f;
    const float wx[2] = {1.0f - a.x, 1.0f + a.x};
    const float wy[2] = {1.0f - a.y, 1.0f + a.y};
    const float wz[2] = {1.0f - a.z, 1.0f + a.z};
    float c[8];
#pragma unroll
    for (int k = 0; k < 8; ++k) c[k] = valid ? ((qw8 * wx[k & 1]) * wy[(k >> 1) & 1]) * wz[k >> 2] : 0.0f;
    const unsigned peers = __match_any_sync(FULL, v);
    const bool big = valid && __popc(peers) >= 4;
    bool done = !valid;
    while (true) {
      const unsigned bal = __ballot_sync(FULL, big && !done);
      if (!bal) break;
      const int seg = __shfl_sync(FULL, v, __ffs(bal) - 1);
      const bool in = !done && v == seg;
      float s[8];
#pragma unroll
      for (int k = 0; k < 8; ++k) s[k] = in ? c[k] : 0.0f;
#pragma unroll
      for (int half = 4, bit = 16; half >= 1; half >>= 1, bit >>= 1) {
        const bool hi = lane & bit;
#pragma unroll
        for (int k = 0; k < half; ++k) {
          const float send = hi ? s[k] : s[k + half];
          const float keep = hi ? s[k + half] : s[k];
          s[k] = keep + __shfl_xor_sync(FULL, send, bit);
        }
      }
      s[0] += __shfl_xor_sync(FULL, s[0], 2);
      s[0] += __shfl_xor_sync(FULL, s[0], 1);
      if ((lane & 3) == 0) {
        const int x = seg % g.sx, y = (seg / g.sx) % g.sy, z = seg / g.sxy;
        red_f32(rho + corner_node(g, per, x, y, z, (lane >> 2) & 7), s[0]);
      }
      done |= in;
    }
    if (!done) {
      const int x = v % g.sx, y = (v / g.sx) % g.sy, z = v / g.sxy;
#pragma unroll
      for (int k = 0; k < 8; ++k) red_f32(rho + corner_node(g, per, x, y, z, k), c[k]);
    }
  }
}

__device__ __forceinline__ void atomic_max_nonneg(float *a, float x) {
  atomicMax(reinterpret_cast<unsigned *>(a), __float_as_uint(x));  // x >= 0: uint order = float order
}

// res = (rho1 - rho0) / (dV dt) + sum_a (j_a(node) - j_a(node - e_a)) / d_a on
// the nodes 1..n (locally periodic axis, node - e_a wraps to n) or 1..n+1;
// out[0] = max |res|, out[1] = max |drho/dt| (the scale).
__global__ void __launch_bounds__(256)
k_continuity(const __grid_constant__ GridK g, const Per per, const float inv_vdt, const float idx,
             const float idy, const float idz, const float *__restrict__ rho0,
             const float *__restrict__ rho1, const float4 *__restrict__ jf, float *__restrict__ out,
             float *__restrict__ res) {
  const int ex = g.nx + (per.px ? 0 : 1), ey = g.ny + (per.py ? 0 : 1), ez = g.nz + (per.pz ? 0 : 1);
  const int64_t total = (int64_t)ex * ey * ez;
  float rmax = 0.0f, smax = 0.0f;
  for (int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; t < total;
       t += (int64_t)gridDim.x * blockDim.x) {
    const int x = 1 + (int)(t % ex), y = 1 + (int)((t / ex) % ey), z = 1 + (int)(t / ((int64_t)ex * ey));
    const int xm = (per.px && x == 1) ? g.nx : x - 1;
    const int ym = (per.py && y == 1) ? g.ny : y - 1;
    const int zm = (per.pz && z == 1) ? g.nz : z - 1;
    auto V = [&](int X, int Y, int Z) -> int64_t { return X + (int64_t)g.sx * (Y + (int64_t)g.sy * Z); };
    const int64_t v = V(x, y, z);
    const float4 j0 = jf[v];
    const float drho = (rho1[v] - rho0[v]) * inv_vdt;
    const float div = (j0.x - jf[V(xm, y, z)].x) * idx + (j0.y - jf[V(x, ym, z)].y) * idy +
                      (j0.z - jf[V(x, y, zm)].z) * idz;
    const float r = drho + div;
    if (res) res[v] = r;
    rmax = fmaxf(rmax, fabsf(r));
    smax = fmaxf(smax, fabsf(drho));
  }
#pragma unroll
  for (int o = 16; o; o >>= 1) {
    rmax = fmaxf(rmax, __shfl_xor_sync(FULL, rmax, o));
    smax = fmaxf(smax, __shfl_xor_sync(FULL, smax, o));
  }
  if ((threadIdx.x & 31) == 0) {
    atomic_max_nonneg(out, rmax);
    atomic_max_nonneg(out + 1, smax);
  }
}

inline unsigned grid_for(int64_t n, int threads, int num_sms) {
  int64_t b = (n + threads - 1) / threads;
  const int64_t cap = (int64_t)num_sms * 16;
  if (b > cap) b = cap;
  if (b < 1) b = 1;
  return (unsigned)b;
}

}  // namespace

cudaError_t launch_accumulate_rho(const vpic_ctx *c, float q, const vpic_particle_t *p, int64_t np,
                                  float *rho, cudaStream_t s) {
  if (np == 0) return cudaSuccess;
  Per per{c->periodic_local[0], c->periodic_local[1], c->periodic_local[2]};
  k_accumulate_rho<<<grid_for(np, 256, c->num_sms), 256, 0, s>>>(
      c->gk, per, q, reinterpret_cast<const float4 *>(p), np, rho); note_launch();
  return cudaGetLastError();
}

cudaError_t launch_continuity(const vpic_ctx *c, const float *rho0, const float *rho1,
                              const float *jf, float *out, float *res, cudaStream_t s) {
  Per per{c->periodic_local[0], c->periodic_local[1], c->periodic_local[2]};
  const vpic_grid_t &g = c->g;
  const float inv_vdt = 1.0f / (g.dx * g.dy * g.dz * g.dt);
  cudaError_t e = cudaMemsetAsync(out, 0, 2 * sizeof(float), s);
  if (e != cudaSuccess) return e;
  const int64_t total = (int64_t)(g.nx + 1) * (g.ny + 1) * (g.nz + 1);
  k_continuity<<<grid_for(total, 256, c->num_sms), 256, 0, s>>>(
      c->gk, per, inv_vdt, 1.0f / g.dx, 1.0f / g.dy, 1.0f / g.dz, rho0, rho1,
      reinterpret_cast<const float4 *>(jf), out, res); note_launch();
  return cudaGetLastError();
}

}  // namespace vpic
