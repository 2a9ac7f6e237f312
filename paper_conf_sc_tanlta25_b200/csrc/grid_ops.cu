// Grid-side kernels of the hot path: ghost fill + load_interpolator (row a5),
// unload_accumulator (row a12).  VPIC reading; the paper
// names only the "gather phase" source.
#include "vpic_internal.cuh"

namespace vpic {
namespace {

struct Per {
  int px, py, pz;  // axis wraps locally
};

// +x/+y/+z ghost planes of locally periodic axes := copy of plane 1 (edges
// and the corner included).  Equivalent to copying plane by plane in axis
// order; no voxel is both read and written.
__global__ void k_fill_ghosts(const GridK g, const Per per, float4 *__restrict__ f) {
  const int64_t nv = g.nv;
  for (int64_t v = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; v < nv;
       v += (int64_t)gridDim.x * blockDim.x) {
    int x = (int)(v % g.sx), y = (int)((v / g.sx) % g.sy), z = (int)(v / g.sxy);
    bool w = false;
    if (per.px && x == g.nx + 1) { x = 1; w = true; }
    if (per.py && y == g.ny + 1) { y = 1; w = true; }
    if (per.pz && z == g.nz + 1) { z = 1; w = true; }
    if (!w) continue;
    const int64_t src = x + (int64_t)g.sx * (y + (int64_t)g.sy * z);
    f[2 * v] = f[2 * src];
    f[2 * v + 1] = f[2 * src + 1];
  }
}

// -x/-y/-z ghost planes of locally periodic axes := copy of plane n (the cB
// neighbours advance_e needs).  Same direct mapping as k_fill_ghosts.
__global__ void k_fill_ghosts_minus(const GridK g, const Per per, float4 *__restrict__ f) {
  const int64_t nv = g.nv;
  for (int64_t v = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; v < nv;
       v += (int64_t)gridDim.x * blockDim.x) {
    int x = (int)(v % g.sx), y = (int)((v / g.sx) % g.sy), z = (int)(v / g.sxy);
    bool w = false;
    if (per.px && x == 0) { x = g.nx; w = true; }
    if (per.py && y == 0) { y = g.ny; w = true; }
    if (per.pz && z == 0) { z = g.nz; w = true; }
    if (!w) continue;
    const int64_t src = x + (int64_t)g.sx * (y + (int64_t)g.sy * z);
    f[2 * v] = f[2 * src];
    f[2 * v + 1] = f[2 * src + 1];
  }
}

// Field solver (VPIC advance_b / advance_e, reading F1):
// one thread per interior voxel, consecutive threads along x.
//   advance_b: cB -= frac c dt curl E   (E at +1 neighbours)
//   advance_e: E  += c dt curl cB - (dt/eps0) jf   (cB at -1 neighbours)
// Same expressions and order as the oracle; compiled without FMA contraction.
__global__ void __launch_bounds__(256)
k_advance_b(const GridK g, const float px, const float py, const float pz, float4 *__restrict__ f) {
  const int64_t ncell = (int64_t)g.nx * g.ny * g.nz;
  for (int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; t < ncell;
       t += (int64_t)gridDim.x * blockDim.x) {
    const int x = 1 + (int)(t % g.nx);
    const int row = (int)(t / g.nx);
    const int y = 1 + row % g.ny, z = 1 + row / g.ny;
    const int64_t v = x + (int64_t)g.sx * (y + (int64_t)g.sy * z);
    const float4 e = f[2 * v];
    float4 b = f[2 * v + 1];
    const float4 ex1 = f[2 * (v + 1)], ey1 = f[2 * (v + g.sx)], ez1 = f[2 * (v + g.sxy)];
    b.x -= py * (ey1.z - e.z) - pz * (ez1.y - e.y);
    b.y -= pz * (ez1.x - e.x) - px * (ex1.z - e.z);
    b.z -= px * (ex1.y - e.y) - py * (ey1.x - e.x);
    f[2 * v + 1] = b;
  }
}

__global__ void __launch_bounds__(256)
k_advance_e(const GridK g, const float px, const float py, const float pz, const float cj,
            float4 *__restrict__ f, const float4 *__restrict__ jf) {
  const int64_t ncell = (int64_t)g.nx * g.ny * g.nz;
  for (int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; t < ncell;
       t += (int64_t)gridDim.x * blockDim.x) {
    const int x = 1 + (int)(t % g.nx);
    const int row = (int)(t / g.nx);
    const int y = 1 + row % g.ny, z = 1 + row / g.ny;
    const int64_t v = x + (int64_t)g.sx * (y + (int64_t)g.sy * z);
    float4 e = f[2 * v];
    const float4 b = f[2 * v + 1];
    const float4 bx1 = f[2 * (v - 1) + 1], by1 = f[2 * (v - g.sx) + 1], bz1 = f[2 * (v - g.sxy) + 1];
    const float4 j = __ldg(jf + v);
    e.x += py * (b.z - by1.z) - pz * (b.y - bz1.y) - cj * j.x;
    e.y += pz * (b.x - bz1.x) - px * (b.z - bx1.z) - cj * j.y;
    e.z += px * (b.y - bx1.y) - py * (b.x - by1.x) - cj * j.z;
    f[2 * v] = e;
  }
}

// One thread per interior voxel; consecutive threads take consecutive x of
// a (y,z) row so the x+1 neighbours come from L1.  interp[v] = 6 x float4
// (96 B, the last 24 B zero) so that a particle's gather is three
// sector-aligned 32-B loads.  Each warp stages its 32 rows in shared memory and
// stores them as consecutive 16-B units (warm: 86 vs 127 us at C2).
__global__ void __launch_bounds__(128)
k_load_interp(const GridK g, const float4 *__restrict__ f, float4 *__restrict__ interp) {
  __shared__ float4 stage[4][32 * 6];
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  const uint32_t nx = (uint32_t)g.nx, ny = (uint32_t)g.ny;
  const int64_t n = (int64_t)g.ny * g.nz * g.nx;   // < 2^32 (host-checked)
  const float fourth = 0.25f, half = 0.5f;
  for (int64_t t0 = ((int64_t)blockIdx.x * blockDim.x + (threadIdx.x & ~31)); t0 < n;
       t0 += (int64_t)gridDim.x * blockDim.x) {
    const int64_t t = t0 + lane;
    const bool act = t < n;
    int64_t v = 0;
    if (act) {
      const uint32_t tt = (uint32_t)t, row = tt / nx;
      const uint32_t x = 1 + (tt - row * nx), y = 1 + row % ny, z = 1 + row / ny;
      v = x + (int64_t)g.sx * (y + (int64_t)g.sy * z);
      const int64_t X = 1, Y = g.sx, Z = g.sxy;
      // E (first float4) and cB (second float4) of the 7 neighbours needed
      const float4 e000 = __ldg(f + 2 * v), b000 = __ldg(f + 2 * v + 1);
      const float4 e100 = __ldg(f + 2 * (v + X)), b100 = __ldg(f + 2 * (v + X) + 1);
      const float4 e010 = __ldg(f + 2 * (v + Y)), b010 = __ldg(f + 2 * (v + Y) + 1);
      const float4 e001 = __ldg(f + 2 * (v + Z)), b001 = __ldg(f + 2 * (v + Z) + 1);
      const float4 e110 = __ldg(f + 2 * (v + X + Y));
      const float4 e011 = __ldg(f + 2 * (v + Y + Z));
      const float4 e101 = __ldg(f + 2 * (v + X + Z));
      float w0, w1, w2, w3;
      float4 o0, o1, o2, o3, o4;
      // ex: bilinear in (y, z)
      w0 = e000.x; w1 = e010.x; w2 = e001.x; w3 = e011.x;
      o0.x = fourth * ((w3 + w0) + (w1 + w2));
      o0.y = fourth * ((w3 - w0) + (w1 - w2));
      o0.z = fourth * ((w3 - w0) - (w1 - w2));
      o0.w = fourth * ((w3 + w0) - (w1 + w2));
      // ey: bilinear in (z, x)
      w0 = e000.y; w1 = e001.y; w2 = e100.y; w3 = e101.y;
      o1.x = fourth * ((w3 + w0) + (w1 + w2));
      o1.y = fourth * ((w3 - w0) + (w1 - w2));
      o1.z = fourth * ((w3 - w0) - (w1 - w2));
      o1.w = fourth * ((w3 + w0) - (w1 + w2));
      // ez: bilinear in (x, y)
      w0 = e000.z; w1 = e100.z; w2 = e010.z; w3 = e110.z;
      o2.x = fourth * ((w3 + w0) + (w1 + w2));
      o2.y = fourth * ((w3 - w0) + (w1 - w2));
      o2.z = fourth * ((w3 - w0) - (w1 - w2));
      o2.w = fourth * ((w3 + w0) - (w1 + w2));
      // cB: linear along the face normal
      o3.x = half * (b100.x + b000.x);
      o3.y = half * (b100.x - b000.x);
      o3.z = half * (b010.y + b000.y);
      o3.w = half * (b010.y - b000.y);
      o4.x = half * (b001.z + b000.z);
      o4.y = half * (b001.z - b000.z);
      o4.z = 0.0f;
      o4.w = 0.0f;
      float4 *o = &stage[w][6 * lane];
      o[0] = o0; o[1] = o1; o[2] = o2; o[3] = o3; o[4] = o4;
      o[5] = make_float4(0.f, 0.f, 0.f, 0.f);
    }
    __syncwarp();
    // staged unit j = component j % 6 of the warp's row j / 6: consecutive
    // lanes store consecutive 16-B units of consecutive voxels
    const int nact = n - t0 < 32 ? (int)(n - t0) : 32;
#pragma unroll
    for (int k = 0; k < 6; ++k) {
      const int j = lane + 32 * k;
      const int src = j / 6;
      const int64_t vj = __shfl_sync(0xffffffffu, v, src);
#if VPIC_INTERP_SPLIT
      const int comp = j - 6 * src;
      if (src < nact) {
        if (comp < 4) {
          interp[4 * vj + comp] = stage[w][j];
        } else if (comp == 4) {   // (cbz, dcbz/dz) into the compact tail
          const float4 q = stage[w][j];
          reinterpret_cast<float2 *>(interp + 4 * g.nv)[vj] = make_float2(q.x, q.y);
        }
      }
#else
      if (src < nact) interp[6 * vj + (j - 6 * src)] = stage[w][j];
#endif
    }
    __syncwarp();
  }
}

// jf on the edges of voxels 1..n+1.  On a locally periodic axis the n+1
// plane aliases plane 1 and the x-1 neighbour of plane 1 is plane n, which
// sums the shared planes directly (the fold of reading c.1) and makes the n+1
// ghost copy identical to plane 1.  Other axes: ghost accumulators are zero.
__global__ void k_unload(const GridK g, const Per per, const float cx, const float cy,
                         const float cz, const float4 *__restrict__ a, float4 *__restrict__ jf) {
  const int64_t ex = g.nx + 1, ey = g.ny + 1, ez = g.nz + 1;
  const int64_t total = ex * ey * ez;
  for (int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; t < total;
       t += (int64_t)gridDim.x * blockDim.x) {
    const int xo = 1 + (int)(t % ex);
    const int yo = 1 + (int)((t / ex) % ey);
    const int zo = 1 + (int)(t / (ex * ey));
    int x = xo, y = yo, z = zo;
    if (per.px && x == g.nx + 1) x = 1;
    if (per.py && y == g.ny + 1) y = 1;
    if (per.pz && z == g.nz + 1) z = 1;
    const int xm = (per.px && x == 1) ? g.nx : x - 1;
    const int ym = (per.py && y == 1) ? g.ny : y - 1;
    const int zm = (per.pz && z == 1) ? g.nz : z - 1;
    auto V = [&](int X, int Y, int Z) -> int64_t { return X + (int64_t)g.sx * (Y + (int64_t)g.sy * Z); };
    const int64_t v0 = V(x, y, z), vy = V(x, ym, z), vz = V(x, y, zm), vyz = V(x, ym, zm);
    const int64_t vx = V(xm, y, z), vzx = V(xm, y, zm), vxy = V(xm, ym, z);
    // jx[q] is float4 #0, jy #1, jz #2 of each accumulator
    const float4 a0x = __ldg(a + 3 * v0), a0y = __ldg(a + 3 * v0 + 1), a0z = __ldg(a + 3 * v0 + 2);
    const float jx = cx * (a0x.x + __ldg(a + 3 * vy).y + __ldg(a + 3 * vz).z + __ldg(a + 3 * vyz).w);
    const float jy = cy * (a0y.x + __ldg(a + 3 * vz + 1).y + __ldg(a + 3 * vx + 1).z +
                           __ldg(a + 3 * vzx + 1).w);
    const float jz = cz * (a0z.x + __ldg(a + 3 * vx + 2).y + __ldg(a + 3 * vy + 2).z +
                           __ldg(a + 3 * vxy + 2).w);
    jf[V(xo, yo, zo)] = make_float4(jx, jy, jz, 0.0f);
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

cudaError_t launch_fill_ghosts(const vpic_ctx *c, float *fields, cudaStream_t s) {
  Per per{c->periodic_local[0], c->periodic_local[1], c->periodic_local[2]};
  if (!per.px && !per.py && !per.pz) return cudaSuccess;
  k_fill_ghosts<<<grid_for(c->gk.nv, 256, c->num_sms), 256, 0, s>>>(
      c->gk, per, reinterpret_cast<float4 *>(fields)); note_launch();
  return cudaGetLastError();
}

cudaError_t launch_load_interp(const vpic_ctx *c, const float *fields, float *interp,
                               cudaStream_t s) {
  const int64_t n = (int64_t)c->gk.nx * c->gk.ny * c->gk.nz;
  if (n >= ((int64_t)1 << 32)) return cudaErrorInvalidValue;   // 32-bit voxel counter
  k_load_interp<<<grid_for(n, 128, c->num_sms), 128, 0, s>>>(
      c->gk, reinterpret_cast<const float4 *>(fields), reinterpret_cast<float4 *>(interp)); note_launch();
  return cudaGetLastError();
}

cudaError_t launch_fill_ghosts_minus(const vpic_ctx *c, float *fields, cudaStream_t s) {
  Per per{c->periodic_local[0], c->periodic_local[1], c->periodic_local[2]};
  if (!per.px && !per.py && !per.pz) return cudaSuccess;
  k_fill_ghosts_minus<<<grid_for(c->gk.nv, 256, c->num_sms), 256, 0, s>>>(
      c->gk, per, reinterpret_cast<float4 *>(fields)); note_launch();
  return cudaGetLastError();
}

cudaError_t launch_advance_b(const vpic_ctx *c, float *fields, float frac, cudaStream_t s) {
  const vpic_grid_t &g = c->g;
  // same expressions as the oracle: frac * c * dt / d
  const float px = frac * g.cvac * g.dt / g.dx;
  const float py = frac * g.cvac * g.dt / g.dy;
  const float pz = frac * g.cvac * g.dt / g.dz;
  const int64_t n = (int64_t)g.nx * g.ny * g.nz;
  k_advance_b<<<grid_for(n, 256, c->num_sms), 256, 0, s>>>(c->gk, px, py, pz,
                                                           reinterpret_cast<float4 *>(fields)); note_launch();
  return cudaGetLastError();
}

cudaError_t launch_advance_e(const vpic_ctx *c, float *fields, const float *jf, float eps0,
                             cudaStream_t s) {
  const vpic_grid_t &g = c->g;
  const float px = g.cvac * g.dt / g.dx;
  const float py = g.cvac * g.dt / g.dy;
  const float pz = g.cvac * g.dt / g.dz;
  const float cj = g.dt / eps0;
  const int64_t n = (int64_t)g.nx * g.ny * g.nz;
  k_advance_e<<<grid_for(n, 256, c->num_sms), 256, 0, s>>>(c->gk, px, py, pz, cj,
                                                           reinterpret_cast<float4 *>(fields),
                                                           reinterpret_cast<const float4 *>(jf)); note_launch();
  return cudaGetLastError();
}

cudaError_t launch_unload(const vpic_ctx *c, const float *acc, float *jf, cudaStream_t s) {
  Per per{c->periodic_local[0], c->periodic_local[1], c->periodic_local[2]};
  const vpic_grid_t &g = c->g;
  const float cx = 0.25f / (g.dy * g.dz * g.dt);
  const float cy = 0.25f / (g.dz * g.dx * g.dt);
  const float cz = 0.25f / (g.dx * g.dy * g.dt);
  const int64_t n = (int64_t)(c->gk.nx + 1) * (c->gk.ny + 1) * (c->gk.nz + 1);
  k_unload<<<grid_for(n, 256, c->num_sms), 256, 0, s>>>(c->gk, per, cx, cy, cz,
                                                        reinterpret_cast<const float4 *>(acc),
                                                        reinterpret_cast<float4 *>(jf)); note_launch();
  return cudaGetLastError();
}

}  // namespace vpic
