// Particle boundary handling and the multi-GPU exchange (row a13 of SURVEY.md
// §8(a)): particle migration across rank faces ("Most MPI communication in
// VPIC is non-blocking point-to-point with up to six neighbors", PAPER.md:55;
// "exchanging particles"), the E/cB ghost-plane halo and the jf
// shared-plane reduction.  Transport: NCCL send/recv (NVLink / NVSwitch) in
// grouped calls; one process per GPU.
#include <nccl.h>
#include <nccl_device.h>

#include <algorithm>
#include <vector>

#include "vpic_internal.cuh"

namespace vpic {

struct Exchange {
  ncclComm_t comm = nullptr;
  // migration buffers (48-B records: particle + remaining displacement)
  float4 *send = nullptr;   // [6][send_cap][3]
  float4 *recv = nullptr;   // [recv_cap][3]
  int64_t send_cap = 0, recv_cap = 0;
  int64_t *d_cnt = nullptr; // [0..5] send counts, [6..11] recv counts
  vpic_mover_t *mv_arr = nullptr, *mv_next = nullptr;  // arrivals' movers, next round's
  int64_t mv_arr_cap = 0, mv_next_cap = 0;
  // plane buffers for halo / jf reduction
  float *plane_send = nullptr, *plane_recv = nullptr;
  size_t plane_bytes = 0;
  // device-initiated exchange (VPIC_OPT_DEVICE_EXCHANGE): inbox window in
  // NCCL symmetric memory, the device communicator for the LSA barrier, and
  // device-count driven arrival / hole bookkeeping (no host sync per round)
  bool di = false;
  void *di_buf = nullptr;
  ncclWindow_t di_win = nullptr;
  ncclDevComm di_dcomm{};
  bool di_dcomm_ok = false;
  int64_t di_cap = 0, di_hcap = 0;
  int64_t *di_ctr = nullptr;          // [0] np [1] H [2] A [3] next movers [4] nlow [5] nsurv [6] np_new [7] base; [8..13] face offsets
  int32_t *di_flag = nullptr;         // bit 0 inbox full (senders), 1 holes overflow, 2 particles overflow
  vpic_mover_t *di_arr = nullptr, *di_next = nullptr;
  uint32_t *di_scr = nullptr;         // hole scratch: tail_dead | low | surv, di_hcap each
  // single-round mode: per-mover direction, packed send records, the
  // accumulator's ghost planes (2 out, 2 in)
  int8_t *g_dir = nullptr;
  int64_t g_dir_cap = 0;
  int64_t *g_pc = nullptr;            // per-peer direction counts: [2][27 peers][27]
  float *acc_plane[4] = {nullptr, nullptr, nullptr, nullptr};
  size_t acc_plane_bytes = 0;
};

namespace {

constexpr int OPP[6] = {3, 4, 5, 0, 1, 2};

#define CKC(x) do { cudaError_t e_ = (x); if (e_ != cudaSuccess) return VPIC_ERR_CUDA; } while (0)
#define CKN(x) do { ncclResult_t r_ = (x); if (r_ != ncclSuccess) return VPIC_ERR_NCCL; } while (0)

struct Ptrs6 { float4 *p[6]; };

// Classify the movers of this round: every mover's particle leaves this rank
// (remote face: packed for the neighbour with its entry voxel and flipped
// offset; absorb face: dropped).  Its slot becomes a hole.
__global__ void k_pack_movers(const GridK g, const vpic_particle_t *__restrict__ p,
                              const vpic_mover_t *__restrict__ mv, const int64_t *__restrict__ Mdev,
                              int64_t Mmax, float4 *__restrict__ send,
                              int64_t send_cap, int64_t *__restrict__ send_cnt,
                              uint32_t *__restrict__ holes, int32_t *__restrict__ flags) {
  const int64_t M = min(*Mdev, Mmax);
  for (int64_t k = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; k < M;
       k += (int64_t)gridDim.x * blockDim.x) {
    const vpic_mover_t m = mv[k];
    holes[k] = (uint32_t)m.idx;
    vpic_particle_t q = p[m.idx];
    const int face = q.i & 7;
    const int32_t v = q.i >> 3;
    if (g.face_kind[face] != FACE_REMOTE) continue;  // absorbed
    int x = v % g.sx, y = (v / g.sx) % g.sy, z = v / g.sxy;
    const int axis = face % 3;
    const bool plus = face >= 3;
    if (axis == 0) { x = plus ? 1 : g.nx; q.dx = -q.dx; }
    else if (axis == 1) { y = plus ? 1 : g.ny; q.dy = -q.dy; }
    else { z = plus ? 1 : g.nz; q.dz = -q.dz; }
    q.i = x + g.sx * (y + g.sy * z);
    const unsigned long long slot = atomicAdd(reinterpret_cast<unsigned long long *>(send_cnt + face), 1ull);
    if ((int64_t)slot >= send_cap) { atomicOr(flags, 2); continue; }
    float4 *r = send + 3 * ((int64_t)face * send_cap + (int64_t)slot);
    r[0] = make_float4(q.dx, q.dy, q.dz, __int_as_float(q.i));
    r[1] = make_float4(q.ux, q.uy, q.uz, q.w);
    r[2] = make_float4(m.dispx, m.dispy, m.dispz, 0.0f);
  }
}

// Back-fill the H holes (distinct indices < np) with the surviving particles
// of the tail [np-H, np).  scratch: 3*H + 2 ints.
__global__ void k_mark_tail(const uint32_t *__restrict__ holes, int64_t H, int64_t np_new,
                            uint32_t *__restrict__ tail_dead, uint32_t *__restrict__ low,
                            unsigned long long *__restrict__ nlow) {
  for (int64_t k = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; k < H;
       k += (int64_t)gridDim.x * blockDim.x) {
    const int64_t h = holes[k];
    if (h >= np_new) tail_dead[h - np_new] = 1;
    else low[atomicAdd(nlow, 1ull)] = (uint32_t)h;
  }
}
__global__ void k_tail_survivors(const uint32_t *__restrict__ tail_dead, int64_t H, int64_t np_new,
                                 uint32_t *__restrict__ surv, unsigned long long *__restrict__ nsurv) {
  for (int64_t j = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; j < H;
       j += (int64_t)gridDim.x * blockDim.x)
    if (!tail_dead[j]) surv[atomicAdd(nsurv, 1ull)] = (uint32_t)(np_new + j);
}
__global__ void k_backfill(vpic_particle_t *__restrict__ p, const uint32_t *__restrict__ low,
                           const uint32_t *__restrict__ surv,
                           const unsigned long long *__restrict__ nlow) {
  const int64_t n = (int64_t)*nlow;
  for (int64_t k = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; k < n;
       k += (int64_t)gridDim.x * blockDim.x)
    p[low[k]] = p[surv[k]];
}

// Append arrivals and build their mover list (remaining displacement).
__global__ void k_unpack(const float4 *__restrict__ recv, int64_t A, vpic_particle_t *__restrict__ p,
                         int64_t np, vpic_mover_t *__restrict__ mv) {
  for (int64_t k = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; k < A;
       k += (int64_t)gridDim.x * blockDim.x) {
    const float4 a = recv[3 * k], b = recv[3 * k + 1], d = recv[3 * k + 2];
    float4 *dst = reinterpret_cast<float4 *>(p + np + k);
    dst[0] = a;
    dst[1] = b;
    vpic_mover_t m;
    m.dispx = d.x; m.dispy = d.y; m.dispz = d.z; m.idx = (int32_t)(np + k);
    mv[k] = m;
  }
}

// ---- planes: (axis, index) plane of an array of nv records of `w` floats,
// over the full extent of the other two axes (ghosts included).
__global__ void k_plane_copy(const GridK g, int axis, int idx, float *__restrict__ a, int w,
                             float *__restrict__ buf, int mode /*0 pack, 1 unpack, 2 add, 3 pack + zero*/) {
  const int sz = g.nv / ((int64_t)g.sx * g.sy);
  const int e0 = axis == 0 ? g.sy : g.sx;
  const int e1 = axis == 2 ? g.sy : sz;
  const int64_t n = (int64_t)e0 * e1 * w;
  for (int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; t < n;
       t += (int64_t)gridDim.x * blockDim.x) {
    const int c = (int)(t % w);
    const int64_t r = t / w;
    const int u = (int)(r % e0), vv = (int)(r / e0);
    int x, y, z;
    if (axis == 0) { x = idx; y = u; z = vv; }
    else if (axis == 1) { x = u; y = idx; z = vv; }
    else { x = u; y = vv; z = idx; }
    float *e = a + (int64_t)w * (x + (int64_t)g.sx * (y + (int64_t)g.sy * z)) + c;
    if (mode == 0) buf[t] = *e;
    else if (mode == 1) *e = buf[t];
    else if (mode == 2) *e += buf[t];
    else { buf[t] = *e; *e = 0.0f; }
  }
}

unsigned blocks_for(int64_t n) {
  int64_t b = (n + 255) / 256;
  return (unsigned)std::max<int64_t>(1, std::min<int64_t>(b, 148 * 16));
}

int ensure(void **ptr, int64_t *cap, int64_t need, size_t rec_bytes) {
  if (need <= *cap) return VPIC_OK;
  if (*ptr) cudaFree(*ptr);
  int64_t nc = std::max<int64_t>(need, *cap * 2);
  nc = std::max<int64_t>(nc, 4096);
  if (cudaMalloc(ptr, (size_t)nc * rec_bytes) != cudaSuccess) { *ptr = nullptr; *cap = 0; return VPIC_ERR_CUDA; }
  *cap = nc;
  return VPIC_OK;
}

int ensure_plane(Exchange *ex, size_t bytes) {
  if (bytes <= ex->plane_bytes) return VPIC_OK;
  if (ex->plane_send) cudaFree(ex->plane_send);
  if (ex->plane_recv) cudaFree(ex->plane_recv);
  if (cudaMalloc(&ex->plane_send, bytes) != cudaSuccess) return VPIC_ERR_CUDA;
  if (cudaMalloc(&ex->plane_recv, bytes) != cudaSuccess) return VPIC_ERR_CUDA;
  ex->plane_bytes = bytes;
  return VPIC_OK;
}

// Scratch of the context used for hole filling (grown on demand).
int ctx_scratch(vpic_ctx *c, size_t bytes) {
  if (bytes <= c->scratch_bytes) return VPIC_OK;
  if (c->scratch) cudaFree(c->scratch);
  c->scratch = nullptr;
  c->scratch_bytes = 0;
  if (cudaMalloc(&c->scratch, bytes) != cudaSuccess) return VPIC_ERR_CUDA;
  c->scratch_bytes = bytes;
  return VPIC_OK;
}

int remove_holes(vpic_ctx *c, vpic_particle_t *p, int64_t np, const uint32_t *holes, int64_t H,
                 cudaStream_t s) {
  if (H == 0) return VPIC_OK;
  const int64_t np_new = np - H;
  uint32_t *sc = static_cast<uint32_t *>(c->scratch) + H;  // after the hole list
  uint32_t *tail_dead = sc, *low = sc + H, *surv = sc + 2 * H;
  unsigned long long *cnt = reinterpret_cast<unsigned long long *>(c->d_count + 4);  // [4], [5]
  CKC(cudaMemsetAsync(tail_dead, 0, 4 * (size_t)H, s));
  CKC(cudaMemsetAsync(cnt, 0, 16, s));
  k_mark_tail<<<blocks_for(H), 256, 0, s>>>(holes, H, np_new, tail_dead, low, cnt); note_launch();
  k_tail_survivors<<<blocks_for(H), 256, 0, s>>>(tail_dead, H, np_new, surv, cnt + 1); note_launch();
  // as many tail survivors as holes below np_new: the device count sizes it
  k_backfill<<<blocks_for(H), 256, 0, s>>>(p, low, surv, cnt); note_launch();
  return cudaGetLastError() == cudaSuccess ? VPIC_OK : VPIC_ERR_CUDA;
}

// ---------------------------------------------------- device-initiated --
struct Peers27 { int lsa[27]; };

__global__ void k_di_peers(ncclWindow_t w, Peers27 pr, int n, unsigned char **out) {
  for (int f = 0; f < n; ++f)
    out[f] = pr.lsa[f] >= 0 ? static_cast<unsigned char *>(ncclGetLsaPointer(w, 0, pr.lsa[f])) : nullptr;
}

// All ranks of the node reach this point; everything any rank stored into a
// peer's inbox before (earlier kernels on its stream) is visible after it.
__global__ void k_lsa_barrier(ncclDevComm dc) {
  ncclLsaBarrierSession<ncclCoopCta> bar(ncclCoopCta(), dc, ncclTeamTagLsa(), 0);
  bar.sync(ncclCoopCta(), cuda::memory_order_acq_rel);
}

__global__ void k_di_set(int64_t *ctr, int64_t np) { ctr[0] = np; ctr[3] = 0; }
__global__ void k_di_set_dev(int64_t *ctr, const int64_t *np_dev) { ctr[0] = *np_dev; ctr[3] = 0; }
// device-count call done: the new count out; the capacity flags (di_flag bit
// 0 inbox full, 1 hole list full, 2 arrivals did not fit; dflag) OR-ed into
// the caller's flags shifted up by one (bit 0 stays advance_p's mover
// overflow) and cleared for the next call
__global__ void k_di_finish(const int64_t *ctr, int64_t *np_dev, int32_t *dflag, int32_t *di_flag,
                            int32_t *flags_dev) {
  *np_dev = ctr[0];
  const int32_t f = *dflag | *di_flag;
  if (f) *flags_dev |= (f << 1);
  *dflag = 0;
  *di_flag = 0;
}

// Holes of this round: H = departures in `mv` (device count *hdev).
// hcap = min(internal hole capacity, the mover list's capacity): a count
// beyond it means movers were dropped (or cannot be holed): flagged, clamped
// so no kernel reads past the list.
__global__ void k_di_holes_prep(int64_t *ctr, const int64_t *hdev, int64_t hcap, int32_t *flag) {
  int64_t H = *hdev;
  if (H > hcap) { atomicOr(flag, 2); H = hcap; }
  ctr[1] = H;
  ctr[6] = ctr[0] - H;
  ctr[0] = ctr[6];
  ctr[4] = 0;
  ctr[5] = 0;
}
__global__ void k_di_mark_tail(const vpic_mover_t *__restrict__ mv, int64_t *ctr,
                               uint32_t *__restrict__ tail_dead, uint32_t *__restrict__ low) {
  const int64_t H = ctr[1], np_new = ctr[6];
  for (int64_t k = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; k < H;
       k += (int64_t)gridDim.x * blockDim.x) {
    const int64_t h = (uint32_t)mv[k].idx;
    if (h >= np_new) tail_dead[h - np_new] = 1;
    else low[atomicAdd(reinterpret_cast<unsigned long long *>(ctr + 4), 1ull)] = (uint32_t)h;
  }
}
__global__ void k_di_clear(uint32_t *__restrict__ a, const int64_t *ctr) {
  const int64_t H = ctr[1];
  for (int64_t k = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; k < H;
       k += (int64_t)gridDim.x * blockDim.x)
    a[k] = 0;
}
__global__ void k_di_tail_surv(const uint32_t *__restrict__ tail_dead, int64_t *ctr,
                               uint32_t *__restrict__ surv) {
  const int64_t H = ctr[1], np_new = ctr[6];
  for (int64_t j = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; j < H;
       j += (int64_t)gridDim.x * blockDim.x)
    if (!tail_dead[j])
      surv[atomicAdd(reinterpret_cast<unsigned long long *>(ctr + 5), 1ull)] = (uint32_t)(np_new + j);
}
__global__ void k_di_backfill(vpic_particle_t *__restrict__ p, const uint32_t *__restrict__ low,
                              const uint32_t *__restrict__ surv, const int64_t *ctr) {
  const int64_t n = ctr[4];
  for (int64_t k = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; k < n;
       k += (int64_t)gridDim.x * blockDim.x)
    p[low[k]] = p[surv[k]];
}

// Arrivals of round r: per-face counts -> offsets, append position, reset.
__global__ void k_di_take(unsigned char *inbox, int r, int64_t cap, int64_t max_np, int64_t *ctr,
                          int32_t *flag) {
  if (threadIdx.x != 0) return;
  int64_t off = 0;
  for (int f = 0; f < 6; ++f) {
    unsigned long long *cf = reinterpret_cast<unsigned long long *>(inbox + di_cnt_off(di_face_slot(r, f)));
    int64_t a = (int64_t)*cf;
    if (a > cap) a = cap;     // the senders flagged the overflow
    ctr[8 + f] = off;
    off += a;
    *cf = 0;
  }
  const int64_t base = ctr[0];
  if (base + off > max_np) {  // no room: drop the round's arrivals, report capacity
    atomicOr(flag, 4);
    off = 0;
    for (int f = 0; f < 6; ++f) ctr[8 + f] = 0;
  }
  ctr[14] = off;              // (per-face ends for the unpack: offsets + counts)
  ctr[2] = off;
  ctr[7] = base;
  ctr[0] = base + off;
}
__global__ void k_di_unpack(const unsigned char *inbox, int r, int64_t cap, const int64_t *ctr,
                            vpic_particle_t *__restrict__ p, vpic_mover_t *__restrict__ mv) {
  const int64_t A = ctr[2], base = ctr[7];
  for (int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; t < A;
       t += (int64_t)gridDim.x * blockDim.x) {
    int f = 0;
    while (f < 5 && t >= ctr[8 + f + 1]) ++f;
    const int64_t k = t - ctr[8 + f];
    const float4 *rec = reinterpret_cast<const float4 *>(inbox + di_rec_off(di_face_slot(r, f), cap, k));
    const float4 a = rec[0], b = rec[1], d = rec[2];
    float4 *dst = reinterpret_cast<float4 *>(p + base + t);
    dst[0] = a;
    dst[1] = b;
    vpic_mover_t m;
    m.dispx = d.x; m.dispy = d.y; m.dispz = d.z; m.idx = (int32_t)(base + t);
    mv[t] = m;
  }
}

// ---- single-round mode (SURVEY.md §8(e) alternative (2)) ----------------
struct Off27 { int64_t o[27]; };

__device__ __forceinline__ int ghost_dir(const GridK &g, int32_t v, int &x, int &y, int &z) {
  x = v % g.sx; y = (v / g.sx) % g.sy; z = v / g.sxy;
  const int ox = x == 0 ? -1 : (x == g.nx + 1 ? 1 : 0);
  const int oy = y == 0 ? -1 : (y == g.ny + 1 ? 1 : 0);
  const int oz = z == 0 ? -1 : (z == g.nz + 1 ? 1 : 0);
  // the voxel as the neighbour sees it: crossed axes enter from its far side
  if (ox) x = ox < 0 ? g.nx : 1;
  if (oy) y = oy < 0 ? g.ny : 1;
  if (oz) z = oz < 0 ? g.nz : 1;
  return dir26(ox, oy, oz);
}

// Departures of this call: every mover's slot becomes a hole; a particle
// marked p.i = -1 - (ghost voxel) leaves for the neighbour in that voxel's
// direction, the others (absorbed) are dropped.  Counts per direction.
__global__ void k_ghost_classify(const GridK g, const vpic_particle_t *__restrict__ p,
                                 const vpic_mover_t *__restrict__ mv, const int64_t *__restrict__ Mdev,
                                 int64_t Mmax, int8_t *__restrict__ dir, int64_t *__restrict__ cnt,
                                 uint32_t *__restrict__ holes) {
  const int64_t M = min(*Mdev, Mmax);
  for (int64_t k = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; k < M;
       k += (int64_t)gridDim.x * blockDim.x) {
    const int32_t idx = mv[k].idx;
    holes[k] = (uint32_t)idx;
    const int32_t i = p[idx].i;
    if (i >= 0) { dir[k] = -1; continue; }
    int x, y, z;
    const int d = ghost_dir(g, -1 - i, x, y, z);
    dir[k] = (int8_t)d;
    atomicAdd(reinterpret_cast<unsigned long long *>(cnt + d), 1ull);
  }
}

__global__ void k_ghost_pack(const GridK g, const vpic_particle_t *__restrict__ p,
                             const vpic_mover_t *__restrict__ mv, int64_t M, const int8_t *__restrict__ dir,
                             Off27 off, unsigned long long *__restrict__ cur, float4 *__restrict__ send) {
  for (int64_t k = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; k < M;
       k += (int64_t)gridDim.x * blockDim.x) {
    const int d = dir[k];
    if (d < 0) continue;
    const vpic_particle_t q = p[mv[k].idx];
    int x, y, z;
    ghost_dir(g, -1 - q.i, x, y, z);
    const int64_t slot = off.o[d] + (int64_t)atomicAdd(cur + d, 1ull);
    float4 *r = send + 3 * slot;
    r[0] = make_float4(q.dx, q.dy, q.dz, __int_as_float(x + g.sx * (y + g.sy * z)));
    r[1] = make_float4(q.ux, q.uy, q.uz, q.w);
    r[2] = make_float4(0.f, 0.f, 0.f, 0.f);
  }
}

struct DirPeer { int p[27]; };

// Per-peer count vectors: out[k][d] = departures in direction d if direction
// d's neighbour is peer k, else 0.
__global__ void k_peer_counts(const int64_t *__restrict__ cnt, DirPeer dp, int npeer, int64_t *__restrict__ out) {
  for (int t = threadIdx.x; t < npeer * 27; t += blockDim.x) {
    const int k = t / 27, d = t % 27;
    out[t] = dp.p[d] == k ? cnt[d] : 0;
  }
}

// Append arrivals (their move is complete).
__global__ void k_ghost_unpack(const float4 *__restrict__ recv, int64_t A, vpic_particle_t *__restrict__ p,
                               int64_t np) {
  for (int64_t k = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; k < A;
       k += (int64_t)gridDim.x * blockDim.x) {
    float4 *dst = reinterpret_cast<float4 *>(p + np + k);
    dst[0] = recv[3 * k];
    dst[1] = recv[3 * k + 1];
  }
}

// Device-initiated: arrivals of epoch parity e from the 26 directions ->
// offsets ctr[16 + a], total ctr[2], append base ctr[7]; counters reset.
__global__ void k_di_take_ghost(unsigned char *inbox, int e, int64_t cap, int64_t max_np, int64_t *ctr,
                                int32_t *flag) {
  if (threadIdx.x != 0) return;
  int64_t off = 0;
  for (int a = 0; a < 27; ++a) {
    unsigned long long *cf = reinterpret_cast<unsigned long long *>(inbox + di_cnt_off(di_ghost_slot(e, a)));
    int64_t n = (int64_t)*cf;
    if (n > cap) n = cap;     // the senders flagged the overflow
    ctr[16 + a] = off;
    off += n;
    *cf = 0;
  }
  const int64_t base = ctr[0];
  if (base + off > max_np) {  // no room: drop the arrivals, report capacity
    atomicOr(flag, 4);
    off = 0;
    for (int a = 0; a < 27; ++a) ctr[16 + a] = 0;
  }
  ctr[2] = off;
  ctr[7] = base;
  ctr[0] = base + off;
}
__global__ void k_di_unpack_ghost(const unsigned char *inbox, int e, int64_t cap, const int64_t *ctr,
                                  vpic_particle_t *__restrict__ p) {
  const int64_t A = ctr[2], base = ctr[7];
  for (int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; t < A;
       t += (int64_t)gridDim.x * blockDim.x) {
    int a = 0;
    while (a < 26 && t >= ctr[16 + a + 1]) ++a;
    const int64_t k = t - ctr[16 + a];
    const float4 *rec = reinterpret_cast<const float4 *>(inbox + di_rec_off(di_ghost_slot(e, a), cap, k));
    float4 *dst = reinterpret_cast<float4 *>(p + base + t);
    dst[0] = rec[0];
    dst[1] = rec[1];
  }
}

}  // namespace

int exchange_create(vpic_ctx *c, const uint8_t *uid) {
  Exchange *ex = new Exchange();
  ncclUniqueId id;
  static_assert(sizeof(id.internal) == 128, "nccl unique id size");
  std::copy(uid, uid + 128, id.internal);
  if (ncclCommInitRank(&ex->comm, c->nranks, id, c->rank) != ncclSuccess) {
    delete ex;
    return VPIC_ERR_NCCL;
  }
  if (cudaMalloc(&ex->d_cnt, 96 * sizeof(int64_t)) != cudaSuccess) {
    ncclCommDestroy(ex->comm);
    delete ex;
    return VPIC_ERR_CUDA;
  }
  c->ex = ex;
  return VPIC_OK;
}

void exchange_destroy(vpic_ctx *c) {
  Exchange *ex = c->ex;
  if (!ex) return;
  if (ex->di_dcomm_ok) ncclDevCommDestroy(ex->comm, &ex->di_dcomm);
  if (ex->di_win) ncclCommWindowDeregister(ex->comm, ex->di_win);
  if (ex->di_buf) ncclMemFree(ex->di_buf);
  if (ex->comm) ncclCommDestroy(ex->comm);
  cudaFree(ex->send);
  cudaFree(ex->recv);
  cudaFree(ex->d_cnt);
  cudaFree(ex->plane_send);
  cudaFree(ex->plane_recv);
  cudaFree(ex->mv_arr);
  cudaFree(ex->mv_next);
  cudaFree(ex->di_ctr);
  cudaFree(ex->di_arr);
  cudaFree(ex->di_next);
  cudaFree(ex->di_scr);
  cudaFree(ex->g_dir);
  cudaFree(ex->g_pc);
  for (float *b : ex->acc_plane) cudaFree(b);
  delete ex;
  c->ex = nullptr;
}

// Collective over the communicator (every rank, same cap): allocate the
// inbox window in NCCL symmetric memory, register it, create the device
// communicator (one LSA barrier) and publish the neighbours' inbox addresses
// to the kernels through GridK.
int device_exchange_enable(vpic_ctx *c, int64_t cap) {
  Exchange *ex = c->ex;
  if (!ex || ex->di || cap <= 0) return VPIC_ERR_INVALID;
  const bool ghost = c->gk.ghost_mig != 0;
  const size_t bytes = (size_t)di_rec_off(ghost ? DI_GHOST_SLOTS : DI_FACE_SLOTS, cap, 0);
  CKN(ncclMemAlloc(&ex->di_buf, bytes));
  CKC(cudaMemset(ex->di_buf, 0, DI_HDR));
  CKN(ncclCommWindowRegister(ex->comm, ex->di_buf, bytes, &ex->di_win, NCCL_WIN_COLL_SYMMETRIC));
  ncclDevCommRequirements req{};
  req.lsaBarrierCount = 1;
  CKN(ncclDevCommCreate(ex->comm, &req, &ex->di_dcomm));
  ex->di_dcomm_ok = true;
  Peers27 pr;
  const ncclTeam_t world = ncclTeamWorld(ex->comm);
  const int npeer = ghost ? 27 : 6;   // single-round mode: 26 directions, else 6 faces
  for (int f = 0; f < npeer; ++f) {
    pr.lsa[f] = -1;
    const int r = ghost ? c->nbr26[f] : (c->gk.face_kind[f] == FACE_REMOTE ? c->g.nbr_rank[f] : -1);
    if (r < 0) continue;
    pr.lsa[f] = ncclTeamRankToLsa(ex->comm, world, r);
    if (pr.lsa[f] < 0) return VPIC_ERR_UNSUPPORTED;   // neighbour not load/store reachable
  }
  unsigned char **d_peers = nullptr;
  CKC(cudaMalloc(&d_peers, 27 * sizeof(void *)));
  k_di_peers<<<1, 1>>>(ex->di_win, pr, npeer, d_peers); note_launch();
  unsigned char *h_peers[27];
  const cudaError_t e = cudaMemcpy(h_peers, d_peers, npeer * sizeof(void *), cudaMemcpyDeviceToHost);
  cudaFree(d_peers);
  CKC(e);
  ex->di_cap = cap;
  ex->di_hcap = std::max<int64_t>(8 * cap, 1 << 16);
  CKC(cudaMalloc(&ex->di_ctr, 64 * sizeof(int64_t)));
  CKC(cudaMemset(ex->di_ctr, 0, 64 * sizeof(int64_t)));
  CKC(cudaMalloc(&ex->di_flag, sizeof(int32_t)));
  CKC(cudaMemset(ex->di_flag, 0, sizeof(int32_t)));
  CKC(cudaMalloc(&ex->di_arr, (size_t)6 * cap * sizeof(vpic_mover_t)));
  CKC(cudaMalloc(&ex->di_next, (size_t)6 * cap * sizeof(vpic_mover_t)));
  CKC(cudaMalloc(&ex->di_scr, (size_t)3 * ex->di_hcap * sizeof(uint32_t)));
  if (ghost) for (int f = 0; f < 27; ++f) c->gk.di_peer26[f] = h_peers[f];
  else for (int f = 0; f < 6; ++f) c->gk.di_peer[f] = h_peers[f];
  c->gk.di_cap = cap;
  c->gk.di_flag = ex->di_flag;
  c->gk.di_round = 0;
  c->gk.di_on = 1;
  ex->di = true;
  return VPIC_OK;
}

namespace {

// Remove this round's departures (device count) by back-filling from the tail.
int di_remove_holes(vpic_ctx *c, vpic_particle_t *p, const vpic_mover_t *mv, const int64_t *hdev,
                    int64_t mcap, cudaStream_t s) {
  Exchange *ex = c->ex;
  const unsigned B = (unsigned)c->num_sms * 4;
  uint32_t *tail_dead = ex->di_scr, *low = ex->di_scr + ex->di_hcap, *surv = ex->di_scr + 2 * ex->di_hcap;
  k_di_holes_prep<<<1, 1, 0, s>>>(ex->di_ctr, hdev, std::min(ex->di_hcap, mcap), ex->di_flag); note_launch();
  k_di_clear<<<B, 256, 0, s>>>(tail_dead, ex->di_ctr); note_launch();
  k_di_mark_tail<<<B, 256, 0, s>>>(mv, ex->di_ctr, tail_dead, low); note_launch();
  k_di_tail_surv<<<B, 256, 0, s>>>(tail_dead, ex->di_ctr, surv); note_launch();
  k_di_backfill<<<B, 256, 0, s>>>(p, low, surv, ex->di_ctr); note_launch();
  return cudaGetLastError() == cudaSuccess ? VPIC_OK : VPIC_ERR_CUDA;
}

}  // namespace

// Device-initiated migration (f4).  The movers' particles were already
// stored into the neighbours' round-0 inboxes by advance_p (REMOTE faces) or
// are absorbed; every round: remove this rank's departures, LSA barrier (all
// round-r stores landed), append the arrivals, continue their move -- whose
// departures k_move_movers stores into the round r+1 inboxes.  Counts stay
// on the device; one host synchronisation at the end (the new np).
int migrate_di(vpic_ctx *c, float qsp, vpic_particle_t *p, int64_t *np_io, int64_t max_np,
               vpic_mover_t *movers, int64_t max_movers, const int64_t *n_movers, float *acc,
               cudaStream_t s) {
  Exchange *ex = c->ex;
  int32_t *d_flags = reinterpret_cast<int32_t *>(c->d_count + 1);
  CKC(cudaMemsetAsync(d_flags, 0, 4, s));
  k_di_set<<<1, 1, 0, s>>>(ex->di_ctr, *np_io); note_launch();
  if (int rc = di_remove_holes(c, p, movers, n_movers, max_movers, s)) return rc;
  const int64_t acap = 6 * ex->di_cap;
  const unsigned B = (unsigned)c->num_sms * 4;
  unsigned char *inbox = static_cast<unsigned char *>(ex->di_buf);
  for (int r = 0; r < DI_ROUNDS; ++r) {
    k_lsa_barrier<<<1, 128, 0, s>>>(ex->di_dcomm); note_launch();
    k_di_take<<<1, 32, 0, s>>>(inbox, r, ex->di_cap, max_np, ex->di_ctr, ex->di_flag); note_launch();
    k_di_unpack<<<B, 256, 0, s>>>(inbox, r, ex->di_cap, ex->di_ctr, p, ex->di_arr); note_launch();
    CKC(cudaMemsetAsync(ex->di_ctr + 3, 0, 8, s));
    // departures of the arrivals go to the round r+1 inboxes (dropped after the last round)
    cudaError_t e = (c->math == MATH_IEEE)
        ? launch_move_movers_ieee(c, qsp, p, ex->di_arr, acap, acc, ex->di_next, acap, ex->di_ctr + 3,
                                  d_flags, s, ex->di_ctr + 2, r + 1)
        : launch_move_movers_fast(c, qsp, p, ex->di_arr, acap, acc, ex->di_next, acap, ex->di_ctr + 3,
                                  d_flags, s, ex->di_ctr + 2, r + 1);
    CKC(e);
    if (int rc = di_remove_holes(c, p, ex->di_next, ex->di_ctr + 3, acap, s)) return rc;
  }
  int64_t h_np = 0;
  int32_t h_fl[2] = {0, 0};
  CKC(cudaMemcpyAsync(&h_np, ex->di_ctr, 8, cudaMemcpyDeviceToHost, s));
  CKC(cudaMemcpyAsync(&h_fl[0], d_flags, 4, cudaMemcpyDeviceToHost, s));
  CKC(cudaMemcpyAsync(&h_fl[1], ex->di_flag, 4, cudaMemcpyDeviceToHost, s));
  CKC(cudaStreamSynchronize(s));
  *np_io = h_np;
  if (h_fl[0] || h_fl[1]) {
    CKC(cudaMemsetAsync(ex->di_flag, 0, 4, s));
    return VPIC_ERR_CAPACITY;
  }
  return VPIC_OK;
}

// ------------------------------------------------- single-round migration --
// The 26 neighbour ranks: direction d reaches the rank found by following the
// face neighbours along x, then y, then z (the ranks' face tables are
// all-gathered; one NCCL all-gather at enable time).  A direction is used only
// if every face it crosses is REMOTE here.
int ghost_migration_enable(vpic_ctx *c) {
  Exchange *ex = c->ex;
  if (!ex || ex->di) return VPIC_ERR_INVALID;   // (before VPIC_OPT_DEVICE_EXCHANGE)
  std::vector<int32_t> tab(6 * (size_t)c->nranks);
  if (c->nranks == 1) {
    for (int f = 0; f < 6; ++f) tab[f] = c->g.nbr_rank[f];
  } else {
    int32_t *d = nullptr;
    CKC(cudaMalloc(&d, sizeof(int32_t) * 6 * (c->nranks + 1)));
    CKC(cudaMemcpy(d, c->g.nbr_rank, 6 * sizeof(int32_t), cudaMemcpyHostToDevice));
    if (ncclAllGather(d, d + 6, 6, ncclInt32, ex->comm, 0) != ncclSuccess) { cudaFree(d); return VPIC_ERR_NCCL; }
    const cudaError_t e = cudaMemcpy(tab.data(), d + 6, tab.size() * sizeof(int32_t), cudaMemcpyDeviceToHost);
    cudaFree(d);
    CKC(e);
  }
  for (int dd = 0; dd < 27; ++dd) {
    const int o[3] = {dd % 3 - 1, (dd / 3) % 3 - 1, dd / 9 - 1};
    int r = c->rank;
    bool ok = dd != 13;
    for (int a = 0; a < 3 && ok; ++a) {
      if (!o[a]) continue;
      const int f = o[a] < 0 ? a : a + 3;
      if (c->gk.face_kind[f] != FACE_REMOTE) ok = false;
      else r = tab[6 * (size_t)r + f];
    }
    c->nbr26[dd] = ok ? r : -1;
  }
  // distinct peers: one count message and one record message per peer
  c->npeer26 = 0;
  for (int r = 0; r < c->nranks; ++r) {
    bool used = false;
    for (int dd = 0; dd < 27; ++dd) used |= c->nbr26[dd] == r;
    if (used) c->peer26[c->npeer26++] = r;
  }
  for (int dd = 0; dd < 27; ++dd) {
    c->dir_peer[dd] = -1;
    for (int k = 0; k < c->npeer26; ++k)
      if (c->nbr26[dd] == c->peer26[k]) c->dir_peer[dd] = k;
  }
  if (!ex->g_pc && cudaMalloc(&ex->g_pc, 2 * 27 * 27 * sizeof(int64_t)) != cudaSuccess) return VPIC_ERR_CUDA;
  c->gk.ghost_mig = 1;
  c->di_epoch = 0;
  return VPIC_OK;
}

// The accumulator's ghost layer holds the currents of streaks this rank's
// particles ran in the neighbours' boundary voxels: axis by axis, plane 0 is
// added into the -face neighbour's plane n and plane n+1 into the +face
// neighbour's plane 1, then zeroed.  Planes span the other axes' ghosts, so
// edge and corner ghosts reach the diagonal neighbours in two or three hops.
// Per peer pair: sends (plane 0, plane n+1) and receives (from +, from -) in
// the same order on both sides.
int reduce_acc_ghosts(vpic_ctx *c, float *acc, cudaStream_t s) {
  Exchange *ex = c->ex;
  if (!ex || !c->gk.ghost_mig) return VPIC_OK;
  const GridK &g = c->gk;
  const int sz = g.nz + 2;
  const size_t maxplane =
      (size_t)std::max({(int64_t)g.sy * sz, (int64_t)g.sx * sz, (int64_t)g.sx * g.sy}) * 12 * 4;
  if (maxplane > ex->acc_plane_bytes) {
    for (float *&b : ex->acc_plane) {
      cudaFree(b);
      b = nullptr;
      CKC(cudaMalloc(&b, maxplane));
    }
    ex->acc_plane_bytes = maxplane;
  }
  float **B = ex->acc_plane;
  for (int axis = 0; axis < 3; ++axis) {
    if (c->periodic_local[axis]) continue;
    const int fm = axis, fp = axis + 3;
    const bool rm = g.face_kind[fm] == FACE_REMOTE, rp = g.face_kind[fp] == FACE_REMOTE;
    if (!rm && !rp) continue;
    const int n = axis == 0 ? g.nx : (axis == 1 ? g.ny : g.nz);
    const int64_t cnt =
        (axis == 0 ? (int64_t)g.sy * sz : axis == 1 ? (int64_t)g.sx * sz : (int64_t)g.sx * g.sy) * 12;
    if (rm) { k_plane_copy<<<blocks_for(cnt), 256, 0, s>>>(g, axis, 0, acc, 12, B[0], 3); note_launch(); }
    if (rp) { k_plane_copy<<<blocks_for(cnt), 256, 0, s>>>(g, axis, n + 1, acc, 12, B[1], 3); note_launch(); }
    CKN(ncclGroupStart());
    if (rm) CKN(ncclSend(B[0], cnt, ncclFloat32, c->g.nbr_rank[fm], ex->comm, s));
    if (rp) CKN(ncclSend(B[1], cnt, ncclFloat32, c->g.nbr_rank[fp], ex->comm, s));
    if (rp) CKN(ncclRecv(B[2], cnt, ncclFloat32, c->g.nbr_rank[fp], ex->comm, s));
    if (rm) CKN(ncclRecv(B[3], cnt, ncclFloat32, c->g.nbr_rank[fm], ex->comm, s));
    CKN(ncclGroupEnd());
    if (rp) { k_plane_copy<<<blocks_for(cnt), 256, 0, s>>>(g, axis, n, acc, 12, B[2], 2); note_launch(); }
    if (rm) { k_plane_copy<<<blocks_for(cnt), 256, 0, s>>>(g, axis, 1, acc, 12, B[3], 2); note_launch(); }
    CKC(cudaGetLastError());
  }
  return VPIC_OK;
}

namespace {

// Single-round mode over NCCL: one exchange of the departures with the (up to)
// 26 neighbours, aggregated per distinct peer rank -- a 27-count vector, one
// host synchronisation, then all records for that peer in one message (the
// send buffer is ordered by (peer, direction)) -- then the accumulator
// ghosts.  One message per peer and phase, so the pairing of sends and
// receives cannot be ambiguous even where one rank is the neighbour in
// several directions.
int migrate_ghost(vpic_ctx *c, vpic_particle_t *p, int64_t *np_io, int64_t max_np,
                  const vpic_mover_t *movers, int64_t max_movers, const int64_t *n_movers, float *acc,
                  cudaStream_t s) {
  Exchange *ex = c->ex;
  int64_t M = 0;
  CKC(cudaMemcpyAsync(&M, n_movers, 8, cudaMemcpyDeviceToHost, s));
  CKC(cudaStreamSynchronize(s));
  int64_t np = *np_io;
  if (M > max_movers) return VPIC_ERR_CAPACITY;   // movers were dropped by advance_p
  if (M > np) return VPIC_ERR_INVALID;
  const int64_t Mpad = std::max<int64_t>(M, 1);
  if (int rc = ctx_scratch(c, 16 * (size_t)Mpad + 64)) return rc;
  uint32_t *holes = static_cast<uint32_t *>(c->scratch);
  if (int rc = ensure(reinterpret_cast<void **>(&ex->g_dir), &ex->g_dir_cap, Mpad, 1)) return rc;
  int64_t *cnt = ex->d_cnt;   // [0,27) sent per direction, [54,81) pack cursors
  CKC(cudaMemsetAsync(cnt, 0, 81 * sizeof(int64_t), s));
  if (M > 0) {
    k_ghost_classify<<<blocks_for(M), 256, 0, s>>>(c->gk, p, movers, n_movers, M, ex->g_dir, cnt, holes); note_launch();
  }
  const int np26 = c->npeer26;
  DirPeer dp;
  for (int d = 0; d < 27; ++d) dp.p[d] = c->dir_peer[d];
  int64_t *pc_out = ex->g_pc, *pc_in = ex->g_pc + 27 * 27;
  k_peer_counts<<<1, 256, 0, s>>>(cnt, dp, np26, pc_out); note_launch();
  CKC(cudaGetLastError());
  CKN(ncclGroupStart());
  for (int k = 0; k < np26; ++k) {
    CKN(ncclSend(pc_out + 27 * k, 27, ncclInt64, c->peer26[k], ex->comm, s));
    CKN(ncclRecv(pc_in + 27 * k, 27, ncclInt64, c->peer26[k], ex->comm, s));
  }
  CKN(ncclGroupEnd());
  std::vector<int64_t> h(27 + 27 * (size_t)np26);
  CKC(cudaMemcpyAsync(h.data(), cnt, 27 * sizeof(int64_t), cudaMemcpyDeviceToHost, s));
  if (np26) CKC(cudaMemcpyAsync(h.data() + 27, pc_in, 27 * np26 * sizeof(int64_t), cudaMemcpyDeviceToHost, s));
  CKC(cudaStreamSynchronize(s));
  Off27 so;
  int64_t pso[27], psz[27], pro[27], prz[27];
  int64_t S = 0, A = 0;
  for (int k = 0; k < np26; ++k) {
    pso[k] = S;
    for (int d = 0; d < 27; ++d)
      if (c->dir_peer[d] == k) { so.o[d] = S; S += h[d]; }
    psz[k] = S - pso[k];
    pro[k] = A;
    for (int d = 0; d < 27; ++d) A += h[27 + 27 * k + d];
    prz[k] = A - pro[k];
  }
  for (int d = 0; d < 27; ++d)
    if (c->dir_peer[d] < 0) so.o[d] = 0;
  int64_t tot = ex->send_cap * 6;
  if (int rc = ensure(reinterpret_cast<void **>(&ex->send), &tot, std::max<int64_t>(S, 1), 48)) return rc;
  ex->send_cap = tot / 6;
  if (int rc = ensure(reinterpret_cast<void **>(&ex->recv), &ex->recv_cap, std::max<int64_t>(A, 1), 48)) return rc;
  if (S > 0) {
    k_ghost_pack<<<blocks_for(M), 256, 0, s>>>(c->gk, p, movers, M, ex->g_dir, so,
                                               reinterpret_cast<unsigned long long *>(cnt + 54), ex->send); note_launch();
    CKC(cudaGetLastError());
  }
  CKN(ncclGroupStart());
  for (int k = 0; k < np26; ++k) {
    CKN(ncclSend(ex->send + 3 * pso[k], (size_t)psz[k] * 12, ncclFloat32, c->peer26[k], ex->comm, s));
    CKN(ncclRecv(ex->recv + 3 * pro[k], (size_t)prz[k] * 12, ncclFloat32, c->peer26[k], ex->comm, s));
  }
  CKN(ncclGroupEnd());
  if (int rc = remove_holes(c, p, np, holes, M, s)) return rc;
  np -= M;
  if (np + A > max_np) return VPIC_ERR_CAPACITY;
  if (A > 0) {
    k_ghost_unpack<<<blocks_for(A), 256, 0, s>>>(ex->recv, A, p, np); note_launch();
    CKC(cudaGetLastError());
    np += A;
  }
  if (int rc = reduce_acc_ghosts(c, acc, s)) return rc;
  *np_io = np;   // (every count was known on the host: no further synchronisation)
  return VPIC_OK;
}

// Single-round mode, device-initiated: advance_p already stored every
// departure into its neighbour's inbox (this epoch's slots); remove the holes,
// one LSA barrier, append the arrivals, reduce the accumulator ghosts.  One
// host synchronisation (the new np and the overflow flags).
int migrate_ghost_di(vpic_ctx *c, vpic_particle_t *p, int64_t *np_io, int64_t max_np,
                     const vpic_mover_t *movers, int64_t max_movers, const int64_t *n_movers,
                     float *acc, cudaStream_t s) {
  Exchange *ex = c->ex;
  const int e = (int)(c->di_epoch & 1);
  int32_t *d_flags = reinterpret_cast<int32_t *>(c->d_count + 1);
  CKC(cudaMemsetAsync(d_flags, 0, 4, s));
  k_di_set<<<1, 1, 0, s>>>(ex->di_ctr, *np_io); note_launch();
  if (int rc = di_remove_holes(c, p, movers, n_movers, max_movers, s)) return rc;
  unsigned char *inbox = static_cast<unsigned char *>(ex->di_buf);
  k_lsa_barrier<<<1, 128, 0, s>>>(ex->di_dcomm); note_launch();
  k_di_take_ghost<<<1, 32, 0, s>>>(inbox, e, ex->di_cap, max_np, ex->di_ctr, ex->di_flag); note_launch();
  k_di_unpack_ghost<<<(unsigned)c->num_sms * 4, 256, 0, s>>>(inbox, e, ex->di_cap, ex->di_ctr, p); note_launch();
  CKC(cudaGetLastError());
  c->di_epoch++;
  if (int rc = reduce_acc_ghosts(c, acc, s)) return rc;
  int64_t h_np = 0;
  int32_t h_fl[2] = {0, 0};
  CKC(cudaMemcpyAsync(&h_np, ex->di_ctr, 8, cudaMemcpyDeviceToHost, s));
  CKC(cudaMemcpyAsync(&h_fl[0], d_flags, 4, cudaMemcpyDeviceToHost, s));
  CKC(cudaMemcpyAsync(&h_fl[1], ex->di_flag, 4, cudaMemcpyDeviceToHost, s));
  CKC(cudaStreamSynchronize(s));
  *np_io = h_np;
  if (h_fl[0] || h_fl[1]) {
    CKC(cudaMemsetAsync(ex->di_flag, 0, 4, s));
    return VPIC_ERR_CAPACITY;
  }
  return VPIC_OK;
}

}  // namespace

// The same with the particle count on the device and no host
// synchronisation: every step is a stream operation (kernels, memsets, NCCL
// plane send/recv), so a PIC step or a whole sort period can be captured in a
// CUDA graph and replayed.  The epoch parity is fixed at enqueue time (each
// call flips it), so a captured sequence must hold an even number of calls.
int migrate_dev(vpic_ctx *c, vpic_particle_t *p, int64_t *np_dev, int64_t max_np,
                const vpic_mover_t *movers, int64_t max_movers, const int64_t *n_movers, float *acc,
                int32_t *flags_dev, cudaStream_t s) {
  Exchange *ex = c->ex;
  if (!ex || !ex->di || !c->gk.ghost_mig) return VPIC_ERR_UNSUPPORTED;
  const int e = (int)(c->di_epoch & 1);
  int32_t *d_flags = reinterpret_cast<int32_t *>(c->d_count + 1);
  CKC(cudaMemsetAsync(d_flags, 0, 4, s));
  k_di_set_dev<<<1, 1, 0, s>>>(ex->di_ctr, np_dev); note_launch();
  if (int rc = di_remove_holes(c, p, movers, n_movers, max_movers, s)) return rc;
  unsigned char *inbox = static_cast<unsigned char *>(ex->di_buf);
  k_lsa_barrier<<<1, 128, 0, s>>>(ex->di_dcomm); note_launch();
  k_di_take_ghost<<<1, 32, 0, s>>>(inbox, e, ex->di_cap, max_np, ex->di_ctr, ex->di_flag); note_launch();
  k_di_unpack_ghost<<<(unsigned)c->num_sms * 4, 256, 0, s>>>(inbox, e, ex->di_cap, ex->di_ctr, p); note_launch();
  CKC(cudaGetLastError());
  c->di_epoch++;
  if (int rc = reduce_acc_ghosts(c, acc, s)) return rc;
  k_di_finish<<<1, 1, 0, s>>>(ex->di_ctr, np_dev, d_flags, ex->di_flag, flags_dev); note_launch();
  return cudaGetLastError() == cudaSuccess ? VPIC_OK : VPIC_ERR_CUDA;
}

// Up to 3 rounds: pack movers per face, exchange counts, exchange records,
// remove departed / absorbed particles, append arrivals, continue their move.
// Host synchronisations: the initial mover count, one per round (the NCCL
// record sizes, which also return the round's mover count), one for flags.
int migrate(vpic_ctx *c, float qsp, float msp, vpic_particle_t *p, int64_t *np_io, int64_t max_np,
            vpic_mover_t *movers, int64_t max_movers, const int64_t *n_movers, float *acc,
            cudaStream_t s) {
  (void)msp;
  if (c->ex && c->gk.ghost_mig) {
    return c->ex->di ? migrate_ghost_di(c, p, np_io, max_np, movers, max_movers, n_movers, acc, s)
                     : migrate_ghost(c, p, np_io, max_np, movers, max_movers, n_movers, acc, s);
  }
  if (c->ex && c->ex->di)
    return migrate_di(c, qsp, p, np_io, max_np, movers, max_movers, n_movers, acc, s);
  int64_t M = 0;
  CKC(cudaMemcpyAsync(&M, n_movers, 8, cudaMemcpyDeviceToHost, s));
  CKC(cudaStreamSynchronize(s));
  int64_t np = *np_io;
  if (M > max_movers) return VPIC_ERR_CAPACITY;   // movers were dropped by advance_p
  if (M > np) return VPIC_ERR_INVALID;
  int32_t *d_flags = reinterpret_cast<int32_t *>(c->d_count + 1);
  CKC(cudaMemsetAsync(d_flags, 0, 4, s));
  Exchange *ex = c->ex;
  const vpic_mover_t *cur = movers;
  const int64_t *Mdev = n_movers;   // device count of the current mover list
  int64_t Mmax = M;                 // host upper bound of it
  const int rounds = ex ? 3 : 1;
  for (int round = 0; round <= rounds; ++round) {
    const bool exchange = ex && round < rounds;
    if (!exchange && Mmax == 0) break;
    const int64_t Mpad = std::max<int64_t>(Mmax, 1);
    if (int rc = ctx_scratch(c, 16 * (size_t)Mpad + 64)) return rc;
    uint32_t *holes = static_cast<uint32_t *>(c->scratch);
    int64_t *cnt = ex ? ex->d_cnt : c->d_count + 3;
    if (exchange) {
      int64_t tot = ex->send_cap * 6;
      if (int rc = ensure(reinterpret_cast<void **>(&ex->send), &tot, 6 * Mpad, 48)) return rc;
      ex->send_cap = tot / 6;
    }
    CKC(cudaMemsetAsync(cnt, 0, (ex ? 12 : 1) * sizeof(int64_t), s));
    if (Mmax > 0) {
      k_pack_movers<<<blocks_for(Mmax), 256, 0, s>>>(c->gk, p, cur, Mdev, Mmax, exchange ? ex->send : nullptr,
                                                      exchange ? ex->send_cap : 0, cnt, holes, d_flags); note_launch();
      CKC(cudaGetLastError());
    }
    int64_t sent[6] = {0, 0, 0, 0, 0, 0}, rcvd[6] = {0, 0, 0, 0, 0, 0}, A = 0;
    if (exchange) {
      // counts: one int64 per face to nbr_rank[f]; the neighbour's count for
      // its face f arrives on my face OPP[f] (posting order matches per pair)
      CKN(ncclGroupStart());
      for (int f = 0; f < 6; ++f)
        if (c->gk.face_kind[f] == FACE_REMOTE)
          CKN(ncclSend(cnt + f, 1, ncclInt64, c->g.nbr_rank[f], ex->comm, s));
      for (int f = 0; f < 6; ++f) {
        const int o = OPP[f];
        if (c->gk.face_kind[o] == FACE_REMOTE)
          CKN(ncclRecv(cnt + 6 + o, 1, ncclInt64, c->g.nbr_rank[o], ex->comm, s));
      }
      CKN(ncclGroupEnd());
      int64_t h[13];
      CKC(cudaMemcpyAsync(h, cnt, 12 * sizeof(int64_t), cudaMemcpyDeviceToHost, s));
      CKC(cudaMemcpyAsync(h + 12, Mdev, sizeof(int64_t), cudaMemcpyDeviceToHost, s));
      CKC(cudaStreamSynchronize(s));
      M = std::min(h[12], Mmax);
      for (int f = 0; f < 6; ++f) {
        sent[f] = h[f];
        rcvd[f] = h[6 + f];
        A += rcvd[f];
        if (sent[f] > ex->send_cap) return VPIC_ERR_CAPACITY;
      }
      if (int rc = ensure(reinterpret_cast<void **>(&ex->recv), &ex->recv_cap, std::max<int64_t>(A, 1), 48))
        return rc;
      float4 *rptr[6];
      int64_t roff = 0;
      for (int f = 0; f < 6; ++f) { rptr[f] = ex->recv + 3 * roff; roff += rcvd[f]; }
      CKN(ncclGroupStart());
      for (int f = 0; f < 6; ++f)
        if (c->gk.face_kind[f] == FACE_REMOTE)
          CKN(ncclSend(ex->send + 3 * (int64_t)f * ex->send_cap, (size_t)sent[f] * 12, ncclFloat32,
                       c->g.nbr_rank[f], ex->comm, s));
      for (int f = 0; f < 6; ++f) {
        const int o = OPP[f];
        if (c->gk.face_kind[o] == FACE_REMOTE)
          CKN(ncclRecv(rptr[o], (size_t)rcvd[o] * 12, ncclFloat32, c->g.nbr_rank[o], ex->comm, s));
      }
      CKN(ncclGroupEnd());
    } else if (round > 0) {  // final clean-up round: the exact count of the leftovers
      CKC(cudaMemcpyAsync(&M, Mdev, 8, cudaMemcpyDeviceToHost, s));
      CKC(cudaStreamSynchronize(s));
      M = std::min(M, Mmax);
    }
    // every mover's particle has left this rank (sent or absorbed)
    if (int rc = remove_holes(c, p, np, holes, M, s)) return rc;
    np -= M;
    if (!exchange) break;
    if (np + A > max_np) return VPIC_ERR_CAPACITY;
    Mmax = 0;
    if (A > 0) {
      if (int rc = ensure(reinterpret_cast<void **>(&ex->mv_arr), &ex->mv_arr_cap, A, 16)) return rc;
      if (int rc = ensure(reinterpret_cast<void **>(&ex->mv_next), &ex->mv_next_cap, A, 16)) return rc;
      k_unpack<<<blocks_for(A), 256, 0, s>>>(ex->recv, A, p, np, ex->mv_arr); note_launch();
      CKC(cudaGetLastError());
      int64_t *d_next = c->d_count + 3;
      CKC(cudaMemsetAsync(d_next, 0, 8, s));
      cudaError_t e = (c->math == MATH_IEEE)
                          ? launch_move_movers_ieee(c, qsp, p, ex->mv_arr, A, acc, ex->mv_next, A, d_next, d_flags, s)
                          : launch_move_movers_fast(c, qsp, p, ex->mv_arr, A, acc, ex->mv_next, A, d_next, d_flags, s);
      CKC(e);
      np += A;
      cur = ex->mv_next;
      Mdev = d_next;
      Mmax = A;     // the arrivals' new movers: at most A, exact count on device
    }
  }
  int32_t hflag = 0;
  CKC(cudaMemcpyAsync(&hflag, d_flags, 4, cudaMemcpyDeviceToHost, s));
  CKC(cudaStreamSynchronize(s));
  *np_io = np;
  if (hflag) return VPIC_ERR_CAPACITY;
  return VPIC_OK;
}

// E/cB ghost planes from the neighbours, axis by axis (edges / corners
// propagate because each plane spans the other axes' ghosts).  dir = +1: my
// plane 1 goes to the -face neighbour, whose plane n+1 it fills; dir = -1: my
// plane n goes to the +face neighbour, whose plane 0 it fills.
int halo_fields(vpic_ctx *c, float *fields, cudaStream_t s, int dir) {
  Exchange *ex = c->ex;
  const GridK &g = c->gk;
  const int sz = g.nz + 2;
  const size_t maxplane = (size_t)std::max({(int64_t)g.sy * sz, (int64_t)g.sx * sz, (int64_t)g.sx * g.sy}) * 8 * 4;
  if (int rc = ensure_plane(ex, maxplane)) return rc;
  for (int axis = 0; axis < 3; ++axis) {
    if (c->periodic_local[axis]) continue;
    const int f_to = dir > 0 ? axis : axis + 3;     // face whose neighbour receives my plane
    const int f_from = dir > 0 ? axis + 3 : axis;   // face whose neighbour fills my ghost
    const bool snd = g.face_kind[f_to] == FACE_REMOTE, rcv = g.face_kind[f_from] == FACE_REMOTE;
    if (!snd && !rcv) continue;
    const int n = axis == 0 ? g.nx : (axis == 1 ? g.ny : g.nz);
    const int src_plane = dir > 0 ? 1 : n, dst_plane = dir > 0 ? n + 1 : 0;
    const int64_t cnt = (axis == 0 ? (int64_t)g.sy * sz : axis == 1 ? (int64_t)g.sx * sz : (int64_t)g.sx * g.sy) * 8;
    if (snd) { k_plane_copy<<<blocks_for(cnt), 256, 0, s>>>(g, axis, src_plane, fields, 8, ex->plane_send, 0); note_launch(); }
    CKN(ncclGroupStart());
    if (snd) CKN(ncclSend(ex->plane_send, cnt, ncclFloat32, c->g.nbr_rank[f_to], ex->comm, s));
    if (rcv) CKN(ncclRecv(ex->plane_recv, cnt, ncclFloat32, c->g.nbr_rank[f_from], ex->comm, s));
    CKN(ncclGroupEnd());
    if (rcv) { k_plane_copy<<<blocks_for(cnt), 256, 0, s>>>(g, axis, dst_plane, fields, 8, ex->plane_recv, 1); note_launch(); }
    CKC(cudaGetLastError());
  }
  return VPIC_OK;
}

// jf shared planes: my plane n+1 partial sums belong to the +face neighbour's
// plane 1 (added there); then the completed plane 1 is sent back to fill the
// -face neighbour's plane n+1.  Axis by axis.
int reduce_jf(vpic_ctx *c, float *jf, cudaStream_t s) {
  Exchange *ex = c->ex;
  const GridK &g = c->gk;
  const int sz = g.nz + 2;
  const size_t maxplane = (size_t)std::max({(int64_t)g.sy * sz, (int64_t)g.sx * sz, (int64_t)g.sx * g.sy}) * 4 * 4;
  if (int rc = ensure_plane(ex, maxplane)) return rc;
  for (int axis = 0; axis < 3; ++axis) {
    if (c->periodic_local[axis]) continue;
    const int fm = axis, fp = axis + 3;
    const bool rm = g.face_kind[fm] == FACE_REMOTE, rp = g.face_kind[fp] == FACE_REMOTE;
    if (!rm && !rp) continue;
    const int n = axis == 0 ? g.nx : (axis == 1 ? g.ny : g.nz);
    const int64_t cnt = (axis == 0 ? (int64_t)g.sy * sz : axis == 1 ? (int64_t)g.sx * sz : (int64_t)g.sx * g.sy) * 4;
    // phase 1: plane n+1 -> +neighbour, add into plane 1
    if (rp) { k_plane_copy<<<blocks_for(cnt), 256, 0, s>>>(g, axis, n + 1, jf, 4, ex->plane_send, 0); note_launch(); }
    CKN(ncclGroupStart());
    if (rp) CKN(ncclSend(ex->plane_send, cnt, ncclFloat32, c->g.nbr_rank[fp], ex->comm, s));
    if (rm) CKN(ncclRecv(ex->plane_recv, cnt, ncclFloat32, c->g.nbr_rank[fm], ex->comm, s));
    CKN(ncclGroupEnd());
    if (rm) { k_plane_copy<<<blocks_for(cnt), 256, 0, s>>>(g, axis, 1, jf, 4, ex->plane_recv, 2); note_launch(); }
    // phase 2: plane 1 -> -neighbour's plane n+1
    if (rm) { k_plane_copy<<<blocks_for(cnt), 256, 0, s>>>(g, axis, 1, jf, 4, ex->plane_send, 0); note_launch(); }
    CKN(ncclGroupStart());
    if (rm) CKN(ncclSend(ex->plane_send, cnt, ncclFloat32, c->g.nbr_rank[fm], ex->comm, s));
    if (rp) CKN(ncclRecv(ex->plane_recv, cnt, ncclFloat32, c->g.nbr_rank[fp], ex->comm, s));
    CKN(ncclGroupEnd());
    if (rp) { k_plane_copy<<<blocks_for(cnt), 256, 0, s>>>(g, axis, n + 1, jf, 4, ex->plane_recv, 1); note_launch(); }
    CKC(cudaGetLastError());
  }
  return VPIC_OK;
}

}  // namespace vpic
