// The C ABI of libvpic.so (include/vpic.h): host-side validation, the
// context, and dispatch to the kernels.  No C++ exception crosses the ABI
// and nothing aborts; every entry point returns a vpic_status.
#include <nccl.h>
#include <nvtx3/nvToolsExt.h>

#include <atomic>
#include <cstring>
#include <new>

#include "vpic_internal.cuh"

using namespace vpic;

namespace {

bool aligned16(const void *p) { return (reinterpret_cast<uintptr_t>(p) & 15u) == 0; }
bool aligned32(const void *p) { return (reinterpret_cast<uintptr_t>(p) & 31u) == 0; }

cudaStream_t S(void *s) { return static_cast<cudaStream_t>(s); }

int cuda_status(cudaError_t e) { return e == cudaSuccess ? VPIC_OK : VPIC_ERR_CUDA; }

bool grid_ok(const vpic_grid_t *g) {
  if (!g) return false;
  if (g->nx < 1 || g->ny < 1 || g->nz < 1) return false;
  const int64_t nv = (int64_t)(g->nx + 2) * (g->ny + 2) * (g->nz + 2);
  if (nv > (int64_t)1 << 28) return false;  // 8*voxel+face must fit int32 (mover encoding)
  if (!(g->dx > 0 && g->dy > 0 && g->dz > 0 && g->dt > 0 && g->cvac > 0)) return false;
  for (int f = 0; f < 6; ++f)
    if (g->pbc[f] < 0 || g->pbc[f] > 2) return false;
  return true;
}

// One NVTX range per C-ABI call (SURVEY.md §5 tracing): visible in nsys /
// ncu --nvtx timelines; a no-op without an attached tool.
struct NvtxRange {
  explicit NvtxRange(const char *name) { nvtxRangePushA(name); }
  ~NvtxRange() { nvtxRangePop(); }
};
#define VPIC_NVTX() NvtxRange nvtx_range_(__func__)

struct DeviceGuard {
  int prev = -1;
  explicit DeviceGuard(int dev) {
    if (cudaGetDevice(&prev) != cudaSuccess) prev = -1;
    if (prev != dev) cudaSetDevice(dev);
  }
  ~DeviceGuard() {
    if (prev >= 0) cudaSetDevice(prev);
  }
};

}  // namespace

namespace vpic {
static std::atomic<int64_t> g_launches{0};
void note_launch(int n) { g_launches.fetch_add(n, std::memory_order_relaxed); }

cudaError_t launch_advance_p(const vpic_ctx *c, float qsp, float msp, vpic_particle_t *p,
                             int64_t np, const float *interp, float *acc, vpic_mover_t *movers,
                             int64_t max_movers, int64_t *n_movers, int32_t *flags,
                             cudaStream_t s, const int64_t *np_dev, uint32_t *keys_out) {
  if (c->math == MATH_IEEE)
    return launch_advance_p_ieee(c, qsp, msp, p, np, interp, acc, movers, max_movers, n_movers,
                                 flags, s, np_dev, keys_out);
  return launch_advance_p_fast(c, qsp, msp, p, np, interp, acc, movers, max_movers, n_movers,
                               flags, s, np_dev, keys_out);
}
}  // namespace vpic

extern "C" {

int64_t vpic_kernel_launches(void) { return vpic::g_launches.load(); }

const char *vpic_status_string(int status) {
  switch (status) {
    case VPIC_OK: return "ok";
    case VPIC_ERR_INVALID: return "invalid argument";
    case VPIC_ERR_CAPACITY: return "capacity exceeded";
    case VPIC_ERR_CUDA: return "CUDA error";
    case VPIC_ERR_NCCL: return "NCCL error";
    case VPIC_ERR_UNSUPPORTED: return "unsupported (needs an sm_100 device)";
    default: return "unknown status";
  }
}

int vpic_get_unique_id(uint8_t uid[128]) {
  if (!uid) return VPIC_ERR_INVALID;
  ncclUniqueId id;
  if (ncclGetUniqueId(&id) != ncclSuccess) return VPIC_ERR_NCCL;
  std::memcpy(uid, id.internal, 128);
  return VPIC_OK;
}

int vpic_ctx_create(vpic_ctx **out, const vpic_grid_t *g, int rank, int nranks,
                    const uint8_t *uid, int device) {
  VPIC_NVTX();
  if (!out || !grid_ok(g) || nranks < 1 || rank < 0 || rank >= nranks) return VPIC_ERR_INVALID;
  *out = nullptr;
  for (int f = 0; f < 6; ++f) {
    if (g->pbc[f] != VPIC_BC_PERIODIC) continue;
    if (g->nbr_rank[f] < 0 || g->nbr_rank[f] >= nranks) return VPIC_ERR_INVALID;
  }
  if (nranks > 1 && !uid) return VPIC_ERR_INVALID;
  int ndev = 0;
  if (cudaGetDeviceCount(&ndev) != cudaSuccess || device < 0 || device >= ndev)
    return VPIC_ERR_UNSUPPORTED;
  DeviceGuard dg(device);   // the caller's current device is restored on return
  cudaDeviceProp prop;
  if (cudaGetDeviceProperties(&prop, device) != cudaSuccess) return VPIC_ERR_CUDA;
  if (prop.major != 10 || prop.minor != 0) return VPIC_ERR_UNSUPPORTED;  // sm_100a code only

  vpic_ctx *c = new (std::nothrow) vpic_ctx();
  if (!c) return VPIC_ERR_CAPACITY;
  c->g = *g;
  c->rank = rank;
  c->nranks = nranks;
  c->device = device;
  c->num_sms = prop.multiProcessorCount;
  c->l2_bytes = prop.l2CacheSize;
  c->tile_sz = 3 * (int64_t)c->num_sms * 128;  // "three times the number of GPU cores"
  c->math = MATH_FAST;
  c->deposit = DEP_AUTO;
  c->adv_kernel = ADV_AUTO;
  c->adv_cps = 0;
  GridK &k = c->gk;
  k.nx = g->nx; k.ny = g->ny; k.nz = g->nz;
  k.sx = g->nx + 2; k.sy = g->ny + 2; k.sxy = k.sx * k.sy;
  k.nv = (int64_t)k.sxy * (g->nz + 2);
  // same expressions, same order as the oracle: (c dt) / dx
  k.cdt_dx = g->cvac * g->dt / g->dx;
  k.cdt_dy = g->cvac * g->dt / g->dy;
  k.cdt_dz = g->cvac * g->dt / g->dz;
  k.dt = g->dt;
  k.cvac = g->cvac;
  set_magic((uint32_t)k.sx, k.mag_sx, k.sh_sx);
  set_magic((uint32_t)k.sxy, k.mag_sxy, k.sh_sxy);
  for (int f = 0; f < 6; ++f) {
    if (g->pbc[f] == VPIC_BC_REFLECT) k.face_kind[f] = FACE_REFLECT;
    else if (g->pbc[f] == VPIC_BC_ABSORB) k.face_kind[f] = FACE_ABSORB;
    else k.face_kind[f] = (g->nbr_rank[f] == rank) ? FACE_LOCAL : FACE_REMOTE;
  }
  for (int a = 0; a < 3; ++a)
    c->periodic_local[a] = k.face_kind[a] == FACE_LOCAL && k.face_kind[a + 3] == FACE_LOCAL;
  if (cudaMalloc(&c->d_count, 8 * sizeof(int64_t)) != cudaSuccess) {
    delete c;
    return VPIC_ERR_CUDA;
  }
  cudaMemset(c->d_count, 0, 8 * sizeof(int64_t));
  if (nranks > 1) {
    const int rc = exchange_create(c, uid);
    if (rc != VPIC_OK) {
      cudaFree(c->d_count);
      delete c;
      return rc;
    }
  }
  *out = c;
  return VPIC_OK;
}

int vpic_ctx_destroy(vpic_ctx *c) {
  VPIC_NVTX();
  if (!c) return VPIC_ERR_INVALID;
  DeviceGuard dg(c->device);
  exchange_destroy(c);
  cudaFree(c->scratch);
  cudaFree(c->d_count);
  delete c;
  return VPIC_OK;
}

int vpic_ctx_set_option(vpic_ctx *c, int option, int64_t value) {
  VPIC_NVTX();
  if (!c) return VPIC_ERR_INVALID;
  switch (option) {
    case VPIC_OPT_MATH:
      if (value != MATH_FAST && value != MATH_IEEE) return VPIC_ERR_INVALID;
      c->math = (int)value;
      return VPIC_OK;
    case VPIC_OPT_DEPOSIT:
      if (value < DEP_AUTO || value > DEP_SMEM) return VPIC_ERR_INVALID;
      c->deposit = (int)value;
      return VPIC_OK;
    case VPIC_OPT_TILE_SZ:
      if (value <= 0) return VPIC_ERR_INVALID;
      c->tile_sz = value;
      return VPIC_OK;
    case VPIC_OPT_ADVANCE_KERNEL:
      if (value < ADV_AUTO || value > ADV_TMA) return VPIC_ERR_INVALID;
      c->adv_kernel = (int)value;
      return VPIC_OK;
    case VPIC_OPT_ADVANCE_CTAS_PER_SM:
      if (value < 0 || value > 2) return VPIC_ERR_INVALID;
      c->adv_cps = (int)value;
      return VPIC_OK;
    case VPIC_OPT_SINGLE_ROUND_MIGRATION: {
      if (value != 1 || !c->ex || c->gk.ghost_mig) return VPIC_ERR_INVALID;
      DeviceGuard dg(c->device);
      return ghost_migration_enable(c);
    }
    case VPIC_OPT_DEVICE_EXCHANGE: {
      if (value < 1 || !c->ex) return VPIC_ERR_INVALID;
      DeviceGuard dg(c->device);
      return device_exchange_enable(c, value == 1 ? ((int64_t)1 << 19) : value);
    }
    case VPIC_OPT_LOOPBACK_EXCHANGE: {
      if (value != 1 || c->nranks != 1 || c->ex) return VPIC_ERR_INVALID;
      DeviceGuard dg(c->device);
      uint8_t uid[128];
      int rc = vpic_get_unique_id(uid);
      if (rc != VPIC_OK) return rc;
      rc = exchange_create(c, uid);
      if (rc != VPIC_OK) return rc;
      for (int f = 0; f < 6; ++f)
        if (c->g.pbc[f] == VPIC_BC_PERIODIC) c->gk.face_kind[f] = FACE_REMOTE;
      for (int a = 0; a < 3; ++a) c->periodic_local[a] = false;
      return VPIC_OK;
    }
    default:
      return VPIC_ERR_INVALID;
  }
}

int vpic_ctx_info(const vpic_ctx *c, int64_t info[8]) {
  if (!c || !info) return VPIC_ERR_INVALID;
  info[0] = c->num_sms;
  info[1] = c->tile_sz;
  info[2] = c->gk.nv;
  info[3] = c->rank;
  info[4] = c->nranks;
  info[5] = c->l2_bytes;
  info[6] = c->math;
  info[7] = c->deposit;
  return VPIC_OK;
}

size_t vpic_sort_workspace_bytes(const vpic_ctx *c, int64_t np, int order) {
  if (!c || np < 0) return 0;
  return sort_workspace_bytes(c, np, order);
}

int vpic_sort_particles(vpic_ctx *c, const vpic_particle_t *p_in, vpic_particle_t *p_out,
                        int64_t np, int order, int64_t tile_sz, void *ws, size_t ws_bytes,
                        int32_t *voxel_counts, int64_t *new_keys, int64_t *perm, void *stream) {
  VPIC_NVTX();
  if (!c || np < 0 || np >= ((int64_t)1 << 32) || order < 0 || order > 3 || tile_sz < 0)
    return VPIC_ERR_INVALID;
  if (np > 0 && (!p_in || !p_out || !aligned16(p_in) || !aligned16(p_out))) return VPIC_ERR_INVALID;
  if (np > 0 && p_in == p_out) return VPIC_ERR_INVALID;
  if (np > 0 && order != VPIC_SORT_NONE) {
    if (!ws) return VPIC_ERR_INVALID;
    if (ws_bytes < sort_workspace_bytes(c, np, order)) return VPIC_ERR_CAPACITY;
  }
  DeviceGuard dg(c->device);
  return cuda_status(launch_sort(c, p_in, p_out, np, order, tile_sz, ws, ws_bytes, voxel_counts,
                                 new_keys, perm, S(stream)));
}

int vpic_sort_particles_keyed(vpic_ctx *c, const vpic_particle_t *p_in, vpic_particle_t *p_out,
                              int64_t np, int order, int64_t tile_sz, const uint32_t *keys, void *ws,
                              size_t ws_bytes, int32_t *voxel_counts, int64_t *new_keys, int64_t *perm,
                              void *stream) {
  VPIC_NVTX();
  if (!c || np < 0 || np >= ((int64_t)1 << 32) || order < 0 || order > 3 || tile_sz < 0)
    return VPIC_ERR_INVALID;
  if (np > 0 && (!p_in || !p_out || !keys || !aligned16(p_in) || !aligned16(p_out) ||
                 (reinterpret_cast<uintptr_t>(keys) & 3u)))
    return VPIC_ERR_INVALID;
  if (np > 0 && p_in == p_out) return VPIC_ERR_INVALID;
  if (np > 0 && order != VPIC_SORT_NONE) {
    if (!ws) return VPIC_ERR_INVALID;
    if (ws_bytes < sort_workspace_bytes(c, np, order)) return VPIC_ERR_CAPACITY;
  }
  DeviceGuard dg(c->device);
  return cuda_status(launch_sort(c, p_in, p_out, np, order, tile_sz, ws, ws_bytes, voxel_counts,
                                 new_keys, perm, S(stream), keys));
}

int vpic_load_interpolator(vpic_ctx *c, float *fields, float *interp, void *stream) {
  VPIC_NVTX();
  if (!c || !fields || !interp || !aligned16(fields) || !aligned32(interp)) return VPIC_ERR_INVALID;
  DeviceGuard dg(c->device);
  cudaError_t e = launch_fill_ghosts(c, fields, S(stream));
  if (e != cudaSuccess) return VPIC_ERR_CUDA;
  if (c->ex) {
    const int rc = halo_fields(c, fields, S(stream), +1);
    if (rc != VPIC_OK) return rc;
  }
  return cuda_status(launch_load_interp(c, fields, interp, S(stream)));
}

int vpic_clear_accumulator(vpic_ctx *c, float *acc, void *stream) {
  VPIC_NVTX();
  if (!c || !acc) return VPIC_ERR_INVALID;
  DeviceGuard dg(c->device);
  return cuda_status(cudaMemsetAsync(acc, 0, (size_t)c->gk.nv * 48, S(stream)));
}

int vpic_advance_p(vpic_ctx *c, float q, float m, vpic_particle_t *p, int64_t np,
                   const float *interp, float *acc, vpic_mover_t *movers, int64_t max_movers,
                   int64_t *n_movers, int32_t *flags, void *stream) {
  VPIC_NVTX();
  if (!c || np < 0 || np >= ((int64_t)1 << 31) || !(m > 0) || max_movers < 0) return VPIC_ERR_INVALID;
  if (np == 0) return VPIC_OK;
  if (!p || !interp || !acc || !n_movers || !aligned16(p) || !aligned32(interp) || !aligned16(acc))
    return VPIC_ERR_INVALID;
  if (max_movers > 0 && (!movers || !aligned16(movers))) return VPIC_ERR_INVALID;
  if ((reinterpret_cast<uintptr_t>(n_movers) & 7u) != 0) return VPIC_ERR_INVALID;
  DeviceGuard dg(c->device);
  return cuda_status(launch_advance_p(c, q, m, p, np, interp, acc, movers, max_movers, n_movers,
                                      flags, S(stream)));
}

int vpic_advance_p_keys(vpic_ctx *c, float q, float m, vpic_particle_t *p, int64_t np,
                        const float *interp, float *acc, vpic_mover_t *movers, int64_t max_movers,
                        int64_t *n_movers, int32_t *flags, uint32_t *keys_out, void *stream) {
  VPIC_NVTX();
  if (!c || np < 0 || np >= ((int64_t)1 << 31) || !(m > 0) || max_movers < 0) return VPIC_ERR_INVALID;
  if (np == 0) return VPIC_OK;
  if (!p || !interp || !acc || !n_movers || !keys_out || !aligned16(p) || !aligned32(interp) ||
      !aligned16(acc) || (reinterpret_cast<uintptr_t>(keys_out) & 3u))
    return VPIC_ERR_INVALID;
  if (max_movers > 0 && (!movers || !aligned16(movers))) return VPIC_ERR_INVALID;
  if ((reinterpret_cast<uintptr_t>(n_movers) & 7u) != 0) return VPIC_ERR_INVALID;
  DeviceGuard dg(c->device);
  return cuda_status(launch_advance_p(c, q, m, p, np, interp, acc, movers, max_movers, n_movers,
                                      flags, S(stream), nullptr, keys_out));
}

int vpic_advance_p_dev(vpic_ctx *c, float q, float m, vpic_particle_t *p, const int64_t *np_dev,
                       int64_t max_np, const float *interp, float *acc, vpic_mover_t *movers,
                       int64_t max_movers, int64_t *n_movers, int32_t *flags, void *stream) {
  VPIC_NVTX();
  if (!c || !np_dev || max_np < 0 || max_np >= ((int64_t)1 << 31) || !(m > 0) || max_movers < 0)
    return VPIC_ERR_INVALID;
  if ((reinterpret_cast<uintptr_t>(np_dev) & 7u) != 0) return VPIC_ERR_INVALID;
  if (max_np == 0) return VPIC_OK;
  if (!p || !interp || !acc || !n_movers || !aligned16(p) || !aligned32(interp) || !aligned16(acc))
    return VPIC_ERR_INVALID;
  if (max_movers > 0 && (!movers || !aligned16(movers))) return VPIC_ERR_INVALID;
  if ((reinterpret_cast<uintptr_t>(n_movers) & 7u) != 0) return VPIC_ERR_INVALID;
  DeviceGuard dg(c->device);
  return cuda_status(launch_advance_p(c, q, m, p, max_np, interp, acc, movers, max_movers, n_movers,
                                      flags, S(stream), np_dev));
}

int vpic_unload_accumulator(vpic_ctx *c, const float *acc, float *jf, void *stream) {
  VPIC_NVTX();
  if (!c || !acc || !jf || !aligned16(acc) || !aligned16(jf)) return VPIC_ERR_INVALID;
  DeviceGuard dg(c->device);
  if (cudaMemsetAsync(jf, 0, (size_t)c->gk.nv * 16, S(stream)) != cudaSuccess) return VPIC_ERR_CUDA;
  cudaError_t e = launch_unload(c, acc, jf, S(stream));
  if (e != cudaSuccess) return VPIC_ERR_CUDA;
  if (c->ex) return reduce_jf(c, jf, S(stream));
  return VPIC_OK;
}

int vpic_advance_b(vpic_ctx *c, float *fields, float frac, void *stream) {
  VPIC_NVTX();
  if (!c || !fields || !aligned16(fields) || !(frac >= 0)) return VPIC_ERR_INVALID;
  DeviceGuard dg(c->device);
  if (launch_fill_ghosts(c, fields, S(stream)) != cudaSuccess) return VPIC_ERR_CUDA;
  if (c->ex) {
    const int rc = halo_fields(c, fields, S(stream), +1);
    if (rc != VPIC_OK) return rc;
  }
  return cuda_status(launch_advance_b(c, fields, frac, S(stream)));
}

int vpic_advance_e(vpic_ctx *c, float *fields, const float *jf, float eps0, void *stream) {
  VPIC_NVTX();
  if (!c || !fields || !jf || !aligned16(fields) || !aligned16(jf) || !(eps0 > 0))
    return VPIC_ERR_INVALID;
  DeviceGuard dg(c->device);
  if (launch_fill_ghosts_minus(c, fields, S(stream)) != cudaSuccess) return VPIC_ERR_CUDA;
  if (c->ex) {
    const int rc = halo_fields(c, fields, S(stream), -1);
    if (rc != VPIC_OK) return rc;
  }
  return cuda_status(launch_advance_e(c, fields, jf, eps0, S(stream)));
}

int vpic_accumulate_rho(vpic_ctx *c, float q, const vpic_particle_t *p, int64_t np, float *rho,
                        void *stream) {
  VPIC_NVTX();
  if (!c || np < 0 || !rho || (np > 0 && (!p || !aligned16(p)))) return VPIC_ERR_INVALID;
  DeviceGuard dg(c->device);
  return cuda_status(launch_accumulate_rho(c, q, p, np, rho, S(stream)));
}

int vpic_continuity_residual(vpic_ctx *c, const float *rho0, const float *rho1, const float *jf,
                             float *out, float *res, void *stream) {
  VPIC_NVTX();
  if (!c || !rho0 || !rho1 || !jf || !out || !aligned16(jf)) return VPIC_ERR_INVALID;
  DeviceGuard dg(c->device);
  return cuda_status(launch_continuity(c, rho0, rho1, jf, out, res, S(stream)));
}

int vpic_gather_scatter(vpic_ctx *c, const int32_t *keys, const double *x, int64_t n,
                        const double *table, double *out, double *acc, int64_t nkeys,
                        int64_t stencil_nx, int aggregate, void *stream) {
  VPIC_NVTX();
  if (!c || n < 0 || nkeys <= 0 || nkeys >= ((int64_t)1 << 31) || stencil_nx < 0) return VPIC_ERR_INVALID;
  if (n > 0 && (!keys || !x || !table || !out || !acc)) return VPIC_ERR_INVALID;
  DeviceGuard dg(c->device);
  return cuda_status(launch_gather_scatter(c, keys, x, n, table, out, acc, nkeys, stencil_nx,
                                           aggregate, S(stream)));
}

int vpic_migrate_particles(vpic_ctx *c, float q, float m, vpic_particle_t *p, int64_t *np,
                           int64_t max_np, vpic_mover_t *movers, int64_t max_movers,
                           const int64_t *n_movers, float *acc, void *stream) {
  VPIC_NVTX();
  if (!c || !np || *np < 0 || max_np < *np || !n_movers || !acc || max_movers < 0)
    return VPIC_ERR_INVALID;
  if (max_np >= ((int64_t)1 << 31)) return VPIC_ERR_INVALID;
  if (*np > 0 && (!p || !aligned16(p))) return VPIC_ERR_INVALID;
  if (max_movers > 0 && (!movers || !aligned16(movers))) return VPIC_ERR_INVALID;
  DeviceGuard dg(c->device);
  return migrate(c, q, m, p, np, max_np, movers, max_movers, n_movers, acc, S(stream));
}

int vpic_migrate_particles_dev(vpic_ctx *c, float q, float m, vpic_particle_t *p, int64_t *np_dev,
                               int64_t max_np, const vpic_mover_t *movers, int64_t max_movers,
                               const int64_t *n_movers, float *acc, int32_t *flags_dev,
                               void *stream) {
  VPIC_NVTX();
  (void)q; (void)m;
  if (!c || !np_dev || max_np < 0 || max_np >= ((int64_t)1 << 31) || !n_movers || !acc || !p ||
      !aligned16(p) || !flags_dev || max_movers < 0)
    return VPIC_ERR_INVALID;
  if (max_movers > 0 && (!movers || !aligned16(movers))) return VPIC_ERR_INVALID;
  DeviceGuard dg(c->device);
  return migrate_dev(c, p, np_dev, max_np, movers, max_movers, n_movers, acc, flags_dev, S(stream));
}

}  // extern "C"
