// Internal declarations shared by the libvpic.so translation units.
// Nothing here is shared with oracle/ (the two are independent by design).
#pragma once

#include <cuda_runtime.h>
#include <stdint.h>

#include <atomic>

#include "../../include/vpic.h"

namespace vpic {

// Grid constants passed by value to kernels (kernel-param constant bank).
// VPIC_CHECK=1 (dev builds only: tools/check_build.sh): device-side bounds
// checks on the hot paths' computed indices -- voxel rows gathered and
// scattered, chunk and record slots, sort positions -- trapping on the first
// violation (the stand-in for compute-sanitizer, closed on the GPU pool).
#ifndef VPIC_CHECK
#define VPIC_CHECK 0
#endif
#define VPIC_ASSERT(cond) do { if (VPIC_CHECK && !(cond)) __trap(); } while (0)

// Interpolator layout (include/vpic.h): VPIC_INTERP_SPLIT = 1 stores the
// first 16 coefficients of every voxel as a 64-B row (two sector-aligned
// 32-B loads) and the last two (cbz, dcbz/dz) in a compact 8-B array after
// the rows (4 voxels per sector), inside the same [nv][24] float buffer.
#ifndef VPIC_INTERP_SPLIT
#define VPIC_INTERP_SPLIT 1
#endif

struct GridK {
  int32_t nx, ny, nz;
  int32_t sx, sy;            // nx+2, ny+2
  int32_t sxy;               // sx*sy
  int64_t nv;
  float cdt_dx, cdt_dy, cdt_dz;
  float dt, cvac;
  // per face: 0 = local neighbour/wrap, 1 = reflect, 2 = absorb, 3 = remote
  int32_t face_kind[6];
  // v / sx and v / sxy for 0 <= v < 2^31 as umulhi(v, mag) >> sh (set_magic)
  uint32_t mag_sx, sh_sx, mag_sxy, sh_sxy;
  // device-initiated exchange (VPIC_OPT_DEVICE_EXCHANGE):
  // a particle stopping on a REMOTE face f is stored straight into the
  // inbox window of nbr_rank[f] (NCCL symmetric memory, LSA address di_peer[f])
  unsigned char *di_peer[6];
  int64_t di_cap;            // records per (round, face) inbox
  int32_t *di_flag;          // local: bit 0 set when an inbox was full
  int32_t di_round;          // migration round of this launch's departures
                             // (single-round mode: the epoch parity)
  int32_t di_on;
  // single-round migration (SURVEY.md §8(e) alternative (2);
  // VPIC_OPT_SINGLE_ROUND_MIGRATION): a particle crossing a REMOTE face keeps
  // moving through this rank's ghost layer (depositing into the ghost
  // accumulators) and leaves, its move complete, from the ghost voxel it
  // ends in -- to one of 26 neighbours, direction d = (ox+1) + 3(oy+1) +
  // 9(oz+1), o = -1 / 0 / +1 for ghost coordinate 0 / interior / n+1
  int32_t ghost_mig;
  unsigned char *di_peer26[27];  // device-initiated: inbox of the direction-d neighbour
  // vpic_advance_p_keys: every particle's voxel after the move, for the next
  // sort (null otherwise; set per launch)
  uint32_t *keys_out;
};

// Round-up reciprocal for exact unsigned division of n < 2^31 by d >= 2:
// s = ceil(log2 d) - 1, m = ceil(2^(32+s) / d) < 2^32; then n / d ==
// umulhi(n, m) >> s (the error e = m d - 2^(32+s) < d <= 2^(s+1) keeps
// n e < 2^(32+s)).
inline void set_magic(uint32_t d, uint32_t &m, uint32_t &s) {
  uint32_t k = 0;
  while ((1ull << (k + 1)) < d) ++k;          // 2^k < d <= 2^(k+1)
  s = k;
  m = (uint32_t)(((1ull << (32 + k)) + d - 1) / d);
}

// inbox window layout: a u64 counter per slot, then records [slot][di_cap] x
// 48 B (position record, momentum record, remaining displacement).  Face
// mode: slot r*6 + f = round r, arrivals through MY face f (18 slots).
// Single-round mode: slot e*27 + a = epoch parity e, arrivals from MY
// direction a (54 slots; the parity keeps a neighbour's next-call stores
// apart from this call's arrivals).
constexpr int DI_ROUNDS = 3;
constexpr int DI_FACE_SLOTS = 18, DI_GHOST_SLOTS = 54;
constexpr int64_t DI_HDR = 512;
__host__ __device__ inline int di_face_slot(int r, int f) { return r * 6 + f; }
__host__ __device__ inline int di_ghost_slot(int e, int a) { return e * 27 + a; }
__host__ __device__ inline int64_t di_cnt_off(int slot) { return 8 * (int64_t)slot; }
__host__ __device__ inline int64_t di_rec_off(int slot, int64_t cap, int64_t k) {
  return DI_HDR + 48 * ((int64_t)slot * cap + k);
}
// direction index of a ghost offset (ox, oy, oz) in {-1, 0, 1}^3; 13 = none
__host__ __device__ inline int dir26(int ox, int oy, int oz) { return (ox + 1) + 3 * (oy + 1) + 9 * (oz + 1); }

enum FaceKind { FACE_LOCAL = 0, FACE_REFLECT = 1, FACE_ABSORB = 2, FACE_REMOTE = 3 };

enum MathMode { MATH_FAST = 0, MATH_IEEE = 1 };
enum DepositMode { DEP_AUTO = 0, DEP_LANE = 1, DEP_WARP = 2, DEP_SMEM = 3 };
enum AdvanceKernel { ADV_AUTO = 0, ADV_DIRECT = 1, ADV_TMA = 2 };

struct Exchange;  // multi-GPU state (migrate.cu)

}  // namespace vpic

struct vpic_ctx {
  vpic_grid_t g;
  vpic::GridK gk;
  int rank, nranks, device;
  int num_sms;
  int64_t l2_bytes;
  int64_t tile_sz;
  int math, deposit, adv_kernel;
  int adv_cps;             // CTAs per SM of k_advance_tma (0 = default)
  bool periodic_local[3];  // axis wraps locally (both faces local periodic)
  vpic::Exchange *ex;      // null when nranks == 1
  // small device scratch owned by the context
  void *scratch;
  size_t scratch_bytes;
  int64_t *d_count;        // device counters [4]
  int nbr26[27];           // single-round mode: rank of the direction-d neighbour (-1: none)
  int npeer26;             // ... its distinct ranks (ascending) and each direction's peer slot
  int peer26[27];
  int dir_peer[27];
  int64_t di_epoch;        // single-round mode: vpic_migrate_particles calls so far
};

namespace vpic {

// process-wide count of kernels launched by the library (vpic_kernel_launches)
void note_launch(int n = 1);

// Run f() (e.g. cudaFuncSetAttribute, a per-device setting) once per device
// for the current device; `done` is the caller's static bitmask of devices.
// Concurrent first calls may both run f() (idempotent); nobody launches
// before it has completed on its device.
template <class F>
inline void once_per_device(std::atomic<uint64_t> &done, F &&f) {
  int dev = 0;
  if (cudaGetDevice(&dev) != cudaSuccess || dev < 0 || dev >= 64) {
    f();
    return;
  }
  const uint64_t bit = 1ull << dev;
  if (done.load(std::memory_order_acquire) & bit) return;
  f();
  done.fetch_or(bit, std::memory_order_release);
}

// ---- launchers implemented in the .cu files (return cudaError_t) ----------
// np_dev (nullable): the live count is read on the device (min(*np_dev, np));
// np then only bounds it and sizes the launch
cudaError_t launch_advance_p(const vpic_ctx *c, float qsp, float msp, vpic_particle_t *p,
                             int64_t np, const float *interp, float *acc, vpic_mover_t *movers,
                             int64_t max_movers, int64_t *n_movers, int32_t *flags,
                             cudaStream_t s, const int64_t *np_dev = nullptr,
                             uint32_t *keys_out = nullptr);
// the two math variants are compiled from the same source (advance_p.cu)
cudaError_t launch_advance_p_fast(const vpic_ctx *c, float qsp, float msp, vpic_particle_t *p,
                                  int64_t np, const float *interp, float *acc,
                                  vpic_mover_t *movers, int64_t max_movers, int64_t *n_movers,
                                  int32_t *flags, cudaStream_t s, const int64_t *np_dev = nullptr,
                                  uint32_t *keys_out = nullptr);
cudaError_t launch_advance_p_ieee(const vpic_ctx *c, float qsp, float msp, vpic_particle_t *p,
                                  int64_t np, const float *interp, float *acc,
                                  vpic_mover_t *movers, int64_t max_movers, int64_t *n_movers,
                                  int32_t *flags, cudaStream_t s, const int64_t *np_dev = nullptr,
                                  uint32_t *keys_out = nullptr);
// move_p of a list of movers (incoming particles after migration)
// n_in_dev (nullable): device count, n_in then only bounds it; di_round: the
// migration round of the departures (device-initiated exchange only)
cudaError_t launch_move_movers_fast(const vpic_ctx *c, float qsp, vpic_particle_t *p,
                                    const vpic_mover_t *in, int64_t n_in, float *acc,
                                    vpic_mover_t *out, int64_t max_out, int64_t *n_out,
                                    int32_t *flags, cudaStream_t s,
                                    const int64_t *n_in_dev = nullptr, int di_round = 0);
cudaError_t launch_move_movers_ieee(const vpic_ctx *c, float qsp, vpic_particle_t *p,
                                    const vpic_mover_t *in, int64_t n_in, float *acc,
                                    vpic_mover_t *out, int64_t max_out, int64_t *n_out,
                                    int32_t *flags, cudaStream_t s,
                                    const int64_t *n_in_dev = nullptr, int di_round = 0);

cudaError_t launch_fill_ghosts(const vpic_ctx *c, float *fields, cudaStream_t s);
cudaError_t launch_load_interp(const vpic_ctx *c, const float *fields, float *interp,
                               cudaStream_t s);
cudaError_t launch_unload(const vpic_ctx *c, const float *acc, float *jf, cudaStream_t s);
cudaError_t launch_fill_ghosts_minus(const vpic_ctx *c, float *fields, cudaStream_t s);
cudaError_t launch_advance_b(const vpic_ctx *c, float *fields, float frac, cudaStream_t s);
cudaError_t launch_advance_e(const vpic_ctx *c, float *fields, const float *jf, float eps0,
                             cudaStream_t s);

cudaError_t launch_accumulate_rho(const vpic_ctx *c, float q, const vpic_particle_t *p, int64_t np,
                                  float *rho, cudaStream_t s);
cudaError_t launch_continuity(const vpic_ctx *c, const float *rho0, const float *rho1,
                              const float *jf, float *out, float *res, cudaStream_t s);
cudaError_t launch_gather_scatter(const vpic_ctx *c, const int32_t *keys, const double *x,
                                  int64_t n, const double *table, double *out, double *acc,
                                  int64_t nkeys, int64_t nx, int aggregate, cudaStream_t s);

size_t sort_workspace_bytes(const vpic_ctx *c, int64_t np, int order);
// keys_in (nullable): the voxel of every input particle, supplied by the
// caller (vpic_advance_p_keys) instead of read from the records
cudaError_t launch_sort(vpic_ctx *c, const vpic_particle_t *p_in, vpic_particle_t *p_out,
                        int64_t np, int order, int64_t tile_sz, void *ws, size_t ws_bytes,
                        int32_t *voxel_counts, int64_t *new_keys, int64_t *perm,
                        cudaStream_t s, const uint32_t *keys_in = nullptr);

int migrate(vpic_ctx *c, float qsp, float msp, vpic_particle_t *p, int64_t *np, int64_t max_np,
            vpic_mover_t *movers, int64_t max_movers, const int64_t *n_movers, float *acc,
            cudaStream_t s);
// single-round, device-initiated migration with the particle count on the
// device: no host synchronisation (capturable in a CUDA graph)
int migrate_dev(vpic_ctx *c, vpic_particle_t *p, int64_t *np_dev, int64_t max_np,
                const vpic_mover_t *movers, int64_t max_movers, const int64_t *n_movers, float *acc,
                int32_t *flags_dev, cudaStream_t s);
int exchange_create(vpic_ctx *c, const uint8_t *uid);
void exchange_destroy(vpic_ctx *c);
// dir = +1: fill the +x/+y/+z ghost planes from the +neighbours' plane 1;
// dir = -1: fill the -x/-y/-z ghost planes from the -neighbours' plane n.
int halo_fields(vpic_ctx *c, float *fields, cudaStream_t s, int dir = +1);
int device_exchange_enable(vpic_ctx *c, int64_t cap);
int reduce_jf(vpic_ctx *c, float *jf, cudaStream_t s);
// single-round mode: the 26 neighbour ranks (collective when nranks > 1)
int ghost_migration_enable(vpic_ctx *c);
// single-round mode: add the accumulator's ghost layer into the neighbours'
// boundary voxels, axis by axis (edges / corners forwarded), and zero it
int reduce_acc_ghosts(vpic_ctx *c, float *acc, cudaStream_t s);

}  // namespace vpic
