/*
 * vpic_oracle.h -- TEST INFRASTRUCTURE ONLY.
 *
 * A plain, slow, serial CPU implementation of the VPIC particle hot path
 * described by Tan et al., SC Workshops '25 and its VPIC reading
 * (SURVEY.md §8(c)).  Only tests/, __graft_entry__.smoke() and bench.py's
 * cpu_baseline / --impl reference legs may load this library.  The product
 * path (paper_conf_sc_tanlta25_b200/) never includes, links or calls it, and
 * this file shares no code with csrc/.
 *
 * Precision: float32 with the operation order written out below, compiled with
 * -O2 -ffp-contract=off (no FMA contraction), matching VPIC's FP32 arithmetic
 * (reading R16).  Where the oracle keeps checking quantities
 * (absolute-contribution sums, rho) it uses double.
 *
 * Pins (tests -m "not gpu"): every function below is pinned to
 * something other than itself -- sort: hand-worked example + exhaustive
 * brute force + the paper's run invariants; interpolator: closed forms;
 * push: bit-exact uniform-E steps, TV2/TV3 golden values (tests/golden/),
 * energy / gyration / E x B closed forms; move_p: geometry invariants and
 * edge cases; deposit: the discrete continuity invariant and totals; unload
 * and rho: single-slot / single-particle closed forms; remove_absorbed:
 * numpy mask multiset; continuity residual: hand cases; field solver: Yee
 * dispersion, div B, Gauss; gather-scatter: bincount / closed forms; the
 * replay (orc_move_deposit) and all-core (orc_advance_p_omp) variants
 * against the serial orc_advance_p.  No function is "parity unpinned".
 */
#ifndef VPIC_ORACLE_H
#define VPIC_ORACLE_H
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

/* Particle: cell-relative offsets dx,dy,dz in [-1,1], voxel index i, momentum
 * u = gamma v / c, weight w.  32 bytes (reading D1). */
typedef struct { float dx, dy, dz; int32_t i; float ux, uy, uz, w; } orc_particle;
/* Mover: remaining half-displacement and particle index (reading D6). */
typedef struct { float dispx, dispy, dispz; int32_t idx; } orc_mover;

/* Face order: 0=-x 1=-y 2=-z 3=+x 4=+y 5=+z.
 * pbc[f]: 0 = PERIODIC (the particle passes into the block owned by
 * nbr_rank[f]; local wrap when nbr_rank[f] == rank), 1 = REFLECT, 2 = ABSORB. */
typedef struct {
  int32_t nx, ny, nz;
  float dx, dy, dz, dt, cvac;
  int32_t pbc[6];
  int32_t nbr_rank[6];
  int32_t rank;
} orc_grid;

enum { ORC_SORT_STANDARD = 0, ORC_SORT_STRIDED = 1, ORC_SORT_TILED = 2, ORC_SORT_NONE = 3 };

/* Alg. 1 / Alg. 2 on a bare key array.  new_keys[i] is the
 * adjusted key of input i (int64); perm[j] = input index of output position j.
 * Either output may be NULL.  Returns 0, or -1 on bad arguments. */
int orc_sort_keys(const int32_t *keys, int64_t n, int order, int64_t tile_sz,
                  int64_t *new_keys, int64_t *perm);

/* Sort particles by voxel key in the requested order (out-of-place).
 * counts[nv] (nullable) receives the voxel histogram. */
int orc_sort_particles(const orc_grid *g, const orc_particle *in, orc_particle *out,
                       int64_t np, int order, int64_t tile_sz, int32_t *counts,
                       int64_t *new_keys, int64_t *perm);

/* Fill the +x/+y/+z ghost planes of fields[nv][8] for locally periodic faces,
 * then compute interp[nv][20] for every interior voxel. */
void orc_load_interpolator(const orc_grid *g, float *fields, float *interp);

/* One advance of np particles of species (q, m).  acc[nv][12] is accumulated
 * into; acc_abs (nullable, double[nv][12]) accumulates |contribution|;
 * acc_cond (nullable, double[nv][12]) accumulates |q uX| of every streak into
 * the 4 entries of its component X (test diagnostic: the scale of a partial's
 * sensitivity to its inputs, for the FAST-mode tolerance T3).
 * Movers (remote/absorb crossings) are appended to movers[]; returns the number
 * appended, or -1 if max_movers was exceeded (excess movers dropped). */
int64_t orc_advance_p(const orc_grid *g, float q, float m, orc_particle *p, int64_t np,
                      const float *interp, float *acc, double *acc_abs, double *acc_cond,
                      orc_mover *movers, int64_t max_movers);

/* orc_advance_p over nthreads contiguous particle blocks (OpenMP), each with
 * a private accumulator summed into acc afterwards (the all-core CPU
 * baseline).  Same particles as orc_advance_p; acc equal up to summation
 * order; movers in block order. */
int64_t orc_advance_p_omp(const orc_grid *g, float q, float m, orc_particle *p, int64_t np,
                          const float *interp, float *acc, orc_mover *movers, int64_t max_movers,
                          int nthreads);

/* The move-and-deposit half of orc_advance_p alone: p[].u must already be
 * the pushed momentum (replay of another implementation's momenta).  acc
 * nullable: trajectories only (no deposit). */
int64_t orc_move_deposit(const orc_grid *g, float qsp, orc_particle *p, int64_t np, float *acc,
                         double *acc_abs, double *acc_cond, orc_mover *movers,
                         int64_t max_movers);

/* move_p for a single mover (exposed for tests). Returns 1 if the mover is
 * still in use (remote / absorb face reached), else 0. */
int orc_move_p(const orc_grid *g, orc_particle *p, orc_mover *pm, float *acc,
               double *acc_abs, double *acc_cond, float qsp);

/* Discrete continuity residual per node (reading D1), in double:
 * res = (rho1-rho0)/(dV dt) + sum_a (jf_a(n) - jf_a(n - e_a))/d_a over nodes
 * 1..n (locally periodic axis, n - e wraps) or 1..n+1; other entries of res
 * untouched.  mag (nullable): sum of the terms' absolute values. */
void orc_continuity_residual(const orc_grid *g, const float *rho0, const float *rho1,
                             const float *jf, double *res, double *mag);

/* jf[nv][4] (jfx,jfy,jfz,0) from acc[nv][12]; locally periodic planes folded. */
void orc_unload_accumulator(const orc_grid *g, const float *acc, float *jf);

/* Same without the c_axis factor and without folding (raw edge sums, double),
 * used by the continuity pin. */
void orc_unload_raw(const orc_grid *g, const float *acc, double *J);

/* rho[nv] (double) += q w (1 +- dx)(1 +- dy)(1 +- dz)/8 on the 8 nodes; node
 * (x,y,z) is the -x-y-z corner of voxel (x,y,z).  Periodic node wrap on
 * locally periodic axes. Test-only diagnostic. */
void orc_accumulate_rho(const orc_grid *g, const orc_particle *p, int64_t np, float q,
                        double *rho);

/* Single-rank particle boundary handling for movers produced by
 * orc_advance_p: absorbed particles are deleted by back-filling from the end
 * (VPIC boundary_p).  Returns the new particle count. */
int64_t orc_remove_absorbed(const orc_grid *g, orc_particle *p, int64_t np,
                            const orc_mover *movers, int64_t n_movers);

/* Field solver (VPIC ref. [3] advance_b / advance_e,
 * reading F1 in DESIGN.md).  fields[nv][8] = ex,ey,ez,0,cbx,cby,cbz,0.
 * Ghost planes of locally periodic axes are refreshed first (E at +1 planes
 * for advance_b, cB at -1 planes for advance_e); interior voxels updated.
 *   advance_b: cB -= frac c dt curl E      (forward differences)
 *   advance_e: E  += c dt curl cB - (dt/eps0) jf   (backward differences) */
void orc_advance_b(const orc_grid *g, float *fields, float frac);
void orc_advance_e(const orc_grid *g, float *fields, const float *jf, float eps0);

/* Gather-scatter microbenchmark of PAPER.md:236-242 (f2, reading F2): for
 * each i, the access set is {k} (stencil_nx == 0) or {k, k-1, k+1, k-nx,
 * k+nx} (mod nkeys), k = keys[i]; out[i] = sum of table over the set (in that
 * order) and acc[k'] += x[i] for every k' of the set.  FP64, serial. */
void orc_gather_scatter(const int32_t *keys, const double *x, int64_t n, const double *table,
                        double *out, double *acc, int64_t nkeys, int64_t stencil_nx);

#ifdef __cplusplus
}
#endif
#endif
