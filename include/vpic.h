/*
 * vpic.h -- C ABI of libvpic.so, the B200-native (sm_100a) VPIC particle hot
 * path of Tan, Luedtke, Taufer & Albright, "Bridging Performance Portability
 * and Scalability for Plasma Simulations on Heterogeneous Systems", SC
 * Workshops '25 ("P:L" below = line L of that paper's text, PAPER.md).
 *
 * Conventions (all calls):
 *  - Every array argument is CALLER-OWNED DEVICE memory (e.g. a PyTorch CUDA
 *    tensor's data_ptr), 16-byte aligned unless stated.  The library never
 *    frees, retains or reallocates a caller pointer after the call returns.
 *  - `stream` is a cudaStream_t passed as void* (NULL = legacy default
 *    stream).  Every call only ENQUEUES work on `stream` and returns without
 *    synchronising, except vpic_migrate_particles (documented below).
 *  - Return value: VPIC_OK (0) or a negative vpic_status.  Arguments are
 *    validated on the host before anything is enqueued; on error nothing is
 *    enqueued.  No call aborts the process and no C++ exception crosses it.
 *  - Layouts (all little-endian, no padding beyond what is written):
 *      voxel index   v = x + (nx+2)*(y + (ny+2)*z), interior x in 1..nx etc.,
 *                    nv = (nx+2)(ny+2)(nz+2) voxels including one ghost layer;
 *      particle      vpic_particle_t, 32 B (AoS);
 *      fields[nv][8] float: ex,ey,ez,0, cbx,cby,cbz,0 (Yee: ex on the x-edge
 *                    from node (x,y,z) to (x+1,y,z), cbx on the -x face);
 *      interp        a buffer of nv x 24 floats holding, per voxel, the
 *                    18 coefficients ex,dexdy,dexdz,d2exdydz, ey,deydz,
 *                    deydx,d2eydzdx, ez,dezdx,dezdy,d2ezdxdy, cbx,dcbxdx,
 *                    cby,dcbydy, cbz,dcbzdz, laid out as nv rows of the
 *                    first 16 (64 B = two 32-B sectors: a gather is two
 *                    256-bit loads) followed by nv pairs (cbz, dcbzdz)
 *                    (8 B, four voxels per sector: one 64-bit load); the
 *                    last nv x 24 B are unused; the array must be 32-B
 *                    aligned (the binding's interp_coefficients() reads it
 *                    back as [nv][18]);
 *      acc[nv][12]   float: jx[4], jy[4], jz[4] quadrant partials
 *                    (48 B = 3 x float4); jx quadrants (-y-z),(+y-z),(-y+z),(+y+z),
 *                    jy cyclic over (z,x), jz over (x,y);
 *      jf[nv][4]     float: jfx, jfy, jfz, 0 on the Yee edges.
 *    The push, move, deposit, interpolation and unload formulas are the VPIC
 *    algorithms the paper relies on (ref. [3]); DESIGN.md "Readings".
 */
#ifndef VPIC_H
#define VPIC_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
  VPIC_OK = 0,
  VPIC_ERR_INVALID = -1,     /* bad argument (null, misaligned, out of range) */
  VPIC_ERR_CAPACITY = -2,    /* a caller buffer is too small (movers, np, ws) */
  VPIC_ERR_CUDA = -3,        /* a CUDA runtime call failed */
  VPIC_ERR_NCCL = -4,        /* an NCCL call failed */
  VPIC_ERR_UNSUPPORTED = -5  /* wrong device (not sm_100) or feature absent */
} vpic_status;

/* Particle boundary condition per face (faces ordered -x,-y,-z,+x,+y,+z).
 * PERIODIC: the particle passes into the block owned by nbr_rank[face]
 * (a local wrap when nbr_rank[face] == the caller's rank).  REFLECT: the
 * momentum and remaining displacement along the face normal are negated.
 * ABSORB: the particle is removed after depositing up to the face. */
enum { VPIC_BC_PERIODIC = 0, VPIC_BC_REFLECT = 1, VPIC_BC_ABSORB = 2 };

/* Sort orders: standard classification by voxel, strided (Alg. 1,
 * P:117-139), tiled strided (Alg. 2), none (input order kept;
 * the paper's "random" order when the input is shuffled, Fig. 7). */
enum { VPIC_SORT_STANDARD = 0, VPIC_SORT_STRIDED = 1, VPIC_SORT_TILED_STRIDED = 2,
       VPIC_SORT_NONE = 3 };

/* Context options (vpic_ctx_set_option). */
enum {
  /* advance_p arithmetic: 0 = FAST (FMA, fast rsqrt/div; within the oracle
   * tolerances), 1 = IEEE (no FMA contraction, correctly rounded div/sqrt:
   * bit-identical to the serial oracle). Default 0. */
  VPIC_OPT_MATH = 0,
  /* current scatter strategy: 0 = AUTO, 1 = LANE (3 x red.global.add.v4.f32 per
   * streak), 2 = WARP (same-voxel contributions reduced across the warp with
   * shuffles before red.global; falls back to LANE for scattered warps),
   * 3 = SMEM (WARP, plus same-voxel groups of 2..6 items of a warp summed
   * through shared memory by their lowest lane before its red.global --
   * faster once particles have diffused a fraction of a cell since their
   * sort, slower right after it; TMA kernel only, the direct kernel treats
   * it as WARP).  Default AUTO (= WARP). */
  VPIC_OPT_DEPOSIT = 1,
  /* default TileSz for VPIC_SORT_TILED_STRIDED when tile_sz == 0.  Default
   * 3 x (#SMs) x 128 ("three times the number of GPU cores"). */
  VPIC_OPT_TILE_SZ = 2,
  /* advance_p kernel variant: 0 = AUTO, 1 = direct global loads,
   * 2 = TMA bulk-copy pipeline (particles staged through shared memory). */
  VPIC_OPT_ADVANCE_KERNEL = 3,
  /* 1 = route every PERIODIC face of a single-rank context through the NCCL
   * exchange with the rank itself as the peer (a one-rank communicator):
   * particle migration, E/cB halos and the jf plane reduction then run the
   * multi-GPU code path on one GPU, and must reproduce the local periodic
   * wrap.  Validation of the exchange; set once, before any other call. */
  VPIC_OPT_LOOPBACK_EXCHANGE = 4,
  /* CTAs per SM of the persistent TMA advance kernel (0 = its default, 2).
   * 1 lets two advance_p calls (e.g. two species on two streams) be
   * co-resident, each on half of every SM. */
  VPIC_OPT_ADVANCE_CTAS_PER_SM = 5,
  /* Device-initiated particle exchange ("GPU-aware MPI
   * will reduce the communication overhead"): value >= 1 enables it
   * with value records per (round, face) inbox (1 = default 2^19).  Needs an
   * exchange (nranks > 1 or VPIC_OPT_LOOPBACK_EXCHANGE) whose neighbours are
   * load/store reachable (one NVLink node).  COLLECTIVE: every rank sets it,
   * with the same value, in the same order of calls.  Then vpic_advance_p
   * stores each particle that stops on a REMOTE face straight into the
   * neighbour's inbox (NCCL symmetric memory, NVLink stores), and
   * vpic_migrate_particles completes the rounds with device-side barriers and
   * counts: one host synchronisation per call instead of one per round.
   * Inbox overflow is reported as VPIC_ERR_CAPACITY. */
  VPIC_OPT_DEVICE_EXCHANGE = 6,
  /* Single-round migration (SURVEY.md §8(e) alternative (2); the paper's
   * exchange is "non-blocking point-to-point with up to six neighbors",
   * P:55): value 1.  Needs an exchange; COLLECTIVE (every rank, same order);
   * set it before VPIC_OPT_DEVICE_EXCHANGE and before any vpic_advance_p.
   * Then a particle crossing a REMOTE face does not stop there: it finishes
   * its move in this rank's ghost layer (the move is < 1 cell per axis),
   * depositing into the ghost voxels of acc, and leaves from the ghost voxel
   * it ends in -- to one of up to 26 neighbours (faces, edges, corners;
   * ranks found by composing the face neighbours x, then y, then z).
   * vpic_migrate_particles then makes ONE exchange (NCCL, or stores into the
   * neighbours' inboxes from advance_p itself with VPIC_OPT_DEVICE_EXCHANGE),
   * appends the arrivals (nothing left to move), and adds acc's ghost layer
   * into the neighbours' boundary voxels (axis by axis, then zeroes it): so
   * call vpic_migrate_particles after EVERY species' vpic_advance_p, before
   * vpic_unload_accumulator.  Reproduces the 3-round path's particles and
   * currents (the latter up to float summation order). */
  VPIC_OPT_SINGLE_ROUND_MIGRATION = 7
};

typedef struct {
  int32_t nx, ny, nz;          /* local interior cells (>= 1 each) */
  float dx, dy, dz, dt, cvac;  /* cell size, time step, speed of light */
  int32_t pbc[6];              /* VPIC_BC_* per face */
  int32_t nbr_rank[6];         /* rank owning the adjacent block (PERIODIC faces) */
  int32_t gx0, gy0, gz0;       /* global offset of this block (cells; informational) */
} vpic_grid_t;

typedef struct { float dx, dy, dz; int32_t i; float ux, uy, uz, w; } vpic_particle_t; /* 32 B */
typedef struct { float dispx, dispy, dispz; int32_t idx; } vpic_mover_t;              /* 16 B */
typedef struct vpic_ctx vpic_ctx;

/* ------------------------------------------------------------- context -- */

/* NCCL unique id for a multi-GPU context (host call, rank 0 only; the caller
 * broadcasts the 128 bytes, e.g. with torch.distributed). */
int vpic_get_unique_id(uint8_t uid[128]);

/* Create a context for one rank on CUDA device `device` (the caller has made
 * it current or it is made current here).  nranks == 1: uid may be NULL, every
 * PERIODIC face must have nbr_rank == rank.  nranks > 1: uid from
 * vpic_get_unique_id; the call is collective over the nranks processes.
 * Fails with VPIC_ERR_UNSUPPORTED on a device that is not compute capability
 * 10.0 (the library holds sm_100a code only). */
int vpic_ctx_create(vpic_ctx **ctx, const vpic_grid_t *g, int rank, int nranks,
                    const uint8_t *uid, int device);
int vpic_ctx_destroy(vpic_ctx *ctx);
int vpic_ctx_set_option(vpic_ctx *ctx, int option, int64_t value);
/* info[0]=#SMs, [1]=default tile size, [2]=nv, [3]=rank, [4]=nranks,
 * [5]=L2 bytes, [6]=math mode, [7]=deposit mode. */
int vpic_ctx_info(const vpic_ctx *ctx, int64_t info[8]);
const char *vpic_status_string(int status);
/* Number of CUDA kernels this process has launched through the library
 * (all contexts; memsets and copies excluded).  Host call, never fails. */
int64_t vpic_kernel_launches(void);

/* ------------------------------------------------------ (a1-a4) sort -- */

/* Bytes of device workspace vpic_sort_particles needs for np particles. */
size_t vpic_sort_workspace_bytes(const vpic_ctx *ctx, int64_t np, int order);

/* Sort particles by voxel key ("VPIC sorts particles according to the cell
 * index") into `order`, out of place: p_out[j] = p_in[perm[j]].
 * STANDARD = stable by voxel (reading R8).  STRIDED = Alg. 1: new key
 * (k - min_k) + r (max_k + 1).  TILED_STRIDED = Alg. 2: new key
 * floor(k/T) T max_r + r T + (k - min_k), T = tile_sz (0: context default).
 * The rank r of a particle among equal keys is the number of EARLIER input
 * particles with the same key (reading R1: deterministic, stable), so keys,
 * counts and permutation are bit-reproducible.
 *   p_in, p_out     [np] particles (must not overlap);
 *   ws, ws_bytes    device workspace, >= vpic_sort_workspace_bytes();
 *   voxel_counts    [nv] int32 out, nullable: particles per voxel;
 *   new_keys        [np] int64 out, nullable: adjusted key of INPUT particle i
 *                   (the raw key for STANDARD / NONE);
 *   perm            [np] int64 out, nullable.
 * np == 0 is valid (nothing enqueued except zeroing voxel_counts).  Keys
 * outside [0, nv) are undefined behaviour (not checked on device). */
int vpic_sort_particles(vpic_ctx *ctx, const vpic_particle_t *p_in, vpic_particle_t *p_out,
                        int64_t np, int order, int64_t tile_sz, void *ws, size_t ws_bytes,
                        int32_t *voxel_counts, int64_t *new_keys, int64_t *perm,
                        void *stream);

/* vpic_sort_particles with the voxel key of every input
 * particle supplied (keys[np] uint32 device, 4-B aligned -- e.g. written by the last
 * vpic_advance_p_keys of a sort period), so the sort does not read a 32-B
 * sector of every record to get its 4-B key (SURVEY.md §8(a) a1 fused into
 * the push).  keys[i] must equal p_in[i].i; otherwise identical to
 * vpic_sort_particles (outputs, workspace, errors, enqueue-only). */
int vpic_sort_particles_keyed(vpic_ctx *ctx, const vpic_particle_t *p_in, vpic_particle_t *p_out,
                              int64_t np, int order, int64_t tile_sz, const uint32_t *keys, void *ws,
                              size_t ws_bytes, int32_t *voxel_counts, int64_t *new_keys,
                              int64_t *perm, void *stream);

/* ---------------------------------------------------- (a5) interpolator -- */

/* Fill the +x/+y/+z ghost planes of fields (locally periodic faces: copy of
 * plane 1; remote faces: received from the neighbour over NCCL) in
 * place, then write interp[v] for every interior voxel v (ghost voxels of
 * interp are left untouched).  Ghost planes of REFLECT/ABSORB faces are the
 * caller's. */
int vpic_load_interpolator(vpic_ctx *ctx, float *fields, float *interp /*[nv][24]*/, void *stream);

/* ------------------------------------------------ (a6) clear accumulator -- */
int vpic_clear_accumulator(vpic_ctx *ctx, float *acc, void *stream);

/* ----------------------------------------------- (a7-a11) particle push -- */

/* One time step of np particles of one species (charge q, mass m): gather E
 * and cB from interp at each particle, relativistic Boris push, move with cell
 * crossing, charge-conserving current scatter into acc ("gather phase, atomic
 * scatter phase, and additional physics computations").  acc is
 * ACCUMULATED into (clear it once per step, before the first species).
 * Particles are updated in place.  A particle that reaches a REMOTE or ABSORB
 * face stops there (offset exactly +-1 on the face, p.i = 8*voxel + face) and
 * appends a mover {remaining displacement, index} at movers[atomic n_movers++];
 * the append order is unspecified.  (VPIC_OPT_SINGLE_ROUND_MIGRATION: a
 * particle ending its move in the ghost layer gets p.i = -1 - ghost voxel and
 * a mover with zero displacement; absorbed ones as above.)
 *   n_movers   device int64, in/out (not reset by this call);
 *   flags      device int32, nullable: bit 0 set if a mover was dropped
 *              because *n_movers reached max_movers. */
int vpic_advance_p(vpic_ctx *ctx, float q, float m, vpic_particle_t *p, int64_t np,
                   const float *interp, float *acc, vpic_mover_t *movers, int64_t max_movers,
                   int64_t *n_movers, int32_t *flags, void *stream);

/* vpic_advance_p that also writes keys_out[i] = p[i].i as the call
 * leaves particle i (keys_out[np] uint32 device, 4-B aligned): the "copy of
 * the keys" the next sort starts from, handed to
 * vpic_sort_particles_keyed, at the cost of a coalesced 4-B store per
 * particle.  Valid for that sort only if the call produced no movers (a
 * mover's record holds its stop code and vpic_migrate_particles reorders the
 * array). */
int vpic_advance_p_keys(vpic_ctx *ctx, float q, float m, vpic_particle_t *p, int64_t np,
                        const float *interp, float *acc, vpic_mover_t *movers, int64_t max_movers,
                        int64_t *n_movers, int32_t *flags, uint32_t *keys_out, void *stream);

/* Same, with the particle count in DEVICE memory (*np_dev, int64, 8-byte
 * aligned; read by the kernels at run time, min(*np_dev, max_np) particles are
 * pushed; max_np sizes the launch).  Lets a PIC step be captured in a CUDA
 * graph and replayed while the count changes (with
 * vpic_migrate_particles_dev).  Same argument rules otherwise. */
int vpic_advance_p_dev(vpic_ctx *ctx, float q, float m, vpic_particle_t *p, const int64_t *np_dev,
                       int64_t max_np, const float *interp, float *acc, vpic_mover_t *movers,
                       int64_t max_movers, int64_t *n_movers, int32_t *flags, void *stream);

/* ------------------------------------------------------ (a12) unload -- */

/* jf on every edge of voxels 1..n+1 from the 4 accumulators sharing it,
 * times c_axis = 1/(4 dA dt); shared boundary planes summed (locally periodic
 * axes: folded; remote faces: summed with the neighbour over NCCL) and the
 * n+1 ghost copies made equal to plane 1.  jf is overwritten. */
int vpic_unload_accumulator(vpic_ctx *ctx, const float *acc, float *jf, void *stream);

/* ------------------------------------------- (f1) field solver (next row) -- */

/* Yee field advance of VPIC (ref. [3]; SURVEY.md §8(f) f1 -- "full simulation"
 * runtime is a paper metric).  fields[nv][8] as above, updated in
 * place on interior voxels; locally periodic ghost planes are refreshed (and
 * remote ones exchanged over NCCL) first.
 *   vpic_advance_b: cB -= frac * c dt curl E (forward differences; needs the
 *                   +x/+y/+z ghost planes of E);
 *   vpic_advance_e: E += c dt curl cB - (dt/eps0) jf (backward differences;
 *                   needs the -x/-y/-z ghost planes of cB), jf[nv][4] from
 *                   vpic_unload_accumulator.
 * A VPIC step is advance_b(1/2), advance_e, advance_b(1/2). */
int vpic_advance_b(vpic_ctx *ctx, float *fields, float frac, void *stream);
int vpic_advance_e(vpic_ctx *ctx, float *fields, const float *jf, float eps0, void *stream);

/* ---------------------------- (f2) gather-scatter microbenchmark kernel -- */

/* The gather-scatter kernel of the paper's sorting study ("one billion
 * double-precision numbers using three key patterns ... Memory bandwidth is
 * calculated based on the total amount of data movement").  For
 * each i < n with k = keys[i] (0 <= k < nkeys), the access set is {k}
 * (stencil_nx == 0) or the 5-point stencil {k, k-1, k+1, k-nx, k+nx} (mod
 * nkeys, reading F2); out[i] = sum of table[] over the set, and x[i] is added
 * to acc[] at every point of the set (aggregate = 0: one red.global.add.f64
 * per lane and point -- the paper's atomic scatter; 1: lanes of a warp that
 * share a point are summed first).  keys[n] int32, x/out[n], table/acc[nkeys]
 * float64, all device memory. */
int vpic_gather_scatter(vpic_ctx *ctx, const int32_t *keys, const double *x, int64_t n,
                        const double *table, double *out, double *acc, int64_t nkeys,
                        int64_t stencil_nx, int aggregate, void *stream);

/* ------------------------- (f4) on-line charge-conservation diagnostics -- */

/* Cloud-in-cell charge on the nodes (VPIC accumulate_rho_p, ref. [3]; reading
 * D1): for each particle, rho[node] += q w (1 +- dx)(1 +- dy)(1 +- dz) / 8 on
 * the 8 nodes (x..x+1, y..y+1, z..z+1) of its voxel, the sign of each factor
 * set by the side of the node.  Node n+1 of a locally periodic axis is node 1;
 * other n+1 nodes are kept (a REMOTE face's shared nodes are NOT summed with
 * the neighbour: single-rank diagnostic).  rho[nv] float32 device memory
 * indexed like voxels, ACCUMULATED into.  np == 0 is a no-op. */
int vpic_accumulate_rho(vpic_ctx *ctx, float q, const vpic_particle_t *p, int64_t np, float *rho,
                        void *stream);

/* Discrete continuity residual of the charge-conserving deposit ("the
 * discrete continuity invariant", BASELINE north_star; deposit P:238):
 *   res(node) = (rho1 - rho0) / (dx dy dz dt) + sum_a (jf_a(node) - jf_a(node - e_a)) / d_a
 * over the nodes 1..n of a locally periodic axis (node - e_a wraps to n) and
 * 1..n+1 otherwise.  rho0/rho1 from vpic_accumulate_rho before/after one
 * vpic_advance_p of every species, jf from vpic_unload_accumulator.
 *   out  device float[2], overwritten: {max |res|, max |drho/dt|};
 *   res  device float[nv] (nullable): res per node, other entries untouched. */
int vpic_continuity_residual(vpic_ctx *ctx, const float *rho0, const float *rho1, const float *jf,
                             float *out, float *res, void *stream);

/* ---------------------------------------------------- (a13) exchange -- */

/* Finish the movers produced by vpic_advance_p for one species: particles on
 * REMOTE faces are sent to the neighbour rank (NCCL send/recv, up to three
 * rounds for corner crossings, "non-blocking point-to-point with up to six
 * neighbors" P:55), received particles continue their move (depositing into
 * acc) and are appended; absorbed and departed particles are removed by
 * back-filling from the end.  *np (HOST) is updated.  SYNCHRONISES `stream`
 * (it reads mover counts).
 *   movers, max_movers  the list vpic_advance_p filled and its capacity (the
 *                       same max_movers): never read past it;
 *   n_movers            device int64, the count vpic_advance_p left.
 * Fails with VPIC_ERR_CAPACITY -- and then the particle array still holds
 * stopped particles (p.i = 8*voxel+face) and must be discarded -- if
 * *n_movers > max_movers (advance_p dropped movers; its flags bit 0) or the
 * arrivals would exceed max_np.  With VPIC_OPT_SINGLE_ROUND_MIGRATION: one
 * exchange with up to 26 neighbours, arrivals appended with their move
 * already complete, then acc's ghost layer added into the neighbours'
 * boundary voxels and zeroed. */
int vpic_migrate_particles(vpic_ctx *ctx, float q, float m, vpic_particle_t *p, int64_t *np,
                           int64_t max_np, vpic_mover_t *movers, int64_t max_movers,
                           const int64_t *n_movers, float *acc, void *stream);

/* vpic_migrate_particles with the count in DEVICE memory and no host
 * synchronisation: every step is a stream operation, so it can be captured in
 * a CUDA graph (a capture must hold an even number of calls: each call flips
 * the inbox epoch, fixed at enqueue time).  Needs
 * VPIC_OPT_SINGLE_ROUND_MIGRATION and VPIC_OPT_DEVICE_EXCHANGE (else
 * VPIC_ERR_UNSUPPORTED).  *np_dev (int64) in/out; flags_dev (int32, device):
 * capacity errors are OR-ed in as bits 1 (an inbox was full: particles lost),
 * 2 (more movers than max_movers or than the internal hole list: the count is
 * clamped, nothing is read past the list, the departures beyond it stay in
 * the array as stopped particles), 3 (arrivals did not fit max_np: dropped)
 * -- check it when the count is read back.  n_movers is not reset. */
int vpic_migrate_particles_dev(vpic_ctx *ctx, float q, float m, vpic_particle_t *p, int64_t *np_dev,
                               int64_t max_np, const vpic_mover_t *movers, int64_t max_movers,
                               const int64_t *n_movers, float *acc, int32_t *flags_dev,
                               void *stream);

/* ------------------------------------ host-buffer driver (end to end) -- */

/* One species of vpic_run_host: its input in pinned HOST memory, four
 * caller-owned DEVICE particle buffers of max_np records each (they rotate
 * through input / sort output / next upload / previous download, so the
 * copies of neighbouring periods overlap the compute). */
typedef struct {
  float q, m;                        /* charge, mass */
  const vpic_particle_t *host_in;    /* [np] pinned host: the period's input */
  vpic_particle_t *host_out;         /* [np] pinned host, nullable: the period's particles */
  int64_t np, max_np;                /* records in host_in; capacity of each dev buffer */
  vpic_particle_t *dev[4];           /* device buffers, 16-B aligned */
} vpic_species_host_t;

/* Device workspace bytes vpic_run_host needs (fields x 2, interpolator,
 * accumulator, jf x 3, mover lists, sort workspace). */
size_t vpic_run_host_workspace_bytes(const vpic_ctx *ctx, int nsp, const vpic_species_host_t *sp,
                                     int order);

/* n_cycles sort periods of the hot path from and to pinned host memory (the
 * end-to-end form of the paper's push + sort loop): every
 * period uploads each species' host_in and fields_host (nv x 8 floats),
 * sorts every species in `order` (tile_sz as in vpic_sort_particles), runs
 * `steps` PIC steps (load interpolator, clear, advance_p per species
 * [+ vpic_migrate_particles when the context exchanges or absorbs],
 * unload [+ advance_b(1/2), advance_e, advance_b(1/2) if field_solve]) and
 * downloads jf (nv x 4 floats) into jf_host and, if host_out, the particles.
 * Period k+1's upload and period k-1's download run on internal copy streams
 * under period k's compute (events order them).  deposit_modes (nullable):
 * [steps][nsp] VPIC_OPT_DEPOSIT values per step and species (the caller's
 * AUTO policy).  *pushes (host, nullable) = particles x PIC steps done.
 * ENQUEUES on `stream` (which finally waits for the copy streams); host
 * buffers must stay valid until `stream` is synchronised.  Synchronises only
 * where vpic_migrate_particles does.  Errors: VPIC_ERR_INVALID (bad
 * argument), VPIC_ERR_CAPACITY (workspace too small), or the error of the
 * failing call (work already enqueued is left on the stream). */
int vpic_run_host(vpic_ctx *ctx, int nsp, const vpic_species_host_t *sp, const float *fields_host,
                  float *jf_host, int order, int64_t tile_sz, int steps, int n_cycles,
                  const int8_t *deposit_modes, int field_solve, float eps0, void *ws, size_t ws_bytes,
                  int64_t *pushes, void *stream);

#ifdef __cplusplus
}
#endif
#endif /* VPIC_H */
