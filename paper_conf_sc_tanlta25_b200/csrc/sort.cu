// Hardware-targeted particle sort by voxel (rows a1-a4 of SURVEY.md §8(a)):
// standard classification, strided (Alg. 1) and
// tiled strided (Alg. 2).
//
// B200 design: the paper adjusts keys in O(N) and then calls
// a generic sort_by_key.  Here every order is produced by stable LSD
// counting passes with no comparison sort and no nondeterministic atomics:
//   standard      = stable radix sort of (voxel, index) pairs, passes of
//                   <= 8-bit digits (one sweep each: decoupled look-back, the
//                   tile staged in shared memory in digit order so that every
//                   digit run is written coalesced), then one gather of the
//                   32-B records;
//   strided       = standard, then one stable counting pass by the rank
//                   r = pos - offset[voxel]        (lexicographic (r, k));
//   tiled strided = standard, then one stable counting pass by
//                   (floor(k/T) - floor(min_k/T)) * max_r + r   (lexicographic
//                   (floor(k/T), r, k)).
// The rank of a particle among equal keys is its stable rank (reading R1), so
// the result equals Alg. 1/2 with the atomic_fetch_add loop run in input
// order: keys, counts and permutation are bit-exact against the oracle.
// Nothing synchronises with the host: the rank passes are launched for the
// worst case the host can bound (8-bit digits from the least significant;
// strided keys r < np in 32 bits, tiled keys (chunk - chunk0) max_r + r in 64
// bits) and every pass above the bits the device finds it needs (max_r, min_k,
// max_k are device values) returns at once; the record gather picks the
// buffer the last live pass wrote.  Every order is stream-ordered and can be
// captured in a CUDA graph.
#include <algorithm>

#include "vpic_internal.cuh"

namespace vpic {
namespace {

#ifndef VPIC_SORT_IPT
#define VPIC_SORT_IPT 12
#endif
#ifndef VPIC_SORT_PERSIST
#define VPIC_SORT_PERSIST 0
#endif
#ifndef VPIC_SORT_MINB
#define VPIC_SORT_MINB 2
#endif
#ifndef VPIC_SORT_NT
#define VPIC_SORT_NT 512
#endif
constexpr int NT = VPIC_SORT_NT;    // threads per radix CTA
constexpr int NW = NT / 32;         // warps
constexpr int IPT = VPIC_SORT_IPT;  // items per thread
constexpr int TILE = NT * IPT;      // 6144 elements per tile
// Launch shape measured on late C2 electrons / ions (sort ms, same box):
// 256 x 16 x 3 CTAs/SM 14.07 / 10.79; 512 x 12 x 2 13.87 / 10.47 (kept);
// 256 x 24 x 2 14.19 / 10.81; 256 x 32 x 2 13.91 / 10.57 (spills);
// 512 x 16 x 1 15.54 / 11.84; persistent 256 x 16 x 2 CTAs/SM (next tile
// loaded during the current one) 14.86 / 12.10, 256 x 8 x 4 16.56 / 13.99
// (another box: 512 x 12 x 2 13.84 / 10.48; 384 x 16 x 2 13.84 / 10.48;
// 512 x 10 x 2 14.40 / 10.99; 1024 x 6 x 1 16.64 / 12.90)
constexpr int MAX_BITS = 8;         // digit width: 256 buckets, one look-back chain per thread
constexpr int MAX_PASSES = 8;       // keys up to 64 bits (tiled-strided composite keys)
constexpr unsigned FULL = 0xffffffffu;

constexpr unsigned long long FLAG_AGG = 1ull << 62;
constexpr unsigned long long FLAG_INC = 2ull << 62;
constexpr unsigned long long VAL_MASK = (1ull << 40) - 1;

__device__ __forceinline__ void st_relaxed(unsigned long long *p, unsigned long long v) {
  asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ unsigned long long ld_relaxed(const unsigned long long *p) {
  unsigned long long v;
  asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ unsigned lanemask_lt() {
  unsigned m;
  asm("mov.u32 %0, %%lanemask_lt;" : "=r"(m));
  return m;
}

struct PassDesc {
  int shift[MAX_PASSES];
  int bits[MAX_PASSES];
  int npass;
};

// keys[i] = p_in[i].i and the voxel histogram count[k] (zeroed by the caller).
// Runs of equal keys within a warp (the input is nearly sorted between sorts)
// are counted with one atomic per run, found with a lane-neighbour compare.
__global__ void __launch_bounds__(256)
k_keys_count(const vpic_particle_t *__restrict__ p, int64_t n, uint32_t *__restrict__ keys,
             uint32_t *__restrict__ count, int64_t *__restrict__ new_keys) {
  const int lane = threadIdx.x & 31;
  const int32_t *pi = reinterpret_cast<const int32_t *>(p) + 3;
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  for (int64_t base = (int64_t)blockIdx.x * blockDim.x + (threadIdx.x & ~31); base < n;
       base += stride) {
    const int64_t i = base + lane;
    const bool valid = i < n;
    uint32_t k = 0xffffffffu;
    if (valid) {
      k = (uint32_t)__ldcs(pi + 8 * i);
      keys[i] = k;
      if (new_keys) new_keys[i] = (int64_t)k;
    }
    const uint32_t prev = __shfl_up_sync(FULL, k, 1);
    const bool head = valid && (lane == 0 || prev != k);
    const unsigned ends = __ballot_sync(FULL, head) | ~__ballot_sync(FULL, valid);
    const unsigned above = lane == 31 ? 0u : (ends & ~((2u << lane) - 1u));
    const int len = (above ? __ffs(above) - 1 : 32) - lane;
    if (head) atomicAdd(&count[k], (uint32_t)len);
  }
}

// The same from keys supplied by the caller (vpic_sort_particles_keyed:
// written by the last advance_p): a coalesced 4-B read per particle instead
// of a 32-B sector of its record.
__global__ void __launch_bounds__(256)
k_count_keys(const uint32_t *__restrict__ keys_in, int64_t n, uint32_t *__restrict__ count,
             int64_t *__restrict__ new_keys) {
  const int lane = threadIdx.x & 31;
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  for (int64_t base = (int64_t)blockIdx.x * blockDim.x + (threadIdx.x & ~31); base < n;
       base += stride) {
    const int64_t i = base + lane;
    const bool valid = i < n;
    uint32_t k = 0xffffffffu;
    if (valid) {
      k = __ldcs(keys_in + i);
      if (new_keys) new_keys[i] = (int64_t)k;
    }
    const uint32_t prev = __shfl_up_sync(FULL, k, 1);
    const bool head = valid && (lane == 0 || prev != k);
    const unsigned ends = __ballot_sync(FULL, head) | ~__ballot_sync(FULL, valid);
    const unsigned above = lane == 31 ? 0u : (ends & ~((2u << lane) - 1u));
    const int len = (above ? __ffs(above) - 1 : 32) - lane;
    if (head) atomicAdd(&count[k], (uint32_t)len);
  }
}

// Digit histograms of every LSD pass from the voxel histogram.
__global__ void k_digit_hist(const uint32_t *__restrict__ count, int64_t nv, PassDesc pd,
                             uint32_t *__restrict__ ghist) {
  __shared__ uint32_t sh[MAX_PASSES << MAX_BITS];
  for (int i = threadIdx.x; i < (MAX_PASSES << MAX_BITS); i += blockDim.x) sh[i] = 0;
  __syncthreads();
  for (int64_t k = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; k < nv;
       k += (int64_t)gridDim.x * blockDim.x) {
    const uint32_t c = count[k];
    if (!c) continue;
    for (int q = 0; q < pd.npass; ++q)
      atomicAdd(&sh[(q << MAX_BITS) + (((uint32_t)k >> pd.shift[q]) & ((1u << pd.bits[q]) - 1))], c);
  }
  __syncthreads();
  for (int q = 0; q < pd.npass; ++q)
    for (int b = threadIdx.x; b < (1 << pd.bits[q]); b += blockDim.x) {
      const uint32_t c = sh[(q << MAX_BITS) + b];
      if (c) atomicAdd(&ghist[(q << MAX_BITS) + b], c);
    }
}

// offs[k] = sum of count[k' < k] over nv voxels (+ offs[nv] = total), in
// three phases over blocks of SCAN_B voxels; max_r = max count.
constexpr int SCAN_B = 4096;
__global__ void k_scan_blocksum(const uint32_t *__restrict__ count, int64_t nv,
                                uint32_t *__restrict__ bsum, unsigned int *__restrict__ max_r) {
  __shared__ uint32_t red[32];
  __shared__ uint32_t redm[32];
  const int64_t b0 = (int64_t)blockIdx.x * SCAN_B;
  uint32_t sum = 0, mx = 0;
  for (int j = threadIdx.x; j < SCAN_B; j += blockDim.x) {
    const int64_t k = b0 + j;
    const uint32_t c = k < nv ? count[k] : 0u;
    sum += c;
    mx = max(mx, c);
  }
  for (int o = 16; o; o >>= 1) {
    sum += __shfl_xor_sync(FULL, sum, o);
    mx = max(mx, __shfl_xor_sync(FULL, mx, o));
  }
  if ((threadIdx.x & 31) == 0) { red[threadIdx.x >> 5] = sum; redm[threadIdx.x >> 5] = mx; }
  __syncthreads();
  if (threadIdx.x == 0) {
    uint32_t t = 0, m = 0;
    for (int w = 0; w < (int)(blockDim.x >> 5); ++w) { t += red[w]; m = max(m, redm[w]); }
    bsum[blockIdx.x] = t;
    if (m) atomicMax(max_r, m);
  }
}
__global__ void k_scan_bsums(uint32_t *__restrict__ bsum, int64_t nb) {
  // one CTA of 1024 threads: exclusive scan in place
  __shared__ uint32_t part[1024];
  const int64_t per = (nb + blockDim.x - 1) / blockDim.x;
  const int64_t j0 = threadIdx.x * per;
  uint32_t t = 0;
  for (int64_t j = j0; j < min(nb, j0 + per); ++j) t += bsum[j];
  part[threadIdx.x] = t;
  __syncthreads();
  if (threadIdx.x == 0) {
    uint32_t run = 0;
    for (int w = 0; w < (int)blockDim.x; ++w) { const uint32_t x = part[w]; part[w] = run; run += x; }
  }
  __syncthreads();
  uint32_t run = part[threadIdx.x];
  for (int64_t j = j0; j < min(nb, j0 + per); ++j) { const uint32_t x = bsum[j]; bsum[j] = run; run += x; }
}
__global__ void __launch_bounds__(256)
k_scan_apply(const uint32_t *__restrict__ count, int64_t nv, const uint32_t *__restrict__ bsum,
             uint32_t *__restrict__ offs, int64_t total) {
  // 256 threads x 16 consecutive voxels each
  __shared__ uint32_t wsum[8];
  const int64_t b0 = (int64_t)blockIdx.x * SCAN_B + threadIdx.x * 16;
  uint32_t c[16], t = 0;
#pragma unroll
  for (int j = 0; j < 16; ++j) { c[j] = (b0 + j < nv) ? count[b0 + j] : 0u; t += c[j]; }
  uint32_t incl = t;
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  for (int o = 1; o < 32; o <<= 1) {
    const uint32_t y = __shfl_up_sync(FULL, incl, o);
    if (lane >= o) incl += y;
  }
  if (lane == 31) wsum[w] = incl;
  __syncthreads();
  uint32_t wpre = 0;
  for (int ww = 0; ww < w; ++ww) wpre += wsum[ww];
  uint32_t run = bsum[blockIdx.x] + wpre + incl - t;
#pragma unroll
  for (int j = 0; j < 16; ++j) {
    if (b0 + j < nv) offs[b0 + j] = run;
    run += c[j];
  }
  if (blockIdx.x == 0 && threadIdx.x == 0) offs[nv] = (uint32_t)total;
}

// Exclusive scan of each pass's digit histogram (one CTA per pass).
__global__ void k_scan_hist(const uint32_t *__restrict__ ghist, uint32_t *__restrict__ goff,
                            PassDesc pd) {
  const int q = blockIdx.x;
  if (q >= pd.npass) return;
  const int nb = 1 << pd.bits[q];
  __shared__ uint32_t part[1024];
  const uint32_t *h = ghist + q * (1 << MAX_BITS);
  uint32_t *o = goff + q * (1 << MAX_BITS);
  const int per = (nb + blockDim.x - 1) / blockDim.x;
  const int b0 = threadIdx.x * per;
  uint32_t s = 0;
  for (int b = b0; b < min(nb, b0 + per); ++b) s += h[b];
  part[threadIdx.x] = s;
  __syncthreads();
  if (threadIdx.x == 0) {
    uint32_t run = 0;
    for (int t = 0; t < (int)blockDim.x; ++t) { const uint32_t x = part[t]; part[t] = run; run += x; }
  }
  __syncthreads();
  uint32_t run = part[threadIdx.x];
  for (int b = b0; b < min(nb, b0 + per); ++b) { o[b] = run; run += h[b]; }
}

// ---------------------------------------------------------------- a3/a4 --
// One stable LSD counting pass over (key, val) with a 2^BITS-bucket digit.
// Tiles are taken in order from an atomic ticket; each tile ranks its
// elements stably (per-warp smem histograms, match_any within a warp),
// publishes its per-digit count and resolves its global offset by decoupled
// look-back over earlier tiles' status words (flag | count in one u64).
// With VPIC_SORT_PERSIST the grid is one wave of resident CTAs that loop over
// tickets, loading the next tile's keys/values while the current one is
// ranked, looked back and scattered.  Deadlock-free: a CTA holds at most two
// tickets, processes them in increasing order, and a tile only waits on
// smaller tickets, all held by resident CTAs.
// live_bits (nullable): the pass returns at once (every CTA) when its digit
// lies above the key width the device found (*live_bits), so the host can
// launch the worst-case number of passes without reading it back.
// REC (the last pass of the standard order): instead of the permutation,
// the pass moves the 32-B records themselves -- out[pos] = in[val] -- in its
// coalesced digit-run scatter (two lanes per record, RILP half-records in
// flight per thread), plus the optional int64 permutation: the record gather
// is fused into the pass (no permutation written and re-read, one launch
// less, the gather's DRAM-bound random reads overlap the ranking).
struct RecMove {
  const vpic_particle_t *in;
  vpic_particle_t *out;
  int64_t *perm64;
};
#ifndef VPIC_SORT_RILP
#define VPIC_SORT_RILP 4
#endif
constexpr int RILP = VPIC_SORT_RILP;

template <int BITS, class KeyT, bool REC = false>
__global__ void __launch_bounds__(NT, VPIC_SORT_MINB)
k_radix_pass(const KeyT *__restrict__ kin, const uint32_t *__restrict__ vin,
             KeyT *__restrict__ kout, uint32_t *__restrict__ vout, int64_t n, int shift,
             const uint32_t *__restrict__ dig_off, unsigned long long *__restrict__ status,
             unsigned int *__restrict__ tile_ctr, const int *__restrict__ live_bits, RecMove rec) {
  if (live_bits) {
    const int nb = *live_bits;
    // the 32-bit and the 64-bit chain of rank passes are both launched; the
    // key width the device found selects the one that runs
    if (sizeof(KeyT) == 4 && nb > 32) return;
    if (sizeof(KeyT) == 8 && nb <= 32) return;
    if (shift > 0 && shift >= nb) return;
  }
  constexpr int NB = 1 << BITS;
  extern __shared__ __align__(16) unsigned char smem[];
  uint16_t *whist = reinterpret_cast<uint16_t *>(smem);                       // [NW][NB]
  uint32_t *tpref = reinterpret_cast<uint32_t *>(smem + NW * NB * 2);          // [NB]
  uint32_t *tstart = tpref + NB;                                               // [NB]
  KeyT *skey = reinterpret_cast<KeyT *>(tstart + NB);                          // [TILE]
  uint32_t *sval = reinterpret_cast<uint32_t *>(skey + TILE);                  // [TILE]
  __shared__ unsigned int s_tile;
  __shared__ uint32_t wsum[NW];
  const int64_t ntiles = (n + TILE - 1) / TILE;
  const int w = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const unsigned lt = lanemask_lt();
  uint16_t *wh = whist + w * NB;
  KeyT key[IPT];
  uint32_t val[IPT];
  auto load_tile = [&](int64_t t, KeyT *k, uint32_t *v) {
    const int64_t wb = t * TILE + (int64_t)w * 32 * IPT;
#pragma unroll
    for (int j = 0; j < IPT; ++j) {
      const int64_t i = wb + j * 32 + lane;
      const bool valid = i < n;
      k[j] = valid ? __ldcs(kin + i) : KeyT(0);
      v[j] = valid ? (vin ? __ldcs(vin + i) : (uint32_t)i) : 0u;
    }
  };
  if (threadIdx.x == 0) s_tile = atomicAdd(tile_ctr, 1u);
  __syncthreads();
  int64_t tile = s_tile;
  if (tile >= ntiles) return;
  load_tile(tile, key, val);
  while (true) {
    for (int i = threadIdx.x; i < NW * NB / 2; i += NT) reinterpret_cast<uint32_t *>(whist)[i] = 0;
#if VPIC_SORT_PERSIST
    if (threadIdx.x == 0) s_tile = atomicAdd(tile_ctr, 1u);
#endif
    __syncthreads();
#if VPIC_SORT_PERSIST
    const int64_t next = s_tile;
#else
    const int64_t next = ntiles;
#endif
    const int64_t wbase = tile * TILE + (int64_t)w * 32 * IPT;
    uint32_t rank[IPT / 2];  // two u16 ranks per register
#pragma unroll
    for (int j = 0; j < IPT; ++j) {
      const int64_t i = wbase + j * 32 + lane;
      const bool valid = i < n;
      const uint32_t d = valid ? (uint32_t)((key[j] >> shift) & (NB - 1)) : (uint32_t)NB;
      const unsigned peers = __match_any_sync(FULL, d);
      uint32_t cur = 0;
      if (valid) cur = wh[d];
      __syncwarp();
      if (valid && (__ffs(peers) - 1) == lane) wh[d] = (uint16_t)(cur + __popc(peers));
      __syncwarp();
      const uint32_t r = cur + __popc(peers & lt);
      if (j & 1) rank[j >> 1] |= r << 16; else rank[j >> 1] = r;
    }
#if VPIC_SORT_PERSIST
    KeyT nkey[IPT];
    uint32_t nval[IPT];
    if (next < ntiles) load_tile(next, nkey, nval);
#endif
    __syncthreads();
    // per-digit: warp exclusive offsets, tile count, look-back
    for (int b = threadIdx.x; b < NB; b += NT) {
      uint32_t run = 0;
#pragma unroll
      for (int ww = 0; ww < NW; ++ww) {
        const uint32_t c = whist[ww * NB + b];
        whist[ww * NB + b] = (uint16_t)run;
        run += c;
      }
      tstart[b] = run;   // tile count of digit b (scanned below)
      unsigned long long *st = status + tile * NB + b;
      uint64_t excl = 0;
      if (tile == 0) {
        st_relaxed(st, FLAG_INC | run);
      } else {
        st_relaxed(st, FLAG_AGG | run);
        int64_t t = tile - 1;
        while (true) {
          const unsigned long long sv = ld_relaxed(status + t * NB + b);
          const unsigned long long f = sv & (3ull << 62);
          if (f == 0) continue;
          excl += sv & VAL_MASK;
          if (f == FLAG_INC) break;
          --t;
        }
        st_relaxed(st, FLAG_INC | (excl + run));
      }
      tpref[b] = dig_off[b] + (uint32_t)excl;
    }
    __syncthreads();
    // tile-local exclusive digit offsets (block scan of the NB tile counts)
    {
      const uint32_t c = threadIdx.x < NB ? tstart[threadIdx.x] : 0u;
      uint32_t incl = c;
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        const uint32_t y = __shfl_up_sync(FULL, incl, o);
        if (lane >= o) incl += y;
      }
      if (lane == 31) wsum[w] = incl;
      __syncthreads();
      uint32_t pre = 0;
      for (int ww = 0; ww < w; ++ww) pre += wsum[ww];
      if (threadIdx.x < NB) tstart[threadIdx.x] = pre + incl - c;
      __syncthreads();
    }
    // stage the tile in digit order in shared memory, then write each digit's
    // run with consecutive threads on consecutive addresses (coalesced: one
    // element-granular scatter per 4 B made the first pass L2-request-bound)
#pragma unroll
    for (int j = 0; j < IPT; ++j) {
      const int64_t i = wbase + j * 32 + lane;
      if (i < n) {
        const uint32_t d = (uint32_t)((key[j] >> shift) & (NB - 1));
        const uint32_t r = (j & 1) ? (rank[j >> 1] >> 16) : (rank[j >> 1] & 0xffffu);
        const uint32_t lp = tstart[d] + whist[w * NB + d] + r;
        skey[lp] = key[j];
        sval[lp] = val[j];
      }
    }
    __syncthreads();
    const int64_t t0 = tile * TILE;
    const int nvalid = (int)(n - t0 < TILE ? n - t0 : (int64_t)TILE);
    if (REC) {
      // half-record h of element e: lanes 2j, 2j+1 move one whole record
      const float4 *src = reinterpret_cast<const float4 *>(rec.in);
      float4 *dst = reinterpret_cast<float4 *>(rec.out);
      for (int tb = 0; tb < 2 * nvalid; tb += NT * RILP) {
        uint32_t sidx[RILP], dpos[RILP];
        float4 v[RILP];
#pragma unroll
        for (int j = 0; j < RILP; ++j) {
          const int t = tb + j * NT + (int)threadIdx.x;
          if (t < 2 * nvalid) {
            const int e = t >> 1;
            const KeyT k = skey[e];
            const uint32_t d = (uint32_t)((k >> shift) & (NB - 1));
            dpos[j] = tpref[d] + (uint32_t)e - tstart[d];
            sidx[j] = sval[e];
            VPIC_ASSERT((int64_t)dpos[j] < n && (int64_t)sidx[j] < n);
          }
        }
#pragma unroll
        for (int j = 0; j < RILP; ++j) {
          const int t = tb + j * NT + (int)threadIdx.x;
          if (t < 2 * nvalid) {
            const float4 *a = src + 2 * (int64_t)sidx[j] + (t & 1);
            asm volatile("ld.global.nc.L2::64B.v4.f32 {%0,%1,%2,%3}, [%4];"
                         : "=f"(v[j].x), "=f"(v[j].y), "=f"(v[j].z), "=f"(v[j].w) : "l"(a));
          }
        }
#pragma unroll
        for (int j = 0; j < RILP; ++j) {
          const int t = tb + j * NT + (int)threadIdx.x;
          if (t < 2 * nvalid) {
            __stcs(dst + 2 * (int64_t)dpos[j] + (t & 1), v[j]);
            if (rec.perm64 && !(t & 1)) rec.perm64[dpos[j]] = sidx[j];
          }
        }
      }
    } else {
      for (int e = threadIdx.x; e < nvalid; e += NT) {
        const KeyT k = skey[e];
        const uint32_t d = (uint32_t)((k >> shift) & (NB - 1));
        const uint32_t pos = tpref[d] + (uint32_t)e - tstart[d];
        VPIC_ASSERT((int64_t)pos < n);
        if (kout) kout[pos] = k;
        vout[pos] = sval[e];
      }
    }
#if VPIC_SORT_PERSIST
    if (next >= ntiles) break;
#pragma unroll
    for (int j = 0; j < IPT; ++j) { key[j] = nkey[j]; val[j] = nval[j]; }
    tile = next;
    __syncthreads();  // smem (whist, tpref, tstart, skey/sval, s_tile) reused next tile
#else
    break;
#endif
  }
}

// Device-side sizing of the rank passes (no host round trip): from max_r
// (k_scan_blocksum), min_k = K[0] and max_k = K[n-1] of the standard order.
struct RankParams {
  int64_t min_k, max_k, chunk0;
  uint64_t max_ck;   // largest rank-pass key
  uint32_t max_r;
  int nbits;         // bits of max_ck (>= 1): passes with shift >= nbits are skipped
  int sel;           // the buffer the last live pass writes (number of live passes & 1)
};
__global__ void k_rank_setup(const uint32_t *__restrict__ K, int64_t n, int order, int64_t T,
                             const unsigned int *__restrict__ max_r_dev, RankParams *rp) {
  RankParams r;
  r.max_r = *max_r_dev;
  r.min_k = K[0];
  r.max_k = K[n - 1];
  r.chunk0 = r.min_k / T;
  const uint64_t rmax = r.max_r ? r.max_r - 1 : 0;
  r.max_ck = order == VPIC_SORT_STRIDED ? rmax
                                        : (uint64_t)(r.max_k / T - r.chunk0) * r.max_r + rmax;
  int b = 1;
  while (b < 64 && (r.max_ck >> b)) ++b;
  r.nbits = b;
  const int live = (b + MAX_BITS - 1) / MAX_BITS;
  r.sel = live & 1;
  *rp = r;
}

// Rank-pass keys (strided: r; tiled: (chunk - chunk0) * max_r + r) with the
// digit histograms of the following (worst-case) passes; optional Alg. 1/2
// new keys scattered to the INPUT index (perm_std[j]).
// ckey: the rank keys as uint32 when they fit 32 bits (rp->nbits <= 32), as
// uint64 otherwise (the buffer holds either).
__global__ void __launch_bounds__(256)
k_rank_keys(const uint32_t *__restrict__ K, const uint32_t *__restrict__ perm_std,
            const uint32_t *__restrict__ offs, int64_t n, int order, int64_t T,
            const RankParams *__restrict__ rp, void *__restrict__ ckey, PassDesc pd,
            uint32_t *__restrict__ ghist, int64_t *__restrict__ new_keys) {
  using KeyT = uint64_t;
  extern __shared__ uint32_t sh[];
  int off[MAX_PASSES];
  int tot = 0;
  for (int q = 0; q < pd.npass; ++q) { off[q] = tot; tot += 1 << pd.bits[q]; }
  for (int i = threadIdx.x; i < tot; i += blockDim.x) sh[i] = 0;
  __syncthreads();
  const int lane = threadIdx.x & 31;
  const int64_t min_k = rp->min_k, max_k = rp->max_k, chunk0 = rp->chunk0;
  const uint64_t max_r = rp->max_r;
  const int nbits = rp->nbits;
  const bool wide = nbits > 32;
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  for (int64_t base = (int64_t)blockIdx.x * blockDim.x + (threadIdx.x & ~31); base < n;
       base += stride) {
    const int64_t j = base + lane;
    const bool valid = j < n;
    KeyT ck = 0;
    if (valid) {
      const int64_t k = K[j];
      const int64_t r = j - (int64_t)offs[k];
      if (order == VPIC_SORT_STRIDED) {
        ck = (KeyT)r;
        if (new_keys) new_keys[perm_std[j]] = (k - min_k) + r * (max_k + 1);
      } else {
        ck = (KeyT)((uint64_t)(k / T - chunk0) * max_r + (uint64_t)r);
        if (new_keys) new_keys[perm_std[j]] = (k / T) * (T * (int64_t)max_r) + r * T + (k - min_k);
      }
      if (wide) static_cast<uint64_t *>(ckey)[j] = ck;
      else static_cast<uint32_t *>(ckey)[j] = (uint32_t)ck;
    }
    for (int q = 0; q < pd.npass; ++q) {
      if (pd.shift[q] > 0 && pd.shift[q] >= nbits) break;   // skipped pass (uniform)
      const uint32_t d = valid ? (uint32_t)((ck >> pd.shift[q]) & ((1u << pd.bits[q]) - 1)) : 0xffffffffu;
      const unsigned peers = __match_any_sync(FULL, d);
      if (valid && (__ffs(peers) - 1) == lane) atomicAdd(&sh[off[q] + d], __popc(peers));
    }
  }
  __syncthreads();
  for (int q = 0; q < pd.npass; ++q)
    for (int b = threadIdx.x; b < (1 << pd.bits[q]); b += blockDim.x) {
      const uint32_t c = sh[off[q] + b];
      if (c) atomicAdd(&ghist[q * (1 << MAX_BITS) + b], c);
    }
}

// ---------------------------------------------------------------- a4 --
#ifndef VPIC_GATHER_ILP
#define VPIC_GATHER_ILP 8
#endif
// half-records in flight per thread (measured at C2, electrons / ions ms:
// 4: 13.9 / 11.1, 8: 14.0 / 10.8, 16: 13.4 / 11.8)
constexpr int GATHER_ILP = VPIC_GATHER_ILP;

// perm_alt / sel (nullable): the permutation is in perm_alt instead when
// sel->sel is 1 (the rank passes' output buffer is known on the device only).
__global__ void __launch_bounds__(256)
k_gather(const vpic_particle_t *__restrict__ pin, vpic_particle_t *__restrict__ pout,
         const uint32_t *__restrict__ perm_main, const uint32_t *__restrict__ perm_alt,
         const RankParams *__restrict__ sel, int64_t n, int64_t *__restrict__ perm64) {
  const uint32_t *__restrict__ perm = (sel && sel->sel) ? perm_alt : perm_main;
  // two lanes per 32-B record (every warp load / store instruction moves 16
  // whole records: sector-complete, stores fully coalesced); each warp owns
  // blocks of 32 x GATHER_ILP half-records and issues all their loads first
  const float4 *src = reinterpret_cast<const float4 *>(pin);
  float4 *dst = reinterpret_cast<float4 *>(pout);
  const int lane = threadIdx.x & 31;
  const int64_t nh = 2 * n;
  const int64_t wid = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t base = wid * 32 * GATHER_ILP; base < nh; base += nw * 32 * GATHER_ILP) {
    float4 v[GATHER_ILP];
    uint32_t sidx[GATHER_ILP];
#pragma unroll
    for (int j = 0; j < GATHER_ILP; ++j) {
      const int64_t t = base + lane + 32 * j;
      sidx[j] = t < nh ? __ldcs(perm + (t >> 1)) : 0u;
    }
#pragma unroll
    for (int j = 0; j < GATHER_ILP; ++j) {
      const int64_t t = base + lane + 32 * j;
      // default (evict-normal) caching on purpose: a source line fetched for
      // one record is re-used by the neighbouring output voxels shortly after
      // (streaming hints made the L2 miss every time).  20 steps after a sort
      // the electrons of one output voxel come from ~5 z-planes of input
      // (~350 MB > L2), so DRAM still reads ~3.6x the records; measured
      // alternatives -- evict_last on these loads, scattering by the inverse
      // permutation (whose inversion costs more than it saves), gathering in
      // (y-tile, z) segment order so that a segment's sources (~50 MB) stay
      // in L2 (still 31 GB read, 5% L2 hits) -- were not faster.
      // 64-B L2 fetch granularity: the neighbouring records of a source line
      // go to other output voxels, rarely still cached (-1% vs default/256 B)
      if (t < nh) {
        VPIC_ASSERT((int64_t)sidx[j] < n);
        const float4 *a = src + 2 * (int64_t)sidx[j] + (t & 1);
        asm volatile("ld.global.nc.L2::64B.v4.f32 {%0,%1,%2,%3}, [%4];"
                     : "=f"(v[j].x), "=f"(v[j].y), "=f"(v[j].z), "=f"(v[j].w) : "l"(a));
      }
    }
#pragma unroll
    for (int j = 0; j < GATHER_ILP; ++j) {
      const int64_t t = base + lane + 32 * j;
      if (t < nh) {
        __stcs(dst + t, v[j]);
        if (perm64 && !(t & 1)) perm64[t >> 1] = sidx[j];
      }
    }
  }
}

__global__ void k_iota64(int64_t *__restrict__ a, int64_t n) {
  for (int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; t < n;
       t += (int64_t)gridDim.x * blockDim.x)
    a[t] = t;
}

__global__ void k_hist_voxels(const vpic_particle_t *__restrict__ p, int64_t n,
                              int32_t *__restrict__ counts, int64_t *__restrict__ new_keys) {
  const int32_t *pi = reinterpret_cast<const int32_t *>(p) + 3;
  const int lane = threadIdx.x & 31;
  for (int64_t base = (int64_t)blockIdx.x * blockDim.x + (threadIdx.x & ~31); base < n;
       base += (int64_t)gridDim.x * blockDim.x) {
    const int64_t i = base + lane;
    const bool valid = i < n;
    const int32_t k = valid ? pi[8 * i] : -1;
    if (valid && new_keys) new_keys[i] = k;
    const unsigned peers = __match_any_sync(FULL, k);
    if (valid && counts && (__ffs(peers) - 1) == lane) atomicAdd(&counts[k], __popc(peers));
  }
}

// ------------------------------------------------------------ host side --
struct WsLayout {
  size_t keysA, keysB, valsA, valsB, offs, count, bsum, ghist, goff, status, ctr, misc, total;
};

inline size_t align_up(size_t x, size_t a) { return (x + a - 1) / a * a; }

// key buffers: u32 voxel keys; 8 B per particle for TILED_STRIDED, whose
// rank-pass keys (chunk - chunk0) max_r + r can need more than 32 bits
WsLayout layout(int64_t np, int64_t nv, int order) {
  WsLayout L{};
  size_t o = 0;
  auto take = [&](size_t bytes) { size_t r = o; o = align_up(o + bytes, 256); return r; };
  const int64_t tiles = (np + TILE - 1) / TILE;
  const size_t kb = order == VPIC_SORT_TILED_STRIDED ? 8 : 4;
  L.keysA = take(kb * (size_t)np);
  L.keysB = take(kb * (size_t)np);
  L.valsA = take(4 * (size_t)np);
  L.valsB = take(4 * (size_t)np);
  L.offs = take(4 * (size_t)(nv + 1));
  L.count = take(4 * (size_t)nv);
  L.bsum = take(4 * (size_t)(nv / SCAN_B + 2));
  L.ghist = take(4 * (size_t)MAX_PASSES * (1 << MAX_BITS));
  L.goff = take(4 * (size_t)MAX_PASSES * (1 << MAX_BITS));
  L.status = take(8 * (size_t)std::max<int64_t>(tiles, 1) * (1 << MAX_BITS));
  L.ctr = take(4 * MAX_PASSES);
  L.misc = take(64 + sizeof(RankParams));
  L.total = o;
  return L;
}

int bits_for(uint64_t max_value) {  // bits needed to hold values 0..max_value
  int b = 0;
  while (b < 64 && (max_value >> b)) ++b;
  return std::max(b, 1);
}

PassDesc make_passes(int nbits) {
  // full MAX_BITS digits for the later passes, the remainder first: the first
  // pass scatters the least ordered input, so fewer buckets keep its output
  // runs long (measured: 6+8+8 beats 8+7+7 for 22-bit voxel keys)
  PassDesc pd{};
  pd.npass = (nbits + MAX_BITS - 1) / MAX_BITS;
  if (pd.npass < 1) pd.npass = 1;
  const int first = nbits - MAX_BITS * (pd.npass - 1);
  int sh = 0;
  for (int q = 0; q < pd.npass; ++q) {
    const int b = q == 0 ? std::max(first, 1) : MAX_BITS;
    pd.bits[q] = b;
    pd.shift[q] = sh;
    sh += b;
  }
  return pd;
}

template <int BITS, class KeyT, bool REC>
cudaError_t radix_pass_bits(const KeyT *kin, const uint32_t *vin, KeyT *kout, uint32_t *vout,
                            int64_t n, int shift, const uint32_t *dig_off,
                            unsigned long long *status, unsigned int *ctr, const int *live_bits,
                            cudaStream_t s, RecMove rec) {
  const size_t smem = (size_t)NW * (1 << BITS) * 2 + (size_t)(1 << BITS) * 8 + (size_t)TILE * (sizeof(KeyT) + 4);
  const int64_t tiles = (n + TILE - 1) / TILE;
  static std::atomic<uint64_t> configured{0};   // > 48 KB only for large tiles; once per device
  once_per_device(configured, [&] {
    cudaFuncSetAttribute(k_radix_pass<BITS, KeyT, REC>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  });
  int64_t grid = tiles;
#if VPIC_SORT_PERSIST
  {
    int dev = 0, sms = 0, per_sm = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k_radix_pass<BITS, KeyT, REC>, NT, smem);
    grid = std::min<int64_t>(tiles, (int64_t)sms * std::max(per_sm, 1));
  }
#endif
  k_radix_pass<BITS, KeyT, REC><<<(unsigned)grid, NT, smem, s>>>(kin, vin, kout, vout, n, shift, dig_off,
                                                                  status, ctr, live_bits, rec); note_launch();
  return cudaGetLastError();
}

template <class KeyT>
cudaError_t radix_pass(int bits, const KeyT *kin, const uint32_t *vin, KeyT *kout, uint32_t *vout,
                       int64_t n, int shift, const uint32_t *dig_off, unsigned long long *status,
                       unsigned int *ctr, const int *live_bits, cudaStream_t s, const RecMove *rec = nullptr) {
  const RecMove r0{nullptr, nullptr, nullptr};
  switch (bits) {
#define VPIC_RP(B) case B: return rec ? radix_pass_bits<B, KeyT, true>(kin, vin, kout, vout, n, shift, dig_off, status, ctr, live_bits, s, *rec) \
                                      : radix_pass_bits<B, KeyT, false>(kin, vin, kout, vout, n, shift, dig_off, status, ctr, live_bits, s, r0);
    VPIC_RP(1) VPIC_RP(2) VPIC_RP(3) VPIC_RP(4) VPIC_RP(5) VPIC_RP(6) VPIC_RP(7) VPIC_RP(8)
#undef VPIC_RP
    default: return cudaErrorInvalidValue;
  }
}

unsigned grid_cap(int64_t n, int threads, int num_sms, int per_sm) {
  int64_t b = (n + threads - 1) / threads;
  const int64_t cap = (int64_t)num_sms * per_sm;
  if (b > cap) b = cap;
  if (b < 1) b = 1;
  return (unsigned)b;
}

#define CK(x) do { cudaError_t e_ = (x); if (e_ != cudaSuccess) return e_; } while (0)

// Run the LSD passes of `pd` over (keys0, vals0 [nullable = iota]).  Returns
// pointers to the final keys / vals (inside the workspace) when every pass
// runs; with live_bits, trailing passes may return at once on the device and
// the vals then end in *v_final (an even number of live passes) or the other
// buffer (odd; RankParams::sel).
template <class KeyT>
cudaError_t lsd_sort(const PassDesc &pd, int64_t n, KeyT *kA, KeyT *kB, uint32_t *vA,
                     uint32_t *vB, const uint32_t *vals0, uint32_t *ghist, uint32_t *goff,
                     unsigned long long *status, unsigned int *ctr, bool need_keys_out,
                     const int *live_bits, KeyT **k_final, uint32_t **v_final, cudaStream_t s,
                     const KeyT *k_first = nullptr /* the first pass's keys, if not in kA */,
                     const RecMove *rec = nullptr /* the last pass moves the records */) {
  CK(cudaMemsetAsync(ctr, 0, 4 * MAX_PASSES, s));
  k_scan_hist<<<pd.npass, 256, 0, s>>>(ghist, goff, pd); note_launch();
  CK(cudaGetLastError());
  const int64_t tiles = (n + TILE - 1) / TILE;
  KeyT *kin = kA, *kout = kB;
  const KeyT *kin0 = k_first ? k_first : kA;
  const uint32_t *vin = vals0;
  uint32_t *vout = (vals0 == vA) ? vB : vA;
  for (int q = 0; q < pd.npass; ++q) {
    CK(cudaMemsetAsync(status, 0, 8 * (size_t)tiles * (1 << pd.bits[q]), s));
    const bool last = q == pd.npass - 1;
    CK(radix_pass<KeyT>(pd.bits[q], q == 0 ? kin0 : kin, vin, (last && !need_keys_out) ? nullptr : kout,
                        vout, n, pd.shift[q], goff + q * (1 << MAX_BITS), status, ctr + q, live_bits, s,
                        last ? rec : nullptr));
    *k_final = kout;
    *v_final = vout;
    std::swap(kin, kout);
    vin = vout;
    vout = (vout == vA) ? vB : vA;
  }
  return cudaSuccess;
}

// Worst-case rank passes: 8-bit digits from the least significant bit.
PassDesc rank_passes(int nbits) {
  PassDesc pd{};
  pd.npass = std::min(MAX_PASSES, std::max(1, (nbits + MAX_BITS - 1) / MAX_BITS));
  for (int q = 0; q < pd.npass; ++q) {
    pd.bits[q] = MAX_BITS;
    pd.shift[q] = MAX_BITS * q;
  }
  return pd;
}

// The rank stage of STRIDED / TILED_STRIDED: keys from the standard order
// (K, P), passes sized on the device; returns the two candidate perm buffers
// (the first when the number of live passes is even).  Rank keys go through
// 32-bit passes when the device finds they fit (always for STRIDED), else
// through 64-bit ones (TILED_STRIDED with (chunks) x max_r >= 2^32): both
// chains are launched, the other one returns at once.
cudaError_t rank_stage(vpic_ctx *c, int64_t np, int order, int64_t T, int worst_bits,
                       const uint32_t *K, uint32_t *P, void *ckA, void *ckB, uint32_t *vfree,
                       const uint32_t *offs, const unsigned int *max_r_dev, RankParams *rp,
                       uint32_t *ghist, uint32_t *goff, unsigned long long *status,
                       unsigned int *ctr, int64_t *new_keys, uint32_t **perm_even,
                       uint32_t **perm_odd, cudaStream_t s) {
  k_rank_setup<<<1, 1, 0, s>>>(K, np, order, T, max_r_dev, rp); note_launch();
  CK(cudaGetLastError());
  const PassDesc pr = rank_passes(worst_bits);
  CK(cudaMemsetAsync(ghist, 0, 4 * (size_t)MAX_PASSES * (1 << MAX_BITS), s));
  int tot = 0;
  for (int q = 0; q < pr.npass; ++q) tot += 1 << pr.bits[q];
  static std::atomic<uint64_t> configured{0};
  once_per_device(configured, [] {
    cudaFuncSetAttribute(k_rank_keys, cudaFuncAttributeMaxDynamicSharedMemorySize,
                         4 * MAX_PASSES * (1 << MAX_BITS));
  });
  k_rank_keys<<<grid_cap(np, 256, c->num_sms, 2), 256, 4 * (size_t)tot, s>>>(
      K, P, offs, np, order, T, rp, ckA, pr, ghist, new_keys); note_launch();
  CK(cudaGetLastError());
  PassDesc p32 = pr;
  p32.npass = std::min(pr.npass, 4);
  uint32_t *k32 = nullptr, *vf = nullptr;
  CK(lsd_sort<uint32_t>(p32, np, static_cast<uint32_t *>(ckA), static_cast<uint32_t *>(ckB), P, vfree, P,
                        ghist, goff, status, ctr, false, &rp->nbits, &k32, &vf, s));
  if (pr.npass > 4) {
    uint64_t *k64 = nullptr;
    CK(lsd_sort<uint64_t>(pr, np, static_cast<uint64_t *>(ckA), static_cast<uint64_t *>(ckB), P, vfree, P,
                          ghist, goff, status, ctr, false, &rp->nbits, &k64, &vf, s));
  }
  *perm_even = P;       // live passes: 2, 4, ...
  *perm_odd = vfree;    //              1, 3, ...
  return cudaSuccess;
}

}  // namespace

size_t sort_workspace_bytes(const vpic_ctx *c, int64_t np, int order) {
  return layout(np, c->gk.nv, order).total;
}

cudaError_t launch_sort(vpic_ctx *c, const vpic_particle_t *p_in, vpic_particle_t *p_out,
                        int64_t np, int order, int64_t tile_sz, void *ws, size_t ws_bytes,
                        int32_t *voxel_counts, int64_t *new_keys, int64_t *perm, cudaStream_t s,
                        const uint32_t *keys_in) {
  const int64_t nv = c->gk.nv;
  const int sms = c->num_sms;
  if (np == 0) {
    if (voxel_counts) CK(cudaMemsetAsync(voxel_counts, 0, 4 * (size_t)nv, s));
    return cudaSuccess;
  }
  if (order == VPIC_SORT_NONE) {
    CK(cudaMemcpyAsync(p_out, p_in, 32 * (size_t)np, cudaMemcpyDeviceToDevice, s));
    if (voxel_counts) CK(cudaMemsetAsync(voxel_counts, 0, 4 * (size_t)nv, s));
    if (voxel_counts || new_keys) {
      k_hist_voxels<<<grid_cap(np, 256, sms, 8), 256, 0, s>>>(p_in, np, voxel_counts, new_keys); note_launch();
      CK(cudaGetLastError());
    }
    if (perm) {
      k_iota64<<<grid_cap(np, 256, sms, 8), 256, 0, s>>>(perm, np); note_launch();
      CK(cudaGetLastError());
    }
    return cudaSuccess;
  }
  const WsLayout L = layout(np, nv, order);
  if (ws_bytes < L.total) return cudaErrorInvalidValue;
  char *w = static_cast<char *>(ws);
  uint32_t *kA = reinterpret_cast<uint32_t *>(w + L.keysA);
  uint32_t *kB = reinterpret_cast<uint32_t *>(w + L.keysB);
  uint32_t *vA = reinterpret_cast<uint32_t *>(w + L.valsA);
  uint32_t *vB = reinterpret_cast<uint32_t *>(w + L.valsB);
  uint32_t *offs = reinterpret_cast<uint32_t *>(w + L.offs);
  uint32_t *ghist = reinterpret_cast<uint32_t *>(w + L.ghist);
  uint32_t *goff = reinterpret_cast<uint32_t *>(w + L.goff);
  unsigned long long *status = reinterpret_cast<unsigned long long *>(w + L.status);
  unsigned int *ctr = reinterpret_cast<unsigned int *>(w + L.ctr);
  unsigned int *misc = reinterpret_cast<unsigned int *>(w + L.misc);
  RankParams *rp = reinterpret_cast<RankParams *>(w + L.misc + 64);

  // ---- voxel histogram (deterministic run counts), digit histograms
  uint32_t *count = voxel_counts ? reinterpret_cast<uint32_t *>(voxel_counts)
                                 : reinterpret_cast<uint32_t *>(w + L.count);
  CK(cudaMemsetAsync(count, 0, 4 * (size_t)nv, s));
  if (keys_in) {   // keys from the caller: histogram only (the first pass reads keys_in)
    k_count_keys<<<grid_cap(np, 256, sms, 8), 256, 0, s>>>(
        keys_in, np, count, (order == VPIC_SORT_STANDARD) ? new_keys : nullptr); note_launch();
  } else {
    k_keys_count<<<grid_cap(np, 256, sms, 8), 256, 0, s>>>(
        p_in, np, kA, count, (order == VPIC_SORT_STANDARD) ? new_keys : nullptr); note_launch();
  }
  CK(cudaGetLastError());
  const PassDesc pd = make_passes(bits_for((uint64_t)(nv - 1)));
  CK(cudaMemsetAsync(ghist, 0, 4 * (size_t)MAX_PASSES * (1 << MAX_BITS), s));
  k_digit_hist<<<grid_cap(nv, 256, sms, 2), 256, 0, s>>>(count, nv, pd, ghist); note_launch();
  CK(cudaGetLastError());
  // ---- standard order: stable LSD radix sort of (voxel, index)
  uint32_t *K = nullptr, *P = nullptr;
  const bool need_offs = order != VPIC_SORT_STANDARD;
  // standard order: the last pass moves the records (no separate gather)
  const RecMove rec{p_in, p_out, perm};
  CK(lsd_sort<uint32_t>(pd, np, kA, kB, vA, vB, nullptr, ghist, goff, status, ctr, need_offs,
                        nullptr, &K, &P, s, keys_in, need_offs ? nullptr : &rec));
  if (!need_offs) return cudaSuccess;
  const RankParams *sel = nullptr;
  uint32_t *P_alt = nullptr;
  if (need_offs) {  // offs[k] = first standard position of voxel k; max_r
    uint32_t *bsum = reinterpret_cast<uint32_t *>(w + L.bsum);
    const int64_t nb = (nv + SCAN_B - 1) / SCAN_B;
    CK(cudaMemsetAsync(misc, 0, 64, s));
    k_scan_blocksum<<<(unsigned)nb, 256, 0, s>>>(count, nv, bsum, misc); note_launch();
    k_scan_bsums<<<1, 1024, 0, s>>>(bsum, nb); note_launch();
    k_scan_apply<<<(unsigned)nb, 256, 0, s>>>(count, nv, bsum, offs, np); note_launch();
    CK(cudaGetLastError());
    const int64_t T = tile_sz > 0 ? tile_sz : c->tile_sz;
    // the standard keys/perm live in (K, P); the rank passes use the other
    // buffers (and K's once the rank keys are written)
    uint32_t *ck = (K == kA) ? kB : kA;
    uint32_t *vfree = (P == vA) ? vB : vA;
    uint32_t *Pe = nullptr, *Po = nullptr;
    // strided: r < max_r <= np < 2^32; tiled: (chunk - chunk0) max_r + r <=
    // ((nv - 1) / T) np + np - 1, up to 64 bits (8-B key buffers)
    const uint64_t worst = order == VPIC_SORT_STRIDED
                               ? (uint64_t)(np - 1)
                               : (uint64_t)((nv - 1) / T) * (uint64_t)np + (uint64_t)(np - 1);
    CK(rank_stage(c, np, order, T, bits_for(worst), K, P, ck, K, vfree, offs, misc, rp, ghist, goff,
                  status, ctr, new_keys, &Pe, &Po, s));
    P = Pe;
    P_alt = Po;
    sel = rp;
  }
  k_gather<<<grid_cap(2 * np / GATHER_ILP + 1, 256, sms, 8), 256, 0, s>>>(p_in, p_out, P, P_alt, sel, np,
                                                                          perm); note_launch();
  return cudaGetLastError();
}

}  // namespace vpic
