// bsort.cu -- request sort for the batch path (Alg.1:10), part 1 of
// 2: distribution of the batch into balanced key-range groups, sm_100a.  group.cu finishes every group with one CTA (sort in shared
// memory, combine, partition).
//
// Requests must end up ordered by (key, logical timestamp); the payload of a
// request is ts<<2 | op and ts is unique, so ordering by (key, payload) is the
// (key, timestamp) order and this pass need not be stable.
//   K0 hist    : histogram of the top bits of key - key_lo (bin_of: 4096 bins in
//                the fused kernel, 16384 above 2^22 requests); the last
//                CTA to finish scans the bins and cuts them into G groups of
//                ~n/G requests each (a bin never straddles two groups):
//                group(bin) = floor((excl(bin) + cnt(bin)/2) * G / n), and
//                sets every group's start and cursor.
//   K1 scatter : request validation; tile histogram over the
//                groups in shared memory, ONE global atomicAdd per (tile,
//                group) on the group cursor, then the scatter.
// Traffic at n = 2^20: key 8 B read twice, op 1 B (+ 8 B value of a write)
// read once, 12 B per request written to the (L2-resident) group array.
#include "eirene_internal.cuh"

namespace eirene {

namespace {

// Request validation: op in range, key != UINT64_MAX and
// inside the shard, upsert value != UINT64_MAX.  A range query R(l, u)
// (op RANGE, key = l, val = u) is valid with any bounds, but only in a batch
// submitted with range outputs (rok).
__device__ __forceinline__ bool request_invalid(uint32_t o, uint64_t k, uint64_t v, bool up, bool rok,
                                                  uint64_t key_lo, uint64_t key_hi) {
  if (o == OP_RANGE) return !rok;
  return o > OP_DELETE || k == KEY_MAX || k < key_lo || k >= key_hi || (up && v == KEY_MAX);
}
__device__ __forceinline__ void count_ranges(uint32_t nr, BatchCtl* ctl) {
  nr = __reduce_add_sync(FULL, nr);
  if (nr && (threadIdx.x & 31) == 0) atomicAdd(&ctl->nrange, nr);
}

// Group of a bin whose requests' midpoint has prefix x: floor(x * G / total),
// clamped.  Any monotone non-decreasing map of x gives a valid cut (a bin never
// straddles groups, groups stay key ranges in order); a float multiply is that
// and costs one instruction instead of a 64-bit division per bin.  Every CTA
// computes it from the same inputs, so all agree.
__device__ __forceinline__ uint32_t group_of(uint32_t x, float gscale, uint32_t G) {
  return min(G - 1u, (uint32_t)__fmul_rz((float)x, gscale));
}

constexpr int H_THREADS = 512;
constexpr int H_ITEMS = 16;                      // 8192 requests per CTA
constexpr int S_THREADS = 256;
constexpr int S_ITEMS = 8;
constexpr int S_TILE = S_THREADS * S_ITEMS;      // 2048

__global__ void __launch_bounds__(H_THREADS) bsort_hist_kernel(const BatchArgs* __restrict__ A, uint32_t n,
                                                               uint32_t G, uint64_t key_lo, uint32_t bshift,
                                                               uint32_t* __restrict__ bcount,
                                                               uint16_t* __restrict__ bin2grp,
                                                               uint32_t* __restrict__ gstart,
                                                               uint32_t* __restrict__ cursor, BatchCtl* ctl) {
  pdl_wait();   // predecessor kernel complete, its writes visible (no-op without PDL)
  pdl_trigger();
  extern __shared__ __align__(16) uint32_t h[];   // [2 * NBINS_L]: counts; the last CTA's cut (groups, prefixes)
  __shared__ uint32_t s_last;
  n = A->n;   // the launch is sized for the graph's size bucket; the batch's own size is on the device
  __shared__ uint32_t wsum[H_THREADS / 32];
  __shared__ uint32_t s_total;
  const tkey_t* __restrict__ keys = A->keys;
  const uint8_t* __restrict__ ops = A->ops;
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  for (uint32_t i = tid; i < NBINS_L; i += H_THREADS) h[i] = 0;
  __syncthreads();
  // grid-stride over tiles of H_THREADS * H_ITEMS requests: one flush of the
  // CTA's histogram for all its tiles
  for (uint32_t t0 = blockIdx.x * (H_THREADS * H_ITEMS); t0 < n; t0 += gridDim.x * (H_THREADS * H_ITEMS)) {
    uint64_t k[H_ITEMS];
    bool pt[H_ITEMS];   // point request (range queries do not enter the sort)
#pragma unroll
    for (int j = 0; j < H_ITEMS; ++j) {
      const uint32_t i = t0 + j * H_THREADS + tid;
      k[j] = i < n ? widen(keys[i]) : 0;
      pt[j] = i < n && ops[i] != OP_RANGE;
    }
#pragma unroll
    for (int j = 0; j < H_ITEMS; ++j)
      if (pt[j]) atomicAdd(&h[bin_of(k[j], key_lo, bshift, NBINS_L)], 1u);
  }
  __syncthreads();
  for (uint32_t i = tid; i < NBINS_L; i += H_THREADS) {
    const uint32_t c = h[i];
    if (c) atomicAdd(&bcount[i], c);
  }
  __syncthreads();
  if (tid == 0) {   // barrier + one fence releases the whole CTA's counts (grid-sync pattern)
    __threadfence();
    s_last = atomicAdd(&ctl->tile_ctr[TC_HIST], 1u) == gridDim.x - 1;
  }
  __syncthreads();
  if (!s_last) return;
  __threadfence();
  // last CTA: exclusive scan of the bins (32 per thread), then the group cut
  constexpr int PER = NBINS_L / H_THREADS;
  uint32_t cnt[PER];
  uint32_t s = 0;
#pragma unroll
  for (int j = 0; j < PER; ++j) {
    cnt[j] = ld_cg(bcount + tid * PER + j);
    s += cnt[j];
  }
  uint32_t x = s;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const uint32_t y = __shfl_up_sync(FULL, x, o);
    if (lane >= o) x += y;
  }
  if (lane == 31) wsum[warp] = x;
  __syncthreads();
  uint32_t run = x - s;
  for (int w = 0; w < warp; ++w) run += wsum[w];
  if (tid == H_THREADS - 1) s_total = run + s;   // point requests in the batch
  __syncthreads();
  const uint32_t total = s_total;
  uint32_t* sg = h;              // group of every bin
  uint32_t* se = h + NBINS_L;    // exclusive prefix of every bin
  const bool identity = G == (uint32_t)NBINS_L;
  const float gscale = (float)G / (float)max(total, 1u);
#pragma unroll
  for (int j = 0; j < PER; ++j) {
    const uint32_t bin = tid * PER + j;
    const uint32_t g = identity ? bin : group_of(run + cnt[j] / 2, gscale, G);
    sg[bin] = g;
    se[bin] = run;
    bin2grp[bin] = (uint16_t)g;
    run += cnt[j];
  }
  __syncthreads();
  // group g starts at the first bin mapped to it (empty groups start where the next one does)
  for (uint32_t bin = tid; bin < (uint32_t)NBINS_L; bin += H_THREADS) {
    const uint32_t g = sg[bin];
    const uint32_t gp = bin ? sg[bin - 1] : 0xFFFFFFFFu;
    for (uint32_t q = gp + 1; q <= g; ++q) {
      gstart[q] = se[bin];
      cursor[q] = se[bin];
    }
    if (bin == NBINS_L - 1)
      for (uint32_t q = g + 1; q <= G; ++q) gstart[q] = total;
  }
}

// One tile of S_TILE requests per CTA: tile-local group histogram with
// shared-memory atomics (the returned count is the request's rank inside the
// tile), ONE global atomicAdd per (tile, group) on the group cursor, then the
// scatter.  Request validation rides on this pass: it reads
// every key and op anyway, and the value only of writes.
__global__ void __launch_bounds__(S_THREADS) bsort_scatter_kernel(
    const BatchArgs* __restrict__ A, uint32_t n, uint32_t G, uint64_t key_lo, uint64_t key_hi, uint32_t bshift,
    const uint16_t* __restrict__ bin2grp, uint32_t* __restrict__ cursor, uint64_t* __restrict__ kout,
    uint32_t* __restrict__ pout, BatchCtl* ctl) {
  pdl_wait();   // predecessor kernel complete, its writes visible (no-op without PDL)
  pdl_trigger();
  extern __shared__ __align__(16) unsigned char smem[];
  uint16_t* s_b2g = reinterpret_cast<uint16_t*>(smem);             // [NBINS_L]
  uint32_t* hist = reinterpret_cast<uint32_t*>(s_b2g + NBINS_L);   // [G] tile counts, then global base
  n = A->n;
  const tkey_t* __restrict__ keys = A->keys;
  const uint8_t* __restrict__ ops = A->ops;
  const tkey_t* __restrict__ vals = A->vals_src;
  tkey_t* __restrict__ vstage = A->vals_stage;
  const int tid = threadIdx.x;
  for (uint32_t i = tid; i < (uint32_t)NBINS_L; i += S_THREADS) s_b2g[i] = bin2grp[i];
  for (uint32_t i = tid; i < G; i += S_THREADS) hist[i] = 0;
  const uint32_t t0 = blockIdx.x * S_TILE;
  uint64_t k[S_ITEMS];
  uint32_t o[S_ITEMS], g[S_ITEMS], r[S_ITEMS];
#pragma unroll
  for (int j = 0; j < S_ITEMS; ++j) {
    const uint32_t i = t0 + j * S_THREADS + tid;
    k[j] = i < n ? widen(keys[i]) : 0;
    o[j] = i < n ? (uint32_t)ops[i] : 0u;
  }
  bool bad = false;
  const bool rok = A->rkeys != nullptr;
  uint32_t nr = 0;
#pragma unroll
  for (int j = 0; j < S_ITEMS; ++j) {
    const uint32_t i = t0 + j * S_THREADS + tid;
    const bool up = (o[j] == OP_UPDATE || o[j] == OP_INSERT);
    const uint64_t v = (i < n && up) ? widen(vals[i]) : 0;
    if (vstage && i < n && up) vstage[i] = v;
    bad |= i < n && request_invalid(o[j], k[j], v, up, rok, key_lo, key_hi);
    nr += i < n && o[j] == OP_RANGE;
  }
  if (__any_sync(FULL, bad) && (tid & 31) == 0) atomicOr(&ctl->invalid, 1u);
  if (rok) count_ranges(nr, ctl);
  __syncthreads();
#pragma unroll
  for (int j = 0; j < S_ITEMS; ++j) {
    const uint32_t i = t0 + j * S_THREADS + tid;
    g[j] = s_b2g[bin_of(k[j], key_lo, bshift, NBINS_L)];
    r[j] = (i < n && o[j] != OP_RANGE) ? atomicAdd(&hist[g[j]], 1u) : 0u;
  }
  __syncthreads();
  for (uint32_t q = tid; q < G; q += S_THREADS) {
    const uint32_t c = hist[q];
    hist[q] = c ? atomicAdd(&cursor[q], c) : 0u;
  }
  __syncthreads();
#pragma unroll
  for (int j = 0; j < S_ITEMS; ++j) {
    const uint32_t i = t0 + j * S_THREADS + tid;
    if (i < n && o[j] != OP_RANGE) {
      const uint32_t pos = hist[g[j]] + r[j];
      kout[pos] = k[j];
      pout[pos] = (i << 2) | o[j];
    }
  }
}

// Fused K0 + K1 for batches that fit in registers (n <= grid * D_THREADS *
// D_ITEMS): one persistent wave (every CTA resident), each CTA owns a
// contiguous slice of the batch and keeps its keys and ops in registers.
// Phase 1: validation + 4096-bin smem histogram -> global bin counts.  Grid
// barrier.  Phase 2: every CTA recomputes the group cut from the global counts
// (CTA 0 also publishes the group starts).  Phase 3: tile histogram over the
// groups, one atomic per (CTA, group) on the group cursor (zeroed per batch,
// relative to the group start), scatter from registers.  One launch and one
// read of the keys instead of two of each.
constexpr int D_THREADS = 512;
constexpr int D_ITEMS = 8;
constexpr int D_TILE = D_THREADS * D_ITEMS;   // >= per_cta
constexpr int D_GMAX = NBINS / 2;             // groups of the fused path
// Dynamic shared memory of the fused kernel (two CTAs per SM).  The tile
// staging arrays overlay the bin arrays, which are dead by the time the tile
// is staged.
struct DSmem {
  union {
    struct {
      uint32_t h[NBINS];        // local bin counts; global counts; then bin -> group
      uint32_t gs[NBINS + 4];   // exclusive bin prefix; then group starts
    } b;
    uint64_t sk[D_TILE];        // the tile's keys in group order (staged scatter)
  } u;
  uint32_t sp[D_TILE];          // ... their payloads
  uint16_t sg[D_TILE];          // ... their groups
  uint32_t th[D_GMAX];          // tile count per group; then local offsets
  uint32_t gb[D_GMAX];          // global position of the tile's first request of each group
  uint32_t wsum[D_THREADS / 32];
  uint32_t total;
};

__global__ void __launch_bounds__(D_THREADS, 2) bsort_dist_kernel(
    const BatchArgs* __restrict__ A, uint32_t n, uint32_t G, uint32_t per_cta, uint64_t key_lo, uint64_t key_hi,
    uint32_t bshift, uint32_t* __restrict__ bcount, uint32_t* __restrict__ gstart, uint32_t* __restrict__ cursor,
    uint64_t* __restrict__ kout, uint32_t* __restrict__ pout, BatchCtl* ctl) {
  pdl_wait();   // predecessor kernel complete, its writes visible (no-op without PDL)
  pdl_trigger();
  extern __shared__ __align__(16) unsigned char dsm_raw[];
  DSmem& S = *reinterpret_cast<DSmem*>(dsm_raw);
  uint32_t* h = S.u.b.h;
  uint32_t* gs = S.u.b.gs;
  n = A->n;   // (per_cta is sized for the graph's size bucket >= n)
  EIRENE_PHASE(A, 0, blockIdx.x, 0);
  const tkey_t* __restrict__ keys = A->keys;
  const uint8_t* __restrict__ ops = A->ops;
  const tkey_t* __restrict__ vals = A->vals_src;
  tkey_t* __restrict__ vstage = A->vals_stage;
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  for (uint32_t i = tid; i < NBINS; i += D_THREADS) h[i] = 0;
  __syncthreads();
  const uint32_t t0 = blockIdx.x * per_cta;
  const uint32_t t1 = min(n, t0 + per_cta);
  uint64_t k[D_ITEMS];
  uint32_t o[D_ITEMS];
#pragma unroll
  for (int j = 0; j < D_ITEMS; ++j) {
    const uint32_t i = t0 + j * D_THREADS + tid;
    k[j] = i < t1 ? widen(keys[i]) : 0;
    o[j] = i < t1 ? (uint32_t)ops[i] : 0u;
  }
  bool bad = false;
  const bool rok = A->rkeys != nullptr;
  uint32_t nr = 0;
#pragma unroll
  for (int j = 0; j < D_ITEMS; ++j) {
    const uint32_t i = t0 + j * D_THREADS + tid;
    const bool up = (o[j] == OP_UPDATE || o[j] == OP_INSERT);
    const uint64_t v = (i < t1 && up) ? widen(vals[i]) : 0;
    if (vstage && i < t1 && up) vstage[i] = v;
    bad |= i < t1 && request_invalid(o[j], k[j], v, up, rok, key_lo, key_hi);
    nr += i < t1 && o[j] == OP_RANGE;
    if (i < t1 && o[j] != OP_RANGE) atomicAdd(&h[bin_of(k[j], key_lo, bshift, NBINS)], 1u);
  }
  if (__any_sync(FULL, bad) && lane == 0) atomicOr(&ctl->invalid, 1u);
  if (rok) count_ranges(nr, ctl);
  __syncthreads();
  EIRENE_PHASE(A, 0, blockIdx.x, 1);
  for (uint32_t i = tid; i < NBINS; i += D_THREADS)
    if (h[i]) atomicAdd(&bcount[i], h[i]);
  // grid barrier (all CTAs are resident: the grid is one occupancy wave)
  __syncthreads();
  EIRENE_PHASE(A, 0, blockIdx.x, 2);
  if (tid == 0) {
    __threadfence();
    atomicAdd(&ctl->gbar, 1u);
    SpinGuard sg;
    while (ld_acquire(&ctl->gbar) < gridDim.x)
      if (sg.stuck(ctl)) break;
  }
  __syncthreads();
  EIRENE_PHASE(A, 0, blockIdx.x, 3);
  // phase 2: the group cut, as in bsort_hist_kernel's last CTA.  Every CTA
  // needs all 4096 global counts: staged into shared memory with coalesced
  // 16 B loads (296 CTAs reading the same 16 KB as strided 4 B loads hammered
  // the same L2 lines: 7-11 us, r2d phase profile)
  for (uint32_t i = tid; i < NBINS / 4; i += D_THREADS)
    reinterpret_cast<uint4*>(h)[i] = __ldcg(reinterpret_cast<const uint4*>(bcount) + i);
  __syncthreads();
  constexpr int PER = NBINS / D_THREADS;
  uint32_t cnt[PER];
  uint32_t sum = 0;
  {
    const uint4 a = reinterpret_cast<const uint4*>(h)[2 * tid], b = reinterpret_cast<const uint4*>(h)[2 * tid + 1];
    cnt[0] = a.x; cnt[1] = a.y; cnt[2] = a.z; cnt[3] = a.w;
    cnt[4] = b.x; cnt[5] = b.y; cnt[6] = b.z; cnt[7] = b.w;
  }
#pragma unroll
  for (int j = 0; j < PER; ++j) sum += cnt[j];
  uint32_t x = sum;
#pragma unroll
  for (int d = 1; d < 32; d <<= 1) {
    const uint32_t y = __shfl_up_sync(FULL, x, d);
    if (lane >= d) x += y;
  }
  if (lane == 31) S.wsum[warp] = x;
  __syncthreads();
  uint32_t run = x - sum;
  for (int w = 0; w < warp; ++w) run += S.wsum[w];
  if (tid == D_THREADS - 1) S.total = run + sum;   // point requests in the batch
  __syncthreads();
  const uint32_t total = S.total;
  const bool identity = G == (uint32_t)NBINS;
  const float gscale = (float)G / (float)max(total, 1u);
  uint32_t gq[PER], ge[PER];
#pragma unroll
  for (int j = 0; j < PER; ++j) {
    const uint32_t bin = tid * PER + j;
    gq[j] = identity ? bin : group_of(run + cnt[j] / 2, gscale, G);
    ge[j] = run;
    h[bin] = gq[j];
    run += cnt[j];
  }
  __syncthreads();
  // group g starts at the prefix of its first bin (empty groups: where the next one does)
  {
    uint32_t gp = tid ? h[tid * PER - 1] : 0xFFFFFFFFu;
#pragma unroll
    for (int j = 0; j < PER; ++j) {
      for (uint32_t q = gp + 1; q <= gq[j]; ++q) gs[q] = ge[j];
      gp = gq[j];
    }
    if (tid == D_THREADS - 1)
      for (uint32_t q = gp + 1; q <= G; ++q) gs[q] = total;
  }
  __syncthreads();
  if (blockIdx.x == 0)
    for (uint32_t q = tid; q <= G; q += D_THREADS) gstart[q] = gs[q];
  EIRENE_PHASE(A, 0, blockIdx.x, 4);
  // phase 3: group of every item; tile histogram over the groups
  uint32_t g[D_ITEMS], r[D_ITEMS];
#pragma unroll
  for (int j = 0; j < D_ITEMS; ++j) g[j] = h[bin_of(k[j], key_lo, bshift, NBINS)];
  for (uint32_t q = tid; q < G; q += D_THREADS) S.th[q] = 0;
  __syncthreads();
#pragma unroll
  for (int j = 0; j < D_ITEMS; ++j) {
    const uint32_t i = t0 + j * D_THREADS + tid;
    r[j] = (i < t1 && o[j] != OP_RANGE) ? atomicAdd(&S.th[g[j]], 1u) : 0u;
  }
  __syncthreads();
  // per group: one global atomic for the tile's base in the group, and the
  // exclusive scan of the tile's counts (local offsets of the group-ordered tile)
  for (uint32_t q = tid; q < G; q += D_THREADS) {   // (one atomic per thread: all in flight together)
    const uint32_t c = S.th[q];
    if (c) S.gb[q] = gs[q] + atomicAdd(&cursor[q], c);
  }
  {
    constexpr int GPER = D_GMAX / D_THREADS;   // 4 groups per thread
    uint32_t c[GPER], lsum = 0;
#pragma unroll
    for (int j = 0; j < GPER; ++j) {
      const uint32_t q = tid * GPER + j;
      c[j] = q < G ? S.th[q] : 0u;
      lsum += c[j];
    }
    uint32_t y = lsum;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
      const uint32_t z = __shfl_up_sync(FULL, y, d);
      if (lane >= d) y += z;
    }
    __syncthreads();   // (S.wsum reuse)
    if (lane == 31) S.wsum[warp] = y;
    __syncthreads();
    uint32_t lr = y - lsum;
    for (int w = 0; w < warp; ++w) lr += S.wsum[w];
#pragma unroll
    for (int j = 0; j < GPER; ++j) {
      const uint32_t q = tid * GPER + j;
      if (q < G) S.th[q] = lr;
      lr += c[j];
    }
  }
  __syncthreads();   // (the bin arrays are dead from here: the staging overlays them)
  EIRENE_PHASE(A, 0, blockIdx.x, 5);
  // staged scatter: the tile in group order in shared memory, then every
  // group's run written out contiguously (coalesced instead of one scattered
  // 8 B + 4 B store per request)
#pragma unroll
  for (int j = 0; j < D_ITEMS; ++j) {
    const uint32_t i = t0 + j * D_THREADS + tid;
    if (i < t1 && o[j] != OP_RANGE) {
      const uint32_t lp = S.th[g[j]] + r[j];
      S.u.sk[lp] = k[j];
      S.sp[lp] = (i << 2) | o[j];
      S.sg[lp] = (uint16_t)g[j];
    }
  }
  __syncthreads();
  uint32_t tcount = 0;   // point requests of the tile
#pragma unroll
  for (int j = 0; j < D_ITEMS; ++j) {
    const uint32_t i = t0 + j * D_THREADS + tid;
    tcount += (i < t1 && o[j] != OP_RANGE) ? 1u : 0u;
  }
  tcount = __reduce_add_sync(FULL, tcount);
  if (lane == 0) S.wsum[warp] = tcount;
  __syncthreads();
  uint32_t tot = 0;
  for (int w = 0; w < D_THREADS / 32; ++w) tot += S.wsum[w];
  for (uint32_t lp = tid; lp < tot; lp += D_THREADS) {
    const uint32_t q = S.sg[lp];
    const uint32_t pos = S.gb[q] + (lp - S.th[q]);
    kout[pos] = S.u.sk[lp];
    pout[pos] = S.sp[lp];
  }
  EIRENE_PHASE(A, 0, blockIdx.x, 6);
}

}  // namespace

static uint32_t dist_grid(int num_sms) {
  static int occ[MAX_DEVICES];
  const int per_sm = per_device(occ, [] {
    int v = 0;
    cudaFuncSetAttribute(bsort_dist_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sizeof(DSmem));
    return cudaOccupancyMaxActiveBlocksPerMultiprocessor(&v, bsort_dist_kernel, D_THREADS, sizeof(DSmem)) ==
                   cudaSuccess
               ? v
               : 0;
  });
  return (uint32_t)num_sms * (uint32_t)std::max(per_sm, 0);
}

// The ONE predicate choosing the distribution path (used by the launcher, the
// group count and the handle's buffer choice in api.cu): the fused kernel
// (4096 bins, keys held in registers by one resident wave) when the batch fits
// that wave, else the two-kernel path (16384 bins, its own zeroed region).
bool bsort_fused(uint32_t n, int num_sms) {
  const uint32_t grid = dist_grid(num_sms);
  return grid > 0 && (uint64_t)grid * D_THREADS * D_ITEMS >= n;
}
uint64_t bsort_fused_capacity(int num_sms) { return (uint64_t)dist_grid(num_sms) * D_THREADS * D_ITEMS; }

uint32_t bsort_groups(uint32_t n, int num_sms) {
  // two resident group CTAs per SM when n allows; ~3.5K requests per group
  // otherwise.  The fused kernel cuts 4096 bins (at most NBINS / 2 groups);
  // the two-kernel path cuts 16384 (every group still fits shared memory
  // unless one key holds more than a group's worth of requests)
  uint32_t g = (n + 3583) / 3584;
  const uint32_t par = std::min<uint32_t>(2u * (uint32_t)num_sms, (n + 255) / 256);
  g = std::max(g, par);
  const uint32_t cap = bsort_fused(n, num_sms) ? (uint32_t)NBINS / 2 : (uint32_t)NBINS_L;
  return std::max(1u, std::min(g, cap));
}

void launch_bucket_sort(const BatchArgs* A, uint32_t n, uint64_t key_lo, uint64_t key_hi, const BSortBufs& b,
                        BatchCtl* ctl, int num_sms, cudaStream_t st, int* launches) {
  const uint32_t G = bsort_groups(n, num_sms);
  const uint32_t grid = dist_grid(num_sms);
  if (bsort_fused(n, num_sms)) {
    uint32_t bshift = bin_shift(key_lo, key_hi, BIN_BITS);
    // fused single launch; slices of whole 512-request rows per CTA
    const uint32_t rows = (n + D_THREADS - 1) / D_THREADS;
    const uint32_t per_cta = ((rows + grid - 1) / grid) * D_THREADS;
    // one resident wave with a grid barrier: every CTA co-resident (a cooperative
    // launch only with EIRENE_COOP=1; see launch_k for why a plain launch is safe here)
    launch_k(bsort_dist_kernel, dim3(grid), dim3(D_THREADS), sizeof(DSmem), st, true, true, A, n, G, per_cta, key_lo, key_hi,
             bshift, b.bcount, b.gstart, b.cursor, b.kA, b.pA, ctl);
    *launches += 1;
    return;
  }
  const uint32_t bshift = bin_shift(key_lo, key_hi, BIN_BITS_L);
  const size_t hsm = 2 * NBINS_L * sizeof(uint32_t);
  const size_t ssm = NBINS_L * sizeof(uint16_t) + (size_t)NBINS_L * sizeof(uint32_t);
  static int attr[MAX_DEVICES];
  per_device(attr, [&] {
    cudaFuncSetAttribute(bsort_hist_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)hsm);
    return (int)cudaFuncSetAttribute(bsort_scatter_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)ssm);
  });
  const uint32_t tiles = (n + H_THREADS * H_ITEMS - 1) / (H_THREADS * H_ITEMS);
  launch_k(bsort_hist_kernel, dim3(std::max(1u, std::min(tiles, (uint32_t)num_sms))), dim3(H_THREADS), hsm, st, true,
           false, A, n, G, key_lo, bshift, b.bcount, b.bin2grp, b.gstart, b.cursor, ctl);
  const size_t sm = NBINS_L * sizeof(uint16_t) + (size_t)G * sizeof(uint32_t);
  launch_k(bsort_scatter_kernel, dim3((n + S_TILE - 1) / S_TILE), dim3(S_THREADS), sm, st, true, false, A, n, G,
           key_lo, key_hi, bshift, (const uint16_t*)b.bin2grp, b.cursor, b.kA, b.pA, ctl);
  *launches += 2;
}

}  // namespace eirene
