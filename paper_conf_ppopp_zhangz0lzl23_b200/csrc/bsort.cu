// bsort.cu -- request sort for the batch path (Alg.1:10), sm_100a.
//
// Requests must end up ordered by (key, logical timestamp).  The payload of a
// request is ts<<2 | op and ts is unique, so ordering by (key, payload) IS the
// (key, timestamp) order and no step needs to be stable.  That lets the sort
// use atomics freely (B200 design):
//   K0 hist    : histogram of the top BB key bits (2^BB buckets, mean <= 4096
//                requests per bucket); the last CTA to finish scans the counts
//                into bucket starts / cursors;
//   K1 scatter : request validation; tile histogram in shared
//                memory and one global atomicAdd per (tile, bucket) on the
//                bucket cursor place every request in its bucket (unordered
//                within the bucket);
// and group.cu finishes each bucket (sort in shared memory, combine,
// partition) with one CTA per bucket.
// Traffic at n = 2^20: input 9 B (+ 8 B value of each write) read once, 12 B
// per request scattered to the (L2-resident) bucket array.
#include "eirene_internal.cuh"

namespace eirene {

namespace {

constexpr int H_THREADS = 256;
constexpr int H_ITEMS = 8;
constexpr int SC_ITEMS = 8;

// K0+K1: tile histogram of the top bb key bits in shared memory (two copies,
// even / odd warps), one global atomicAdd per (tile, bucket); the last tile to
// finish (threadfence + done counter) scans the bucket counts into bucket
// starts (== cursor starts), so no separate plan launch is needed.
__global__ void __launch_bounds__(H_THREADS) bsort_hist_kernel(const BatchArgs* __restrict__ A, uint32_t n, int bb, int bsh,
                                                               uint32_t* __restrict__ bcount,
                                                               uint32_t* __restrict__ bstart,
                                                               uint32_t* __restrict__ cursor, BatchCtl* ctl) {
  extern __shared__ uint32_t h[];   // [2][1 << bb]
  __shared__ uint32_t s_last;
  __shared__ uint32_t wsum[H_THREADS / 32];
  const uint64_t* __restrict__ keys = A->keys;
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const uint32_t nb = 1u << bb;
  for (uint32_t i = tid; i < 2 * nb; i += H_THREADS) h[i] = 0;
  __syncthreads();
  uint32_t* hw = h + (warp & 1) * nb;
  constexpr int HI = H_ITEMS;
  const uint32_t t0 = blockIdx.x * (H_THREADS * HI);
  uint64_t k[HI];
#pragma unroll
  for (int j = 0; j < HI; ++j) {
    const uint32_t i = t0 + j * H_THREADS + tid;
    k[j] = i < n ? keys[i] : 0;
  }
#pragma unroll
  for (int j = 0; j < HI; ++j)
    if (t0 + j * H_THREADS + tid < n) atomicAdd(&hw[(uint32_t)(k[j] >> (64 - bb))], 1u);
  __syncthreads();
  for (uint32_t i = tid; i < nb; i += H_THREADS) {
    const uint32_t c = h[i] + h[nb + i];
    if (c) atomicAdd(&bcount[i << bsh], c);
  }
  __syncthreads();
  if (tid == 0) {   // barrier + one fence releases the whole CTA's counts (grid-sync pattern)
    __threadfence();
    s_last = atomicAdd(&ctl->tile_ctr[TC_HIST], 1u) == gridDim.x - 1;
  }
  __syncthreads();
  if (!s_last) return;
  __threadfence();
  // exclusive scan of bcount[0..nb) (nb <= 4096: <= 16 per thread)
  const uint32_t per = (nb + H_THREADS - 1) / H_THREADS;
  uint32_t loc[16];
  uint32_t s = 0;
#pragma unroll
  for (uint32_t j = 0; j < 16; ++j) {
    const uint32_t i = tid * per + j;
    loc[j] = (j < per && i < nb) ? ld_cg(bcount + (i << bsh)) : 0u;
    s += loc[j];
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
#pragma unroll
  for (uint32_t j = 0; j < 16; ++j) {
    const uint32_t i = tid * per + j;
    if (j < per && i < nb) {
      bstart[i] = run;
      cursor[i << bsh] = run;
    }
    run += loc[j];
  }
}

// One tile of SC_ITEMS x 256 requests per CTA: tile-local bucket histogram
// with shared-memory atomics (the returned count is the request's rank inside
// the tile), ONE global atomicAdd per (tile, bucket) on the bucket cursor, then
// the scatter.  Global atomics per bucket address = number of tiles (256 at
// n = 2^20) instead of one per request.  Request validation rides on this pass: it reads every key
// and op anyway, and the value only of writes.
__global__ void __launch_bounds__(256) bsort_scatter_kernel(const BatchArgs* __restrict__ A, uint32_t n, int bb, int bsh,
                                                            uint64_t key_lo, uint64_t key_hi,
                                                            uint32_t* __restrict__ cursor, uint64_t* __restrict__ kout,
                                                            uint32_t* __restrict__ pout, BatchCtl* ctl) {
  extern __shared__ uint32_t sh[];   // [2 << bb]: tile histogram, then global base per bucket
  const uint64_t* __restrict__ keys = A->keys;
  const uint8_t* __restrict__ ops = A->ops;
  const uint64_t* __restrict__ vals = A->vals;
  const int tid = threadIdx.x;
  const uint32_t nb = 1u << bb;
  uint32_t* hist = sh;
  uint32_t* gbase = sh + nb;
  for (uint32_t i = tid; i < nb; i += 256) hist[i] = 0;
  __syncthreads();
  const uint32_t t0 = blockIdx.x * (256 * SC_ITEMS);
  uint64_t k[SC_ITEMS];
  uint32_t r[SC_ITEMS];
  uint32_t o[SC_ITEMS];
#pragma unroll
  for (int j = 0; j < SC_ITEMS; ++j) {
    const uint32_t i = t0 + j * 256 + tid;
    k[j] = i < n ? keys[i] : 0;
    o[j] = i < n ? (uint32_t)ops[i] : 0u;
  }
  bool bad = false;
#pragma unroll
  for (int j = 0; j < SC_ITEMS; ++j) {
    const uint32_t i = t0 + j * 256 + tid;
    const bool up = (o[j] == OP_UPDATE || o[j] == OP_INSERT);
    const uint64_t v = (i < n && up) ? vals[i] : 0;
    bad |= i < n && (o[j] > OP_DELETE || k[j] == KEY_MAX || k[j] < key_lo || k[j] >= key_hi || (up && v == KEY_MAX));
  }
  if (__any_sync(FULL, bad) && (tid & 31) == 0) atomicOr(&ctl->invalid, 1u);
#pragma unroll
  for (int j = 0; j < SC_ITEMS; ++j) {
    const uint32_t i = t0 + j * 256 + tid;
    r[j] = i < n ? atomicAdd(&hist[(uint32_t)(k[j] >> (64 - bb))], 1u) : 0u;
  }
  __syncthreads();
  for (uint32_t b = tid; b < nb; b += 256) {
    const uint32_t c = hist[b];
    gbase[b] = c ? atomicAdd(&cursor[b << bsh], c) : 0u;
  }
  __syncthreads();
#pragma unroll
  for (int j = 0; j < SC_ITEMS; ++j) {
    const uint32_t i = t0 + j * 256 + tid;
    if (i < n) {
      const uint32_t pos = gbase[(uint32_t)(k[j] >> (64 - bb))] + r[j];
      kout[pos] = k[j];
      pout[pos] = (i << 2) | o[j];
    }
  }
}

}  // namespace

int bsort_bits(uint32_t n) {
  int bb = 8;
  while (bb < 12 && ((uint64_t)n >> bb) > 4096) ++bb;
  return bb;
}

int bsort_ctr_shift(int bb) {
  int bsh = 0;
  while (bsh < 5 && ((1 << bb) << (bsh + 1)) <= BSORT_CTR_WORDS) ++bsh;
  return bsh;
}

void launch_bucket_sort(const BatchArgs* A, uint32_t n, uint64_t key_lo, uint64_t key_hi, const BSortBufs& b,
                        BatchCtl* ctl, int num_sms, cudaStream_t st, int* launches) {
  (void)num_sms;
  const int bb = bsort_bits(n);
  const uint32_t nb = 1u << bb;
  // bucket counters / cursors are spread over BSORT_CTR_WORDS words so the
  // per-(tile, bucket) atomics hit many L2 slices instead of a few lines
  const int bsh = bsort_ctr_shift(bb);
  const size_t hsm = 2 * nb * sizeof(uint32_t);
  bsort_hist_kernel<<<(n + H_THREADS * H_ITEMS - 1) / (H_THREADS * H_ITEMS), H_THREADS, hsm, st>>>(
      A, n, bb, bsh, b.bcount, b.bstart, b.cursor, ctl);
  bsort_scatter_kernel<<<(n + 256 * SC_ITEMS - 1) / (256 * SC_ITEMS), 256, hsm, st>>>(A, n, bb, bsh, key_lo, key_hi,
                                                                                    b.cursor, b.kA, b.pA, ctl);
  *launches += 2;
}

}  // namespace eirene
