// bsort.cu -- request sort for the batch path (Alg.1:10), sm_100a.
//
// Requests must end up ordered by (key, logical timestamp).  The payload of a
// request is ts<<2 | op and ts is unique, so ordering by (key, payload) IS the
// (key, timestamp) order and no step needs to be stable.  That lets the sort
// use atomics freely (B200 design):
//   K0 hist    : histogram of the top BB key bits (2^BB buckets, mean <= 4096
//                requests per bucket) + request validation;
//   K1 plan    : one CTA scans the bucket counts -> bucket starts / cursors;
//   K2 scatter : warp-aggregated atomicAdd on the bucket cursor places every
//                request in its bucket (unordered within the bucket);
//   K3 local   : one CTA per bucket.  Small buckets (the uniform case) are
//                sorted in shared memory: sub-bucket by the next 12 key bits
//                (smem atomics + block scan + scatter) and finish each
//                sub-bucket (~1 request on average) by insertion sort on
//                (key, payload).  Oversized buckets (skewed / Zipf keys) are
//                sorted by the same CTA with a stable in-L2 LSD radix sort on
//                (payload, then the low key bits).
// Traffic at n = 2^20: input 9 B + 2 x 12 B scatter/gather + 12 B output per
// request, all L2-resident except the first read of the input.
#include "eirene_internal.cuh"

namespace eirene {

namespace {

constexpr int SB_BITS = 12;                    // sub-bucket bits inside a bucket
constexpr int SB_N = 1 << SB_BITS;
constexpr int LOC_THREADS = 512;
constexpr int LOC_ITEMS = 12;
constexpr int LOC_CAP = LOC_THREADS * LOC_ITEMS;   // 6144 requests sorted in smem
constexpr int H_THREADS = 256;

__device__ __forceinline__ bool kp_less(uint64_t ka, uint32_t pa, uint64_t kb, uint32_t pb) {
  return ka < kb || (ka == kb && pa < pb);
}

__global__ void __launch_bounds__(H_THREADS) bsort_hist_kernel(const BatchArgs* __restrict__ A, uint32_t n,
                                                               int bb, uint64_t key_lo, uint64_t key_hi,
                                                               uint32_t* __restrict__ bcount, BatchCtl* ctl) {
  extern __shared__ uint32_t h[];   // [2][1 << bb]: two copies (even / odd warps) halve contention
  const uint64_t* __restrict__ keys = A->keys;
  const uint8_t* __restrict__ ops = A->ops;
  const uint64_t* __restrict__ vals = A->vals;
  const int tid = threadIdx.x, lane = tid & 31;
  const uint32_t nb = 1u << bb;
  for (uint32_t i = tid; i < 2 * nb; i += H_THREADS) h[i] = 0;
  __syncthreads();
  uint32_t* hw = h + ((tid >> 5) & 1) * nb;
  bool bad = false;
  // one tile of 16 x 256 requests per CTA, all loads issued before any atomic
  constexpr int HI = 16;
  const uint32_t t0 = blockIdx.x * (H_THREADS * HI);
  uint64_t k[HI];
  uint32_t o[HI];
#pragma unroll
  for (int j = 0; j < HI; ++j) {
    const uint32_t i = t0 + j * H_THREADS + tid;
    k[j] = i < n ? keys[i] : 0;
    o[j] = (ops && i < n) ? (uint32_t)ops[i] : 0u;
  }
#pragma unroll
  for (int j = 0; j < HI; ++j) {
    const uint32_t i = t0 + j * H_THREADS + tid;
    if (i < n) {
      atomicAdd(&hw[(uint32_t)(k[j] >> (64 - bb))], 1u);
      if (ops) {
        const bool up = (o[j] == OP_UPDATE || o[j] == OP_INSERT);
        bad |= o[j] > OP_DELETE || k[j] == KEY_MAX || k[j] < key_lo || k[j] >= key_hi || (up && vals[i] == KEY_MAX);
      }
    }
  }
  if (__any_sync(FULL, bad) && lane == 0) atomicOr(&ctl->invalid, 1u);
  __syncthreads();
  for (uint32_t i = tid; i < nb; i += H_THREADS) {
    const uint32_t c = h[i] + h[nb + i];
    if (c) atomicAdd(&bcount[i], c);
  }
}

// one CTA: exclusive scan of the bucket counts -> bstart (== cursor start)
__global__ void __launch_bounds__(1024) bsort_plan_kernel(const uint32_t* __restrict__ bcount, int bb,
                                                          uint32_t* __restrict__ bstart,
                                                          uint32_t* __restrict__ cursor) {
  __shared__ uint32_t wsum[32];
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const uint32_t nb = 1u << bb;
  const uint32_t per = (nb + 1023) / 1024;
  uint32_t loc[4];
  uint32_t s = 0;
  for (uint32_t j = 0; j < per; ++j) {
    const uint32_t i = tid * per + j;
    loc[j] = i < nb ? bcount[i] : 0;
    s += loc[j];
  }
  uint32_t x = s;
  for (int o = 1; o < 32; o <<= 1) {
    const uint32_t y = __shfl_up_sync(FULL, x, o);
    if (lane >= o) x += y;
  }
  if (lane == 31) wsum[warp] = x;
  __syncthreads();
  uint32_t wp = 0;
  for (int w = 0; w < warp; ++w) wp += wsum[w];
  uint32_t run = wp + x - s;
  for (uint32_t j = 0; j < per; ++j) {
    const uint32_t i = tid * per + j;
    if (i < nb) {
      bstart[i] = run;
      cursor[i] = run;
    }
    run += loc[j];
  }
  if (tid == 0) bstart[nb] = 0;   // unused sentinel slot
}

// One tile of SC_ITEMS x 256 requests per CTA: tile-local bucket histogram
// with shared-memory atomics (the returned count is the request's rank inside
// the tile), ONE global atomicAdd per (tile, bucket) on the bucket cursor, then
// the scatter.  Global atomics per bucket address = number of tiles (256 at
// n = 2^20) instead of one per request.
constexpr int SC_ITEMS = 16;
__global__ void __launch_bounds__(256) bsort_scatter_kernel(const BatchArgs* __restrict__ A, uint32_t n, int bb,
                                                            uint32_t* __restrict__ cursor, uint64_t* __restrict__ kout,
                                                            uint32_t* __restrict__ pout, const BatchCtl* ctl) {
  extern __shared__ uint32_t sh[];   // [2 << bb]: tile histogram, then global base per bucket
  const uint64_t* __restrict__ keys = A->keys;
  const uint8_t* __restrict__ ops = A->ops;
  if (ctl->invalid) return;
  const int tid = threadIdx.x;
  const uint32_t nb = 1u << bb;
  uint32_t* hist = sh;
  uint32_t* gbase = sh + nb;
  for (uint32_t i = tid; i < nb; i += 256) hist[i] = 0;
  __syncthreads();
  const uint32_t t0 = blockIdx.x * (256 * SC_ITEMS);
  uint64_t k[SC_ITEMS];
  uint32_t r[SC_ITEMS];
#pragma unroll
  for (int j = 0; j < SC_ITEMS; ++j) {
    const uint32_t i = t0 + j * 256 + tid;
    k[j] = i < n ? keys[i] : 0;
  }
#pragma unroll
  for (int j = 0; j < SC_ITEMS; ++j) {
    const uint32_t i = t0 + j * 256 + tid;
    r[j] = i < n ? atomicAdd(&hist[(uint32_t)(k[j] >> (64 - bb))], 1u) : 0u;
  }
  __syncthreads();
  for (uint32_t b = tid; b < nb; b += 256) {
    const uint32_t c = hist[b];
    gbase[b] = c ? atomicAdd(&cursor[b], c) : 0u;
  }
  __syncthreads();
#pragma unroll
  for (int j = 0; j < SC_ITEMS; ++j) {
    const uint32_t i = t0 + j * 256 + tid;
    if (i < n) {
      const uint32_t pos = gbase[(uint32_t)(k[j] >> (64 - bb))] + r[j];
      kout[pos] = k[j];
      pout[pos] = (i << 2) | (uint32_t)ops[i];
    }
  }
}

struct LocSmem {
  uint64_t k[LOC_CAP];
  uint32_t p[LOC_CAP];
  uint32_t sb[SB_N + 1];
  uint32_t wsum[LOC_THREADS / 32];
  uint32_t hist[256];
  uint32_t off[256];
};

// Stable LSD pass over [0, cnt) of (ks, ps) -> (kd, pd) by an 8-bit digit, by
// one CTA walking the bucket in LOC_THREADS-sized tiles; warps of a tile take
// their offsets in warp order, lanes in lane order, so the pass is stable.
template <class DigitFn>
__device__ void cta_lsd_pass(const uint64_t* ks, const uint32_t* ps, uint64_t* kd, uint32_t* pd, uint32_t cnt,
                             DigitFn dig, LocSmem& S) {
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  if (tid < 256) S.hist[tid] = 0;
  __syncthreads();
  for (uint32_t i = tid; i < cnt; i += LOC_THREADS) atomicAdd(&S.hist[dig(ks[i], ps[i])], 1u);
  __syncthreads();
  if (tid == 0) {
    uint32_t r = 0;
    for (int d = 0; d < 256; ++d) {
      S.off[d] = r;
      r += S.hist[d];
    }
  }
  __syncthreads();
  for (uint32_t base = 0; base < cnt; base += LOC_THREADS) {
    const uint32_t i = base + tid;
    const bool act = i < cnt;
    const uint64_t k = act ? ks[i] : 0;
    const uint32_t p = act ? ps[i] : 0;
    const uint32_t d = act ? dig(k, p) : 256u;
    const uint32_t peers = __match_any_sync(FULL, d);
    uint32_t before = 0;
    for (int w = 0; w < LOC_THREADS / 32; ++w) {
      if (warp == w && act) before = S.off[d];
      __syncthreads();
      if (warp == w && act && lane == 31 - __clz(peers)) S.off[d] += __popc(peers);
      __syncthreads();
    }
    if (act) {
      const uint32_t pos = before + __popc(peers & lanemask_lt());
      kd[pos] = k;
      pd[pos] = p;
    }
  }
  __syncthreads();
}

__global__ void __launch_bounds__(LOC_THREADS) bsort_local_kernel(uint64_t* __restrict__ ka, uint32_t* __restrict__ pa,
                                                                  uint64_t* __restrict__ kb, uint32_t* __restrict__ pb,
                                                                  const uint32_t* __restrict__ bcount,
                                                                  const uint32_t* __restrict__ bstart, int bb,
                                                                  const BatchCtl* ctl) {
  extern __shared__ __align__(16) unsigned char smem_raw[];
  LocSmem& S = *reinterpret_cast<LocSmem*>(smem_raw);
  if (ctl->invalid) return;
  const int tid = threadIdx.x;
  const uint32_t b = blockIdx.x;
  const uint32_t cnt = bcount[b];
  const uint32_t base = bstart[b];
  if (cnt == 0) return;
  uint64_t* ks = ka + base;
  uint32_t* ps = pa + base;
  uint64_t* kd = kb + base;
  uint32_t* pd = pb + base;
  if (cnt == 1) {
    if (tid == 0) {
      kd[0] = ks[0];
      pd[0] = ps[0];
    }
    return;
  }
  const int sb_shift = 64 - bb - SB_BITS;
  if (cnt <= LOC_CAP) {
    for (int i = tid; i <= SB_N; i += LOC_THREADS) S.sb[i] = 0;
    __syncthreads();
    uint32_t r[LOC_ITEMS];
#pragma unroll
    for (int j = 0; j < LOC_ITEMS; ++j) {
      const uint32_t i = tid + j * LOC_THREADS;
      r[j] = 0;
      if (i < cnt) r[j] = atomicAdd(&S.sb[(uint32_t)(ks[i] >> sb_shift) & (SB_N - 1)], 1u);
    }
    __syncthreads();
    // exclusive scan of S.sb[0..SB_N) (8 per thread)
    {
      constexpr int PER = SB_N / LOC_THREADS;
      uint32_t loc[PER], s = 0;
#pragma unroll
      for (int j = 0; j < PER; ++j) {
        loc[j] = S.sb[tid * PER + j];
        s += loc[j];
      }
      const int lane = tid & 31, warp = tid >> 5;
      uint32_t x = s;
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        const uint32_t y = __shfl_up_sync(FULL, x, o);
        if (lane >= o) x += y;
      }
      if (lane == 31) S.wsum[warp] = x;
      __syncthreads();
      uint32_t wp = 0;
      for (int w = 0; w < warp; ++w) wp += S.wsum[w];
      uint32_t run = wp + x - s;
#pragma unroll
      for (int j = 0; j < PER; ++j) {
        S.sb[tid * PER + j] = run;
        run += loc[j];
      }
      if (tid == 0) S.sb[SB_N] = cnt;
    }
    __syncthreads();
#pragma unroll
    for (int j = 0; j < LOC_ITEMS; ++j) {
      const uint32_t i = tid + j * LOC_THREADS;
      if (i < cnt) {
        const uint64_t k = ks[i];
        const uint32_t pos = S.sb[(uint32_t)(k >> sb_shift) & (SB_N - 1)] + r[j];
        S.k[pos] = k;
        S.p[pos] = ps[i];
      }
    }
    __syncthreads();
    // finish every sub-bucket by insertion sort on (key, payload)
    for (int s = tid; s < SB_N; s += LOC_THREADS) {
      const uint32_t lo = S.sb[s], hi = S.sb[s + 1];
      for (uint32_t a = lo + 1; a < hi; ++a) {
        const uint64_t k = S.k[a];
        const uint32_t p = S.p[a];
        uint32_t c = a;
        while (c > lo && kp_less(k, p, S.k[c - 1], S.p[c - 1])) {
          S.k[c] = S.k[c - 1];
          S.p[c] = S.p[c - 1];
          --c;
        }
        S.k[c] = k;
        S.p[c] = p;
      }
    }
    __syncthreads();
    for (uint32_t i = tid; i < cnt; i += LOC_THREADS) {
      kd[i] = S.k[i];
      pd[i] = S.p[i];
    }
    return;
  }
  // Oversized bucket: stable LSD in L2 on the payload (4 x 8 bits) and then the
  // key bits below the bucket prefix; 4 + ceil((64-bb)/8) passes ping-pong
  // between (ks, ps) and (kd, pd); an odd number of passes ends in (kd, pd).
  const int key_passes = (64 - bb + 7) / 8;
  int total = 4 + key_passes;
  uint64_t* k0 = ks;
  uint32_t* p0 = ps;
  uint64_t* k1 = kd;
  uint32_t* p1 = pd;
  if ((total & 1) == 0) {   // make the count odd with a copy pass into (kd, pd) first
    for (uint32_t i = tid; i < cnt; i += LOC_THREADS) {
      kd[i] = ks[i];
      pd[i] = ps[i];
    }
    __syncthreads();
    k0 = kd; p0 = pd; k1 = ks; p1 = ps;
  }
  for (int pass = 0; pass < total; ++pass) {
    if (pass < 4) {
      const int sh = pass * 8;
      cta_lsd_pass(k0, p0, k1, p1, cnt, [sh](uint64_t, uint32_t p) { return (p >> sh) & 0xFFu; }, S);
    } else {
      const int sh = (pass - 4) * 8;
      cta_lsd_pass(k0, p0, k1, p1, cnt, [sh](uint64_t k, uint32_t) { return (uint32_t)(k >> sh) & 0xFFu; }, S);
    }
    uint64_t* tk = k0; k0 = k1; k1 = tk;
    uint32_t* tp = p0; p0 = p1; p1 = tp;
  }
}

}  // namespace

int bsort_bits(uint32_t n) {
  int bb = 8;
  while (bb < 12 && ((uint64_t)n >> bb) > 4096) ++bb;
  return bb;
}

void launch_bucket_sort(const BatchArgs* A, uint32_t n, uint64_t key_lo, uint64_t key_hi, const BSortBufs& b,
                        BatchCtl* ctl, int num_sms, cudaStream_t st, int* launches) {
  (void)num_sms;
  static bool attr = false;
  if (!attr) {
    cudaFuncSetAttribute(bsort_local_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sizeof(LocSmem));
    attr = true;
  }
  const int bb = bsort_bits(n);
  const uint32_t nb = 1u << bb;
  const uint32_t hb = (n + H_THREADS * 16 - 1) / (H_THREADS * 16);
  bsort_hist_kernel<<<hb, H_THREADS, 2 * nb * sizeof(uint32_t), st>>>(A, n, bb, key_lo, key_hi, b.bcount, ctl);
  bsort_plan_kernel<<<1, 1024, 0, st>>>(b.bcount, bb, b.bstart, b.cursor);
  const uint32_t sbk = (n + 256 * SC_ITEMS - 1) / (256 * SC_ITEMS);
  bsort_scatter_kernel<<<sbk, 256, 2 * nb * sizeof(uint32_t), st>>>(A, n, bb, b.cursor, b.kA, b.pA, ctl);
  bsort_local_kernel<<<nb, LOC_THREADS, sizeof(LocSmem), st>>>(b.kA, b.pA, b.kB, b.pB, b.bcount, b.bstart, bb, ctl);
  *launches += 4;
}

}  // namespace eirene
