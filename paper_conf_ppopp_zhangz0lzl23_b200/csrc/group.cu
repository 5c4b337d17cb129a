// group.cu -- per-bucket end of the request sort (Alg.1:10) fused with
// combining (Alg.1:11) and partition (Alg.1:3), sm_100a.
//
// The bucket sort (bsort.cu) leaves every request in the bucket of its top key
// bits.  Buckets are key ranges, so no key segment ever crosses a bucket: once
// a CTA has sorted its bucket in shared memory it can combine it completely.
// The only cross-bucket information is two counts -- the key segments (issued
// requests) and the issued writes of all earlier buckets -- which a decoupled
// look-back over the buckets provides.  One kernel therefore replaces the
// sort's last pass, the combine pass and the partition pass, and the sorted
// keys never go back to memory (only the sorted payloads do: RESULT_CAL needs
// the request order of each segment).
//
// Definitions, for bucket position x (the bucket sorted by (key, payload) =
// (key, timestamp), payload = ts<<2|op):
//   head(x) = x == 0 or key[x] != key[x-1]          (a new key segment)
//   tail(x) = x == cnt-1 or key[x+1] != key[x]
//   seg(x)  = SEG0 + #heads in [0, x] - 1           (issued-request index)
//   lw(x)   = last write position <= x               (same segment iff same key)
// Early result (nearest write P:834-835): a non-head request whose
// nearest earlier write is in its segment returns that write's value (null for
// a delete) now.  Issue rule (§8(c) 5-6): at the tail, the segment's
// last write if it has one, else its last query.  Partition (Alg.1:3): write
// segments go to the write list at index W0 + #write segments before, query
// segments to the query list at seg - that index.
//
// Layout: one CTA (16 warps) per bucket, taken in ticket order; a "round" of
// up to G_CAP positions is split into 16 contiguous warp chunks walked 32
// positions per step (lane = position), with ballots for the in-step scans,
// register carries across steps and a 16-entry shared scan across warps.  A
// bucket larger than G_CAP (skewed keys) is sorted in L2 and walked in several
// rounds with a carry; a round-walk is repeated after the look-back to emit.
#include "eirene_internal.cuh"
#include <cstdio>
#include <cstdlib>


namespace eirene {

namespace {

#define GROUP_PRAGMA(x) _Pragma(#x)
#define GROUP_UNROLL_(n) GROUP_PRAGMA(unroll n)

constexpr int G_THREADS = 512;
constexpr int G_WARPS = G_THREADS / 32;
constexpr int G_ITEMS = 8;
constexpr int G_CAP = G_THREADS * G_ITEMS;    // 4096 positions sorted in smem
constexpr int SB_BITS = 12;                   // sub-bucket bits inside a bucket
constexpr int SB_N = 1 << SB_BITS;

constexpr unsigned long long F_AGG = 1ull << 62;
constexpr unsigned long long F_INC = 2ull << 62;
constexpr unsigned long long F_VAL = (1ull << 62) - 1;

struct GSmem {
  uint64_t k[G_CAP];
  uint32_t p[G_CAP];
  uint32_t sb[SB_N + 1];       // sub-bucket starts; per-warp digit counters of the L2 passes
  uint32_t whist[G_CAP / 32];  // list of the sub-buckets larger than FAST_SB
  uint32_t wsum[G_WARPS];
  unsigned long long wmin[G_WARPS], wmax[G_WARPS];
  uint32_t wcmax[G_WARPS];
  uint64_t kmin, kmax;
  uint32_t cmax;
  uint32_t dhist[256];         // digit counts / running offsets of the L2 passes
  // per-warp aggregates and exclusive carries of the current round
  uint32_t w_nh[G_WARPS], w_lw[G_WARPS], w_nw[G_WARPS];
  uint32_t c_nh[G_WARPS], c_lw[G_WARPS], c_nw[G_WARPS];
  uint32_t r_nh, r_lw, r_nw;   // round carry-out
  uint32_t seg0, w0, ticket;
  uint32_t h_cnt[G_WARPS], h_lw[G_WARPS], h_lp[G_WARPS];   // hot_pass1 per-warp results
  uint64_t hk;                 // split-off hot key of an oversized group
  unsigned long long prof_t[2];  // EIRENE_GROUP_PROF timestamps (diagnostic)
  unsigned long long prof_l[4];  // ... inside l2_sort: range pass, split pass, rest sorted
  uint32_t* hot_bits;          // its timestamp bitmap slot (null: none free)
  // hot_run_sort: timestamp-bucket counters, provisional payloads, the run's other keys
  uint32_t tcnt[SB_N + 1];
  uint32_t tpay[G_CAP];
  uint64_t ck[32];
  uint32_t cp[32];
  uint32_t hr_lt, hr_eq, hr_nc, hr_cm;
  uint32_t hot_lastw, hot_lastp, hot_slot;   // split-off hot key: last write / last payload, bitmap slot
};

__device__ __forceinline__ bool kp_less(uint64_t ka, uint32_t pa, uint64_t kb, uint32_t pb) {
  return ka < kb || (ka == kb && pa < pb);
}
__device__ __forceinline__ uint32_t lanemask_le() { return lanemask_lt() | (1u << lane_id()); }

// Block-wide min / max of the group's keys -> S.kmin, S.kmax.
__device__ void key_range(uint64_t mn, uint64_t mx, GSmem& S) {
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) {
    mn = min(mn, (uint64_t)__shfl_xor_sync(FULL, mn, o));
    mx = max(mx, (uint64_t)__shfl_xor_sync(FULL, mx, o));
  }
  if (lane == 0) {
    S.wmin[warp] = mn;
    S.wmax[warp] = mx;
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    uint64_t a = S.wmin[0], z = S.wmax[0];
    for (int w = 1; w < G_WARPS; ++w) {
      a = min(a, (uint64_t)S.wmin[w]);
      z = max(z, (uint64_t)S.wmax[w]);
    }
    S.kmin = a;
    S.kmax = z;
  }
  __syncthreads();
}

// Bitonic sort of S.k / S.p [lo, lo + m) by (key, payload), in place, by the
// threads [t0, t0 + nt) of a warp (nt = 32, warp sync) or of the CTA (nt =
// G_THREADS, block sync).  The network is the "flip" variant whose merges all
// run ascending, so positions >= m act as +infinity and are simply skipped.
template <bool CTA>
__device__ void bitonic_run(uint32_t lo, uint32_t m, int t, int nt, GSmem& S) {
  uint32_t N = 2;
  while (N < m) N <<= 1;
  for (uint32_t k = 2; k <= N; k <<= 1) {
    for (uint32_t sdist = k >> 1; sdist > 0; sdist >>= 1) {
      const bool flip = sdist == (k >> 1);
      for (uint32_t q = t; q < N / 2; q += nt) {
        // q-th pair of this step: i has bit log2(sdist) clear
        const uint32_t i = ((q & ~(sdist - 1)) << 1) | (q & (sdist - 1));
        const uint32_t j = flip ? (i ^ (k - 1)) : (i | sdist);
        if (j < m) {
          const uint64_t ki = S.k[lo + i], kj = S.k[lo + j];
          const uint32_t pi = S.p[lo + i], pj = S.p[lo + j];
          if (kp_less(kj, pj, ki, pi)) {
            S.k[lo + i] = kj;
            S.k[lo + j] = ki;
            S.p[lo + i] = pj;
            S.p[lo + j] = pi;
          }
        }
      }
      if (CTA)
        __syncthreads();
      else
        __syncwarp();
    }
  }
}

// Sort a group of 2 <= cnt <= G_CAP requests (in no particular order) into
// S.k / S.p by (key, payload).  Items live in registers in warp-contiguous
// order (position = warp * C + 32 j + lane).  Sub-bucket index =
// (key - kmin) >> shift, SB_BITS wide, so sub-buckets adapt to the group's key
// range.  Requests are scattered to their sub-bucket by smem-atomic rank;
// a request of a sub-bucket of <= FAST_SB requests then moves to sub-bucket
// start + number of smaller (key, payload) in it (uniform keys: all of them).
// Larger sub-buckets (hot keys: a key's requests always share one) are
// sorted by a bitonic network, one warp per sub-bucket up to WARP_SB
// requests, the whole CTA above, so no distribution costs O(m^2).
#ifndef GROUP_FAST_SB
#define GROUP_FAST_SB 32   // A/B builds: -DGROUP_FAST_SB=n
#endif
constexpr uint32_t FAST_SB = GROUP_FAST_SB;
#ifndef GROUP_WARP_SB
#define GROUP_WARP_SB 256   // A/B builds: -DGROUP_WARP_SB=n; cfg3 1024 -> 256: 3.43 -> 3.64 Greq/s
#endif
constexpr uint32_t WARP_SB = GROUP_WARP_SB;
// Exclusive scan of a[0..SB_N) in place (SB_N / G_THREADS per thread), a[SB_N] = total.
__device__ void block_scan_sbn(uint32_t* a, GSmem& S) {
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  constexpr int PER = SB_N / G_THREADS;
  uint32_t loc[PER], sum = 0;
#pragma unroll
  for (int j = 0; j < PER; ++j) {
    loc[j] = a[tid * PER + j];
    sum += loc[j];
  }
  uint32_t x = sum;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const uint32_t y = __shfl_up_sync(FULL, x, o);
    if (lane >= o) x += y;
  }
  if (lane == 31) S.wsum[warp] = x;
  __syncthreads();
  uint32_t run = x - sum;
  for (int w = 0; w < warp; ++w) run += S.wsum[w];
#pragma unroll
  for (int j = 0; j < PER; ++j) {
    a[tid * PER + j] = run;
    run += loc[j];
  }
  if (tid == G_THREADS - 1) a[SB_N] = run;
  __syncthreads();
}

// A big sub-bucket S.k/S.p[lo, lo + m) (m <= G_CAP) dominated by one key hk
// (a hot key: Zipf).  hk's requests -- equal keys -- only need timestamp
// order: a counting sort on the top SB_BITS bits of the timestamp, then a rank
// fix inside each timestamp bucket; the few other requests of the sub-bucket
// (<= 32) are ranked against each other directly.  About ten CTA barriers
// instead of a bitonic network's log2(m)(log2(m)+1)/2 (78 at m = 4096).
// Returns false, having changed nothing, if the sub-bucket holds more than 32
// other requests or a timestamp bucket more than FAST_SB (the caller then
// sorts it with the bitonic network).  CTA-uniform.
constexpr uint32_t FAST_SB_ = 32;
__device__ __noinline__ bool hot_run_sort(uint32_t lo, uint32_t m, int tsbits, GSmem& S) {
  const int tid = threadIdx.x, lane = tid & 31;
  const uint64_t hk = S.k[lo + m / 2];   // a member: the dominant key with high probability
  uint64_t kr[G_ITEMS];
  uint32_t pr[G_ITEMS], r[G_ITEMS];
  uint32_t lt = 0, eq = 0;
#pragma unroll
  for (int j = 0; j < G_ITEMS; ++j) {
    const uint32_t i = tid + j * G_THREADS;
    const bool v = i < m;
    kr[j] = v ? S.k[lo + i] : hk;
    pr[j] = v ? S.p[lo + i] : 0u;
    lt += (v && kr[j] < hk) ? 1u : 0u;
    eq += (v && kr[j] == hk) ? 1u : 0u;
  }
  if (tid == 0) {
    S.hr_lt = 0;
    S.hr_eq = 0;
    S.hr_nc = 0;
    S.hr_cm = 0;
  }
  for (int i = tid; i <= SB_N; i += G_THREADS) S.tcnt[i] = 0;
  __syncthreads();
  lt = __reduce_add_sync(FULL, lt);
  eq = __reduce_add_sync(FULL, eq);
  if (lane == 0) {
    if (lt) atomicAdd(&S.hr_lt, lt);
    if (eq) atomicAdd(&S.hr_eq, eq);
  }
  const int tsh = tsbits > SB_BITS ? tsbits - SB_BITS : 0;
  uint32_t cm = 0;
#pragma unroll
  for (int j = 0; j < G_ITEMS; ++j) {
    const uint32_t i = tid + j * G_THREADS;
    r[j] = 0;
    if (i < m) {
      if (kr[j] == hk) {
        r[j] = atomicAdd(&S.tcnt[(pr[j] >> 2) >> tsh], 1u);
        cm = max(cm, r[j] + 1);
      } else {
        const uint32_t c = atomicAdd(&S.hr_nc, 1u);
        if (c < 32) {
          S.ck[c] = kr[j];
          S.cp[c] = pr[j];
        }
      }
    }
  }
  cm = __reduce_max_sync(FULL, cm);
  if (lane == 0 && cm) atomicMax(&S.hr_cm, cm);
  __syncthreads();
  const uint32_t nlt = S.hr_lt, neq = S.hr_eq, nc = S.hr_nc;
  if (nc > 32 || S.hr_cm > FAST_SB_) {
    __syncthreads();   // (everyone read the verdict before the caller reuses S)
    return false;
  }
  block_scan_sbn(S.tcnt, S);   // timestamp bucket starts among hk's requests
#pragma unroll
  for (int j = 0; j < G_ITEMS; ++j)
    if (tid + j * G_THREADS < m && kr[j] == hk) S.tpay[S.tcnt[(pr[j] >> 2) >> tsh] + r[j]] = pr[j];
  __syncthreads();
  uint32_t pos[G_ITEMS];
#pragma unroll
  for (int j = 0; j < G_ITEMS; ++j) {
    const uint32_t i = tid + j * G_THREADS;
    pos[j] = 0xFFFFFFFFu;
    if (i >= m) continue;
    if (kr[j] == hk) {
      const uint32_t b = (pr[j] >> 2) >> tsh, s0 = S.tcnt[b], s1 = S.tcnt[b + 1];
      uint32_t less = 0;
      for (uint32_t x = s0; x < s1; ++x) less += S.tpay[x] < pr[j];
      pos[j] = lo + nlt + s0 + less;
    } else {
      const bool low = kr[j] < hk;
      uint32_t less = 0;
      for (uint32_t x = 0; x < nc; ++x)
        less += ((S.ck[x] < hk) == low && kp_less(S.ck[x], S.cp[x], kr[j], pr[j])) ? 1u : 0u;
      pos[j] = (low ? lo : lo + nlt + neq) + less;
    }
  }
  __syncthreads();   // every read of the run done before it is rewritten
#pragma unroll
  for (int j = 0; j < G_ITEMS; ++j)
    if (pos[j] != 0xFFFFFFFFu) {
      S.k[pos[j]] = kr[j];
      S.p[pos[j]] = pr[j];
    }
  __syncthreads();
  return true;
}

#ifdef EIRENE_RANK_UNROLL   // A/B: the in-sub-bucket rank loop of smem_sort unrolled (loads in flight together)
#define RANK_UNROLL GROUP_UNROLL_(EIRENE_RANK_UNROLL)
#else
#define RANK_UNROLL
#endif
// (A, b: the phase stamps of diagnostic builds, -DEIRENE_PHASE_PROF; null elsewhere)
__device__ void smem_sort(const uint64_t* ks, const uint32_t* ps, uint32_t cnt, int tsbits, GSmem& S,
                          const BatchArgs* A = nullptr, uint32_t b = 0) {
#ifdef EIRENE_PHASE_PROF
#define SS_PHASE(i) \
  if (A) EIRENE_PHASE(A, 1, b, i)
#else
#define SS_PHASE(i) (void)A, (void)b
#endif
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const uint32_t C = 32u * ((cnt + G_THREADS - 1) / G_THREADS);
  const uint32_t wb = warp * C;
  uint64_t kr[G_ITEMS];
  uint32_t pr[G_ITEMS], r[G_ITEMS];
  uint64_t mn = KEY_MAX, mx = 0;
#pragma unroll
  for (int j = 0; j < G_ITEMS; ++j) {
    const uint32_t i = wb + 32 * j + lane;
    const bool v = 32u * j < C && i < cnt;
    kr[j] = v ? ks[i] : 0;
    pr[j] = v ? ps[i] : 0;
    if (v) {
      mn = min(mn, kr[j]);
      mx = max(mx, kr[j]);
    }
  }
  for (int i = tid; i <= SB_N; i += G_THREADS) S.sb[i] = 0;
  key_range(mn, mx, S);   // (its barriers also order the sb zeroing)
  SS_PHASE(5);
  const uint64_t kmin = S.kmin, range = S.kmax - S.kmin;
  const int bits = 64 - __clzll((long long)range);
  const int shift = bits > SB_BITS ? bits - SB_BITS : 0;
  uint32_t cm = 0;
#pragma unroll
  for (int j = 0; j < G_ITEMS; ++j) {
    const uint32_t i = wb + 32 * j + lane;
    r[j] = 0;
    if (32u * j < C && i < cnt) {
      r[j] = atomicAdd(&S.sb[(uint32_t)((kr[j] - kmin) >> shift)], 1u);
      cm = max(cm, r[j] + 1);
    }
  }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) cm = max(cm, __shfl_xor_sync(FULL, cm, o));
  if (lane == 0) S.wcmax[warp] = cm;
  __syncthreads();
  if (tid == 0) {
    uint32_t c = 0;
    for (int w = 0; w < G_WARPS; ++w) c = max(c, S.wcmax[w]);
    S.cmax = c;
  }
  {   // exclusive scan of S.sb[0..SB_N) (8 per thread)
    constexpr int PER = SB_N / G_THREADS;
    uint32_t loc[PER], sum = 0;
#pragma unroll
    for (int j = 0; j < PER; ++j) {
      loc[j] = S.sb[tid * PER + j];
      sum += loc[j];
    }
    uint32_t x = sum;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const uint32_t y = __shfl_up_sync(FULL, x, o);
      if (lane >= o) x += y;
    }
    if (lane == 31) S.wsum[warp] = x;
    __syncthreads();
    uint32_t run = x - sum;
    for (int w = 0; w < warp; ++w) run += S.wsum[w];
#pragma unroll
    for (int j = 0; j < PER; ++j) {
      S.sb[tid * PER + j] = run;
      run += loc[j];
    }
    if (tid == 0) S.sb[SB_N] = cnt;
  }
  __syncthreads();
  SS_PHASE(6);
#pragma unroll
  for (int j = 0; j < G_ITEMS; ++j) {
    const uint32_t i = wb + 32 * j + lane;
    if (32u * j < C && i < cnt) {
      const uint32_t pos = S.sb[(uint32_t)((kr[j] - kmin) >> shift)] + r[j];
      S.k[pos] = kr[j];
      S.p[pos] = pr[j];
    }
  }
  __syncthreads();
#pragma unroll
  for (int j = 0; j < G_ITEMS; ++j) {
    const uint32_t i = wb + 32 * j + lane;
    r[j] = 0xFFFFFFFFu;
    if (32u * j < C && i < cnt) {
      const uint32_t x = (uint32_t)((kr[j] - kmin) >> shift);
      const uint32_t lo = S.sb[x], hi = S.sb[x + 1];
      if (hi - lo <= FAST_SB) {
        uint32_t less = 0;
        RANK_UNROLL
        for (uint32_t m = lo; m < hi; ++m) less += kp_less(S.k[m], S.p[m], kr[j], pr[j]);
        r[j] = lo + less;
      }
    }
  }
  __syncthreads();
#pragma unroll
  for (int j = 0; j < G_ITEMS; ++j) {
    if (r[j] != 0xFFFFFFFFu) {
      S.k[r[j]] = kr[j];
      S.p[r[j]] = pr[j];
    }
  }
  __syncthreads();
  SS_PHASE(7);
#undef SS_PHASE
  if (S.cmax <= FAST_SB) return;
  // big sub-buckets: list them, then bitonic-sort each in place
  if (tid == 0) S.r_nh = 0;
  __syncthreads();
  for (uint32_t x = tid; x < (uint32_t)SB_N; x += G_THREADS) {
    const uint32_t m = S.sb[x + 1] - S.sb[x];
    if (m > FAST_SB) S.whist[atomicAdd(&S.r_nh, 1u)] = x;   // <= G_CAP / FAST_SB entries
  }
  __syncthreads();
  const uint32_t nbig = S.r_nh;
  for (uint32_t e = warp; e < nbig; e += G_WARPS) {
    const uint32_t x = S.whist[e], lo = S.sb[x], m = S.sb[x + 1] - lo;
    if (m <= WARP_SB) bitonic_run<false>(lo, m, lane, 32, S);
  }
  __syncthreads();
  for (uint32_t e = 0; e < nbig; ++e) {
    const uint32_t x = S.whist[e], lo = S.sb[x], m = S.sb[x + 1] - lo;
    if (m > WARP_SB && !hot_run_sort(lo, m, tsbits, S)) bitonic_run<true>(lo, m, tid, G_THREADS, S);
  }
  __syncthreads();
}

// One stable LSD pass in L2 over [0, cnt) of (ks, ps) -> (kd, pd) by an 8-bit
// digit -- of the timestamp (ts) or of key - kmin: digit counts, then tiles of
// G_THREADS * 8 requests ranked by match_any and per-warp counters
// (S.sb as [digit][warp]) with running per-digit offsets in S.dhist.
__device__ __forceinline__ uint32_t l2_digit(uint64_t k, uint32_t p, bool ts, uint64_t kmin, int sh) {
  return (ts ? (uint32_t)((p >> 2) >> sh) : (uint32_t)((k - kmin) >> sh)) & 255u;
}
__device__ void l2_pass(const uint64_t* ks, const uint32_t* ps, uint64_t* kd, uint32_t* pd, uint32_t cnt, bool ts,
                        uint64_t kmin, int sh, GSmem& S) {
  constexpr int IT = 8;
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  if (tid < 256) S.dhist[tid] = 0;
  __syncthreads();
  for (uint32_t i0 = tid; i0 < cnt; i0 += 8 * G_THREADS) {   // 8 loads in flight per thread
    uint32_t d[8];
#pragma unroll
    for (int u = 0; u < 8; ++u) {
      const uint32_t i = i0 + u * G_THREADS;
      d[u] = i < cnt ? l2_digit(ks[i], ps[i], ts, kmin, sh) : 256u;
    }
#pragma unroll
    for (int u = 0; u < 8; ++u)
      if (d[u] < 256u) atomicAdd(&S.dhist[d[u]], 1u);
  }
  __syncthreads();
  if (tid == 0) {
    uint32_t run = 0;
    for (int d = 0; d < 256; ++d) {
      const uint32_t c = S.dhist[d];
      S.dhist[d] = run;
      run += c;
    }
  }
  __syncthreads();
  uint32_t* wh = S.sb;   // [256][G_WARPS]
  for (uint32_t t0 = 0; t0 < cnt; t0 += G_THREADS * IT) {
    for (int i = tid; i < 256 * G_WARPS; i += G_THREADS) wh[i] = 0;
    __syncthreads();
    uint64_t k[IT];
    uint32_t p[IT], d[IT], r[IT];
    const uint32_t wb = t0 + warp * 32 * IT;
#pragma unroll
    for (int j = 0; j < IT; ++j) {
      const uint32_t i = wb + 32 * j + lane;
      const bool v = i < cnt;
      k[j] = v ? ks[i] : 0;
      p[j] = v ? ps[i] : 0;
      d[j] = v ? l2_digit(k[j], p[j], ts, kmin, sh) : 256u;
    }
#pragma unroll
    for (int j = 0; j < IT; ++j) {
      const bool v = d[j] < 256u;
      const uint32_t peers = __match_any_sync(FULL, d[j]);
      const uint32_t base = v ? wh[d[j] * G_WARPS + warp] : 0u;
      r[j] = base + __popc(peers & lanemask_lt());
      __syncwarp();
      if (v && lane == 31 - __clz(peers)) wh[d[j] * G_WARPS + warp] = base + __popc(peers);
      __syncwarp();
    }
    __syncthreads();
    if (tid < 256) {   // per digit: exclusive over warps, tile total
      uint32_t c = 0;
#pragma unroll
      for (int w = 0; w < G_WARPS; ++w) {
        const uint32_t x = wh[tid * G_WARPS + w];
        wh[tid * G_WARPS + w] = c + S.dhist[tid];
        c += x;
      }
      S.dhist[tid] += c;
    }
    __syncthreads();
#pragma unroll
    for (int j = 0; j < IT; ++j) {
      if (d[j] < 256u) {
        const uint32_t pos = wh[d[j] * G_WARPS + warp] + r[j];
        kd[pos] = k[j];
        pd[pos] = p[j];
      }
    }
    __syncthreads();
  }
}

// One stable LSD pass in L2 over a payload-only array (one key's requests):
// digit = 8 bits of the timestamp at sh.
__device__ void l2_pass_pay(const uint32_t* ps, uint32_t* pd, uint32_t cnt, int sh, GSmem& S) {
  constexpr int IT = 8;
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  if (tid < 256) S.dhist[tid] = 0;
  __syncthreads();
  for (uint32_t i0 = tid; i0 < cnt; i0 += 8 * G_THREADS) {   // 8 loads in flight per thread
    uint32_t d[8];
#pragma unroll
    for (int u = 0; u < 8; ++u) {
      const uint32_t i = i0 + u * G_THREADS;
      d[u] = i < cnt ? ((ps[i] >> 2) >> sh) & 255u : 256u;
    }
#pragma unroll
    for (int u = 0; u < 8; ++u)
      if (d[u] < 256u) atomicAdd(&S.dhist[d[u]], 1u);
  }
  __syncthreads();
  if (tid == 0) {
    uint32_t run = 0;
    for (int d = 0; d < 256; ++d) {
      const uint32_t c = S.dhist[d];
      S.dhist[d] = run;
      run += c;
    }
  }
  __syncthreads();
  uint32_t* wh = S.sb;   // [256][G_WARPS]
  for (uint32_t t0 = 0; t0 < cnt; t0 += G_THREADS * IT) {
    for (int i = tid; i < 256 * G_WARPS; i += G_THREADS) wh[i] = 0;
    __syncthreads();
    uint32_t p[IT], d[IT], r[IT];
    const uint32_t wb = t0 + warp * 32 * IT;
#pragma unroll
    for (int j = 0; j < IT; ++j) {
      const uint32_t i = wb + 32 * j + lane;
      p[j] = i < cnt ? ps[i] : 0u;
      d[j] = i < cnt ? ((p[j] >> 2) >> sh) & 255u : 256u;
    }
#pragma unroll
    for (int j = 0; j < IT; ++j) {
      const bool v = d[j] < 256u;
      const uint32_t peers = __match_any_sync(FULL, d[j]);
      const uint32_t base = v ? wh[d[j] * G_WARPS + warp] : 0u;
      r[j] = base + __popc(peers & lanemask_lt());
      __syncwarp();
      if (v && lane == 31 - __clz(peers)) wh[d[j] * G_WARPS + warp] = base + __popc(peers);
      __syncwarp();
    }
    __syncthreads();
    if (tid < 256) {
      uint32_t c = 0;
#pragma unroll
      for (int w = 0; w < G_WARPS; ++w) {
        const uint32_t x = wh[tid * G_WARPS + w];
        wh[tid * G_WARPS + w] = c + S.dhist[tid];
        c += x;
      }
      S.dhist[tid] += c;
    }
    __syncthreads();
#pragma unroll
    for (int j = 0; j < IT; ++j)
      if (d[j] < 256u) pd[wh[d[j] * G_WARPS + warp] + r[j]] = p[j];
    __syncthreads();
  }
}

// Oversized group (cnt > G_CAP): hot keys.  One pass finds the key range and
// counts three sampled candidates; the most frequent one, hk, is split off
// when the rest fits in shared memory: the rest is sorted there (smem_sort),
// hk's payloads are sorted by timestamp with payload-only LSD passes in L2,
// and the group is laid out as [rest < hk][hk in timestamp order][rest > hk]
// in (kd, pd).  Otherwise: stable LSD on the timestamp bits, then on the bits
// of key - kmin, ping-pong between the group's two L2 ranges.  Returns the
// range that holds the result (0: ks/ps, 1: kd/pd).
// An oversized group with no dominant key (cnt > G_CAP, its largest key run
// leaves more than G_CAP others): cut its key range [kmin, kmax] into parts of
// <= G_CAP requests with a histogram of (k - kmin) >> shift over SB_N bins --
// part(bin) = floor(prefix(bin) / T), T = G_CAP - largest bin, so a part never
// exceeds T + largest bin -- scatter the requests into their parts (key
// ranges, ascending) in kd / pd, then sort every part in shared memory and
// write it back in place: three passes over the group instead of up to 11
// LSD passes.  Returns false (nothing written) if it would take more than
// PART_MAX parts (a bin of nearly G_CAP requests).
constexpr uint32_t PART_MAX = 64;
__device__ bool range_partition_sort(const uint64_t* ks, const uint32_t* ps, uint64_t* kd, uint32_t* pd,
                                     uint32_t cnt, uint64_t kmin, uint64_t range, int tsbits, GSmem& S) {
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const int bits = 64 - __clzll((long long)range);
  const int shift = bits > SB_BITS ? bits - SB_BITS : 0;
  for (int i = tid; i <= SB_N; i += G_THREADS) S.sb[i] = 0;
  __syncthreads();
  for (uint32_t i0 = tid; i0 < cnt; i0 += 8 * G_THREADS) {   // 8 loads in flight per thread
    uint64_t kk[8];
#pragma unroll
    for (int u = 0; u < 8; ++u) {
      const uint32_t i = i0 + u * G_THREADS;
      kk[u] = i < cnt ? ks[i] : kmin;
    }
#pragma unroll
    for (int u = 0; u < 8; ++u)
      if (i0 + u * G_THREADS < cnt) atomicAdd(&S.sb[(uint32_t)((kk[u] - kmin) >> shift)], 1u);
  }
  __syncthreads();
  // exclusive prefix of the bins (8 per thread) and the largest bin
  constexpr int PER = SB_N / G_THREADS;
  uint32_t loc[PER], sum = 0, mx = 0;
#pragma unroll
  for (int j = 0; j < PER; ++j) {
    loc[j] = S.sb[tid * PER + j];
    sum += loc[j];
    mx = max(mx, loc[j]);
  }
  uint32_t x = sum;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const uint32_t y = __shfl_up_sync(FULL, x, o);
    if (lane >= o) x += y;
  }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) mx = max(mx, __shfl_xor_sync(FULL, mx, o));
  if (lane == 31) S.wsum[warp] = x;
  if (lane == 0) S.wcmax[warp] = mx;
  __syncthreads();
  uint32_t run = x - sum, big = 0;
  for (int w = 0; w < G_WARPS; ++w) {
    if (w < warp) run += S.wsum[w];
    big = max(big, S.wcmax[w]);
  }
  const uint32_t T = big < (uint32_t)G_CAP ? (uint32_t)G_CAP - big : 0u;
  const uint32_t parts = T ? (cnt + T - 1) / T : 0xFFFFFFFFu;
  if (parts > PART_MAX) return false;   // (uniform: every thread computed the same)
  // part starts: the prefix of the first bin of each part
  if (tid <= (int)PART_MAX) S.dhist[tid] = cnt;   // empty parts start at the end
  __syncthreads();
#pragma unroll
  for (int j = 0; j < PER; ++j) {
    const uint32_t q = min(run / T, parts - 1);
    if (loc[j]) atomicMin(&S.dhist[q], run);   // part start = prefix of its first nonempty bin
    S.sb[tid * PER + j] = q;                              // bin -> part
    run += loc[j];
  }
  __syncthreads();
  if (tid == 0) {   // empty parts start where the next nonempty one does
    for (int q = (int)parts - 1; q >= 0; --q) S.dhist[q] = min(S.dhist[q], S.dhist[q + 1]);
    for (uint32_t q = 0; q < parts; ++q) S.whist[q] = S.dhist[q];   // fill cursors
  }
  __syncthreads();
  for (uint32_t i0 = tid; i0 < cnt; i0 += 4 * G_THREADS) {   // scatter into the parts (order inside a part: any)
    uint64_t kk[4];
    uint32_t pp[4];
#pragma unroll
    for (int u = 0; u < 4; ++u) {
      const uint32_t i = i0 + u * G_THREADS;
      kk[u] = i < cnt ? ks[i] : 0;
      pp[u] = i < cnt ? ps[i] : 0;
    }
#pragma unroll
    for (int u = 0; u < 4; ++u) {
      if (i0 + u * G_THREADS < cnt) {
        const uint32_t q = S.sb[(uint32_t)((kk[u] - kmin) >> shift)];
        const uint32_t pos = atomicAdd(&S.whist[q], 1u);
        kd[pos] = kk[u];
        pd[pos] = pp[u];
      }
    }
  }
  __threadfence_block();
  __syncthreads();
  for (uint32_t q = 0; q < parts; ++q) {
    const uint32_t b0 = S.dhist[q], m = S.dhist[q + 1] - b0;
    __syncthreads();   // (every thread read the part bounds before smem_sort reuses S)
    if (m < 2) continue;
    smem_sort(kd + b0, pd + b0, m, tsbits, S);
    for (uint32_t i = tid; i < m; i += G_THREADS) {
      kd[b0 + i] = S.k[i];
      pd[b0 + i] = S.p[i];
    }
    __syncthreads();
  }
  return true;
}

__device__ int l2_sort(uint64_t* ks, uint32_t* ps, uint64_t* kd, uint32_t* pd, uint32_t cnt, int tsbits, GSmem& S,
                       uint32_t* hot_base, uint32_t* hot_ctr, uint32_t nreq, uint32_t hot_words) {
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const uint64_t c0 = ks[0], c1 = ks[cnt / 3], c2 = ks[(2 * (uint64_t)cnt) / 3];
  uint64_t mn = KEY_MAX, mx = 0;
  uint32_t n0 = 0, n1 = 0, n2 = 0;
  for (uint32_t i0 = tid; i0 < cnt; i0 += 8 * G_THREADS) {   // 8 loads in flight per thread
    uint64_t kk[8];
#pragma unroll
    for (int u = 0; u < 8; ++u) {
      const uint32_t i = i0 + u * G_THREADS;
      kk[u] = i < cnt ? ks[i] : ks[0];
    }
#pragma unroll
    for (int u = 0; u < 8; ++u) {
      if (i0 + u * G_THREADS < cnt) {
        mn = min(mn, kk[u]);
        mx = max(mx, kk[u]);
        n0 += kk[u] == c0;
        n1 += kk[u] == c1;
        n2 += kk[u] == c2;
      }
    }
  }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) {
    n0 += __shfl_xor_sync(FULL, n0, o);
    n1 += __shfl_xor_sync(FULL, n1, o);
    n2 += __shfl_xor_sync(FULL, n2, o);
  }
  if (lane == 0) {
    S.w_nh[warp] = n0;
    S.w_lw[warp] = n1;
    S.w_nw[warp] = n2;
  }
  key_range(mn, mx, S);   // (its barriers publish the per-warp counts)
#ifdef EIRENE_GROUP_PROF_BUILD
  if (tid == 0) S.prof_l[0] = gtime_ns();
#endif
  n0 = n1 = n2 = 0;
  for (int w = 0; w < G_WARPS; ++w) {
    n0 += S.w_nh[w];
    n1 += S.w_lw[w];
    n2 += S.w_nw[w];
  }
  const uint64_t kmin = S.kmin, range = S.kmax - S.kmin;
  const uint64_t hk = (n0 >= n1 && n0 >= n2) ? c0 : (n1 >= n2 ? c1 : c2);
  const uint32_t hcnt = max(n0, max(n1, n2));
  if (cnt - hcnt <= (uint32_t)G_CAP) {
    // split: the rest into S.k / S.p, hk's payloads into kd (as u32 scratch).
    // A timestamp bitmap costs O(n / 32) words whatever hk's count; LSD passes
    // over hk's payloads cost O(hcnt): the bitmap (a slot of HOT_SLOTS) only
    // for keys holding more than n / 128 requests -- at most 128 of them
    if (tid == 0) {
      uint32_t* b = nullptr;
      S.hot_slot = 0xFFFFFFFFu;
      if (hot_base && hcnt > max((uint32_t)G_CAP, nreq >> 7)) {
        const uint32_t slot = atomicAdd(hot_ctr, 1u);
        if (slot < (uint32_t)HOT_SLOTS) {
          b = hot_base + (size_t)slot * 3 * hot_words;
          S.hot_slot = slot;
        }
      }
      S.hot_bits = b;
    }
    __syncthreads();
    uint32_t* bits = S.hot_bits;
    uint32_t* hs = reinterpret_cast<uint32_t*>(kd);
    if (tid == 0) {
      S.r_nh = 0;   // rest
      S.r_lw = 0;   // hk
      S.r_nw = 0;   // rest below hk
      S.hot_lastw = 0;   // hk's last write payload (0: none; a write's op bits are never 0)
      S.hot_lastp = 0;   // hk's last payload
    }
    __syncthreads();
    uint32_t my_lw = 0, my_lp = 0;
    for (uint32_t b0 = 0; b0 < cnt; b0 += 8 * G_THREADS) {   // 8 loads in flight per thread
      uint64_t kk[8];
      uint32_t pp[8];
#pragma unroll
      for (int u = 0; u < 8; ++u) {
        const uint32_t i = b0 + u * G_THREADS + tid;
        kk[u] = i < cnt ? ks[i] : 0;
        pp[u] = i < cnt ? ps[i] : 0;
      }
#pragma unroll
      for (int u = 0; u < 8; ++u) {
        const bool v = b0 + u * G_THREADS + tid < cnt;
        const uint64_t k = kk[u];
        const uint32_t p = pp[u];
        const bool hot = v && k == hk;
        const uint32_t mh = __ballot_sync(FULL, hot), mo = __ballot_sync(FULL, v && !hot);
        const uint32_t below = __popc(__ballot_sync(FULL, v && !hot && k < hk));
        uint32_t bh = 0, bo = 0;
        if (lane == 0) {
          if (mh) bh = atomicAdd(&S.r_lw, __popc(mh));
          if (mo) bo = atomicAdd(&S.r_nh, __popc(mo));
          if (below) atomicAdd(&S.r_nw, below);
        }
        bh = __shfl_sync(FULL, bh, 0);
        bo = __shfl_sync(FULL, bo, 0);
        if (hot) {
          my_lp = max(my_lp, p);
          if (p & 3) my_lw = max(my_lw, p);
          if (bits) {   // timestamp bitmaps: the set bits ARE the hot key's requests in timestamp order
            const uint32_t ts = p >> 2, wd = ts >> 5, bit = 1u << (ts & 31);
            atomicOr(bits + wd, bit);
            if (p & 1) atomicOr(bits + hot_words + wd, bit);
            if (p & 2) atomicOr(bits + 2 * hot_words + wd, bit);
          }
          else
            hs[bh + __popc(mh & lanemask_lt())] = p;
        }
        if (v && !hot) {
          const uint32_t x = bo + __popc(mo & lanemask_lt());
          S.k[x] = k;
          S.p[x] = p;
        }
      }
    }
    my_lw = __reduce_max_sync(FULL, my_lw);
    my_lp = __reduce_max_sync(FULL, my_lp);
    if (lane == 0) {
      if (my_lw) atomicMax(&S.hot_lastw, my_lw);
      if (my_lp) atomicMax(&S.hot_lastp, my_lp);
    }
    __syncthreads();
#ifdef EIRENE_GROUP_PROF_BUILD
    if (tid == 0) S.prof_l[1] = gtime_ns();
#endif
    const uint32_t o = S.r_nh, h = S.r_lw, lo = S.r_nw;
    if (o > 1) smem_sort(S.k, S.p, o, tsbits, S);
    __syncthreads();
#ifdef EIRENE_GROUP_PROF_BUILD
    if (tid == 0) S.prof_l[2] = gtime_ns();
#endif
    if (bits) {   // SPLIT: the rest stays sorted in S.k / S.p, hk in the bitmap
      if (tid == 0) {
        S.r_nh = o;
        S.r_lw = h;
        S.r_nw = lo;
        S.hk = hk;
      }
      __syncthreads();
      return 2;
    }
    // hk's payloads by timestamp: hs -> ps -> hs ... -> pd + lo (last pass)
    const int tpass = max(1, (tsbits + 7) / 8);
    for (int pass = 0; pass < tpass; ++pass) {
      const uint32_t* src = (pass & 1) ? ps : hs;
      uint32_t* dst = pass + 1 == tpass ? pd + lo : ((pass & 1) ? hs : ps);
      l2_pass_pay(src, dst, h, 8 * pass, S);
    }
    for (uint32_t x = tid; x < h; x += G_THREADS) kd[lo + x] = hk;
    for (uint32_t x = tid; x < o; x += G_THREADS) {
      const uint32_t d = x < lo ? x : x + h;
      kd[d] = S.k[x];
      pd[d] = S.p[x];
    }
    __syncthreads();
    return 1;
  }
  if (range && range_partition_sort(ks, ps, kd, pd, cnt, kmin, range, tsbits, S)) return 1;
  const int tpass = (tsbits + 7) / 8;
  const int passes = tpass + (range ? (64 - __clzll((long long)range) + 7) / 8 : 0);
  for (int pass = 0; pass < passes; ++pass) {
    const bool ts = pass < tpass;
    const int sh = 8 * (ts ? pass : pass - tpass);
    if (pass & 1)
      l2_pass(kd, pd, ks, ps, cnt, ts, kmin, sh, S);
    else
      l2_pass(ks, ps, kd, pd, cnt, ts, kmin, sh, S);
  }
  return passes & 1;
}

struct GroupArgs {
  const BatchArgs* A;
  uint64_t* kA;                 // bucketed requests (bsort scatter output)
  uint32_t* pA;
  uint64_t* kB;                 // L2 scratch for oversized buckets
  uint32_t* pB;                 // sorted payloads (output, read by RESULT_CAL)
  const uint32_t* gstart;       // [G + 1]
  uint32_t n, nb;               // requests, groups
  int tsbits;                   // bits of the largest timestamp (n - 1)
  uint32_t* pinfo;
  uint32_t* istart;
  uint64_t* qkey;
  uint32_t* qseg;
  uint64_t* wkey;
  uint8_t* wop;
  uint64_t* wval;
  uint32_t* wseg;
  unsigned long long* status;   // [nb] look-back words (zeroed per batch)
  uint32_t* hot_bits;           // [HOT_SLOTS][hot_words] timestamp bitmaps, zero between uses
  uint32_t hot_words;
  uint32_t* hot_seg;            // [HOT_SLOTS] segment of each deferred hot key (result phase)
  int prof;                     // EIRENE_GROUP_PROF: print the phases of slow groups (diagnostic)
  int phase;                    // 0: one kernel; 1: phase 1 of the two-phase group stage
  uint4* grec;                  // [nb] GroupRec (two-phase)
  Tree t;
  BatchCtl* ctl;
};

// The sorted group as seen by the combine passes: positions [c0, c1) from a
// shared-memory copy (the whole group when it fits, else the current round of
// an oversized group), the rest (a round's neighbours) from L2.
struct GView {
  const uint64_t* Kg;
  const uint32_t* Pg;
  const uint64_t* Ks;
  const uint32_t* Ps;
  uint32_t c0, c1;
  __device__ __forceinline__ uint64_t k(uint32_t x) const { return x - c0 < c1 - c0 ? Ks[x - c0] : Kg[x]; }
  __device__ __forceinline__ uint32_t p(uint32_t x) const { return x - c0 < c1 - c0 ? Ps[x - c0] : Pg[x]; }
};

// A/B switch: unrolling of the warps' 32-position steps (independent smem loads
// of several steps in flight); EIRENE_GROUP_UNROLL=n
#ifndef EIRENE_GROUP_UNROLL
#define EIRENE_GROUP_UNROLL 2   // (A/B r2s: 2 > 1, 4)
#endif
#if EIRENE_GROUP_UNROLL > 1
#define GROUP_UNROLL GROUP_UNROLL_(EIRENE_GROUP_UNROLL)
#else
#define GROUP_UNROLL
#endif

// Round [r0, r1) of a bucket walked by 16 warps: pass 1 (heads, last write per
// warp), warp scan, pass 2 (write segments ending in each warp), warp scan.
// Leaves the exclusive per-warp carries in S.c_* and the carry-out in S.r_*.
__device__ void round_scan(const GView& V, uint32_t cnt, uint32_t r0, uint32_t r1,
                           uint32_t cin_nh, uint32_t cin_lw, uint32_t cin_nw, GSmem& S) {
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const uint32_t len = r1 - r0;
  const uint32_t C = 32u * ((len + G_THREADS - 1) / G_THREADS);
  const uint32_t wb = r0 + warp * C;
  const uint32_t we = min(r1, wb + C);
  uint32_t nh = 0, lw = 0;
  GROUP_UNROLL
  for (uint32_t b = wb; b < we; b += 32) {
    const uint32_t x = b + lane;
    const bool valid = x < we;
    const uint64_t k = valid ? V.k(x) : 0;
    const bool head = valid && (x == 0 || V.k(x - 1) != k);
    const uint32_t W = __ballot_sync(FULL, valid && is_write(V.p(valid ? x : 0) & 3));
    nh += __popc(__ballot_sync(FULL, head));
    if (W) lw = b + (31 - __clz(W)) + 1;
  }
  if (lane == 0) {
    S.w_nh[warp] = nh;
    S.w_lw[warp] = lw;
  }
  __syncthreads();
  if (tid == 0) {
    uint32_t a = cin_nh, l = cin_lw;
    for (int w = 0; w < G_WARPS; ++w) {
      S.c_nh[w] = a;
      S.c_lw[w] = l;
      a += S.w_nh[w];
      l = max(l, S.w_lw[w]);
    }
    S.r_nh = a;
    S.r_lw = l;
  }
  __syncthreads();
  uint32_t lwc = S.c_lw[warp], nwt = 0;
  GROUP_UNROLL
  for (uint32_t b = wb; b < we; b += 32) {
    const uint32_t x = b + lane;
    const bool valid = x < we;
    const uint64_t k = valid ? V.k(x) : 0;
    const uint32_t W = __ballot_sync(FULL, valid && is_write(V.p(valid ? x : 0) & 3));
    const uint32_t wle = W & lanemask_le();
    const uint32_t lwi = wle ? b + (31 - __clz(wle)) + 1 : lwc;
    const bool tail = valid && (x + 1 == cnt || V.k(x + 1) != k);
    const bool hasw = tail && lwi && V.k(lwi - 1) == k;
    nwt += __popc(__ballot_sync(FULL, hasw));
    if (W) lwc = b + (31 - __clz(W)) + 1;
  }
  if (lane == 0) S.w_nw[warp] = nwt;
  __syncthreads();
  if (tid == 0) {
    uint32_t a = cin_nw;
    for (int w = 0; w < G_WARPS; ++w) {
      S.c_nw[w] = a;
      a += S.w_nw[w];
    }
    S.r_nw = a;
  }
  __syncthreads();
}

// Pass 3 of round [r0, r1): every output of the combine and the partition.
__device__ void round_emit(const GroupArgs& g, const GView& V, uint32_t cnt, uint32_t gbase,
                           uint32_t r0, uint32_t r1, bool write_spay, GSmem& S,
                           uint32_t split_lo = 0xFFFFFFFFu, uint32_t split_h = 0, uint32_t split_w = 0) {
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const tkey_t* __restrict__ vals = g.A->vals;
  tkey_t* __restrict__ results = g.A->results;
  const uint32_t len = r1 - r0;
  const uint32_t C = 32u * ((len + G_THREADS - 1) / G_THREADS);
  const uint32_t wb = r0 + warp * C;
  const uint32_t we = min(r1, wb + C);
  const uint32_t seg0 = S.seg0, w0 = S.w0;
  uint32_t nh = S.c_nh[warp], lwc = S.c_lw[warp], nwc = S.c_nw[warp];
  GROUP_UNROLL
  for (uint32_t b = wb; b < we; b += 32) {
    const uint32_t x = b + lane;
    const bool valid = x < we;
    const uint64_t k = valid ? V.k(x) : 0;
    const uint32_t p = valid ? V.p(x) : 0;
    const bool head = valid && (x == 0 || V.k(x - 1) != k);
    const uint32_t H = __ballot_sync(FULL, head);
    const uint32_t W = __ballot_sync(FULL, valid && is_write(p & 3));
    // SPLIT groups: positions >= split_lo come after the hot key's segment
    // (split_h positions, one segment, split_w issued writes)
    const bool after = x >= split_lo;
    const uint32_t seg = seg0 + nh + __popc(H & lanemask_le()) - 1u + (after ? 1u : 0u);
    const uint32_t gx = gbase + x + (after ? split_h : 0u);
    // nearest write strictly before x, and at or before x (bucket positions + 1)
    const uint32_t wl = W & lanemask_lt();
    const uint32_t lwb = wl ? b + (31 - __clz(wl)) + 1 : lwc;
    const uint32_t wle = W & lanemask_le();
    const uint32_t lwi = wle ? b + (31 - __clz(wle)) + 1 : lwc;
    const bool done = valid && !head && lwb && V.k(lwb - 1) == k;
    if (done) {
      const uint32_t pw = V.p(lwb - 1);
      results[p >> 2] = ((pw & 3) == OP_DELETE) ? KEY_MAX : vals[pw >> 2];
    }
    if (valid) {
      g.pinfo[gx] = seg | (done ? DONE_BIT : 0u);
      if (write_spay) g.pB[gx] = p;
    }
    if (head) g.istart[seg] = gx;
    const bool tail = valid && (x + 1 == cnt || V.k(x + 1) != k);
    const bool hasw = tail && lwi && V.k(lwi - 1) == k;
    const uint32_t WT = __ballot_sync(FULL, hasw);
    if (tail) {
      const uint32_t wi = w0 + nwc + __popc(WT & lanemask_lt()) + (after ? split_w : 0u);
      if (hasw) {   // issue rule: the segment's last write
        const uint32_t pw = V.p(lwi - 1);
        const uint32_t opw = pw & 3;
        g.wkey[wi] = k;
        g.wop[wi] = (uint8_t)opw;
        g.wval[wi] = pw >> 2;   // its timestamp: the query kernel's locate gathers the value (WVAL_TS)
        g.wseg[wi] = seg;
      } else {      // all-query segment: its last query
        const uint32_t qi = seg - wi;
        g.qkey[qi] = k;
        // a one-request segment (head and tail) carries its timestamp instead of
        // its segment index: the query kernel writes results[ts] directly, with
        // no istart / sorted-payload reads and no old[seg] (RESULT_CAL)
        g.qseg[qi] = head ? (Q_SINGLE | (p >> 2)) : seg;
      }
    }
    nh += __popc(H);
    nwc += __popc(WT);
    if (W) lwc = b + (31 - __clz(W)) + 1;
  }
}


// ---------------------------------------------------------------- hot key
// The split-off hot key hk of an oversized group is one key segment.  Its
// requests were recorded by l2_sort in the group's timestamp bitmap slot --
// three bitmaps over [0, n): present, op bit 0, op bit 1 -- so walking the
// bitmaps in ts order visits them in timestamp order: the (key, ts) sort of
// that segment for O(n / 32) word reads instead of radix passes over its
// requests, and the ops come with the bits (no gather of the batch's ops).
// Thread t owns the contiguous words [t*PW, (t+1)*PW) (PW a multiple of 4,
// read as uint4).
//   pass 1: per thread, requests and last write / last request payload;
//           CTA scan -> the thread's rank carry and nearest-write carry;
//   pass 2: sorted payload, pinfo (seg | DONE) and, in the group's unused
//           kB range, the payload of each position's nearest earlier write;
//           words are cleared as they are read;
//   results: the early results (nearest write P:834-835) of the
//           DONE positions, all positions in parallel.
struct HotCarry {
  uint32_t rank, lw;       // this thread's exclusive carries
  uint32_t total, last_w, last_p;
};
__device__ __forceinline__ uint32_t hot_pw(uint32_t W) { return 4u * ((W + 4u * G_THREADS - 1) / (4u * G_THREADS)); }

__device__ HotCarry hot_pass1(const GroupArgs& g, const uint32_t* bits, GSmem& S) {
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const uint32_t W = g.hot_words, PW = hot_pw(W);
  const uint32_t w0 = min(W, tid * PW), w1 = min(W, w0 + PW);
  uint32_t cnt = 0, lw = 0, lp = 0;   // payload 0 = none (a write has op != 0)
  for (uint32_t x = w0; x < w1; x += 4) {
    const uint4 P = __ldcg(reinterpret_cast<const uint4*>(bits + x));
    const uint4 B0 = __ldcg(reinterpret_cast<const uint4*>(bits + W + x));
    const uint4 B1 = __ldcg(reinterpret_cast<const uint4*>(bits + 2 * W + x));
    const uint32_t pw[4] = {P.x, P.y, P.z, P.w}, b0[4] = {B0.x, B0.y, B0.z, B0.w}, b1[4] = {B1.x, B1.y, B1.z, B1.w};
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      cnt += __popc(pw[j]);
      const uint32_t base = (x + j) * 32;
      if (pw[j]) {
        const uint32_t t = 31 - __clz(pw[j]);
        lp = ((base + t) << 2) | ((b0[j] >> t) & 1u) | (((b1[j] >> t) & 1u) << 1);
      }
      const uint32_t wm = b0[j] | b1[j];
      if (wm) {
        const uint32_t t = 31 - __clz(wm);
        lw = ((base + t) << 2) | ((b0[j] >> t) & 1u) | (((b1[j] >> t) & 1u) << 1);
      }
    }
  }
  // CTA scan: exclusive sum of cnt, exclusive max of lw (ascending chunks)
  uint32_t inc = cnt, mx = lw;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const uint32_t y = __shfl_up_sync(FULL, inc, o), z = __shfl_up_sync(FULL, mx, o);
    if (lane >= o) {
      inc += y;
      mx = max(mx, z);
    }
  }
  if (lane == 31) {
    S.h_cnt[warp] = inc;
    S.h_lw[warp] = mx;
  }
  uint32_t lpw = lp;
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) lpw = max(lpw, __shfl_xor_sync(FULL, lpw, o));
  if (lane == 0) S.h_lp[warp] = lpw;
  __syncthreads();
  HotCarry c;
  uint32_t rb = 0, mb = 0;
  c.total = 0;
  c.last_w = 0;
  c.last_p = 0;
  for (int w = 0; w < G_WARPS; ++w) {
    if (w < warp) {
      rb += S.h_cnt[w];
      mb = max(mb, S.h_lw[w]);
    }
    c.total += S.h_cnt[w];
    c.last_w = max(c.last_w, S.h_lw[w]);
    c.last_p = max(c.last_p, S.h_lp[w]);
  }
  const uint32_t ex_inc = __shfl_up_sync(FULL, inc, 1), ex_mx = __shfl_up_sync(FULL, mx, 1);
  c.rank = rb + (lane ? ex_inc : 0u);
  c.lw = max(mb, lane ? ex_mx : 0u);
  __syncthreads();
  return c;
}

// Pass 2 + results; sH = the hot segment's index, pos0 = its first sorted position.
// The early results of the DONE positions are written here only for a short
// segment; a long one's positions are marked DEFER and the result phase,
// which spreads long segments over many CTAs, writes them.
// Pass 2 walks the bitmaps warp-contiguously (warp w owns the words of
// threads [32w, 32w + 32) of pass 1, lanes read consecutive words), so the
// positions written by a warp step are contiguous and the stores coalesce;
// the lane carries come from a warp scan of the words' counts and last writes.
__device__ void hot_pass2(const GroupArgs& g, uint32_t* bits, const HotCarry& c, uint32_t sH, uint32_t pos0) {
  const int tid = threadIdx.x, lane = tid & 31;
  const uint32_t W = g.hot_words, PW = hot_pw(W);
  const uint32_t wbeg = min(W, (uint32_t)(tid & ~31) * PW), wend = min(W, wbeg + 32u * PW);
  // the warp's carries = those of its lane 0 in pass 1
  uint32_t rank = __shfl_sync(FULL, c.rank, 0), prev = __shfl_sync(FULL, c.lw, 0);
  // a long hot segment's early results are left to the result phase (many CTAs)
  const bool defer = c.total > SHORT_SEG;
  const uint32_t dbits = DONE_BIT | (defer ? DEFER_BIT : 0u);
  constexpr int D = 4;   // steps whose loads are issued together
  for (uint32_t xb = wbeg; xb < wend; xb += 32 * D) {
    uint32_t P[D], B0[D], B1[D];
#pragma unroll
    for (int k = 0; k < D; ++k) {
      const uint32_t x = xb + 32 * k + lane;
      const bool v = x < wend;
      P[k] = v ? __ldcg(bits + x) : 0u;
      B0[k] = v ? __ldcg(bits + W + x) : 0u;
      B1[k] = v ? __ldcg(bits + 2 * W + x) : 0u;
    }
#pragma unroll
    for (int k = 0; k < D; ++k) {
      const uint32_t x = xb + 32 * k + lane;
      const uint32_t word = P[k];
      if (!__any_sync(FULL, word)) continue;
      const uint32_t wm = word & (B0[k] | B1[k]);   // write requests of this word
      const uint32_t pc = __popc(word);
      uint32_t mylw = 0;
      if (wm) {
        const uint32_t t = 31 - __clz(wm);
        mylw = ((x * 32 + t) << 2) | ((B0[k] >> t) & 1u) | (((B1[k] >> t) & 1u) << 1);
      }
      uint32_t inc = pc, mx = mylw;
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        const uint32_t y = __shfl_up_sync(FULL, inc, o), z = __shfl_up_sync(FULL, mx, o);
        if (lane >= o) {
          inc += y;
          mx = max(mx, z);
        }
      }
      const uint32_t tot = __shfl_sync(FULL, inc, 31), mxall = __shfl_sync(FULL, mx, 31);
      const uint32_t ex_mx = __shfl_up_sync(FULL, mx, 1);
      uint32_t pv = max(prev, lane ? ex_mx : 0u);
      uint32_t pos = pos0 + rank + inc - pc;
      for (uint32_t m = word; m; m &= m - 1) {
        const uint32_t t = __ffs(m) - 1;
        const uint32_t op = ((B0[k] >> t) & 1u) | (((B1[k] >> t) & 1u) << 1);
        const uint32_t pay = ((x * 32 + t) << 2) | op;
        g.pB[pos] = pay;
        g.pinfo[pos] = sH | (pv ? dbits : 0u);
        g.kB[pos] = pv;   // nearest earlier write (0: none)
        ++pos;
        if (op) pv = pay;
      }
      if (word) {   // leave the slot clean for the next batch
        bits[x] = 0u;
        bits[W + x] = 0u;
        bits[2 * W + x] = 0u;
      }
      rank += tot;
      prev = max(prev, mxall);
    }
  }
  __syncthreads();
  const tkey_t* __restrict__ vals = g.A->vals;
  tkey_t* __restrict__ results = g.A->results;
  const uint32_t e = pos0 + c.total;
  for (uint32_t q0 = pos0 + tid; q0 < e && !defer; q0 += 8 * G_THREADS) {   // 8 in flight per thread
    uint32_t pw[8], py[8];
#pragma unroll
    for (int u = 0; u < 8; ++u) {
      const uint32_t q = q0 + u * G_THREADS;
      pw[u] = q < e ? (uint32_t)__ldcg(reinterpret_cast<const unsigned long long*>(g.kB + q)) : 0u;
      py[u] = q < e ? __ldcg(g.pB + q) : 0u;
    }
#pragma unroll
    for (int u = 0; u < 8; ++u)
      if (pw[u]) results[py[u] >> 2] = ((pw[u] & 3) == OP_DELETE) ? KEY_MAX : vals[pw[u] >> 2];
  }
}

// Per-group record from phase 1 to phase 2 of the two-phase group stage.
struct alignas(16) GroupRec {
  uint64_t hk;          // SPLIT: the hot key
  uint32_t where;       // 0: sorted in kA / pA, 1: in kB / pB, 2: SPLIT (the rest sorted in kB / pB [0, sp_o))
  uint32_t c_nh, c_nw;  // the group's key segments and issued writes (its look-back aggregate)
  uint32_t sp_o, sp_h, sp_lo, a_nh, a_nw, hot_w, hot_last, hot_slot;
};
static_assert(sizeof(GroupRec) == 4 * sizeof(uint4), "grec holds 4 uint4 per group");

// Round [r0, r1) of a group sorted in L2 (K, P), copied to shared memory.
__device__ GView load_round(const uint64_t* K, const uint32_t* P, uint32_t r0, uint32_t r1, GSmem& S) {
  const int tid = threadIdx.x;
  __syncthreads();
  for (uint32_t i0 = r0 + tid; i0 < r1; i0 += 8 * G_THREADS) {   // 8 loads in flight per thread
    uint64_t kk[8];
    uint32_t pp[8];
#pragma unroll
    for (int u = 0; u < 8; ++u) {
      const uint32_t i = i0 + u * G_THREADS;
      kk[u] = i < r1 ? K[i] : 0;
      pp[u] = i < r1 ? P[i] : 0;
    }
#pragma unroll
    for (int u = 0; u < 8; ++u) {
      const uint32_t i = i0 + u * G_THREADS;
      if (i < r1) {
        S.k[i - r0] = kk[u];
        S.p[i - r0] = pp[u];
      }
    }
  }
  __syncthreads();
  return GView{K, P, S.k, S.p, r0, r1};
}

// Decoupled look-back over the buckets (ticket order) on (heads << 31 | writes)
// -> S.seg0, S.w0 (the last bucket also writes the batch totals).
__device__ void group_lookback(const GroupArgs& g, uint32_t b, uint32_t c_nh, uint32_t c_nw, GSmem& S) {
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  BatchCtl* ctl = g.ctl;
  if (warp == 0) {
    const unsigned long long tot = ((unsigned long long)c_nh << 31) | c_nw;
    unsigned long long* my = g.status + b;
    unsigned long long excl = 0;
    if (b == 0) {
      if (lane == 0) st_relaxed64(my, F_INC | tot);
    } else {
      if (lane == 0) st_relaxed64(my, F_AGG | tot);
      SpinGuard sg;
      int32_t pt = (int32_t)b - 1;
      for (;;) {
        const int32_t idx = pt - lane;
        const unsigned long long w = idx >= 0 ? ld_relaxed64(g.status + idx) : F_INC;
        const uint32_t fl = (uint32_t)(w >> 62);
        const uint32_t inc = __ballot_sync(FULL, fl == 2);
        const uint32_t need = inc ? ((2u << (__ffs(inc) - 1)) - 1u) : FULL;
        if (__ballot_sync(FULL, fl == 0) & need) {
          // a predecessor has not published: back off (a waiting group's spin
          // would otherwise keep the L2 busy under the slow groups it waits for)
          __nanosleep(256);
          if (sg.stuck(ctl)) break;
          continue;
        }
        unsigned long long a = ((need >> lane) & 1u) ? (w & F_VAL) : 0ull;
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) a += __shfl_xor_sync(FULL, a, o);
        excl += a;
        if (inc) break;
        pt -= 32;
      }
      if (lane == 0) st_relaxed64(my, F_INC | (excl + tot));
    }
    if (lane == 0) {
      const uint32_t seg0 = (uint32_t)(excl >> 31), w0 = (uint32_t)(excl & ((1u << 31) - 1));
      S.seg0 = seg0;
      S.w0 = w0;
      if (b + 1 == g.nb) {   // last bucket: batch totals (the pool headroom is checked by the query kernel)
        const uint32_t nseg = seg0 + c_nh, nw = w0 + c_nw;
        ctl->nseg = nseg;
        ctl->nw = nw;
        ctl->nq = nseg - nw;
        g.istart[nseg] = g.gstart[g.nb];   // point requests (range queries are not sorted)
      }
    }
  }
  __syncthreads();
}

// Sweep 2 of a SPLIT group: the rest (sorted in S.k / S.p [0, sp_o)) around the
// hot key's segment (sp_h positions after the sp_lo smaller ones).
__device__ void emit_split(const GroupArgs& g, GSmem& S, uint32_t base, uint32_t sp_o, uint32_t sp_lo, uint32_t sp_h,
                           uint32_t hot_w, uint32_t hot_last, uint32_t a_nh, uint32_t a_nw, bool deferred,
                           const HotCarry& hc) {
  const int tid = threadIdx.x;
  const GView V{S.k, S.p, S.k, S.p, 0, sp_o};
  if (sp_o) {
    round_scan(V, sp_o, 0, sp_o, 0, 0, 0, S);
    round_emit(g, V, sp_o, base, 0, sp_o, true, S, sp_lo, sp_h, hot_w);
  }
  __syncthreads();
  const uint32_t sH = S.seg0 + a_nh, wH = S.w0 + a_nw, pos0 = base + sp_lo;
  if ((g.prof & 1) && tid == 0) S.prof_t[0] = gtime_ns();
  if (!deferred) hot_pass2(g, S.hot_bits, hc, sH, pos0);
  if ((g.prof & 1) && tid == 0) S.prof_t[1] = gtime_ns();
  if (tid == 0) {
    const uint64_t hk = S.hk;
    g.istart[sH] = pos0;
    // deferred: the segment's positions (pinfo, sorted payloads) are not
    // written; every result of it comes from the result phase's walk of the
    // bitmap slot, spread over many CTAs (result_phase, eirene_internal.cuh)
    if (deferred) g.hot_seg[S.hot_slot] = sH;
    if (hot_w) {   // issue rule: the segment's last write
      const uint32_t opw = hot_last & 3;
      g.wkey[wH] = hk;
      g.wop[wH] = (uint8_t)opw;
      g.wval[wH] = hot_last >> 2;   // (timestamp, as above)
      g.wseg[wH] = sH;
    } else {       // all-query segment: its last query
      g.qkey[sH - wH] = hk;
      g.qseg[sH - wH] = sH;
    }
  }
}

// Sweep 2 of a group sorted in L2 (K, P), walked in rounds of G_CAP positions.
__device__ void emit_rounds(const GroupArgs& g, GSmem& S, const uint64_t* K, const uint32_t* P, uint32_t cnt,
                            uint32_t base) {
  const bool write_spay = P != g.pB + base;
  uint32_t c_nh = 0, c_lw = 0, c_nw = 0;
  for (uint32_t r0 = 0; r0 < cnt; r0 += G_CAP) {
    const uint32_t r1 = min(cnt, r0 + (uint32_t)G_CAP);
    const GView V = load_round(K, P, r0, r1, S);
    round_scan(V, cnt, r0, r1, c_nh, c_lw, c_nw, S);
    round_emit(g, V, cnt, base, r0, r1, write_spay, S);
    c_nh = S.r_nh;
    c_lw = S.r_lw;
    c_nw = S.r_nw;
    __syncthreads();
  }
}

// Phase 2 of the two-phase group stage: look-back on the aggregates phase 1
// published, then the emit sweep over the group phase 1 left sorted in L2.
__device__ void group_phase2(const GroupArgs& g, GSmem& S, uint32_t b) {
  const int tid = threadIdx.x;
  const GroupRec r = reinterpret_cast<const GroupRec*>(g.grec)[b];
  const uint32_t base = g.gstart[b];
  const uint32_t cnt = g.gstart[b + 1] - base;
  if (r.where == 2) {
    for (uint32_t i = tid; i < r.sp_o; i += G_THREADS) {
      S.k[i] = __ldcg(g.kB + base + i);
      S.p[i] = __ldcg(g.pB + base + i);
    }
    if (tid == 0) {
      S.hk = r.hk;
      S.hot_slot = r.hot_slot;
    }
  }
  group_lookback(g, b, r.c_nh, r.c_nw, S);   // (ends with a barrier)
  if (r.where == 2)
    emit_split(g, S, base, r.sp_o, r.sp_lo, r.sp_h, r.hot_w, r.hot_last, r.a_nh, r.a_nw, true, HotCarry{});
  else
    emit_rounds(g, S, (r.where ? g.kB : g.kA) + base, (r.where ? g.pB : g.pA) + base, cnt, base);
}

// Phase 2 of the two-phase group stage (its own kernel: its register budget
// stays out of group_kernel's).
__global__ void __launch_bounds__(G_THREADS, 2) group_emit_kernel(GroupArgs g) {
  pdl_wait();
  pdl_trigger();
  extern __shared__ __align__(16) unsigned char smem_raw[];
  GSmem& S = *reinterpret_cast<GSmem*>(smem_raw);
  if (g.ctl->invalid) return;
  if (threadIdx.x == 0) S.ticket = atomicAdd(&g.ctl->tile_ctr[TC_GROUP2], 1u);
  __syncthreads();
  group_phase2(g, S, S.ticket);
}

// g.phase 0: the whole group stage in one kernel; 1: phase 1 of the two-phase
// stage of a multi-wave batch (phase 1 never waits for another group, so a
// slow group holds only its own SM slot; phase 2's look-back finds every
// aggregate published).
__global__ void __launch_bounds__(G_THREADS, 2) group_kernel(GroupArgs g) {
  pdl_wait();   // predecessor kernel complete, its writes visible (no-op without PDL)
  pdl_trigger();
  extern __shared__ __align__(16) unsigned char smem_raw[];
  GSmem& S = *reinterpret_cast<GSmem*>(smem_raw);
  BatchCtl* ctl = g.ctl;
  if (ctl->invalid) return;
  const int tid = threadIdx.x;
  if (tid == 0) S.ticket = atomicAdd(&ctl->tile_ctr[TC_GROUP], 1u);
  __syncthreads();
  const uint32_t b = S.ticket;
  EIRENE_PHASE(g.A, 1, b, 0);
  const unsigned long long tp0 = g.prof ? gtime_ns() : 0;
  const uint32_t base = g.gstart[b];
  const uint32_t cnt = g.gstart[b + 1] - base;
  const bool small = cnt <= (uint32_t)G_CAP;
  const uint64_t* K;
  const uint32_t* P;
  if (small) {
    if (cnt == 1 && tid == 0) {
      S.k[0] = g.kA[base];
      S.p[0] = g.pA[base];
    } else if (cnt > 1) {
      smem_sort(g.kA + base, g.pA + base, cnt, g.tsbits, S, g.A, b);
    }
    __syncthreads();
    K = S.k;
    P = S.p;
  }
  int mode = 0;   // 0: small / L2-sorted group, 2: SPLIT (rest in smem, hot key in a bitmap)
  // SPLIT groups of a batch without range queries hand the hot key's bitmap to
  // the result phase (multi-CTA); range batches need the segment's positions
  // (artificial queries binary-search them) and walk it here (hot_pass2)
#ifdef EIRENE_NO_HOTDEFER
  const bool deferred = false;
#else
  const bool deferred = g.A->rkeys == nullptr;
#endif
  uint32_t sp_o = 0, sp_h = 0, sp_lo = 0;
  if (!small) {
    const int where = l2_sort(g.kA + base, g.pA + base, g.kB + base, g.pB + base, cnt, g.tsbits, S, g.hot_bits,
                              &ctl->hot_ctr, g.A->n, g.hot_words);
    if (where == 2) {
      mode = 2;
      sp_o = S.r_nh;
      sp_h = S.r_lw;
      sp_lo = S.r_nw;
      K = S.k;
      P = S.p;
    } else {
      K = (where ? g.kB : g.kA) + base;
      P = (where ? g.pB : g.pA) + base;
    }
  }
  EIRENE_PHASE(g.A, 1, b, 1);
  const unsigned long long tp1 = g.prof ? gtime_ns() : 0;
  // sweep 1: bucket totals (heads, write segments)
  uint32_t c_nh = 0, c_lw = 0, c_nw = 0;
  uint32_t a_nh = 0, a_nw = 0, hot_w = 0, hot_last = 0;   // SPLIT: rest below hk; hk's issue
  HotCarry hc{};
  if (mode == 2) {
    const GView V{K, P, K, P, 0, sp_o};
    if (sp_lo) {   // the part of the rest below hk, alone (its tail ends at hk)
      round_scan(V, sp_lo, 0, sp_lo, 0, 0, 0, S);
      a_nh = S.r_nh;
      a_nw = S.r_nw;
    }
    if (sp_o) {
      round_scan(V, sp_o, 0, sp_o, 0, 0, 0, S);
      c_nh = S.r_nh;
      c_nw = S.r_nw;
    }
    __syncthreads();
    if (deferred) {   // the aggregate came with the split scan; the bitmap walk is the result phase's
      hot_w = S.hot_lastw ? 1u : 0u;
      hot_last = S.hot_lastw ? S.hot_lastw : S.hot_lastp;
    } else {
      hc = hot_pass1(g, S.hot_bits, S);
      hot_w = hc.last_w ? 1u : 0u;
      hot_last = hc.last_w ? hc.last_w : hc.last_p;   // issue rule: the last write, else the last query
    }
    c_nh += 1;
    c_nw += hot_w;
    __syncthreads();
  }
  for (uint32_t r0 = 0; mode == 0 && r0 < cnt; r0 += G_CAP) {
    const uint32_t r1 = min(cnt, r0 + (uint32_t)G_CAP);
    const GView V = small ? GView{K, P, K, P, 0, cnt} : load_round(K, P, r0, r1, S);
    round_scan(V, cnt, r0, r1, c_nh, c_lw, c_nw, S);
    c_nh = S.r_nh;
    c_lw = S.r_lw;
    c_nw = S.r_nw;
  }
  EIRENE_PHASE(g.A, 1, b, 2);
  const unsigned long long tp2 = g.prof ? gtime_ns() : 0;
  if (g.phase == 1) {
    // phase 1 of two (batches without range queries: deferred hot keys): leave
    // the sorted group in L2 for phase 2 and publish the aggregate -- no wait
    const uint32_t where = mode == 2 ? 2u : (small || K == g.kB + base) ? 1u : 0u;
    if (small || mode == 2) {
      const uint32_t m = small ? cnt : sp_o;
      for (uint32_t i = tid; i < m; i += G_THREADS) {
        g.kB[base + i] = S.k[i];
        g.pB[base + i] = S.p[i];
      }
    }
    if (tid == 0) {
      GroupRec r;
      r.hk = mode == 2 ? S.hk : 0;
      r.where = where;
      r.c_nh = c_nh;
      r.c_nw = c_nw;
      r.sp_o = sp_o;
      r.sp_h = sp_h;
      r.sp_lo = sp_lo;
      r.a_nh = a_nh;
      r.a_nw = a_nw;
      r.hot_w = hot_w;
      r.hot_last = hot_last;
      r.hot_slot = mode == 2 ? S.hot_slot : 0u;
      reinterpret_cast<GroupRec*>(g.grec)[b] = r;
      st_relaxed64(g.status + b, F_AGG | (((unsigned long long)c_nh << 31) | c_nw));
    }
    return;
  }
  group_lookback(g, b, c_nh, c_nw, S);
  EIRENE_PHASE(g.A, 1, b, 3);
  const unsigned long long tp3 = g.prof ? gtime_ns() : 0;
  // sweep 2: emit (a small bucket reuses the carries of its single round)
  if (mode == 2)
    emit_split(g, S, base, sp_o, sp_lo, sp_h, hot_w, hot_last, a_nh, a_nw, deferred, hc);
  else if (small) {
    if (cnt) round_emit(g, GView{K, P, K, P, 0, cnt}, cnt, base, 0, cnt, true, S);
  } else
    emit_rounds(g, S, K, P, cnt, base);
  EIRENE_PHASE(g.A, 1, b, 4);
#ifdef EIRENE_GROUP_PROF_BUILD   // diagnostic builds only: printf in a kernel costs on every launch
  if ((g.prof & 1) && tid == 0) {
    const unsigned long long tp4 = gtime_ns();
    if (tp4 - tp0 > 20000)
      printf("[group prof] ticket %u cnt %u mode %d sort %.1f (range %.1f split %.1f rest %.1f, rest %u hot %u) "
             "sweep1 %.1f lookback %.1f emit %.1f us hot2 %.1f\n", b,
             cnt, mode, (tp1 - tp0) * 1e-3, small ? 0.0 : (S.prof_l[0] - tp0) * 1e-3,
             mode == 2 ? (S.prof_l[1] - S.prof_l[0]) * 1e-3 : 0.0, mode == 2 ? (S.prof_l[2] - S.prof_l[1]) * 1e-3 : 0.0,
             sp_o, sp_h, (tp2 - tp1) * 1e-3, (tp3 - tp2) * 1e-3, (tp4 - tp3) * 1e-3,
             mode == 2 ? (S.prof_t[1] - S.prof_t[0]) * 1e-3 : 0.0);
  }
#else
  (void)tp0; (void)tp1; (void)tp2; (void)tp3;
#endif
}

}  // namespace

bool group_two_phase(uint32_t n, int num_sms) { return bsort_groups(n, num_sms) > 2u * (uint32_t)num_sms; }

void launch_group(const BatchArgs* A, uint32_t n, const BSortBufs& b, const CombBufs& c, Tree t, BatchCtl* ctl,
                  int num_sms, bool two_phase, cudaStream_t st, int* launches) {
  static int attr[MAX_DEVICES];
  per_device(attr, [] {
    return (int)cudaFuncSetAttribute(group_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sizeof(GSmem));
  });
  GroupArgs g;
  g.A = A;
  g.kA = b.kA;
  g.pA = b.pA;
  g.kB = b.kB;
  g.pB = b.pB;
  g.gstart = b.gstart;
  g.n = n;
  g.nb = bsort_groups(n, num_sms);
  g.tsbits = n > 1 ? 32 - __builtin_clz(n - 1) : 0;
  g.pinfo = c.pinfo;
  g.istart = c.istart;
  g.qkey = c.qkey;
  g.qseg = c.qseg;
  g.wkey = c.wkey;
  g.wop = c.wop;
  g.wval = c.wval;
  g.wseg = c.wseg;
  g.status = c.group_status;
  g.hot_bits = c.hot_bits;
  g.hot_words = c.hot_words;
  g.hot_seg = c.hot_seg;
  static const int prof = std::getenv("EIRENE_GROUP_PROF") ? std::atoi(std::getenv("EIRENE_GROUP_PROF")) : 0;
  g.prof = prof;
  g.grec = c.grec;
  g.t = t;
  g.ctl = ctl;
  if (!two_phase) {
    g.phase = 0;
    launch_k(group_kernel, dim3(g.nb), dim3(G_THREADS), sizeof(GSmem), st, true, false, g);
    ++*launches;
    return;
  }
  static int attr2[MAX_DEVICES];
  per_device(attr2, [] {
    return (int)cudaFuncSetAttribute(group_emit_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                     (int)sizeof(GSmem));
  });
  g.phase = 1;
  launch_k(group_kernel, dim3(g.nb), dim3(G_THREADS), sizeof(GSmem), st, true, false, g);
  launch_k(group_emit_kernel, dim3(g.nb), dim3(G_THREADS), sizeof(GSmem), st, true, false, g);
  *launches += 2;
}

}  // namespace eirene
