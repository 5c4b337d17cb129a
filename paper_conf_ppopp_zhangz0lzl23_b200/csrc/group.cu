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

namespace eirene {

namespace {

constexpr int G_THREADS = 512;
constexpr int G_WARPS = G_THREADS / 32;
constexpr int G_ITEMS = 12;
constexpr int G_CAP = G_THREADS * G_ITEMS;    // 6144 positions sorted in smem
constexpr int SB_BITS = 12;                   // sub-bucket bits inside a bucket
constexpr int SB_N = 1 << SB_BITS;

constexpr unsigned long long F_AGG = 1ull << 62;
constexpr unsigned long long F_INC = 2ull << 62;
constexpr unsigned long long F_VAL = (1ull << 62) - 1;

struct GSmem {
  uint64_t k[G_CAP];
  uint32_t p[G_CAP];
  uint32_t sb[SB_N + 1];
  uint32_t wsum[G_WARPS];
  uint32_t hist[256];
  uint32_t off[256];
  // per-warp aggregates and exclusive carries of the current round
  uint32_t w_nh[G_WARPS], w_lw[G_WARPS], w_nw[G_WARPS];
  uint32_t c_nh[G_WARPS], c_lw[G_WARPS], c_nw[G_WARPS];
  uint32_t r_nh, r_lw, r_nw;   // round carry-out
  uint32_t seg0, w0, ticket;
};

__device__ __forceinline__ bool kp_less(uint64_t ka, uint32_t pa, uint64_t kb, uint32_t pb) {
  return ka < kb || (ka == kb && pa < pb);
}
__device__ __forceinline__ uint32_t lanemask_le() { return lanemask_lt() | (1u << lane_id()); }

// Stable LSD pass over [0, cnt) of (ks, ps) -> (kd, pd) by an 8-bit digit, by
// one CTA walking the bucket in G_THREADS-sized tiles; warps of a tile take
// their offsets in warp order, lanes in lane order, so the pass is stable.
template <class DigitFn>
__device__ void cta_lsd_pass(const uint64_t* ks, const uint32_t* ps, uint64_t* kd, uint32_t* pd, uint32_t cnt,
                             DigitFn dig, GSmem& S) {
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  if (tid < 256) S.hist[tid] = 0;
  __syncthreads();
  for (uint32_t i = tid; i < cnt; i += G_THREADS) atomicAdd(&S.hist[dig(ks[i], ps[i])], 1u);
  __syncthreads();
  if (tid == 0) {
    uint32_t r = 0;
    for (int d = 0; d < 256; ++d) {
      S.off[d] = r;
      r += S.hist[d];
    }
  }
  __syncthreads();
  for (uint32_t base = 0; base < cnt; base += G_THREADS) {
    const uint32_t i = base + tid;
    const bool act = i < cnt;
    const uint64_t k = act ? ks[i] : 0;
    const uint32_t p = act ? ps[i] : 0;
    const uint32_t d = act ? dig(k, p) : 256u;
    const uint32_t peers = __match_any_sync(FULL, d);
    uint32_t before = 0;
    for (int w = 0; w < G_WARPS; ++w) {
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

// Sort a bucket of cnt <= G_CAP requests into S.k / S.p: sub-bucket by the
// next SB_BITS key bits (smem atomics + block scan + scatter), then finish
// each sub-bucket (~1 request on average) by insertion sort on (key, payload).
__device__ void smem_sort(const uint64_t* __restrict__ ks, const uint32_t* __restrict__ ps, uint32_t cnt, int sb_shift,
                          GSmem& S) {
  const int tid = threadIdx.x;
  for (int i = tid; i <= SB_N; i += G_THREADS) S.sb[i] = 0;
  __syncthreads();
  uint64_t kr[G_ITEMS];
  uint32_t r[G_ITEMS];
#pragma unroll
  for (int j = 0; j < G_ITEMS; ++j) {
    const uint32_t i = tid + j * G_THREADS;
    kr[j] = i < cnt ? ks[i] : 0;
  }
#pragma unroll
  for (int j = 0; j < G_ITEMS; ++j) {
    const uint32_t i = tid + j * G_THREADS;
    r[j] = i < cnt ? atomicAdd(&S.sb[(uint32_t)(kr[j] >> sb_shift) & (SB_N - 1)], 1u) : 0u;
  }
  __syncthreads();
  {   // exclusive scan of S.sb[0..SB_N) (8 per thread)
    constexpr int PER = SB_N / G_THREADS;
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
    uint32_t run = x - s;
    for (int w = 0; w < warp; ++w) run += S.wsum[w];
#pragma unroll
    for (int j = 0; j < PER; ++j) {
      S.sb[tid * PER + j] = run;
      run += loc[j];
    }
    if (tid == 0) S.sb[SB_N] = cnt;
  }
  __syncthreads();
#pragma unroll
  for (int j = 0; j < G_ITEMS; ++j) {
    const uint32_t i = tid + j * G_THREADS;
    if (i < cnt) {
      const uint32_t pos = S.sb[(uint32_t)(kr[j] >> sb_shift) & (SB_N - 1)] + r[j];
      S.k[pos] = kr[j];
      S.p[pos] = ps[i];
    }
  }
  __syncthreads();
  for (int s = tid; s < SB_N; s += G_THREADS) {
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
}

// Oversized bucket: stable LSD in L2 on the payload (4 x 8 bits) and then the
// key bits below the bucket prefix; an odd number of passes ends in (kd, pd).
__device__ void l2_sort(uint64_t* ks, uint32_t* ps, uint64_t* kd, uint32_t* pd, uint32_t cnt, int bb, GSmem& S) {
  const int tid = threadIdx.x;
  const int key_passes = (64 - bb + 7) / 8;
  const int total = 4 + key_passes;
  uint64_t* k0 = ks;
  uint32_t* p0 = ps;
  uint64_t* k1 = kd;
  uint32_t* p1 = pd;
  if ((total & 1) == 0) {   // make the count odd with a copy pass into (kd, pd) first
    for (uint32_t i = tid; i < cnt; i += G_THREADS) {
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

// Worst-case node demand of the update kernel (EFULL pre-check, SURVEY
// §8(b)): new leaves <= issued writes; new inner nodes at level l+1 <=
// min(N_l, (I_l + N_l) / 8) because every node created by an even multi-way
// split keeps >= 8 children, plus root growth.
__device__ bool headroom_ok(const Tree& t, uint32_t nw) {
  const TreeHdr* h = t.hdr;
  const uint32_t height = (uint32_t)(h->root_word >> 32);
  unsigned long long need_leaf = nw;
  unsigned long long N = nw, inner = 0;
  for (uint32_t l = 0; l + 1 < height && N > 0; ++l) {
    unsigned long long I = h->level_count[l];
    unsigned long long Nn = min(N, (I + N) / 8 + 1);
    inner += Nn;
    N = Nn;
  }
  inner += 2 * (N + 1) + 64;   // new root levels
  return (unsigned long long)h->leaf_count + need_leaf <= t.leaf_cap &&
         (unsigned long long)h->inner_count + inner <= t.inner_cap;
}

struct GroupArgs {
  const BatchArgs* A;
  uint64_t* kA;                 // bucketed requests (bsort scatter output)
  uint32_t* pA;
  uint64_t* kB;                 // L2 scratch for oversized buckets
  uint32_t* pB;                 // sorted payloads (output, read by RESULT_CAL)
  const uint32_t* bcount;
  const uint32_t* bstart;
  int bb, bsh;
  uint32_t n, nb;
  uint32_t* pinfo;
  uint32_t* istart;
  uint64_t* qkey;
  uint32_t* qseg;
  uint64_t* wkey;
  uint8_t* wop;
  uint64_t* wval;
  uint32_t* wseg;
  unsigned long long* status;   // [nb] look-back words (zeroed per batch)
  Tree t;
  BatchCtl* ctl;
};

// Round [r0, r1) of a bucket walked by 16 warps: pass 1 (heads, last write per
// warp), warp scan, pass 2 (write segments ending in each warp), warp scan.
// Leaves the exclusive per-warp carries in S.c_* and the carry-out in S.r_*.
__device__ void round_scan(const uint64_t* K, const uint32_t* P, uint32_t cnt, uint32_t r0, uint32_t r1,
                           uint32_t cin_nh, uint32_t cin_lw, uint32_t cin_nw, GSmem& S) {
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const uint32_t len = r1 - r0;
  const uint32_t C = 32u * ((len + G_THREADS - 1) / G_THREADS);
  const uint32_t wb = r0 + warp * C;
  const uint32_t we = min(r1, wb + C);
  uint32_t nh = 0, lw = 0;
  for (uint32_t b = wb; b < we; b += 32) {
    const uint32_t x = b + lane;
    const bool valid = x < we;
    const uint64_t k = valid ? K[x] : 0;
    const bool head = valid && (x == 0 || K[x - 1] != k);
    const uint32_t W = __ballot_sync(FULL, valid && is_write(P[valid ? x : 0] & 3));
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
  for (uint32_t b = wb; b < we; b += 32) {
    const uint32_t x = b + lane;
    const bool valid = x < we;
    const uint64_t k = valid ? K[x] : 0;
    const uint32_t W = __ballot_sync(FULL, valid && is_write(P[valid ? x : 0] & 3));
    const uint32_t wle = W & lanemask_le();
    const uint32_t lwi = wle ? b + (31 - __clz(wle)) + 1 : lwc;
    const bool tail = valid && (x + 1 == cnt || K[x + 1] != k);
    const bool hasw = tail && lwi && K[lwi - 1] == k;
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
__device__ void round_emit(const GroupArgs& g, const uint64_t* K, const uint32_t* P, uint32_t cnt, uint32_t gbase,
                           uint32_t r0, uint32_t r1, bool write_spay, GSmem& S) {
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const uint64_t* __restrict__ vals = g.A->vals;
  uint64_t* __restrict__ results = g.A->results;
  const uint32_t len = r1 - r0;
  const uint32_t C = 32u * ((len + G_THREADS - 1) / G_THREADS);
  const uint32_t wb = r0 + warp * C;
  const uint32_t we = min(r1, wb + C);
  const uint32_t seg0 = S.seg0, w0 = S.w0;
  uint32_t nh = S.c_nh[warp], lwc = S.c_lw[warp], nwc = S.c_nw[warp];
  for (uint32_t b = wb; b < we; b += 32) {
    const uint32_t x = b + lane;
    const bool valid = x < we;
    const uint64_t k = valid ? K[x] : 0;
    const uint32_t p = valid ? P[x] : 0;
    const bool head = valid && (x == 0 || K[x - 1] != k);
    const uint32_t H = __ballot_sync(FULL, head);
    const uint32_t W = __ballot_sync(FULL, valid && is_write(p & 3));
    const uint32_t seg = seg0 + nh + __popc(H & lanemask_le()) - 1u;
    // nearest write strictly before x, and at or before x (bucket positions + 1)
    const uint32_t wl = W & lanemask_lt();
    const uint32_t lwb = wl ? b + (31 - __clz(wl)) + 1 : lwc;
    const uint32_t wle = W & lanemask_le();
    const uint32_t lwi = wle ? b + (31 - __clz(wle)) + 1 : lwc;
    const bool done = valid && !head && lwb && K[lwb - 1] == k;
    if (done) {
      const uint32_t pw = P[lwb - 1];
      results[p >> 2] = ((pw & 3) == OP_DELETE) ? KEY_MAX : vals[pw >> 2];
    }
    if (valid) {
      g.pinfo[gbase + x] = seg | (done ? DONE_BIT : 0u);
      if (write_spay) g.pB[gbase + x] = p;
    }
    if (head) g.istart[seg] = gbase + x;
    const bool tail = valid && (x + 1 == cnt || K[x + 1] != k);
    const bool hasw = tail && lwi && K[lwi - 1] == k;
    const uint32_t WT = __ballot_sync(FULL, hasw);
    if (tail) {
      const uint32_t wi = w0 + nwc + __popc(WT & lanemask_lt());
      if (hasw) {   // issue rule: the segment's last write
        const uint32_t pw = P[lwi - 1];
        const uint32_t opw = pw & 3;
        g.wkey[wi] = k;
        g.wop[wi] = (uint8_t)opw;
        g.wval[wi] = (opw == OP_DELETE) ? KEY_MAX : vals[pw >> 2];
        g.wseg[wi] = seg;
      } else {      // all-query segment: its last query
        const uint32_t qi = seg - wi;
        g.qkey[qi] = k;
        g.qseg[qi] = seg;
      }
    }
    nh += __popc(H);
    nwc += __popc(WT);
    if (W) lwc = b + (31 - __clz(W)) + 1;
  }
}

__global__ void __launch_bounds__(G_THREADS) group_kernel(GroupArgs g) {
  extern __shared__ __align__(16) unsigned char smem_raw[];
  GSmem& S = *reinterpret_cast<GSmem*>(smem_raw);
  BatchCtl* ctl = g.ctl;
  if (ctl->invalid) return;
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  if (tid == 0) S.ticket = atomicAdd(&ctl->tile_ctr[TC_GROUP], 1u);
  __syncthreads();
  const uint32_t b = S.ticket;
  const uint32_t cnt = g.bcount[b << g.bsh];
  const uint32_t base = g.bstart[b];
  const bool small = cnt <= (uint32_t)G_CAP;
  const uint64_t* K;
  const uint32_t* P;
  if (small) {
    if (cnt) smem_sort(g.kA + base, g.pA + base, cnt, 64 - g.bb - SB_BITS, S);
    K = S.k;
    P = S.p;
  } else {
    l2_sort(g.kA + base, g.pA + base, g.kB + base, g.pB + base, cnt, g.bb, S);
    K = g.kB + base;
    P = g.pB + base;
  }
  // sweep 1: bucket totals (heads, write segments)
  uint32_t c_nh = 0, c_lw = 0, c_nw = 0;
  for (uint32_t r0 = 0; r0 < cnt; r0 += G_CAP) {
    const uint32_t r1 = min(cnt, r0 + (uint32_t)G_CAP);
    round_scan(K, P, cnt, r0, r1, c_nh, c_lw, c_nw, S);
    c_nh = S.r_nh;
    c_lw = S.r_lw;
    c_nw = S.r_nw;
  }
  // decoupled look-back over the buckets (ticket order) on (heads << 31 | writes)
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
      if (b + 1 == g.nb) {   // last bucket: batch totals + headroom check
        const uint32_t nseg = seg0 + c_nh, nw = w0 + c_nw;
        ctl->nseg = nseg;
        ctl->nw = nw;
        ctl->nq = nseg - nw;
        g.istart[nseg] = g.n;
        if (!headroom_ok(g.t, nw)) ctl->status = EIRENE_EFULL;
      }
    }
  }
  __syncthreads();
  // sweep 2: emit (a small bucket reuses the carries of its single round)
  if (small) {
    if (cnt) round_emit(g, K, P, cnt, base, 0, cnt, true, S);
  } else {
    c_nh = c_lw = c_nw = 0;
    for (uint32_t r0 = 0; r0 < cnt; r0 += G_CAP) {
      const uint32_t r1 = min(cnt, r0 + (uint32_t)G_CAP);
      round_scan(K, P, cnt, r0, r1, c_nh, c_lw, c_nw, S);
      round_emit(g, K, P, cnt, base, r0, r1, false, S);
      c_nh = S.r_nh;
      c_lw = S.r_lw;
      c_nw = S.r_nw;
      __syncthreads();
    }
  }
}

}  // namespace

void launch_group(const BatchArgs* A, uint32_t n, const BSortBufs& b, const CombBufs& c, Tree t, BatchCtl* ctl,
                  cudaStream_t st, int* launches) {
  static bool attr = false;
  if (!attr) {
    cudaFuncSetAttribute(group_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sizeof(GSmem));
    attr = true;
  }
  const int bb = bsort_bits(n);
  GroupArgs g;
  g.A = A;
  g.kA = b.kA;
  g.pA = b.pA;
  g.kB = b.kB;
  g.pB = b.pB;
  g.bcount = b.bcount;
  g.bstart = b.bstart;
  g.bb = bb;
  g.bsh = bsort_ctr_shift(bb);
  g.n = n;
  g.nb = 1u << bb;
  g.pinfo = c.pinfo;
  g.istart = c.istart;
  g.qkey = c.qkey;
  g.qseg = c.qseg;
  g.wkey = c.wkey;
  g.wop = c.wop;
  g.wval = c.wval;
  g.wseg = c.wseg;
  g.status = c.group_status;
  g.t = t;
  g.ctl = ctl;
  group_kernel<<<g.nb, G_THREADS, sizeof(GSmem), st>>>(g);
  ++*launches;
}

}  // namespace eirene
