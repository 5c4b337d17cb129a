// combine.cu -- combining (Alg.1:11), partition (Alg.1:3) and the
// long-segment part of RESULT_CAL (Alg.1:6), sm_100a.
//
// combine_kernel: one pass over the sorted requests ("each GPU
// thread scans one request with its neighbours"), here as segmented scans.
// For sorted position i:
//   head(i)  = i == 0 or key[i] != key[i-1]            (a new key segment)
//   seg(i)   = (#heads in [0, i]) - 1                   (issued-request index)
//   lw(i)    = 1 + max{ j <= i : op[j] is a write }      (0 = none)
// The nearest earlier write j of i is in i's segment iff key[j] == key[i]
// (the array is sorted).  Then i's result is that write's value, or null for a
// delete (nearest write P:834-835) and is written now ("early
// result"); otherwise i waits for the value its segment's issued request
// retrieves.  At the segment tail the issued request is chosen:
// the last write if the segment has one, else the last query (§8(c) 5-6).
//
// Layout (B200): a 2048-request tile per CTA; each warp walks 256 consecutive
// requests in 8 steps of 32, lane = request, so every load and store of a step
// is one coalesced 32-element access; in-step scans are ballots/popc and
// shuffles, and a register carry runs across steps.  Pass 1 reduces each warp
// (heads, last write), a block scan + decoupled look-back (warp 0, 32 tiles per
// probe) gives the tile prefix, pass 2 produces the outputs.
#include "eirene_internal.cuh"

namespace eirene {

namespace {

constexpr unsigned long long F_AGG = 1ull << 62;
constexpr unsigned long long F_INC = 2ull << 62;
constexpr unsigned long long M31 = (1ull << 31) - 1;
constexpr int CW = COMB_THREADS / 32;          // warps per tile
constexpr int CSTEPS = COMB_ITEMS;             // steps of 32 requests per warp

struct Agg {
  uint32_t nh;   // heads
  uint32_t lw;   // 1 + last write position (0 = none)
};
__device__ __forceinline__ Agg agg_op(Agg a, Agg b) { return {a.nh + b.nh, max(a.lw, b.lw)}; }
__device__ __forceinline__ unsigned long long agg_pack(Agg a, unsigned long long f) {
  return f | ((unsigned long long)a.nh << 31) | a.lw;
}
__device__ __forceinline__ Agg agg_unpack(unsigned long long w) {
  return {(uint32_t)((w >> 31) & M31), (uint32_t)(w & M31)};
}

__device__ __forceinline__ uint32_t lanemask_le() { return lanemask_lt() | (1u << lane_id()); }

__global__ void __launch_bounds__(COMB_THREADS) combine_kernel(
    const uint64_t* __restrict__ skey, const uint32_t* __restrict__ spay, const BatchArgs* __restrict__ A,
    uint32_t n, uint32_t* __restrict__ pinfo, uint64_t* __restrict__ ikey,
    uint8_t* __restrict__ iop, uint64_t* __restrict__ ival, uint32_t* __restrict__ istart,
    unsigned long long* __restrict__ status, BatchCtl* __restrict__ ctl) {
  const uint64_t* __restrict__ vals = A->vals;
  uint64_t* __restrict__ results = A->results;
  __shared__ uint32_t s_tile;
  __shared__ Agg s_w[CW];
  __shared__ Agg s_prefix;
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  if (ctl->invalid) return;
  if (tid == 0) s_tile = atomicAdd(&ctl->tile_ctr[TC_COMB], 1u);
  __syncthreads();
  const uint32_t tile = s_tile;
  const uint32_t wb = tile * COMB_TILE + warp * (32 * CSTEPS);   // warp base position

  uint64_t K[CSTEPS];
  uint32_t P[CSTEPS];
#pragma unroll
  for (int j = 0; j < CSTEPS; ++j) {
    const uint32_t p = wb + 32 * j + lane;
    K[j] = p < n ? skey[p] : KEY_MAX;
    P[j] = p < n ? spay[p] : 0u;
  }
  const uint64_t kbefore = (wb > 0 && wb <= n) ? skey[wb - 1] : 0;   // key before the warp's range
  const uint64_t kafter = (wb + 32 * CSTEPS < n) ? skey[wb + 32 * CSTEPS] : KEY_MAX;

  // ---- pass 1: warp aggregate (heads, last write)
  uint32_t heads[CSTEPS], writes[CSTEPS];
  Agg wagg = {0, 0};
#pragma unroll
  for (int j = 0; j < CSTEPS; ++j) {
    const uint32_t p = wb + 32 * j + lane;
    const bool valid = p < n;
    const uint64_t up = __shfl_up_sync(FULL, K[j], 1);
    const uint64_t last_prev = j == 0 ? kbefore : __shfl_sync(FULL, K[j > 0 ? j - 1 : 0], 31);
    const uint64_t kp = lane == 0 ? last_prev : up;
    heads[j] = __ballot_sync(FULL, valid && (p == 0 || K[j] != kp));
    writes[j] = __ballot_sync(FULL, valid && is_write(P[j] & 3));
    wagg.nh += __popc(heads[j]);
    if (writes[j]) wagg.lw = wb + 32 * j + (31 - __clz(writes[j])) + 1;
  }
  if (lane == 0) s_w[warp] = wagg;
  __syncthreads();
  // ---- tile aggregate, decoupled look-back by warp 0 (32 predecessors per probe)
  if (warp == 0) {
    Agg tot = {0, 0};
#pragma unroll
    for (int w = 0; w < CW; ++w) tot = agg_op(tot, s_w[w]);
    unsigned long long* my = status + tile;
    Agg excl = {0, 0};
    if (tile == 0) {
      if (lane == 0) st_relaxed64(my, agg_pack(tot, F_INC));
    } else {
      if (lane == 0) st_relaxed64(my, agg_pack(tot, F_AGG));
      SpinGuard sg;
      int32_t pt = (int32_t)tile - 1;
      for (;;) {
        const int32_t idx = pt - lane;
        const unsigned long long w = idx >= 0 ? ld_relaxed64(status + idx) : F_INC;
        const uint32_t fl = (uint32_t)(w >> 62);
        const uint32_t inc = __ballot_sync(FULL, fl == 2);
        const uint32_t need = inc ? ((2u << (__ffs(inc) - 1)) - 1u) : FULL;
        if (__ballot_sync(FULL, fl == 0) & need) {
          if (sg.stuck(ctl)) break;
          continue;
        }
        Agg a = ((need >> lane) & 1u) ? agg_unpack(w) : Agg{0, 0};
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) a = agg_op(a, Agg{__shfl_xor_sync(FULL, a.nh, o), __shfl_xor_sync(FULL, a.lw, o)});
        excl = agg_op(a, excl);
        if (inc) break;
        pt -= 32;
      }
      if (lane == 0) st_relaxed64(my, agg_pack(agg_op(excl, tot), F_INC));
    }
    if (lane == 0) s_prefix = excl;
  }
  __syncthreads();
  Agg carry = s_prefix;
  for (int w = 0; w < warp; ++w) carry = agg_op(carry, s_w[w]);

  // ---- pass 2: per-request outputs with a register carry across steps
  // last write before the warp's range: its key and payload (for the same-segment test)
  bool cw_valid = carry.lw > 0;
  uint64_t cw_key = cw_valid ? skey[carry.lw - 1] : 0;
  uint32_t cw_pay = cw_valid ? spay[carry.lw - 1] : 0;
  uint32_t nh = carry.nh;
#pragma unroll
  for (int j = 0; j < CSTEPS; ++j) {
    const uint32_t p = wb + 32 * j + lane;
    const bool valid = p < n;
    const uint64_t key = K[j];
    const bool head = (heads[j] >> lane) & 1u;
    const uint32_t seg = nh + __popc(heads[j] & lanemask_le()) - 1u;
    // nearest write strictly before me
    const uint32_t wl = writes[j] & lanemask_lt();
    const int q = wl ? 31 - __clz(wl) : lane;
    const uint64_t kq = __shfl_sync(FULL, key, q);
    const uint32_t pq = __shfl_sync(FULL, P[j], q);
    const bool has_before = wl ? true : cw_valid;
    const uint64_t kw = wl ? kq : cw_key;
    const uint32_t pw = wl ? pq : cw_pay;
    bool done = false;
    if (valid && !head && has_before && kw == key) {
      results[P[j] >> 2] = ((pw & 3) == OP_DELETE) ? KEY_MAX : vals[pw >> 2];
      done = true;
    }
    if (valid) pinfo[p] = seg | (done ? DONE_BIT : 0u);
    if (head) istart[seg] = p;
    // tail: the next request has another key
    const uint64_t dn = __shfl_down_sync(FULL, key, 1);
    const uint64_t first_next = j + 1 < CSTEPS ? __shfl_sync(FULL, K[j + 1 < CSTEPS ? j + 1 : j], 0) : kafter;
    const uint64_t kn = lane == 31 ? first_next : dn;
    const bool tail = valid && (p == n - 1 || kn != key);
    // nearest write at or before me (the issued write if it is in my segment)
    const uint32_t wle = writes[j] & lanemask_le();
    const int q2 = wle ? 31 - __clz(wle) : lane;
    const uint64_t kq2 = __shfl_sync(FULL, key, q2);
    const uint32_t pq2 = __shfl_sync(FULL, P[j], q2);
    if (tail) {
      const bool has = wle ? true : cw_valid;
      const uint64_t k2 = wle ? kq2 : cw_key;
      const uint32_t p2 = wle ? pq2 : cw_pay;
      ikey[seg] = key;
      if (has && k2 == key) {   // issue rule: the last write of the segment
        const uint32_t opw = p2 & 3;
        iop[seg] = (uint8_t)opw;
        ival[seg] = (opw == OP_DELETE) ? KEY_MAX : vals[p2 >> 2];
      } else {                  // all-query segment: this (last) query
        iop[seg] = OP_QUERY;
      }
      if (p == n - 1) {
        ctl->nseg = seg + 1;
        istart[seg + 1] = n;
      }
    }
    // carry to the next step
    nh += __popc(heads[j]);
    if (writes[j]) {
      const int ql = 31 - __clz(writes[j]);
      cw_key = __shfl_sync(FULL, key, ql);
      cw_pay = __shfl_sync(FULL, P[j], ql);
      cw_valid = true;
    }
  }
}

// ---------------------------------------------------------------- partition
constexpr unsigned long long P_AGG = 1ull << 62;
constexpr unsigned long long P_INC = 2ull << 62;
constexpr unsigned long long P_VAL = (1ull << 62) - 1;

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

// Alg.1:3 PARTITION: stable split of the issued list (one entry per segment,
// key order) into the query list and the write list; the write index of a
// segment is the number of write segments before it.  Same warp-striped
// layout and look-back as combine_kernel.
__global__ void __launch_bounds__(COMB_THREADS) partition_kernel(
    const uint64_t* __restrict__ ikey, const uint8_t* __restrict__ iop, const uint64_t* __restrict__ ival,
    uint64_t* __restrict__ qkey, uint32_t* __restrict__ qseg, uint64_t* __restrict__ wkey, uint8_t* __restrict__ wop,
    uint64_t* __restrict__ wval, uint32_t* __restrict__ wseg, unsigned long long* __restrict__ status, Tree t,
    BatchCtl* __restrict__ ctl) {
  __shared__ uint32_t s_tile, s_w[CW], s_prefix;
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  if (ctl->invalid) return;
  const uint32_t nseg = ctl->nseg;
  if (tid == 0) s_tile = atomicAdd(&ctl->tile_ctr[TC_PART], 1u);
  __syncthreads();
  const uint32_t tile = s_tile;
  if (tile * COMB_TILE >= nseg) return;
  const uint32_t wb = tile * COMB_TILE + warp * (32 * CSTEPS);
  uint8_t o[CSTEPS];
  uint32_t wm[CSTEPS];
  uint32_t cnt = 0;
#pragma unroll
  for (int j = 0; j < CSTEPS; ++j) {
    const uint32_t s = wb + 32 * j + lane;
    o[j] = s < nseg ? iop[s] : (uint8_t)0;
    wm[j] = __ballot_sync(FULL, s < nseg && is_write(o[j]));
    cnt += __popc(wm[j]);
  }
  if (lane == 0) s_w[warp] = cnt;
  __syncthreads();
  if (warp == 0) {
    uint32_t tot = 0;
#pragma unroll
    for (int w = 0; w < CW; ++w) tot += s_w[w];
    unsigned long long* my = status + tile;
    uint32_t excl = 0;
    if (tile == 0) {
      if (lane == 0) st_relaxed64(my, P_INC | tot);
    } else {
      if (lane == 0) st_relaxed64(my, P_AGG | tot);
      SpinGuard sg;
      int32_t pt = (int32_t)tile - 1;
      for (;;) {
        const int32_t idx = pt - lane;
        const unsigned long long w = idx >= 0 ? ld_relaxed64(status + idx) : P_INC;
        const uint32_t fl = (uint32_t)(w >> 62);
        const uint32_t inc = __ballot_sync(FULL, fl == 2);
        const uint32_t need = inc ? ((2u << (__ffs(inc) - 1)) - 1u) : FULL;
        if (__ballot_sync(FULL, fl == 0) & need) {
          if (sg.stuck(ctl)) break;
          continue;
        }
        uint32_t a = ((need >> lane) & 1u) ? (uint32_t)(w & P_VAL) : 0u;
#pragma unroll
        for (int off = 16; off > 0; off >>= 1) a += __shfl_xor_sync(FULL, a, off);
        excl += a;
        if (inc) break;
        pt -= 32;
      }
      if (lane == 0) st_relaxed64(my, P_INC | (excl + tot));
    }
    if (lane == 0) {
      s_prefix = excl;
      if ((tile + 1) * COMB_TILE >= nseg) {   // last tile: totals + headroom check
        const uint32_t nw = excl + tot;
        ctl->nw = nw;
        ctl->nq = nseg - nw;
        if (!headroom_ok(t, nw)) ctl->status = EIRENE_EFULL;
      }
    }
  }
  __syncthreads();
  uint32_t wbase = s_prefix;
  for (int w = 0; w < warp; ++w) wbase += s_w[w];
#pragma unroll
  for (int j = 0; j < CSTEPS; ++j) {
    const uint32_t s = wb + 32 * j + lane;
    if (s < nseg) {
      const uint32_t wi = wbase + __popc(wm[j] & lanemask_lt());
      const uint64_t key = ikey[s];
      if (is_write(o[j])) {
        wkey[wi] = key;
        wop[wi] = o[j];
        wval[wi] = ival[s];
        wseg[wi] = s;
      } else {
        const uint32_t qi = s - wi;
        qkey[qi] = key;
        qseg[qi] = s;
      }
    }
    wbase += __popc(wm[j]);
  }
}

// RESULT_CAL is fused into the query kernel: every issued request scatters
// the value it retrieved to the pending positions of its own segment.  The
// segments longer than SHORT_SEG (hot keys) are queued instead and finished
// here with one CTA per segment, so a 56K-request Zipf key does not serialise
// one thread.
__global__ void __launch_bounds__(256) result_long_kernel(const uint32_t* __restrict__ spay,
                                                           const uint32_t* __restrict__ pinfo,
                                                           const uint32_t* __restrict__ istart,
                                                           const uint32_t* __restrict__ longseg,
                                                           const uint64_t* __restrict__ old,
                                                           const BatchArgs* __restrict__ A,
                                                           const BatchCtl* __restrict__ ctl) {
  if (ctl->invalid || ctl->status != 0) return;
  uint64_t* __restrict__ results = A->results;
  const uint32_t nl = ctl->nlong;
  for (uint32_t x = blockIdx.x; x < nl; x += gridDim.x) {
    const uint32_t s = longseg[x];
    const uint64_t v = old[s];
    const uint32_t e = istart[s + 1];
    for (uint32_t p = istart[s] + threadIdx.x; p < e; p += blockDim.x)
      if (!(pinfo[p] & DONE_BIT)) results[spay[p] >> 2] = v;
  }
}

}  // namespace

void launch_combine(const uint64_t* skey, const uint32_t* spay, const BatchArgs* A, uint32_t n,
                    const CombBufs& c, BatchCtl* ctl, cudaStream_t st, int* launches) {
  const uint32_t tiles = (n + COMB_TILE - 1) / COMB_TILE;
  combine_kernel<<<tiles, COMB_THREADS, 0, st>>>(skey, spay, A, n, c.pinfo, c.ikey, c.iop, c.ival,
                                                 c.istart, c.comb_status, ctl);
  ++*launches;
}

void launch_partition(uint32_t n, const CombBufs& c, Tree t, BatchCtl* ctl, cudaStream_t st, int* launches) {
  const uint32_t tiles = (n + COMB_TILE - 1) / COMB_TILE;
  partition_kernel<<<tiles, COMB_THREADS, 0, st>>>(c.ikey, c.iop, c.ival, c.qkey, c.qseg, c.wkey, c.wop, c.wval,
                                                   c.wseg, c.part_status, t, ctl);
  ++*launches;
}

void launch_result(const uint32_t* spay, uint32_t n, const CombBufs& c, const BatchArgs* A, BatchCtl* ctl,
                   cudaStream_t st, int* launches) {
  (void)n;
  result_long_kernel<<<148, 256, 0, st>>>(spay, c.pinfo, c.istart, c.longseg, c.old, A, ctl);
  ++*launches;
}

}  // namespace eirene
