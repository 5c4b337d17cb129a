// combine.cu -- combining (Alg.1:11), partition (Alg.1:3) and
// RESULT_CAL (Alg.1:6) kernels, sm_100a.
//
// combine_kernel: one pass over the sorted requests ("each GPU
// thread scans one request with its neighbours"), here as segmented scans with
// a decoupled look-back across 2048-request tiles.  For sorted position i:
//   head(i)  = i == 0 or key[i] != key[i-1]            (a new key segment)
//   seg(i)   = (#heads in [0, i]) - 1                   (issued-request index)
//   lw(i)    = 1 + max{ j <= i : op[j] is a write }      (0 = none)
// The nearest earlier write j = lw(i-1)-1 is in i's segment iff key[j] == key[i]
// (the array is sorted).  Then i's result is that write's value, or null for a
// delete (nearest write P:834-835) and is written now ("early
// result"); otherwise i waits for the value its segment's issued request
// retrieves.  At the segment tail the issued request is chosen:
// the last write if the segment has one, else the last query (§8(c) 5-6).
#include "eirene_internal.cuh"

namespace eirene {

namespace {

constexpr unsigned long long F_AGG = 1ull << 62;
constexpr unsigned long long F_INC = 2ull << 62;
constexpr unsigned long long M31 = (1ull << 31) - 1;

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

template <int NT>
__device__ __forceinline__ Agg block_excl_scan_agg(Agg v, Agg* tmp, Agg* total) {
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  Agg x = v;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    Agg y = {__shfl_up_sync(FULL, x.nh, o), __shfl_up_sync(FULL, x.lw, o)};
    if (lane >= o) x = agg_op(y, x);
  }
  // exclusive within warp
  Agg ex = {__shfl_up_sync(FULL, x.nh, 1), __shfl_up_sync(FULL, x.lw, 1)};
  if (lane == 0) ex = {0, 0};
  if (lane == 31) tmp[warp] = x;
  __syncthreads();
  Agg wpre = {0, 0}, tot = {0, 0};
#pragma unroll
  for (int w = 0; w < NT / 32; ++w) {
    Agg t = tmp[w];
    if (w < warp) wpre = agg_op(wpre, t);
    tot = agg_op(tot, t);
  }
  __syncthreads();
  *total = tot;
  return agg_op(wpre, ex);
}

__global__ void __launch_bounds__(COMB_THREADS) combine_kernel(
    const uint64_t* __restrict__ skey, const uint32_t* __restrict__ spay, const uint64_t* __restrict__ vals,
    uint64_t* __restrict__ results, uint32_t n, uint32_t* __restrict__ pinfo, uint64_t* __restrict__ ikey,
    uint8_t* __restrict__ iop, uint64_t* __restrict__ ival, uint32_t* __restrict__ istart,
    unsigned long long* __restrict__ status,
    BatchCtl* __restrict__ ctl) {
  __shared__ uint32_t s_tile;
  __shared__ Agg s_tmp[COMB_THREADS / 32];
  __shared__ Agg s_prefix;
  const int tid = threadIdx.x;
  if (ctl->invalid) return;
  if (tid == 0) s_tile = atomicAdd(&ctl->tile_ctr[TC_COMB], 1u);
  __syncthreads();
  const uint32_t tile = s_tile;
  const uint32_t p0 = tile * COMB_TILE + tid * COMB_ITEMS;   // blocked arrangement

  uint64_t k[COMB_ITEMS];
  uint32_t pay[COMB_ITEMS];
#pragma unroll
  for (int j = 0; j < COMB_ITEMS; ++j) {
    uint32_t p = p0 + j;
    k[j] = p < n ? skey[p] : KEY_MAX;
    pay[j] = p < n ? spay[p] : 0;
  }
  const uint64_t kprev = (p0 > 0 && p0 <= n) ? skey[p0 - 1] : ~k[0];
  const uint64_t knext = (p0 + COMB_ITEMS < n) ? skey[p0 + COMB_ITEMS] : KEY_MAX;

  Agg mine = {0, 0};
#pragma unroll
  for (int j = 0; j < COMB_ITEMS; ++j) {
    uint32_t p = p0 + j;
    if (p < n) {
      uint64_t kp = j == 0 ? kprev : k[j - 1];
      if (p == 0 || k[j] != kp) mine.nh++;
      if (is_write(pay[j] & 3)) mine.lw = p + 1;
    }
  }
  Agg tile_tot;
  Agg bex = block_excl_scan_agg<COMB_THREADS>(mine, s_tmp, &tile_tot);

  // decoupled look-back, warp 0: 32 predecessors per step (the operator --
  // sum of heads, max of write positions -- is commutative, so a window is
  // reduced with warp shuffles once every tile up to the nearest inclusive
  // prefix has published)
  if (tid < 32) {
    const int lane = tid;
    unsigned long long* my = status + tile;
    Agg excl = {0, 0};
    if (tile == 0) {
      if (lane == 0) st_relaxed64(my, agg_pack(tile_tot, F_INC));
    } else {
      if (lane == 0) st_relaxed64(my, agg_pack(tile_tot, F_AGG));
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
      if (lane == 0) st_relaxed64(my, agg_pack(agg_op(excl, tile_tot), F_INC));
    }
    if (lane == 0) s_prefix = excl;
  }
  __syncthreads();
  Agg run = agg_op(s_prefix, bex);   // state before my first item

#pragma unroll
  for (int j = 0; j < COMB_ITEMS; ++j) {
    const uint32_t p = p0 + j;
    if (p >= n) break;
    const uint64_t key = k[j];
    const uint64_t kp = j == 0 ? kprev : k[j - 1];
    const bool head = (p == 0) || key != kp;
    const uint32_t op = pay[j] & 3;
    const uint32_t ts = pay[j] >> 2;
    run.nh += head ? 1 : 0;
    const uint32_t seg = run.nh - 1;
    // nearest earlier write in the same segment -> early result
    bool done = false;
    if (!head && run.lw > 0) {
      const uint32_t jw = run.lw - 1;
      uint64_t kw;
      uint32_t pw;
      if (jw >= p0) {           // inside my items (always same segment if no head in between)
        kw = k[jw - p0];
        pw = pay[jw - p0];
      } else {
        kw = skey[jw];
        pw = spay[jw];
      }
      if (kw == key) {
        const uint32_t opw = pw & 3;
        results[ts] = (opw == OP_DELETE) ? KEY_MAX : vals[pw >> 2];
        done = true;
      }
    }
    pinfo[p] = seg | (done ? DONE_BIT : 0u);
    if (head) istart[seg] = p;
    if (is_write(op)) run.lw = p + 1;
    const uint64_t kn = (j + 1 < COMB_ITEMS) ? k[j + 1] : knext;
    const bool tail = (p == n - 1) || kn != key;
    if (tail) {
      // issue rule: last write of the segment, else this (last) query
      bool wr = false;
      uint32_t pw = 0;
      if (run.lw > 0) {
        const uint32_t jw = run.lw - 1;
        uint64_t kw;
        if (jw >= p0) {
          kw = k[jw - p0];
          pw = pay[jw - p0];
        } else {
          kw = skey[jw];
          pw = spay[jw];
        }
        wr = (kw == key);
      }
      ikey[seg] = key;
      if (wr) {
        const uint32_t opw = pw & 3;
        iop[seg] = (uint8_t)opw;
        ival[seg] = (opw == OP_DELETE) ? KEY_MAX : vals[pw >> 2];
      } else {
        iop[seg] = OP_QUERY;
      }
      if (p == n - 1) {
        ctl->nseg = seg + 1;
        istart[seg + 1] = n;
      }
    }
  }
}

// ---------------------------------------------------------------- partition
constexpr unsigned long long P_AGG = 1ull << 62;
constexpr unsigned long long P_INC = 2ull << 62;
constexpr unsigned long long P_VAL = (1ull << 62) - 1;

__device__ __forceinline__ uint32_t block_excl_scan_u32(uint32_t v, uint32_t* tmp, uint32_t* total) {
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  uint32_t x = v;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    uint32_t y = __shfl_up_sync(FULL, x, o);
    if (lane >= o) x += y;
  }
  if (lane == 31) tmp[warp] = x;
  __syncthreads();
  uint32_t wpre = 0, tot = 0;
#pragma unroll
  for (int w = 0; w < COMB_THREADS / 32; ++w) {
    uint32_t t = tmp[w];
    if (w < warp) wpre += t;
    tot += t;
  }
  __syncthreads();
  *total = tot;
  return wpre + x - v;
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

__global__ void __launch_bounds__(COMB_THREADS) partition_kernel(
    const uint64_t* __restrict__ ikey, const uint8_t* __restrict__ iop, const uint64_t* __restrict__ ival,
    uint64_t* __restrict__ qkey, uint32_t* __restrict__ qseg, uint64_t* __restrict__ wkey, uint8_t* __restrict__ wop,
    uint64_t* __restrict__ wval, uint32_t* __restrict__ wseg, unsigned long long* __restrict__ status, Tree t,
    BatchCtl* __restrict__ ctl) {
  __shared__ uint32_t s_tile, s_tmp[COMB_THREADS / 32], s_prefix;
  const int tid = threadIdx.x;
  if (ctl->invalid) return;
  const uint32_t nseg = ctl->nseg;
  if (tid == 0) s_tile = atomicAdd(&ctl->tile_ctr[TC_PART], 1u);
  __syncthreads();
  const uint32_t tile = s_tile;
  if (tile * COMB_TILE >= nseg) return;
  const uint32_t s0 = tile * COMB_TILE + tid * COMB_ITEMS;
  uint8_t o[COMB_ITEMS];
  uint32_t mine = 0;
#pragma unroll
  for (int j = 0; j < COMB_ITEMS; ++j) {
    o[j] = (s0 + j < nseg) ? iop[s0 + j] : 0;
    mine += (s0 + j < nseg && is_write(o[j])) ? 1 : 0;
  }
  uint32_t tot;
  uint32_t bex = block_excl_scan_u32(mine, s_tmp, &tot);
  if (tid < 32) {   // warp-parallel decoupled look-back (see combine_kernel)
    const int lane = tid;
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
        for (int o = 16; o > 0; o >>= 1) a += __shfl_xor_sync(FULL, a, o);
        excl += a;
        if (inc) break;
        pt -= 32;
      }
      if (lane == 0) st_relaxed64(my, P_INC | (excl + tot));
    }
    if (lane == 0) s_prefix = excl;
    if (lane == 0 && (tile + 1) * COMB_TILE >= nseg) {   // last tile: totals + headroom check
      const uint32_t nw = excl + tot;
      ctl->nw = nw;
      ctl->nq = nseg - nw;
      if (!headroom_ok(t, nw)) ctl->status = EIRENE_EFULL;
    }
  }
  __syncthreads();
  uint32_t wb = s_prefix + bex;
#pragma unroll
  for (int j = 0; j < COMB_ITEMS; ++j) {
    const uint32_t s = s0 + j;
    if (s >= nseg) break;
    if (is_write(o[j])) {
      wkey[wb] = ikey[s];
      wop[wb] = o[j];
      wval[wb] = ival[s];
      wseg[wb] = s;
      ++wb;
    } else {
      const uint32_t q = s - wb;
      qkey[q] = ikey[s];
      qseg[q] = s;
    }
  }
}

// ---------------------------------------------------------------- RESULT_CAL
// Alg.1:6: positions without an earlier write in their segment take the value
// their segment's issued request retrieved (old[seg]); results are scattered
// back to submission (timestamp) order.
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
                                                           uint64_t* __restrict__ results,
                                                           const BatchCtl* __restrict__ ctl) {
  if (ctl->invalid || ctl->status != 0) return;
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

void launch_combine(const uint64_t* skey, const uint32_t* spay, const uint64_t* vals, uint64_t* results, uint32_t n,
                    const CombBufs& c, BatchCtl* ctl, cudaStream_t st, int* launches) {
  const uint32_t tiles = (n + COMB_TILE - 1) / COMB_TILE;
  combine_kernel<<<tiles, COMB_THREADS, 0, st>>>(skey, spay, vals, results, n, c.pinfo, c.ikey, c.iop, c.ival,
                                                 c.istart, c.comb_status, ctl);
  ++*launches;
}

void launch_partition(uint32_t n, const CombBufs& c, Tree t, BatchCtl* ctl, cudaStream_t st, int* launches) {
  const uint32_t tiles = (n + COMB_TILE - 1) / COMB_TILE;
  partition_kernel<<<tiles, COMB_THREADS, 0, st>>>(c.ikey, c.iop, c.ival, c.qkey, c.qseg, c.wkey, c.wop, c.wval,
                                                   c.wseg, c.part_status, t, ctl);
  ++*launches;
}

void launch_result(const uint32_t* spay, uint32_t n, const CombBufs& c, uint64_t* results, BatchCtl* ctl,
                   cudaStream_t st, int* launches) {
  (void)n;
  result_long_kernel<<<148, 256, 0, st>>>(spay, c.pinfo, c.istart, c.longseg, c.old, results, ctl);
  ++*launches;
}

}  // namespace eirene
