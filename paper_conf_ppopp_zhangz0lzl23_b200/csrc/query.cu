// query.cu -- QUERY_KERNEL (Alg.1:15-21), leaf locate for the issued writes,
// and the fused RESULT_CAL (Alg.1:6) for short segments.
//
// Issued queries run with no concurrency control: the tree is
// quiescent (the update kernel of the previous batch has finished, and this
// batch's update kernel runs after this one).  Each thread owns
// one issued request; the issued list is key-sorted, so the 32 lanes of a warp
// walk overlapping root-to-leaf paths and their 256-bit loads of shared upper
// nodes coalesce into one L1/L2 request per distinct node (the B200 analogue
// of Harmonia's path sharing / NTG).  Inner levels (<= 18 MB at
// 2^24 keys) stay L2-resident across batches; leaves (256 MiB) come from HBM:
// one 128 B key line plus one 32 B value sector per issued query.
//
// The same traversal gives each issued write its target leaf and slot (a4,
// the input of the leaf-run regrouping in the update kernel) and the value
// its key holds before the batch ("the old (original) value ... retrieved by
// the issued request").  Issued keys are distinct, so no other
// request of the batch can change that value before the update kernel runs.
//
// RESULT_CAL: the un-issued requests of a segment that have no
// earlier write take the retrieved value.  The thread that retrieved it
// scatters it to its segment's pending positions (results in timestamp
// order); segments longer than SHORT_SEG are queued for result_long_kernel.
#include "eirene_internal.cuh"
#include <cstdio>

namespace eirene {

namespace {

__device__ __forceinline__ ulonglong4 ldg256(const uint64_t* p) {
  ulonglong4 v;
  asm volatile("ld.global.nc.v4.u64 {%0,%1,%2,%3}, [%4];" : "=l"(v.x), "=l"(v.y), "=l"(v.z), "=l"(v.w) : "l"(p));
  return v;
}
// Slot of key k in a 16-key leaf line (4 x 256-bit loads), -1 if absent.
__device__ __forceinline__ int slot16(const uint64_t* __restrict__ line, uint64_t k) {
  ulonglong4 v[4];
#pragma unroll
  for (int i = 0; i < 4; ++i) v[i] = ldg256(line + 4 * i);
  int s = -1;
#pragma unroll
  for (int i = 0; i < 4; ++i) {
    if (v[i].x == k) s = 4 * i;
    if (v[i].y == k) s = 4 * i + 1;
    if (v[i].z == k) s = 4 * i + 2;
    if (v[i].w == k) s = 4 * i + 3;
  }
  return s;
}

__global__ void __launch_bounds__(256, 8) query_kernel(const uint64_t* __restrict__ qkey,
                                                        const uint32_t* __restrict__ qseg,
                                                        const uint64_t* __restrict__ wkey,
                                                        const uint32_t* __restrict__ wseg, uint32_t* __restrict__ wleaf,
                                                        uint8_t* __restrict__ wslot, uint64_t* __restrict__ old,
                                                        const uint32_t* __restrict__ spay,
                                                        const uint32_t* __restrict__ pinfo,
                                                        const uint32_t* __restrict__ istart,
                                                        uint32_t* __restrict__ longseg, const BatchArgs* __restrict__ A,
                                                        Tree t, BatchCtl* __restrict__ ctl) {
  if (ctl->invalid || ctl->status != 0) return;
  uint64_t* __restrict__ results = A->results;
  const uint32_t nq = ctl->nq, nw = ctl->nw, total = nq + nw;
  const unsigned long long rw = t.hdr->root_word;
  const uint32_t height = (uint32_t)(rw >> 32), root = (uint32_t)rw;
  const uint32_t stride = gridDim.x * blockDim.x;
  for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < total; i += stride) {
    const bool isq = i < nq;
    const uint64_t k = isq ? qkey[i] : wkey[i - nq];
    uint32_t node = root;
    for (uint32_t lvl = height - 1; lvl > 0; --lvl) {
      // a 128 B separator line is four 256-bit loads (LDG.E.ENL2.256), then
      // the one child pointer: loading the whole child line alongside the keys
      // (one round trip per level instead of two) measured slower, as did two
      // or four interleaved traversals per thread (tools/ab.py)
      const uint64_t* kl = t.ikeys + (size_t)node * FAN;
      ulonglong4 kv[4];
#pragma unroll
      for (int x = 0; x < 4; ++x) kv[x] = ldg256(kl + 4 * x);
      uint32_t c = 0;
#pragma unroll
      for (int x = 0; x < 4; ++x) c += (kv[x].x <= k) + (kv[x].y <= k) + (kv[x].z <= k) + (kv[x].w <= k);
      node = __ldg(t.ichild + (size_t)node * FAN + c);
    }
    const int s = slot16(t.lkeys + (size_t)node * LSTRIDE, k);
    const uint64_t v = s >= 0 ? __ldg(t.lvals + (size_t)node * LSTRIDE + s) : KEY_MAX;
    uint32_t seg;
    if (isq) {
      seg = qseg[i];
    } else {
      const uint32_t w = i - nq;
      seg = wseg[w];
      wleaf[w] = node;
      wslot[w] = s >= 0 ? (uint8_t)s : (uint8_t)255;
    }
    old[seg] = v;
    const uint32_t p0 = istart[seg], p1 = istart[seg + 1];
    if (p1 - p0 <= SHORT_SEG) {
      if (isq) {   // an all-query segment: every position is pending
        for (uint32_t p = p0; p < p1; ++p) results[spay[p] >> 2] = v;
      } else {     // positions up to (and including) the first write are pending
        for (uint32_t p = p0; p < p1; ++p)
          if (!(pinfo[p] & DONE_BIT)) results[spay[p] >> 2] = v;
      }
    } else {
      longseg[atomicAdd(&ctl->nlong, 1u)] = seg;
    }
  }
}

// RESULT_CAL is fused into the query kernel: every issued request scatters
// the value it retrieved to the pending positions of its own segment.  The
// segments longer than SHORT_SEG (hot keys) are queued instead and finished
// here with one CTA per segment, so a 56K-request Zipf key does not serialise
// one thread.
__global__ void __launch_bounds__(1024) result_long_kernel(const uint32_t* __restrict__ spay,
                                                            const uint32_t* __restrict__ pinfo,
                                                            const uint32_t* __restrict__ istart,
                                                            const uint32_t* __restrict__ longseg,
                                                            const uint64_t* __restrict__ old,
                                                            const BatchArgs* __restrict__ A,
                                                            BatchCtl* __restrict__ ctl, const TreeHdr* hdr,
                                                            int dbgprint) {
  if (blockIdx.x == 0 && threadIdx.x == 0) {
    // end of the batch (the last kernel; nothing below changes ctl): final
    // status and height, then the whole BatchCtl to the batch's ring slot
    if (ctl->invalid) ctl->status = EIRENE_EINVAL;
    ctl->height = (uint32_t)(hdr->root_word >> 32);
    *A->ctl_out = *ctl;
    if (dbgprint)
      printf("[eirene dbg] %u %u %u %u %u %u %u %u\n", ctl->dbg[0], ctl->dbg[1], ctl->dbg[2], ctl->dbg[3],
             ctl->dbg[4], ctl->dbg[5], ctl->dbg[6], ctl->dbg[7]);
  }
  if (ctl->invalid || ctl->status != 0) return;
  uint64_t* __restrict__ results = A->results;
  const uint32_t nl = ctl->nlong;
  for (uint32_t x = blockIdx.x; x < nl; x += gridDim.x) {
    const uint32_t s = longseg[x];
    const uint64_t v = old[s];
    const uint32_t e = istart[s + 1];
    for (uint32_t p0 = istart[s] + threadIdx.x; p0 < e; p0 += 8 * blockDim.x) {   // 8 loads in flight
      uint32_t pi[8], py[8];
#pragma unroll
      for (int u = 0; u < 8; ++u) {
        const uint32_t p = p0 + u * blockDim.x;
        pi[u] = p < e ? pinfo[p] : DONE_BIT;
        py[u] = p < e ? spay[p] : 0u;
      }
#pragma unroll
      for (int u = 0; u < 8; ++u)
        if (!(pi[u] & DONE_BIT)) results[py[u] >> 2] = v;
    }
  }
}

// ---------------------------------------------------------------- range queries
// R(l, u) at timestamp t (§4.1.2).  Range queries are
// not sorted or combined; each one reads the pre-batch tree (this kernel runs
// after the query kernel and before the update kernel, the query-kernel phase
// of P:1066-1074) and merges two key-ordered streams:
//   * the tree's pairs in [l, u]: leaf of l by the same descent as the query
//     kernel, then the leaf chain until a leaf's hi fence
//     passes u -- the range's result "in the original manner";
//   * the batch's written keys in [l, u]: the issued-write list is
//     key-sorted (one entry per key with update requests), found by binary
//     search.  Each such key k takes the result of the "artificial query"
//     Qr(k)@t: k's segment is timestamp-ordered, so a binary
//     search finds where t would be inserted; the request just before that
//     point decides -- a write gives its value (NOT_FOUND for a delete), a
//     query gives its own result (its early result when a write precedes it
//     in the segment, else the pre-batch value), no request gives the
//     pre-batch value.  NOT_FOUND drops k from the range, a value adds or
//     replaces it (reading R2).
// The first `cap` merged pairs are written to the request's row of the range
// output; results[t] = pairs written.  One thread per range query.
__device__ __forceinline__ uint64_t artificial_query(uint32_t w, uint32_t t, uint64_t pre,
                                                     const uint32_t* __restrict__ wseg,
                                                     const uint32_t* __restrict__ istart,
                                                     const uint32_t* __restrict__ spay,
                                                     const uint32_t* __restrict__ pinfo,
                                                     const uint64_t* __restrict__ vals,
                                                     const uint64_t* __restrict__ results) {
  const uint32_t seg = wseg[w];
  uint32_t lo = istart[seg], hi = istart[seg + 1];
  const uint32_t p0 = lo;
  while (lo < hi) {   // first position with timestamp > t
    const uint32_t mid = (lo + hi) >> 1;
    if ((spay[mid] >> 2) < t) lo = mid + 1;
    else hi = mid;
  }
  if (lo == p0) return pre;
  const uint32_t pj = spay[lo - 1];
  const uint32_t op = pj & 3;
  if (op == OP_DELETE) return KEY_MAX;
  if (op != OP_QUERY) return vals[pj >> 2];
  return (pinfo[lo - 1] & DONE_BIT) ? ld_cg(results + (pj >> 2)) : pre;
}

__global__ void __launch_bounds__(256) range_kernel(uint32_t n, const uint64_t* __restrict__ wkey,
                                                    const uint32_t* __restrict__ wseg,
                                                    const uint32_t* __restrict__ spay,
                                                    const uint32_t* __restrict__ pinfo,
                                                    const uint32_t* __restrict__ istart,
                                                    const BatchArgs* __restrict__ A, Tree t, BatchCtl* __restrict__ ctl) {
  if (ctl->invalid || ctl->status != 0 || ctl->nrange == 0) return;
  const uint8_t* __restrict__ ops = A->ops;
  const uint64_t* __restrict__ keys = A->keys;
  const uint64_t* __restrict__ vals = A->vals;
  uint64_t* __restrict__ results = A->results;
  uint64_t* __restrict__ rkeys = A->rkeys;
  uint64_t* __restrict__ rvals = A->rvals;
  const uint32_t cap = A->rcap;
  const uint32_t nw = ctl->nw;
  const unsigned long long rw = t.hdr->root_word;
  const uint32_t height = (uint32_t)(rw >> 32), root = (uint32_t)rw;
  uint32_t nart = 0;
  const uint32_t stride = gridDim.x * blockDim.x;
  for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += stride) {
    if (ops[i] != OP_RANGE) continue;
    const uint64_t l = keys[i], u = vals[i];
    uint64_t* __restrict__ ok = rkeys + (size_t)i * cap;
    uint64_t* __restrict__ ov = rvals + (size_t)i * cap;
    uint32_t c = 0;
    if (l <= u && l != KEY_MAX) {   // (no key is UINT64_MAX; the descent needs l < the separator padding)
      // written keys >= l: lower_bound over the key-sorted issued writes
      uint32_t w = 0, whi = nw;
      while (w < whi) {
        const uint32_t mid = (w + whi) >> 1;
        if (wkey[mid] < l) w = mid + 1;
        else whi = mid;
      }
      uint64_t wk = w < nw ? wkey[w] : KEY_MAX;
      // leaf of l
      uint32_t node = root;
      for (uint32_t lvl = height - 1; lvl > 0; --lvl) {
        const uint64_t* kl = t.ikeys + (size_t)node * FAN;
        ulonglong4 kv[4];
#pragma unroll
        for (int x = 0; x < 4; ++x) kv[x] = ldg256(kl + 4 * x);
        uint32_t cc = 0;
#pragma unroll
        for (int x = 0; x < 4; ++x) cc += (kv[x].x <= l) + (kv[x].y <= l) + (kv[x].z <= l) + (kv[x].w <= l);
        node = __ldg(t.ichild + (size_t)node * FAN + cc);
      }
      // merge the leaf chain with the written keys
      bool more = true;
      while (more && c < cap) {
        const uint64_t* lk = t.lkeys + (size_t)node * LSTRIDE;
        ulonglong4 kv[4];
#pragma unroll
        for (int x = 0; x < 4; ++x) kv[x] = ldg256(lk + 4 * x);
        uint32_t s = 0;   // first slot with key >= l (keys ascending, KEY_MAX padded)
#pragma unroll
        for (int x = 0; x < 4; ++x) s += (kv[x].x < l) + (kv[x].y < l) + (kv[x].z < l) + (kv[x].w < l);
        for (; s < FAN && c < cap; ++s) {
          const uint64_t k = __ldg(lk + s);
          if (k == KEY_MAX) break;   // end of this leaf's keys: go on to the next leaf
          if (k > u) {
            more = false;
            break;
          }
          // written keys before k are absent from the pre-batch tree
          while (wk < k && c < cap) {
            const uint64_t v = artificial_query(w, i, KEY_MAX, wseg, istart, spay, pinfo, vals, results);
            ++nart;
            if (v != KEY_MAX) {
              ok[c] = wk;
              ov[c] = v;
              ++c;
            }
            ++w;
            wk = w < nw ? wkey[w] : KEY_MAX;
          }
          if (c >= cap) break;
          uint64_t v = __ldg(t.lvals + (size_t)node * LSTRIDE + s);
          if (wk == k) {
            v = artificial_query(w, i, v, wseg, istart, spay, pinfo, vals, results);
            ++nart;
            ++w;
            wk = w < nw ? wkey[w] : KEY_MAX;
          }
          if (v != KEY_MAX) {
            ok[c] = k;
            ov[c] = v;
            ++c;
          }
        }
        if (!more || c >= cap) break;
        const NodeMeta* m = t.lmeta + node;
        const uint64_t hi = __ldg(&m->hi);
        const uint32_t nx = __ldg(&m->next);
        if (hi > u || hi == KEY_MAX || nx == NIL) break;   // every later key is > u
        node = nx;
      }
      // written keys after the last tree key in range
      while (w < nw && wk <= u && c < cap) {   // (u may be UINT64_MAX, the no-more-writes sentinel)
        const uint64_t v = artificial_query(w, i, KEY_MAX, wseg, istart, spay, pinfo, vals, results);
        ++nart;
        if (v != KEY_MAX) {
          ok[c] = wk;
          ov[c] = v;
          ++c;
        }
        ++w;
        wk = w < nw ? wkey[w] : KEY_MAX;
      }
    }
    results[i] = c;
  }
  nart = __reduce_add_sync(FULL, nart);
  if (nart && (threadIdx.x & 31) == 0) atomicAdd(&ctl->nart, nart);
}

}  // namespace

void launch_query(uint32_t n, const CombBufs& c, const uint32_t* spay, const BatchArgs* A, Tree t, BatchCtl* ctl,
                  int num_sms, cudaStream_t st, int* launches) {
  // one resident wave: 8 CTAs of 256 threads per SM at <= 32 registers
  int blocks = (int)std::min<uint32_t>((n + 255) / 256, (uint32_t)num_sms * 8u);
  if (blocks < 1) blocks = 1;
  query_kernel<<<blocks, 256, 0, st>>>(c.qkey, c.qseg, c.wkey, c.wseg, c.wleaf, c.wslot, c.old, spay, c.pinfo,
                                       c.istart, c.longseg, A, t, ctl);
  ++*launches;
}

void launch_range(uint32_t n, const CombBufs& c, const uint32_t* spay, const BatchArgs* A, Tree t, BatchCtl* ctl,
                  int num_sms, cudaStream_t st, int* launches) {
  int blocks = (int)std::min<uint32_t>((n + 255) / 256, (uint32_t)num_sms * 8u);
  if (blocks < 1) blocks = 1;
  range_kernel<<<blocks, 256, 0, st>>>(n, c.wkey, c.wseg, spay, c.pinfo, c.istart, A, t, ctl);
  ++*launches;
}

void launch_result(const uint32_t* spay, uint32_t n, const CombBufs& c, const BatchArgs* A, BatchCtl* ctl,
                   const TreeHdr* hdr, int dbgprint, cudaStream_t st, int* launches) {
  (void)n;
  result_long_kernel<<<64, 1024, 0, st>>>(spay, c.pinfo, c.istart, c.longseg, c.old, A, ctl, hdr, dbgprint);
  ++*launches;
}

}  // namespace eirene
