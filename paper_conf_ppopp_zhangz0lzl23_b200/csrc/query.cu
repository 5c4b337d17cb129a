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
// order); segments longer than SHORT_SEG are queued for the update kernel's result phase.
#include "eirene_internal.cuh"
#include <cstdio>
#include <cstdlib>

namespace eirene {

namespace {

// Child index of key k in inner node `node`: its separator line (Line16:
// 256-bit loads, L1-allocating -- lanes of neighbouring warps walk shared upper
// nodes -- with an L2 policy, evict_last: re-read every batch).
__device__ __forceinline__ uint32_t child_slot(const Tree& t, uint32_t node, uint64_t k, uint64_t pol) {
  Line16 l;
  l.load_l1(t.ikeys + (size_t)node * FAN, pol);
  return l.count_le(k);
}
// The value of a located key (one 32 B value sector of its leaf).  A/B builds:
// -DEIRENE_VAL_LOAD=1: L1 no-allocate; 2: plain coherent load; 0 (default):
// read-only path with the evict_first L2 policy.
#ifndef EIRENE_CHILD_PF
#define EIRENE_CHILD_PF 0   // A/B: prefetch each inner node's child line into L1 with its separators
#endif
#ifndef EIRENE_QRUN
#define EIRENE_QRUN 0       // A/B: contiguous per-thread runs of the issued list instead of a grid stride
#endif
#ifndef EIRENE_VAL_LOAD
#define EIRENE_VAL_LOAD 4   // r2u: the default fetch of a value sector was 128 B (207 -> 174 MB per cfg2 launch)
#endif
__device__ __forceinline__ uint64_t load_value(const tkey_t* p, uint64_t pol) {
#if EIRENE_VAL_LOAD == 1
  if constexpr (sizeof(tkey_t) == 8) {
    uint64_t v;
    asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.u64 %0, [%1], %2;" : "=l"(v) : "l"(p), "l"(pol));
    return v;
  } else {
    uint32_t v;
    asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.u32 %0, [%1], %2;" : "=r"(v) : "l"(p), "l"(pol));
    return v;
  }
#elif EIRENE_VAL_LOAD == 4
  return ldg64_pol_64b(p, pol);
#elif EIRENE_VAL_LOAD == 2
  (void)pol;
  return *p;
#else
  return ldg64_pol(p, pol);
#endif
}

// Slot of key k in a 16-key leaf line (256-bit loads, L2 evict_first: leaves
// are touched once per batch), -1 if absent.
__device__ __forceinline__ int slot16(const tkey_t* __restrict__ line, uint64_t k, uint64_t pol) {
  Line16 l;
  l.load(line, pol);
  return l.find(k);
}

#ifndef EIRENE_QCOOP
#ifdef EIRENE_KEY32
#define EIRENE_QCOOP 0   // (32-bit keys: a leaf line is two sectors; A/B pending)
#else
#define EIRENE_QCOOP 1   // warp-cooperative leaf search (r3h: cfg2 query 56.8 -> 54.6 us; 0 = per-lane line loads)
#endif
#endif
// Warp-cooperative leaf search: the 32 lanes' leaves are read KPL lanes per
// leaf line (each lane one 32 B sector), 32/KPL leaves per 256-bit load
// instruction, so every L1 tag lookup of a leaf load serves a whole line
// instead of one sector of 32 different lines; the KPL lanes of a leaf compare
// their keys with the owner's key (shuffled) and the owner collects the slot
// by ballot.  All KPL loads are issued before any compare.
__device__ __forceinline__ int slot16_coop(const tkey_t* __restrict__ lkeys, uint32_t node, uint64_t k, uint64_t pol) {
  constexpr int KPL = FAN * (int)sizeof(tkey_t) / 32;   // lanes per leaf line: 4 (u64 keys) or 2 (u32)
  constexpr int LPR = 32 / KPL;                          // leaves per round
  constexpr int KPW = 32 / (int)sizeof(tkey_t);          // keys per 32 B sector
  const uint32_t lane = threadIdx.x & 31u, g = lane / KPL, part = lane % KPL;
  ulonglong4 q[KPL];
  uint64_t kt[KPL];
#pragma unroll
  for (int r = 0; r < KPL; ++r) {
    const uint32_t src = LPR * r + g;
    const uint32_t leaf = __shfl_sync(FULL, node, src);
    kt[r] = __shfl_sync(FULL, k, src);
    q[r] = ldg256_pol(reinterpret_cast<const uint64_t*>(lkeys + (size_t)leaf * LSTRIDE) + 4 * part, pol);
  }
  int s = -1;
  const uint32_t my_r = lane / LPR, my_g = lane % LPR;
#pragma unroll
  for (int r = 0; r < KPL; ++r) {
    const uint64_t w[4] = {q[r].x, q[r].y, q[r].z, q[r].w};
    int li = -1;
#pragma unroll
    for (int y = 0; y < 4; ++y) {
      if constexpr (sizeof(tkey_t) == 8) {
        if (w[y] == kt[r]) li = y;
      } else {
        if ((w[y] & 0xFFFFFFFFull) == kt[r]) li = 2 * y;
        if ((w[y] >> 32) == kt[r]) li = 2 * y + 1;
      }
    }
    const uint32_t b = __ballot_sync(FULL, li >= 0);
    const uint32_t bits = (b >> (KPL * my_g)) & ((1u << KPL) - 1u);
    const int sub = bits ? __ffs(bits) - 1 : 0;
    const int lsrc = __shfl_sync(FULL, li, KPL * my_g + sub);
    if ((int)my_r == r && bits) s = sub * KPW + lsrc;
  }
  return s;
}

// Everything after the locate of issued request i (list position i < nq:
// query, else write i - nq) at leaf `node`, slot s (-1 = absent), value v:
// the write's leaf/slot for the update kernel, the segment's old value, and
// the fused RESULT_CAL of its pending positions (long segments queued).
struct QueryIO {
  const uint32_t* __restrict__ qseg;
  const uint32_t* __restrict__ wseg;
  const uint8_t* __restrict__ wop;
  uint64_t* __restrict__ wval;      // in: the issued write's timestamp; out: its value (WVAL_TS)
  const tkey_t* __restrict__ vals;  // the batch's values
  uint32_t* __restrict__ wleaf;
  uint8_t* __restrict__ wslot;
  uint64_t* __restrict__ old;
  const uint32_t* __restrict__ spay;
  const uint32_t* __restrict__ pinfo;
  const uint32_t* __restrict__ istart;
  uint32_t* __restrict__ longseg;
};

// A/B switch for the query kernel's result stores (EIRENE_RES_ST): 0 plain,
// 1 L2 evict_last (a result sector stays in L2 until its four results are
// written instead of being written back partially), 2 none (diagnostic:
// wrong results, traffic only)
#ifndef EIRENE_RES_ST
#define EIRENE_RES_ST 0
#endif
__device__ __forceinline__ void st_result(tkey_t* p, uint64_t v) {
#if EIRENE_RES_ST == 1
  st64_pol(p, v, pol_evict_last());
#elif EIRENE_RES_ST == 2
  (void)p; (void)v;
#else
  *p = (tkey_t)v;
#endif
}

// The CTA's structural-write counts (nins, ndelp): zeroed by q_zero before the
// first retire, added to the BatchCtl by q_flush after the last (both by every
// thread of the CTA: they synchronise it).
__device__ __forceinline__ uint32_t* q_counts() {
  __shared__ uint32_t qc[2];
  return qc;
}
__device__ __forceinline__ void q_zero() {
  if (threadIdx.x < 2) q_counts()[threadIdx.x] = 0;
  __syncthreads();
}
__device__ __forceinline__ void q_flush(BatchCtl* ctl) {
  __syncthreads();
  const uint32_t* qc = q_counts();
  if (threadIdx.x == 0) {
    if (qc[0]) atomicAdd(&ctl->nins, qc[0]);
    if (qc[1]) atomicAdd(&ctl->ndelp, qc[1]);
  }
}

__device__ __forceinline__ void retire(const QueryIO& io, uint32_t i, bool isq, uint32_t nq, uint32_t node, int s,
                                       uint64_t v, tkey_t* __restrict__ results, BatchCtl* __restrict__ ctl,
                                       tkey_t* __restrict__ lvals) {
  const uint32_t* __restrict__ qseg = io.qseg;
  const uint32_t* __restrict__ wseg = io.wseg;
  const uint8_t* __restrict__ wop = io.wop;
  uint32_t* __restrict__ wleaf = io.wleaf;
  uint8_t* __restrict__ wslot = io.wslot;
  uint64_t* __restrict__ old = io.old;
  const uint32_t* __restrict__ spay = io.spay;
  const uint32_t* __restrict__ pinfo = io.pinfo;
  const uint32_t* __restrict__ istart = io.istart;
  uint32_t* __restrict__ longseg = io.longseg;
  uint32_t seg;
  bool ins = false;    // an upsert of an absent key: the only request that can split a leaf
  bool delp = false;   // a delete of a present key: removes a key from its leaf
  if (isq) {
    seg = qseg[i];
    if (seg & Q_SINGLE) {   // the segment's only request: its result, nothing else
      st_result(results + (seg & ~Q_SINGLE), v);
      return;
    }
  } else {
    const uint32_t w = i - nq;
    seg = wseg[w];
    wleaf[w] = node;
    wslot[w] = s >= 0 ? (uint8_t)s : (uint8_t)255;
    const uint32_t op = wop[w];
    ins = s < 0 && op != OP_DELETE;
    delp = s >= 0 && op == OP_DELETE;
    // WVAL_TS: the group kernel left the issued write's timestamp in wval; its
    // value is gathered from the batch here (off the group kernel's critical
    // path) and stored back for the update kernel
    const uint64_t wv = op == OP_DELETE ? KEY_MAX : ldg64_64b(io.vals + io.wval[w]);
    io.wval[w] = wv;
    // A value overwrite (upsert of a present key) changes one value slot and
    // nothing else, so it is applied here, by the thread that located it: the
    // structure is quiescent during this kernel (the update kernel runs after
    // it), issued keys are distinct (one issued request per key,
    // P:728-745), so no concurrent issued query reads this slot, and v above
    // is already the pre-batch value the write returns.  The update kernel
    // then only has the structural writes (inserts of absent keys, deletes of
    // present ones) to do, and re-applies overwrites idempotently.
    if (s >= 0 && op != OP_DELETE) lvals[(size_t)node * LSTRIDE + s] = wv;
  }
  {   // counted per CTA in shared memory (q_counts), added to ctl once per CTA (q_flush): one global
      // atomic per warp on the same word serialised in L2 under insert-heavy batches
    const uint32_t am = __activemask();
    const uint32_t m = __ballot_sync(am, ins), md = __ballot_sync(am, delp);
    uint32_t* qc = q_counts();
    if (m && (threadIdx.x & 31) == __ffs(m) - 1) atomicAdd(&qc[0], (uint32_t)__popc(m));
    if (md && (threadIdx.x & 31) == __ffs(md) - 1) atomicAdd(&qc[1], (uint32_t)__popc(md));
  }
  // old[seg] (the pre-batch value) is read by the result phase for long
  // segments and by the range kernel for written keys only
  if (!isq) old[seg] = v;
  const uint32_t p0 = istart[seg], p1 = istart[seg + 1];
  if (p1 - p0 <= SHORT_SEG) {
    if (isq) {   // an all-query segment: every position is pending
      for (uint32_t p = p0; p < p1; ++p) st_result(results + (spay[p] >> 2), v);
    } else {     // positions up to (and including) the first write are pending
      for (uint32_t p = p0; p < p1; ++p)
        if (!(pinfo[p] & DONE_BIT)) st_result(results + (spay[p] >> 2), v);
    }
  } else {   // work items of RCHUNK positions: (segment, chunk) pairs
    if (isq) old[seg] = v;
    const uint32_t nc = (p1 - p0 + RCHUNK - 1) / RCHUNK;
    const uint32_t at = atomicAdd(&ctl->nlong, nc);
    for (uint32_t c = 0; c < nc; ++c) {
      longseg[2 * (at + c)] = seg;
      longseg[2 * (at + c) + 1] = c;
    }
  }
}

__device__ __forceinline__ void query_body(const uint64_t* __restrict__ qkey,
                                                        const uint32_t* __restrict__ qseg,
                                                        const uint64_t* __restrict__ wkey,
                                                        const uint32_t* __restrict__ wseg,
                                                        const uint8_t* __restrict__ wop,
                                                        uint64_t* __restrict__ wval, uint32_t* __restrict__ wleaf,
                                                        uint8_t* __restrict__ wslot, uint32_t* __restrict__ wparent,
                                                        uint64_t* __restrict__ old,
                                                        const uint32_t* __restrict__ spay,
                                                        const uint32_t* __restrict__ pinfo,
                                                        const uint32_t* __restrict__ istart,
                                                        uint32_t* __restrict__ longseg, const BatchArgs* __restrict__ A,
                                                        Tree t, BatchCtl* __restrict__ ctl) {
  if (ctl->invalid || ctl->status != 0) return;
  tkey_t* __restrict__ results = A->results;
  const uint32_t nq = ctl->nq, nw = ctl->nw, total = nq + nw;
  // pool headroom for the batch's worst case (every CTA computes the same
  // answer from the same tree header: none of them changes anything if it fails)
  if (!headroom_ok(t, nw)) {
    if (blockIdx.x == 0 && threadIdx.x == 0) ctl->status = EIRENE_EFULL;
    return;
  }
  q_zero();
  const unsigned long long rw = t.hdr->root_word;
  const uint32_t height = (uint32_t)(rw >> 32), root = (uint32_t)rw;
  const uint64_t pl = pol_evict_last(), pf = pol_evict_first();
#if EIRENE_QCOOP
  // Warp-uniform steps of 32 consecutive issued requests (lanes with i >= total
  // ride along with a dummy key, so the leaf search can shuffle over the warp)
  const uint32_t lane = threadIdx.x & 31u;
  const uint32_t wstride = gridDim.x * blockDim.x;
  for (uint32_t i0 = blockIdx.x * blockDim.x + (threadIdx.x & ~31u); i0 < total; i0 += wstride) {
    const uint32_t i = i0 + lane;
    const bool valid = i < total;
    const bool isq = i < nq;
    const uint64_t k = !valid ? 0ull : isq ? qkey[i] : wkey[i - nq];
#elif EIRENE_QRUN
  // every thread takes a contiguous run of the key-sorted list: its next key
  // is the neighbour of the last one, so the inner nodes it walks again (the
  // level-1 and level-2 nodes, L2 round trips on a first visit) are L1 hits
  const uint32_t nth = gridDim.x * blockDim.x, per = (total + nth - 1) / nth;
  const uint32_t i0 = (blockIdx.x * blockDim.x + threadIdx.x) * per, i1 = min(total, i0 + per);
  for (uint32_t i = i0; i < i1; ++i) {
#else
  const uint32_t stride = gridDim.x * blockDim.x;
  for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < total; i += stride) {
#endif
#if !EIRENE_QCOOP
    const bool isq = i < nq;
    const uint64_t k = isq ? qkey[i] : wkey[i - nq];
#endif
    uint32_t node = root, parent = NIL;
    for (uint32_t lvl = height - 1; lvl > 0; --lvl) {
      parent = node;   // after the loop: the leaf's parent (the level-1 node)
#if EIRENE_CHILD_PF
      // the node's 64 B child line into L1 while its separators are in flight,
      // so the dependent child load below is an L1 hit, not a second L2 round trip
      asm volatile("prefetch.global.L1 [%0];" ::"l"(t.ichild + (size_t)node * FAN));
#endif
      // a 128 B separator line is four 256-bit loads (LDG.E.ENL2.256), then
      // the one child pointer: loading the whole child line alongside the keys
      // (one round trip per level instead of two) measured slower, as did two
      // or four interleaved traversals per thread (tools/ab.py)
      node = ldg32_pol(t.ichild + (size_t)node * FAN + child_slot(t, node, k, pl), pl);
    }
#if defined(EIRENE_QDIAG) && EIRENE_QDIAG == 2   // diagnostic (traffic only, wrong results): no leaf loads
    const int s = -1;
#elif EIRENE_QCOOP
    const int s = slot16_coop(t.lkeys, node, k, pf);
#else
    const int s = slot16(t.lkeys + (size_t)node * LSTRIDE, k, pf);
#endif
#if defined(EIRENE_QDIAG) && EIRENE_QDIAG == 1   // diagnostic: no value load
    const uint64_t v = s >= 0 ? 0ull : KEY_MAX;
#else
    const uint64_t v = s >= 0 ? load_value(t.lvals + (size_t)node * LSTRIDE + s, pf) : KEY_MAX;
#endif
#if EIRENE_QCOOP
    if (!valid) continue;
#endif
    if (!isq) wparent[i - nq] = parent;   // (the parent hint of the update kernel's first level)
    retire(QueryIO{qseg, wseg, wop, wval, A->vals, wleaf, wslot, old, spay, pinfo, istart, longseg}, i, isq, nq, node, s, v,
           results, ctl, t.lvals);
  }
  q_flush(ctl);
}

// End of the query kernel in graph mode (cond != 0): its last CTA decides
// whether the batch's update kernel -- a conditional graph node -- runs at all
// (structural writes, long segments or deferred hot keys left); if not, it ends
// the batch itself (publish_batch), so a read-mostly batch is four kernels.
__device__ __forceinline__ void query_end(BatchCtl* ctl, const BatchArgs* A, const TreeHdr* hdr,
                                          cudaGraphConditionalHandle cond) {
  if (!last_cta(ctl->qfin_sub, &ctl->qfin_ctr)) return;
  __shared__ uint32_t s_need;
  if (threadIdx.x == 0) {
    s_need = update_needed(ctl, A) ? 1u : 0u;
    if (s_need) cudaGraphSetConditional(cond, 1u);
  }
  __syncthreads();
  if (!s_need) publish_batch(ctl, A, hdr);
}

// The graph-mode variant with the conditional update node (EIRENE_COND) is a
// kernel of its own: a kernel that references the device graph API is not
// profiled by ncu inside a graph, and the default path should be.
#ifndef EIRENE_QTHREADS
#define EIRENE_QTHREADS 256   // query-kernel CTA size (A/B builds: 768 with EIRENE_QMINB=2)
#endif
#ifndef EIRENE_QMINB
#ifdef EIRENE_KEY32
#define EIRENE_QMINB 8   // resident CTAs per SM the query kernel's registers are fitted to (8: 32 registers)
#else
#define EIRENE_QMINB 6   // (64-bit keys, cooperative leaf search: 40 registers; r3r: 8 / 6 / 5 / 4 CTAs per SM ->
                         // cfg2 9.20 / 9.26 / 9.12 / 9.13 G req/s, cfg3 query 43.4 -> 40.9 us at 6)
#endif
#endif
__global__ void __launch_bounds__(EIRENE_QTHREADS, EIRENE_QMINB) query_kernel(const uint64_t* __restrict__ qkey,
                                                        const uint32_t* __restrict__ qseg,
                                                        const uint64_t* __restrict__ wkey,
                                                        const uint32_t* __restrict__ wseg,
                                                        const uint8_t* __restrict__ wop,
                                                        uint64_t* __restrict__ wval, uint32_t* __restrict__ wleaf,
                                                        uint8_t* __restrict__ wslot, uint32_t* __restrict__ wparent,
                                                        uint64_t* __restrict__ old,
                                                        const uint32_t* __restrict__ spay,
                                                        const uint32_t* __restrict__ pinfo,
                                                        const uint32_t* __restrict__ istart,
                                                        uint32_t* __restrict__ longseg, const BatchArgs* __restrict__ A,
                                                        Tree t, BatchCtl* __restrict__ ctl) {
  pdl_wait();   // predecessor kernel complete, its writes visible (no-op without PDL)
  pdl_trigger();
  query_body(qkey, qseg, wkey, wseg, wop, wval, wleaf, wslot, wparent, old, spay, pinfo, istart, longseg, A, t, ctl);
}
__global__ void __launch_bounds__(EIRENE_QTHREADS, EIRENE_QMINB) query_cond_kernel(const uint64_t* __restrict__ qkey,
                                                        const uint32_t* __restrict__ qseg,
                                                        const uint64_t* __restrict__ wkey,
                                                        const uint32_t* __restrict__ wseg,
                                                        const uint8_t* __restrict__ wop,
                                                        uint64_t* __restrict__ wval, uint32_t* __restrict__ wleaf,
                                                        uint8_t* __restrict__ wslot, uint32_t* __restrict__ wparent,
                                                        uint64_t* __restrict__ old,
                                                        const uint32_t* __restrict__ spay,
                                                        const uint32_t* __restrict__ pinfo,
                                                        const uint32_t* __restrict__ istart,
                                                        uint32_t* __restrict__ longseg, const BatchArgs* __restrict__ A,
                                                        Tree t, BatchCtl* __restrict__ ctl,
                                                        cudaGraphConditionalHandle cond) {
  pdl_wait();
  pdl_trigger();
  query_body(qkey, qseg, wkey, wseg, wop, wval, wleaf, wslot, wparent, old, spay, pinfo, istart, longseg, A, t, ctl);
  query_end(ctl, A, t.hdr, cond);
}

// Locality-aware warp reorganisation the paper's way (§5, P:1380-1512,
// Fig.6): an ablation of the default traversal above (EIRENE_F_ITERWARP).
// Request groups (RGs) are 32 consecutive issued requests of the key-sorted
// query list, then of the write list; an ITERATION WARP runs `iter` adjacent
// RGs one after the other -- iter = iter_rgs, or with 0 the RGs
// evenly spread over the resident warps.  The warp keeps a
// buffer (leaf, RF): the first RG, or one whose MAXIMAL key exceeds the
// buffered RF, descends from the root (vertical, `height`
// nodes); otherwise every lane walks the leaf links from the buffered leaf
// (horizontal, 1 + links nodes).  The buffer then holds the leaf
// of the RG's maximal key and its RF.  RF(leaf) = lo fence of
// the leaf `height` links to the right (reading 22, set at bulk load and
// inherited by split-off leaves); a walk longer than `height` repairs the
// start leaf's RF lazily.  Correctness never depends on RF: a
// horizontal walk starts at the leaf of a smaller key of the same sorted list
// and follows B-link `next` pointers until k < hi, so RF only chooses the
// cheaper way.  With EIRENE_F_STATS the kernel counts vertical / horizontal
// RGs and traversal steps (Fig.10).
__device__ __forceinline__ void query_iterwarp_body(const uint64_t* __restrict__ qkey,
                                                                 const uint64_t* __restrict__ wkey,
                                                                 uint32_t* __restrict__ wparent, QueryIO io,
                                                                 const BatchArgs* __restrict__ A, Tree t,
                                                                 BatchCtl* __restrict__ ctl, uint32_t iter_rgs,
                                                                 uint32_t stats) {
  if (ctl->invalid || ctl->status != 0) return;
  tkey_t* __restrict__ results = A->results;
  io.vals = A->vals;   // (the batch's pointers live on the device)
  const uint32_t nq = ctl->nq, nw = ctl->nw;
  if (!headroom_ok(t, nw)) {
    if (blockIdx.x == 0 && threadIdx.x == 0) ctl->status = EIRENE_EFULL;
    return;
  }
  const uint32_t rq = (nq + 31) / 32, nrg = rq + (nw + 31) / 32;
  q_zero();
  const unsigned long long rw = t.hdr->root_word;
  const uint32_t height = (uint32_t)(rw >> 32), root = (uint32_t)rw;
  const uint32_t lane = threadIdx.x & 31;
  const uint32_t nwarps = (gridDim.x * blockDim.x) >> 5;
  const uint32_t iter = iter_rgs ? iter_rgs : max(1u, (nrg + nwarps - 1) / nwarps);
  const uint64_t pl = pol_evict_last(), pf = pol_evict_first();
  unsigned long long nsteps = 0;
  uint32_t nvert = 0, nhor = 0;
  for (uint32_t w = (blockIdx.x * blockDim.x + threadIdx.x) >> 5; (uint64_t)w * iter < nrg; w += nwarps) {
    uint32_t buf_leaf = NIL;   // empty buffer: the first RG traverses vertically
    uint64_t buf_rf = 0;
    const uint64_t rend = (uint64_t)w * iter + iter;
    const uint32_t r1 = rend < nrg ? (uint32_t)rend : nrg;
    for (uint32_t r = w * iter; r < r1; ++r) {
      const bool isq = r < rq;
      if (r == rq) buf_leaf = NIL;   // the write list starts over at small keys
      const uint32_t base = (isq ? r : r - rq) * 32;
      const uint32_t cnt = min(32u, (isq ? nq : nw) - base);
      const bool act = lane < cnt;
      const uint64_t* __restrict__ kl = isq ? qkey : wkey;
      const uint64_t kmax = kl[base + cnt - 1];   // sorted list: the RG's maximal key
      const uint64_t k = act ? kl[base + lane] : kmax;
      const bool vertical = buf_leaf == NIL || kmax > buf_rf;
      uint32_t node, steps, parent = NIL;   // parent: known after a vertical descent only
      uint64_t rep = 0;
      if (vertical) {
        node = root;
        for (uint32_t lvl = height - 1; lvl > 0; --lvl) {
          parent = node;
          node = ldg32_pol(t.ichild + (size_t)node * FAN + child_slot(t, node, k, pl), pl);
        }
        steps = height;
      } else {
        node = buf_leaf;
        steps = 1;
        while (k >= t.lmeta[node].hi) {   // the tree is quiescent here
          node = t.lmeta[node].next;
          if (++steps == height + 1) rep = t.lmeta[node].lo;   // the leaf `height` links right of the start
        }
      }
      const int s = slot16(t.lkeys + (size_t)node * LSTRIDE, k, pf);
      const uint64_t v = s >= 0 ? load_value(t.lvals + (size_t)node * LSTRIDE + s, pf) : KEY_MAX;
      if (act && !isq) wparent[base + lane] = parent;
      if (act) retire(io, isq ? base + lane : nq + base + lane, isq, nq, node, s, v, results, ctl, t.lvals);
      __syncwarp();
      const uint32_t top = __shfl_sync(FULL, node, cnt - 1);
      const uint32_t rm = __ballot_sync(FULL, act && steps > height);
      if (rm) {   // lazy RF repair of the start leaf; every such lane found the same leaf
        rep = shfl64(rep, __ffs(rm) - 1);
        if (lane == 0) t.lrf[buf_leaf] = rep;
      }
      buf_rf = (rm && top == buf_leaf) ? rep : __ldcg(reinterpret_cast<const unsigned long long*>(t.lrf + top));
      buf_leaf = top;
      if (stats) {
        nsteps += __reduce_add_sync(FULL, act ? steps : 0u);
        nvert += vertical ? 1u : 0u;
        nhor += vertical ? 0u : 1u;
      }
    }
  }
  if (stats && lane == 0 && (nvert | nhor)) {
    atomicAdd(&ctl->trav_steps, nsteps);
    atomicAdd(&ctl->rg_vertical, nvert);
    atomicAdd(&ctl->rg_horizontal, nhor);
  }
  q_flush(ctl);
}

__global__ void __launch_bounds__(256, 4) query_iterwarp_kernel(const uint64_t* __restrict__ qkey,
                                                                 const uint64_t* __restrict__ wkey,
                                                                 uint32_t* __restrict__ wparent, QueryIO io,
                                                                 const BatchArgs* __restrict__ A, Tree t,
                                                                 BatchCtl* __restrict__ ctl, uint32_t iter_rgs,
                                                                 uint32_t stats) {
  pdl_wait();   // predecessor kernel complete, its writes visible (no-op without PDL)
  pdl_trigger();
  query_iterwarp_body(qkey, wkey, wparent, io, A, t, ctl, iter_rgs, stats);
}
__global__ void __launch_bounds__(256, 4) query_iterwarp_cond_kernel(const uint64_t* __restrict__ qkey,
                                                                      const uint64_t* __restrict__ wkey,
                                                                      uint32_t* __restrict__ wparent, QueryIO io,
                                                                      const BatchArgs* __restrict__ A, Tree t,
                                                                      BatchCtl* __restrict__ ctl, uint32_t iter_rgs,
                                                                      uint32_t stats, cudaGraphConditionalHandle cond) {
  pdl_wait();
  pdl_trigger();
  query_iterwarp_body(qkey, wkey, wparent, io, A, t, ctl, iter_rgs, stats);
  query_end(ctl, A, t.hdr, cond);
}

// Diagnostics (EIRENE_DEBUG_SYNC / EIRENE_UPDATE_PROF only): printf lives in
// its own kernel, launched after the batch, not in the batch's kernels.
__global__ void debug_print_kernel(const BatchCtl* __restrict__ ctl, int dbgprint) {
  if (dbgprint)
    printf("[eirene dbg] %u %u %u %u %u %u %u %u\n", ctl->dbg[0], ctl->dbg[1], ctl->dbg[2], ctl->dbg[3],
           ctl->dbg[4], ctl->dbg[5], ctl->dbg[6], ctl->dbg[7]);
  if (ctl->uprof[0]) {   // EIRENE_UPDATE_PROF: update-kernel phases (us since its start)
    printf("[upd prof] entries %u %u %u %u %u | t:", ctl->lvl_ent[0], ctl->lvl_ent[1], ctl->lvl_ent[2],
           ctl->lvl_ent[3], ctl->lvl_ent[4]);
    for (int i = 1; i < 24 && ctl->uprof[i]; ++i) printf(" %.1f", (ctl->uprof[i] - ctl->uprof[0]) * 1e-3);
    printf("\n");
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
                                                     const uint64_t* __restrict__ kB,
                                                     const tkey_t* __restrict__ vals,
                                                     const tkey_t* __restrict__ results) {
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
  const uint32_t pi = pinfo[lo - 1];
  if (!(pi & DONE_BIT)) return pre;
  if (pi & DEFER_BIT) {   // hot key: its early results are written later; the nearest write decides
    const uint32_t pw = (uint32_t)kB[lo - 1];
    return ((pw & 3) == OP_DELETE) ? KEY_MAX : vals[pw >> 2];
  }
  return widen(ld_cg(results + (pj >> 2)));
}

__global__ void __launch_bounds__(256, 4) range_kernel(uint32_t n, const uint64_t* __restrict__ wkey,
                                                    const uint32_t* __restrict__ wseg,
                                                    const uint32_t* __restrict__ spay,
                                                    const uint32_t* __restrict__ pinfo,
                                                    const uint32_t* __restrict__ istart,
                                                    const uint64_t* __restrict__ kB,
                                                    const uint64_t* __restrict__ old,
                                                    const BatchArgs* __restrict__ A, Tree t, BatchCtl* __restrict__ ctl) {
  pdl_wait();   // predecessor kernel complete, its writes visible (no-op without PDL)
  pdl_trigger();
  if (ctl->invalid || ctl->status != 0 || ctl->nrange == 0) return;
  n = A->n;   // (the grid is sized for the graph's size bucket)
  const uint8_t* __restrict__ ops = A->ops;
  const tkey_t* __restrict__ keys = A->keys;
  const tkey_t* __restrict__ vals = A->vals;
  tkey_t* __restrict__ results = A->results;
  tkey_t* __restrict__ rkeys = A->rkeys;
  tkey_t* __restrict__ rvals = A->rvals;
  const uint32_t cap = A->rcap;
  const uint32_t nw = ctl->nw;
  const unsigned long long rw = t.hdr->root_word;
  const uint32_t height = (uint32_t)(rw >> 32), root = (uint32_t)rw;
  uint32_t nart = 0;
  const uint64_t pl = pol_evict_last(), pf = pol_evict_first();
  const uint32_t stride = gridDim.x * blockDim.x;
  for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += stride) {
    if (ops[i] != OP_RANGE) continue;
    const uint64_t l = widen(keys[i]), u = widen(vals[i]);
    tkey_t* __restrict__ ok = rkeys + (size_t)i * cap;
    tkey_t* __restrict__ ov = rvals + (size_t)i * cap;
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
        node = ldg32_pol(t.ichild + (size_t)node * FAN + child_slot(t, node, l, pl), pl);
      }
      // walk the leaf chain, merged with the written keys
      for (;;) {
        const tkey_t* lk = t.lkeys + (size_t)node * LSTRIDE;
        const tkey_t* lv = lk + FAN;
        Line16 kv;
        kv.load(lk, pf);
        // slots [s0, s1) hold the leaf's keys in [l, u] (keys ascending, padding last)
        uint32_t s0 = 0, s1 = 0, nk = 0;
#pragma unroll
        for (uint32_t j = 0; j < (uint32_t)FAN; ++j) {
          const uint64_t q = widen((tkey_t)kv.at(j));
          s0 += q < l;
          s1 += q <= u && q != KEY_MAX;
          nk += q != KEY_MAX;
        }
        if (wk > u) {
          // no written key left in [l, u]: the pairs come straight from the leaf;
          // the value sectors needed are loaded together, then written out
          const uint32_t take = s1 > s0 ? min(s1 - s0, cap - c) : 0u;
          const uint32_t e = s0 + take;
          // keys first (their registers die), then the value chunks that hold slots [s0, e)
#pragma unroll
          for (uint32_t j = 0; j < (uint32_t)FAN; ++j)
            if (j >= s0 && j < e) st64_pol(ok + c + (j - s0), kv.at(j), pf);
          // the value chunks (256 bits each) that hold slots [s0, e)
          constexpr uint32_t PER = 32 / sizeof(tkey_t);
#pragma unroll
          for (int x = 0; x < Line16::NW; ++x) {
            kv.w[x] = make_ulonglong4(0, 0, 0, 0);
            if (PER * x < e && PER * x + PER > s0)
              kv.w[x] = ldg256_pol(reinterpret_cast<const uint64_t*>(lv) + 4 * x, pf);
          }
#pragma unroll
          for (uint32_t j = 0; j < (uint32_t)FAN; ++j)
            if (j >= s0 && j < e) st64_pol(ov + c + (j - s0), kv.at(j), pf);
          c += take;
        } else {
          for (uint32_t s = s0; s < s1 && c < cap; ++s) {
            const uint64_t k = kv.at(s);
            // written keys before k are absent from the pre-batch tree
            while (wk < k && c < cap) {
              const uint64_t v = artificial_query(w, i, KEY_MAX, wseg, istart, spay, pinfo, kB, vals, results);
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
            uint64_t v;
            if (wk == k) {
              // a written key: its pre-batch value is the one its issued write's
              // locate retrieved (old[seg]); the slot may already hold the write's
              // value (overwrites are applied in place by the query kernel)
              v = artificial_query(w, i, old[wseg[w]], wseg, istart, spay, pinfo, kB, vals, results);
              ++nart;
              ++w;
              wk = w < nw ? wkey[w] : KEY_MAX;
            } else {
              v = ldg64_pol(lv + s, pf);
            }
            if (v != KEY_MAX) {
              ok[c] = k;
              ov[c] = v;
              ++c;
            }
          }
        }
        // a key > u in this leaf ends the walk; so does a full output row
        if (s1 < nk || c >= cap) break;
        const NodeMeta* m = t.lmeta + node;
        const uint64_t hi = __ldg(&m->hi);
        const uint32_t nx = __ldg(&m->next);
        if (hi > u || hi == KEY_MAX || nx == NIL) break;   // every later key is > u
        node = nx;
      }
      // written keys after the last tree key in range
      while (w < nw && wk <= u && c < cap) {   // (u may be UINT64_MAX, the no-more-writes sentinel)
        const uint64_t v = artificial_query(w, i, KEY_MAX, wseg, istart, spay, pinfo, kB, vals, results);
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
    st64_pol(results + i, c, pf);
  }
  nart = __reduce_add_sync(FULL, nart);
  if (nart && (threadIdx.x & 31) == 0) atomicAdd(&ctl->nart, nart);
}

}  // namespace

void launch_query(uint32_t n, const CombBufs& c, const uint32_t* spay, const BatchArgs* A, Tree t, BatchCtl* ctl,
                  int num_sms, uint32_t flags, uint32_t iter_rgs, cudaGraphConditionalHandle cond, int use_cond,
                  cudaStream_t st, int* launches) {
  // one resident wave: EIRENE_QMINB (8) CTAs of 256 threads per SM at <= 32 registers
  int blocks = (int)std::min<uint32_t>((n + EIRENE_QTHREADS - 1) / EIRENE_QTHREADS,
                                       (uint32_t)num_sms * (uint32_t)EIRENE_QMINB);
  if (blocks < 1) blocks = 1;
  if (flags & EIRENE_F_ITERWARP) {
    // <= 64 registers (the RG loop keeps the buffer and the lane's state): 4 resident CTAs per SM
    const int iblocks = (int)std::min<uint32_t>((n + 255) / 256, (uint32_t)num_sms * 4u);
    const dim3 g(iblocks < 1 ? 1 : iblocks);
    const QueryIO io{c.qseg, c.wseg, c.wop, c.wval, nullptr, c.wleaf, c.wslot, c.old, spay, c.pinfo, c.istart, c.longseg};
    const uint32_t stats = (flags & EIRENE_F_STATS) ? 1u : 0u;
    if (use_cond)
      launch_k(query_iterwarp_cond_kernel, g, dim3(256), 0, st, true, false, c.qkey, c.wkey, c.wparent, io, A, t, ctl,
               iter_rgs, stats, cond);
    else
      launch_k(query_iterwarp_kernel, g, dim3(256), 0, st, true, false, c.qkey, c.wkey, c.wparent, io, A, t, ctl,
               iter_rgs, stats);
  } else if (use_cond) {
    launch_k(query_cond_kernel, dim3(blocks), dim3(EIRENE_QTHREADS), 0, st, true, false, c.qkey, c.qseg, c.wkey, c.wseg, c.wop,
             c.wval, c.wleaf, c.wslot, c.wparent, c.old, spay, c.pinfo, c.istart, c.longseg, A, t, ctl, cond);
  } else {
    launch_k(query_kernel, dim3(blocks), dim3(EIRENE_QTHREADS), 0, st, true, false, c.qkey, c.qseg, c.wkey, c.wseg, c.wop, c.wval,
             c.wleaf, c.wslot, c.wparent, c.old, spay, c.pinfo, c.istart, c.longseg, A, t, ctl);
  }
  ++*launches;
}

void launch_range(uint32_t n, const CombBufs& c, const uint32_t* spay, const uint64_t* kB, const BatchArgs* A, Tree t,
                  BatchCtl* ctl, int num_sms, cudaStream_t st, int* launches) {
  int blocks = (int)std::min<uint32_t>((n + 255) / 256, (uint32_t)num_sms * 8u);
  if (blocks < 1) blocks = 1;
  launch_k(range_kernel, dim3(blocks), dim3(256), 0, st, true, false, n, c.wkey, c.wseg, spay, c.pinfo, c.istart, kB, c.old, A, t, ctl);
  ++*launches;
}

void launch_result(const BatchCtl* ctl, int dbgprint, cudaStream_t st) {
  // (RESULT_CAL of the long segments and the batch's BatchCtl are the update
  // kernel's last phase, result_phase; only the diagnostics print is left here)
  static const bool uprof = std::getenv("EIRENE_UPDATE_PROF") != nullptr;
  if (dbgprint || uprof) debug_print_kernel<<<1, 1, 0, st>>>(ctl, dbgprint);
}

}  // namespace eirene
