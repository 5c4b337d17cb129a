// update.cu -- UPDATE_KERNEL (Alg.1:23-46) with leaf-bucketed warp regrouping
// (P:1334-1416), optimistic traversal, version validation and an
// eager-conflict-detection STM fallback past THRESHOLD (Alg.1:28-33).
//
// Work unit (regrouping, a4): the issued writes are key-sorted and carry the
// leaf the query-kernel traversal located (an unprotected findLeaf, Alg.1:29).
// Equal leaf ids are contiguous, so each warp takes whole LEAF RUNS: a run is
// merged into its leaf by one warp in one transaction, and no two warps ever
// target the same leaf (the B200 form of the paper's iteration warps: the
// locality is exploited by construction instead of by a horizontal walk).
// With EIRENE_F_REGROUP off every issued write is its own run (one warp per
// request, as in Alg.1:24), and leaf conflicts + retries appear.
//
// Per run (Alg.1:27-45):
//   RETRY: leaf = hint (first try) | findLeaf optimistic (retry < THRESHOLD)
//                                 | TX{findLeaf} with a read log (otherwise)
//          leafvers = leaf.version                                  (Alg.1:35)
//          TX_BEGIN: eager write ownership = CAS(version, v, v|1)    (Alg.1:37)
//          if key in [leaf.lo, leaf.hi): merge the run (upsert/erase), split
//            into ceil(t/16) leaves if it overflows, version += 2 on split
//          else abort: retry_count++, goto RETRY                     (Alg.1:40-43)
// Structure changes propagate upward (B-link tree: every node has a right link
// and [lo, hi) fences, so a warp holds at most one lock at a time and never
// waits while holding one -> no deadlock).  Inserting separators into a parent
// repeats the same optimistic / STM protocol at the parent level; a root split
// installs the new root while the old root is still owned.
#include <cstdio>
#include <cstdlib>

#include "eirene_internal.cuh"

#ifndef UPD_THREADS
#define UPD_THREADS 128   // update-kernel CTA: 4 warps, six per SM (r3w: one 768-thread CTA per SM: cfg1 update 103 -> 111 us)
#endif

namespace eirene {

namespace {

struct Ctx {
  Tree t;
  const uint64_t* wkey;
  const uint8_t* wop;
  const uint64_t* wval;
  const uint32_t* wseg;
  const uint32_t* wleaf;
  const uint8_t* wslot;
  const uint32_t* wparent;   // the leaf's parent at locate time (level-0 parent hints), NIL if unknown
  uint64_t* old;
  uint64_t* eK[2];    // entry ping-pong buffers: separators to insert at the next level
  uint32_t* eC[2];
  uint32_t threshold;
  bool force_stm;
  bool regroup;
  bool stats;
  BatchCtl* ctl;
  uint2* slots[2];      // level-synchronous propagation: per producer unit (base, n)
  uint32_t* eparent;    // parent found for each entry position (lookup step)
  uint64_t* flat_key;   // upper levels: the level's entries concatenated in key order
  uint32_t* flat_child;
  uint32_t* flat_off;   // per producer warp: offset of its entries in the flat list
};

struct WarpStats {
  unsigned long long runs = 0, retries = 0, stm = 0, leaf_splits = 0, inner_splits = 0, new_leaves = 0,
                     new_inner = 0;
  unsigned long long t0 = 0;
  bool dead = false;
  bool leaf_root = true;   // the tree had height 1 at the kernel's start (else no leaf is ever the root)
};

// Watchdog (see eirene_internal.cuh): true if this warp must give up.
__device__ bool watchdog(const Ctx& C, WarpStats& ws, uint32_t where, uint32_t a, uint32_t b, uint32_t c,
                         uint32_t d) {
  if (ws.dead) return true;
  if (*(volatile int32_t*)&C.ctl->status == EIRENE_EINTERNAL || gtime_ns() - ws.t0 > WATCHDOG_NS) {
    ws.dead = true;
    if ((threadIdx.x & 31) == 0 && atomicCAS(reinterpret_cast<int*>(&C.ctl->status), 0, EIRENE_EINTERNAL) == 0) {
      C.ctl->dbg[0] = where;
      C.ctl->dbg[1] = a;
      C.ctl->dbg[2] = b;
      C.ctl->dbg[3] = c;
      C.ctl->dbg[4] = d;
      C.ctl->dbg[5] = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    }
    return true;
  }
  return false;
}

constexpr uint32_t LEAF_TAG = 0x80000000u;

__device__ __forceinline__ void backoff(uint32_t retry) {
  uint32_t ns = 32u << (retry < 5 ? retry : 5);   // <= 1 us: lock holders finish in about that
  __nanosleep(ns);
}

__device__ __forceinline__ uint32_t shfl32(uint32_t v, int src) { return __shfl_sync(FULL, v, src); }

__device__ __forceinline__ NodeMeta* meta_of(const Tree& t, uint32_t node, bool leaf) {
  return leaf ? t.lmeta + node : t.imeta + node;
}

// Warp-collective lock acquisition: TX_BEGIN with eager conflict detection.
// Returns true and the pre-lock version in *v if the node was free.
// Acquire: lane 0's CAS has acquire semantics and __syncwarp orders the other
// lanes' subsequent (L2-coherent) reads after it.
__device__ __forceinline__ bool try_lock(uint32_t* vp, uint32_t* v_out) {
  uint32_t v = 0, ok = 0;
  if (lane_id() == 0) {   // test-and-set: one round trip (setting an already set lock bit changes nothing)
    v = atom_or_acquire(vp, 1u);
    ok = (v & 1u) ? 0u : 1u;
  }
  ok = shfl32(ok, 0);
  v = shfl32(v, 0);
  __syncwarp();
  *v_out = v;
  return ok != 0;
}

// Release: __syncwarp makes every lane's writes happen-before lane 0's
// release store (release is cumulative in the PTX memory model).
__device__ __forceinline__ void unlock(uint32_t* vp, uint32_t newv) {
  __syncwarp();
  if (lane_id() == 0) st_release(vp, newv);
  __syncwarp();
}

// findLeaf / find-node-at-level (warp-collective, uniform arguments).
// Optimistic mode reads without any protection (Alg.1:29).  STM mode (Alg.1:31-33)
// is a read-only transaction: every node read records (node, version) in a
// per-lane read log, aborts eagerly on a node owned by a writer (odd version)
// or a version change during the read, and validates the whole log at TX_END.
// B-link move-right (k >= hi -> follow next) keeps descents correct across
// concurrent splits whose separators are not yet in the parent.
__device__ uint32_t descend(const Ctx& C, uint64_t k, uint32_t target, bool stm) {
  const int lane = lane_id();
  const Tree& t = C.t;
  const unsigned long long rw = ld_acquire64(&t.hdr->root_word);
  const uint32_t height = (uint32_t)(rw >> 32);
  uint32_t node = (uint32_t)rw;
  if (height == 0 || target + 1 > height) return NIL;
  uint32_t lvl = height - 1;
  uint32_t log_node = NIL, log_ver = 0;
  int nlog = 0;
  for (int steps = 0; steps < 1024; ++steps) {
    const bool leaf = (lvl == 0);
    if (node >= (leaf ? t.leaf_cap : t.inner_cap)) return NIL;
    NodeMeta* m = meta_of(t, node, leaf);
    uint32_t v1 = 0;
    if (stm) {
      v1 = ld_acquire(&m->version);
      if (v1 & 1u) return NIL;   // eager conflict: the node is owned by a writer
    }
    const uint64_t hi = ld_cg(&m->hi);
    const uint32_t nxt = ld_cg(&m->next);
    const bool right = (k >= hi) && nxt != NIL;
    uint32_t child = NIL;
    if (!right && lvl > target) {
      const size_t nb = (size_t)node * FAN;
      const uint64_t key = lane < FAN ? widen(ld_cg(t.ikeys + nb + lane)) : KEY_MAX;
      const uint32_t ch = lane < FAN ? ld_cg(t.ichild + nb + lane) : NIL;
      const uint32_t idx = __popc(__ballot_sync(FULL, lane < FAN - 1 && key <= k));
      child = shfl32(ch, idx);
    }
    if (stm) {
      __threadfence();
      const uint32_t v2 = ld_acquire(&m->version);
      if (v2 != v1 || nlog >= 32) return NIL;
      if (lane == nlog) {
        log_node = node | (leaf ? LEAF_TAG : 0u);
        log_ver = v1;
      }
      ++nlog;
    }
    if (right) {
      node = nxt;
      continue;
    }
    if (lvl == target) {
      if (stm) {   // TX_END of the traversal: validate the read set
        bool okl = true;
        if (lane < nlog) {
          const bool lf = (log_node & LEAF_TAG) != 0;
          okl = ld_acquire(&meta_of(t, log_node & ~LEAF_TAG, lf)->version) == log_ver;
        }
        if (!__all_sync(FULL, okl)) return NIL;
      }
      return node;
    }
    if (child == NIL) return NIL;
    node = child;
    --lvl;
  }
  return NIL;
}

__device__ __forceinline__ bool is_root(const Tree& t, uint32_t node, uint32_t level) {
  const unsigned long long rw = ld_acquire64(&t.hdr->root_word);
  return (uint32_t)rw == node && (uint32_t)(rw >> 32) == level + 1;
}

__device__ __forceinline__ uint32_t warp_alloc(uint32_t* ctr, uint32_t n) {
  uint32_t f = 0;
  if (lane_id() == 0) f = atomicAdd(ctr, n);
  return shfl32(f, 0);
}

// New root level(s) above a list of nodes at level L: element 0 is (id0, lo0),
// elements 1..m are the entries (K, Ch)[eb ..].  Called while the old root is
// still owned, so the root word cannot change underneath (P:1196-1202 regions).
__device__ void build_root(const Ctx& C, uint32_t L, uint32_t id0, uint64_t lo0, uint64_t hi_all, uint64_t* K,
                           uint32_t* Ch, uint64_t* K2, uint32_t* Ch2, uint32_t eb, uint32_t m, WarpStats& ws) {
  const int lane = lane_id();
  const Tree& t = C.t;
  uint32_t cnt = m + 1;
  for (;;) {
    const uint32_t nn = (cnt + FAN - 1) / FAN;
    const uint32_t first = warp_alloc(&t.hdr->inner_count, nn);
    if (lane == 0) atomicAdd(&t.hdr->level_count[L + 1], nn);
    const uint32_t bs = cnt / nn, rem = cnt % nn;
    for (uint32_t q0 = 0; q0 < nn; q0 += 2) {
      const uint32_t q = q0 + (lane >> 4), i = lane & 15;
      if (q < nn) {
        const uint32_t size = bs + (q < rem ? 1u : 0u);
        const uint32_t start = q * bs + min(q, rem);
        const uint32_t g = start + i;
        const uint32_t id = first + q;
        const uint32_t child = i < size ? (g == 0 ? id0 : ld_cg(Ch + eb + g - 1)) : NIL;
        const uint64_t key = (i + 1 < size) ? ld_cg(K + eb + g) : KEY_MAX;
        t.ichild[(size_t)id * FAN + i] = child;
        t.ikeys[(size_t)id * FAN + i] = key;
        if (i == 0) {
          NodeMeta mt;
          mt.version = 0;
          mt.lo = g == 0 ? lo0 : ld_cg(K + eb + g - 1);
          const uint32_t nstart = (q + 1) * bs + min(q + 1, rem);
          mt.hi = (q + 1 < nn) ? ld_cg(K + eb + nstart - 1) : hi_all;
          mt.next = (q + 1 < nn) ? id + 1 : NIL;
          mt.count = size;
          mt.level = L + 1;
          t.imeta[id] = mt;
          if (q >= 1) {
            K2[eb + q - 1] = mt.lo;
            Ch2[eb + q - 1] = id;
          }
        }
      }
    }
    __threadfence();
    __syncwarp();
    ws.new_inner += nn;
    if (nn == 1) {
      if (lane == 0) atomicExch(&t.hdr->root_word, ((unsigned long long)(L + 2) << 32) | first);
      __threadfence();
      __syncwarp();
      return;
    }
    id0 = first;
    cnt = nn;
    ++L;
    uint64_t* tk = K; K = K2; K2 = tk;
    uint32_t* tc = Ch; Ch = Ch2; Ch2 = tc;
  }
}

// The merge of writes [b, e) into a leaf whose c keys are okey (slot `lane`,
// lanes < 16): which of the leaf's keys the writes hit (mmask), how many
// upserts (U), per leaf key the upserts before it (ups_before, lanes < c), and
// whether every write is a value overwrite of a present key (inplace).
struct LeafPlan {
  uint32_t c = 0, mmask = 0, U = 0, ups_before = 0;
  bool inplace = true;
};
// #leaf keys < wk: the leaf's keys sit sorted in lanes 0..15 (KEY_MAX padding
// above), so a 5-step binary search over shuffles
__device__ __forceinline__ uint32_t rank16(uint64_t okey, uint64_t wk) {
  uint32_t lo = 0;
#pragma unroll
  for (uint32_t s = 8; s > 0; s >>= 1)
    if (shfl64(okey, lo + s - 1) < wk) lo += s;
  if (shfl64(okey, lo) < wk) ++lo;   // (only reachable at lo == 15)
  return lo;
}
// #active write lanes whose key < ok (the step's write keys are ascending over the lanes, KEY_MAX when inactive)
__device__ __forceinline__ uint32_t rank32(uint64_t wk, uint64_t ok) {
  uint32_t lo = 0;
#pragma unroll
  for (uint32_t s = 16; s > 0; s >>= 1)
    if (shfl64(wk, lo + s - 1) < ok) lo += s;
  if (shfl64(wk, lo & 31u) < ok) ++lo;   // (only reachable at lo == 31)
  return lo;
}
__device__ __forceinline__ LeafPlan leaf_plan(const Ctx& C, uint32_t b, uint32_t e, uint64_t okey) {
  const int lane = lane_id();
  LeafPlan L;
  L.c = __popc(__ballot_sync(FULL, okey != KEY_MAX));
  for (uint32_t base = b; base < e; base += 32) {
    const uint32_t j = base + lane;
    const bool act = j < e;
    const uint64_t wk = act ? C.wkey[j] : KEY_MAX;
    const uint32_t wo = act ? C.wop[j] : 0;
    const uint32_t lo = rank16(okey, wk);
    const uint64_t at = shfl64(okey, lo & 15u);
    const bool match = act && lo < L.c && at == wk;
    const bool ups = act && wo != OP_DELETE;
    L.mmask |= __reduce_or_sync(FULL, match ? (1u << lo) : 0u);
    const uint32_t um = __ballot_sync(FULL, ups);
    L.U += __popc(um);
    if (__any_sync(FULL, act && !(match && ups))) L.inplace = false;
    if (L.c > 0 && um) {   // upserts before leaf key `lane`: the writes below it, counted over um
      const uint32_t p = rank32(wk, okey);
      if (lane < (int)L.c) L.ups_before += __popc(p >= 32 ? um : (um & ((1u << p) - 1u)));
    }
  }
  return L;
}

// Only value overwrites of present keys: no structural change.
__device__ __forceinline__ void leaf_overwrite(const Ctx& C, uint32_t X, uint32_t b, uint32_t e, uint64_t okey) {
  const int lane = lane_id();
  for (uint32_t base = b; base < e; base += 32) {
    const uint32_t j = base + lane;
    const bool act = j < e;
    const uint64_t wk = act ? C.wkey[j] : KEY_MAX;
    const uint32_t lo = rank16(okey, wk);
    if (act) C.t.lvals[(size_t)X * LSTRIDE + lo] = C.wval[j];
  }
}

// The merged sequence (tout keys) written over X and k-1 fresh leaves
// first.. (even multi-way split); entries (first key, leaf) for the parent
// to (Ek, Ec)[b .. b+k-2] if Ek != null.  Returns, in every lane, the first
// key of the second leaf (k > 1).
__device__ uint64_t leaf_place(const Ctx& C, uint32_t X, uint32_t first, uint32_t b, uint32_t e, uint64_t okey,
                               uint64_t oval, const LeafPlan& L, uint32_t tout, uint32_t k, uint64_t* Ek,
                               uint32_t* Ec) {
  const int lane = lane_id();
  const Tree& t = C.t;
  const uint32_t bs = tout / k, rem = tout % k, big = rem * (bs + 1);
  const uint32_t mmask = L.mmask;
  uint64_t k1 = 0;   // this lane placed slot 0 of leaf 1
  bool has1 = false;
  auto place = [&](uint32_t f, uint64_t key, uint64_t val) {
    uint32_t q, start;
    if (f < big) {
      q = f / (bs + 1);
      start = q * (bs + 1);
    } else {
      q = rem + (f - big) / bs;
      start = big + (q - rem) * bs;
    }
    const uint32_t slot = f - start;
    const uint32_t id = q == 0 ? X : first + q - 1;
    t.lkeys[(size_t)id * LSTRIDE + slot] = key;
    t.lvals[(size_t)id * LSTRIDE + slot] = val;
    if (q > 0 && slot == 0) {
      if (Ek) {
        Ek[b + q - 1] = key;
        Ec[b + q - 1] = id;
      }
      if (q == 1) {
        k1 = key;
        has1 = true;
      }
    }
  };
  if (lane < (int)L.c && !((mmask >> lane) & 1u))
    place(lane - __popc(mmask & ((1u << lane) - 1u)) + L.ups_before, okey, oval);
  uint32_t urun = 0;
  for (uint32_t base = b; base < e; base += 32) {
    const uint32_t j = base + lane;
    const bool act = j < e;
    const uint64_t wk = act ? C.wkey[j] : KEY_MAX;
    const uint32_t wo = act ? C.wop[j] : 0;
    const uint32_t lo = rank16(okey, wk);
    const bool ups = act && wo != OP_DELETE;
    const uint32_t um = __ballot_sync(FULL, ups);
    if (ups) place(lo - __popc(mmask & ((1u << lo) - 1u)) + urun + __popc(um & lanemask_lt()), wk, C.wval[j]);
    urun += __popc(um);
  }
  for (uint32_t q0 = 0; q0 < k; q0 += 2) {   // pad unused slots with KEY_MAX
    const uint32_t q = q0 + (lane >> 4), s = lane & 15;
    if (q < k) {
      const uint32_t sz = bs + (q < rem ? 1u : 0u);
      if (s >= sz) t.lkeys[(size_t)(q == 0 ? X : first + q - 1) * LSTRIDE + s] = KEY_MAX;
    }
  }
  const uint32_t h1 = __ballot_sync(FULL, has1);
  return h1 ? shfl64(k1, __ffs(h1) - 1) : 0ull;
}

// Merge writes [b, e) (key-sorted, all inside the locked leaf X's fences) into
// X.  Every write returns the value X held for its key (old[seg], retrieved by
// the query kernel), NOT_FOUND if absent.  Result t keys; t <= 16 stays in X,
// else an even multi-way split into k = ceil(t/16) leaves (X + k-1 fresh),
// entries (first key, leaf) for the parent written to (Ek, Ec)[b .. b+k-2].
// Returns k.
__device__ uint32_t leaf_apply(const Ctx& C, uint32_t X, uint32_t b, uint32_t e, uint64_t X_hi, uint32_t X_next,
                               uint64_t okey, uint64_t oval, uint64_t* Ek, uint32_t* Ec, WarpStats& ws) {
  // okey / oval: X's key and value of slot `lane` (lanes < 16), loaded by the caller under the lock
  const int lane = lane_id();
  const Tree& t = C.t;
  const LeafPlan L = leaf_plan(C, b, e, okey);
  if (L.inplace) {   // only value overwrites of present keys: no structural change
    leaf_overwrite(C, X, b, e, okey);
    return 1;   // ordered before the release by unlock()
  }
  const uint32_t tout = L.c - __popc(L.mmask) + L.U;
  const uint32_t k = tout <= FAN ? 1u : (tout + FAN - 1) / FAN;
  const uint32_t first = k > 1 ? warp_alloc(&t.hdr->leaf_count, k - 1) : 0u;
  const uint32_t bs = tout / k, rem = tout % k;
  leaf_place(C, X, first, b, e, okey, oval, L, tout, k, Ek, Ec);
  // (no fence here: the new leaves are unreachable until X links them below,
  // X itself is read only under its lock; __syncwarp orders the lanes' Ek
  // writes before the meta loop reads them)
  __syncwarp();
  if (k > 1) {
    for (uint32_t q = 1 + lane; q < k; q += 32) {
      const uint32_t id = first + q - 1;
      NodeMeta mt;
      mt.version = 0;
      mt.lo = ld_cg(Ek + b + q - 1);
      mt.hi = (q + 1 < k) ? ld_cg(Ek + b + q) : X_hi;
      mt.next = (q + 1 < k) ? id + 1 : X_next;
      mt.count = bs + (q < rem ? 1u : 0u);
      mt.level = 0;
      t.lmeta[id] = mt;
      t.lrf[id] = t.lrf[X];   // split-off leaves inherit the RF (repaired lazily)
    }
    __threadfence();
    __syncwarp();
    if (lane == 0) {
      t.lmeta[X].hi = ld_cg(Ek + b);
      t.lmeta[X].next = first;
      t.lmeta[X].count = bs + (rem > 0 ? 1u : 0u);
    }
    ws.leaf_splits += 1;
    ws.new_leaves += k - 1;
  } else if (lane == 0) {
    t.lmeta[X].count = tout;
  }
  __syncwarp();   // published by the caller's unlock (a release)
  return k;
}

// Merge m entries (K, Ch)[eb ..] (sorted separators, all inside [plo, phi))
// into the locked parent P (level L, snapshot pk/pc in lanes 0..15) by key:
// the children of P and the new nodes form one sequence sorted by their left
// separator ("lowsep"; P's first child has lowsep plo < every entry).  t <= 16
// elements stay in P; otherwise an even multi-way split into ceil(t/16) nodes
// whose (lo, id) entries for P's parent are written to (K2, Ch2)[eb ..].
// Returns the number of those entries (0 if P did not split).
__device__ uint32_t inner_apply(const Ctx& C, uint32_t P, uint32_t L, uint64_t pk, uint32_t pc, uint32_t cP,
                                uint64_t plo, uint64_t phi, uint32_t pnext, const uint64_t* K, const uint32_t* Ch,
                                uint64_t* K2, uint32_t* Ch2, uint32_t eb, uint32_t m, WarpStats& ws) {
  const int lane = lane_id();
  const Tree& t = C.t;
  const uint32_t tout = cP + m;
  const uint32_t kp = tout <= FAN ? 1u : (tout + FAN - 1) / FAN;
  const uint32_t first = kp > 1 ? warp_alloc(&t.hdr->inner_count, kp - 1) : 0u;
  if (kp > 1 && lane == 0) atomicAdd(&t.hdr->level_count[L], kp - 1);
  const uint32_t bs = tout / kp, rem = tout % kp, big = rem * (bs + 1);
  // element at merged position g -> (node, slot); slot 0 of node q >= 1 is that node's lo
  auto place = [&](uint32_t g, uint32_t child, uint64_t lowsep) {
    uint32_t q, start;
    if (g < big) {
      q = g / (bs + 1);
      start = q * (bs + 1);
    } else {
      q = rem + (g - big) / bs;
      start = big + (q - rem) * bs;
    }
    const uint32_t slot = g - start;
    const uint32_t id = q == 0 ? P : first + q - 1;
    t.ichild[(size_t)id * FAN + slot] = child;
    if (slot > 0) {
      t.ikeys[(size_t)id * FAN + slot - 1] = lowsep;
    } else if (q > 0) {
      K2[eb + q - 1] = lowsep;
      Ch2[eb + q - 1] = id;
    }
  };
  // P's children: position i + #(entries < lowsep_i)
  const uint64_t left_sep = shfl64(pk, (lane + 31) & 31);
  const uint64_t my_low = lane == 0 ? plo : left_sep;
  uint32_t below = 0;
  for (uint32_t base = 0; base < m; base += 32) {
    const uint32_t x = base + lane;
    const uint64_t ek = x < m ? ld_cg(K + eb + x) : KEY_MAX;
    // child i >= 1: the entries below its left separator pk[i-1] (entries are
    // > plo, so child 0 stays first); the entries ascend over the lanes
    const uint32_t p = rank32(ek, my_low);
    if (lane >= 1 && lane < (int)cP) below += p;
  }
  // padding first (disjoint from the element slots below)
  for (uint32_t q0 = 0; q0 < kp; q0 += 2) {
    const uint32_t q = q0 + (lane >> 4), s = lane & 15;
    if (q < kp) {
      const uint32_t size = bs + (q < rem ? 1u : 0u);
      const uint32_t id = q == 0 ? P : first + q - 1;
      if (s >= size) t.ichild[(size_t)id * FAN + s] = NIL;
      if (s + 1 >= size) t.ikeys[(size_t)id * FAN + s] = KEY_MAX;
    }
  }
  __syncwarp();
  if (lane < (int)cP) place(lane + below, pc, my_low);
  // entries: position x + 1 + #(P separators < key)
  for (uint32_t base = 0; base < m; base += 32) {
    const uint32_t x = base + lane;
    const bool act = x < m;
    const uint64_t ek = act ? ld_cg(K + eb + x) : KEY_MAX;
    const uint32_t ec = act ? ld_cg(Ch + eb + x) : NIL;
    const uint32_t lt = rank16(pk, ek);   // pk[>= cP-1] == KEY_MAX
    if (act) place(x + 1 + lt, ec, ek);
  }
  __threadfence();
  __syncwarp();
  if (kp == 1) {
    if (lane == 0) t.imeta[P].count = tout;
    __threadfence();
    __syncwarp();
    return 0;
  }
  for (uint32_t q = 1 + lane; q < kp; q += 32) {
    const uint32_t id = first + q - 1;
    NodeMeta mt;
    mt.version = 0;
    mt.lo = ld_cg(K2 + eb + q - 1);
    mt.hi = (q + 1 < kp) ? ld_cg(K2 + eb + q) : phi;
    mt.next = (q + 1 < kp) ? id + 1 : pnext;
    mt.count = bs + (q < rem ? 1u : 0u);
    mt.level = L;
    t.imeta[id] = mt;
  }
  __threadfence();
  __syncwarp();
  if (lane == 0) {
    t.imeta[P].count = bs + (rem > 0 ? 1u : 0u);
    t.imeta[P].hi = ld_cg(K2 + eb);
    t.imeta[P].next = first;
  }
  __threadfence();
  __syncwarp();
  ws.inner_splits += 1;
  ws.new_inner += kp - 1;
  return kp - 1;
}

// Insert m entries (separator, new node) produced by splits at level L into
// level L+1, repeating upward while parents split.  Entries are merged into a
// parent BY KEY, so two splits of the same node whose parent insertions arrive
// in either order still leave the separators sorted.  Pending lists form a
// depth-first stack; a list produced from a consumed chunk [eb, eb+c) is at
// most c long and lives at [eb, ..) of the other ping-pong buffer, so the
// stacked lists never overlap.
__device__ void insert_up(const Ctx& C, uint32_t L0, uint32_t eb0, uint32_t m0, WarpStats& ws) {
  const int lane = lane_id();
  const Tree& t = C.t;
  uint32_t st_L[MAX_LEVELS], st_eb[MAX_LEVELS], st_m[MAX_LEVELS];
  int sp = 0;
  st_L[0] = L0;
  st_eb[0] = eb0;
  st_m[0] = m0;
  while (sp >= 0) {
    if (st_m[sp] == 0) {
      --sp;
      continue;
    }
    const uint32_t L = st_L[sp], eb = st_eb[sp], m = st_m[sp];
    if (sp + 1 >= MAX_LEVELS) {
      watchdog(C, ws, 3, L, eb, m, 0);
      return;
    }
    uint64_t* K = C.eK[L & 1];
    uint32_t* Ch = C.eC[L & 1];
    uint64_t* K2 = C.eK[(L + 1) & 1];
    uint32_t* Ch2 = C.eC[(L + 1) & 1];
    const uint64_t s = ld_cg(K + eb);
    uint32_t retry = 0, next_m = 0, P = NIL, consumed = 0;
    for (;;) {
      const bool stm = C.force_stm || retry >= C.threshold;
      if (stm) ws.stm += 1;
      P = descend(C, s, L + 1, stm);
      if (P != NIL) {
        uint32_t* vp = &t.imeta[P].version;
        uint32_t v;
        if (try_lock(vp, &v)) {
          const size_t pb = (size_t)P * FAN;
          const uint64_t pk = lane < FAN ? widen(ld_cg(t.ikeys + pb + lane)) : KEY_MAX;
          const uint32_t pc = lane < FAN ? ld_cg(t.ichild + pb + lane) : NIL;
          const uint32_t cP = ld_cg(&t.imeta[P].count);
          const uint64_t plo = ld_cg(&t.imeta[P].lo), phi = ld_cg(&t.imeta[P].hi);
          const uint32_t pnext = ld_cg(&t.imeta[P].next);
          if (s >= plo && s < phi) {   // P covers s: "key in range(node)" (Alg.1:38)
            // the prefix of the entries that P covers; the rest belongs to P's right siblings
            uint32_t m1 = m;
            for (uint32_t base = 0; base < m; base += 32) {
              const uint32_t x = base + lane;
              const uint32_t mk = __ballot_sync(FULL, x < m && ld_cg(K + eb + x) >= phi);
              if (mk) {
                m1 = base + __ffs(mk) - 1;
                break;
              }
            }
            next_m = inner_apply(C, P, L + 1, pk, pc, cP, plo, phi, pnext, K, Ch, K2, Ch2, eb, m1, ws);
            if (next_m > 0 && is_root(t, P, L + 1)) {   // root: phi is the top fence, so m1 == m
              build_root(C, L + 1, P, plo, phi, K2, Ch2, K, Ch, eb, next_m, ws);
              next_m = 0;
            }
            unlock(vp, v + 2u);
            consumed = m1;
            break;
          }
          unlock(vp, v);   // validation failed: P does not cover s (any more)
        }
      }
      ++retry;
      ws.retries += 1;
      if (watchdog(C, ws, 2, L, eb, P, retry)) return;
      backoff(retry);
    }
    // depth first: the entries P's split produced (level L+2 list, at the same
    // offset eb) go before the rest of this level's list
    st_eb[sp] = eb + consumed;
    st_m[sp] = m - consumed;
    if (next_m > 0) {
      ++sp;
      st_L[sp] = L + 1;
      st_eb[sp] = eb;
      st_m[sp] = next_m;
    }
  }
}

// Separator entries of a warp's leaf splits, gathered at [base, base + n) of
// the level-0 entry buffer and inserted into the parents together (one parent
// lock per parent instead of one per split leaf).  Each leaf_apply writes its
// k-1 entries at [b, b+k-1) inside its own run [b, e); runs are processed in
// key order, so the entries are compacted leftwards in key order.
struct SepAcc {
  uint32_t base = NIL, n = 0;
};
__device__ void acc_entries_buf(uint64_t* EK, uint32_t* EC, SepAcc& A, uint32_t b, uint32_t cnt) {
  const int lane = lane_id();
  if (A.base == NIL) A.base = b;
  const uint32_t dst = A.base + A.n;
  if (dst != b) {
    for (uint32_t x0 = 0; x0 < cnt; x0 += 32) {   // dst < b: a forward copy in warp chunks is safe
      const uint32_t x = x0 + lane;
      uint64_t k = 0;
      uint32_t c = 0;
      if (x < cnt) {
        k = ld_cg(EK + b + x);
        c = ld_cg(EC + b + x);
      }
      __syncwarp();
      if (x < cnt) {
        EK[dst + x] = k;
        EC[dst + x] = c;
      }
      __syncwarp();
    }
    // (no fence: the entries are read by this warp, or by others after a grid barrier)
  }
  A.n += cnt;
}
// Level-0 entries of a split leaf, with their parent hint for the level-
// synchronous lookup (the leaf's parent recorded by the locate traversal; the
// inner levels do not change before that lookup, and the apply step validates
// the parent's fences anyway).
__device__ __forceinline__ void acc_entries(const Ctx& C, SepAcc& A, uint32_t b, uint32_t cnt, uint32_t parent) {
  const uint32_t dst = (A.base == NIL ? b : A.base + A.n);
  acc_entries_buf(C.eK[0], C.eC[0], A, b, cnt);
  if (C.eparent)
    for (uint32_t x = lane_id(); x < cnt; x += 32) C.eparent[dst + x] = parent;
}

// One run of writes [b, e) whose first key was located in leaf `hint`.
// Separators of its leaf splits are added to `acc` (inserted by the caller).
__device__ void process_run(const Ctx& C, uint32_t b, uint32_t e, uint32_t hint, WarpStats& ws, SepAcc& acc) {
  const int lane = lane_id();
  const Tree& t = C.t;
  const uint32_t hint0 = hint, b0 = b;   // the run's located leaf and first write
  uint32_t retry = 0;
  while (b < e && !ws.dead) {
    const uint64_t k0 = C.wkey[b];
    const bool stm = C.force_stm || retry >= C.threshold;
    uint32_t X;
    if (retry == 0 && !stm) {
      X = hint;   // the unprotected traversal already done by the locate pass (Alg.1:29)
    } else {
      if (stm) ws.stm += 1;
      X = descend(C, k0, 0, stm);
    }
    if (X != NIL && X < t.leaf_cap) {
      uint32_t* vp = &t.lmeta[X].version;
      uint32_t v;
      if (try_lock(vp, &v)) {   // leafvers = the version the lock saw (Alg.1:35-38)
        // every read of X the run needs, issued together (one round trip)
        const uint64_t lo = ld_cg(&t.lmeta[X].lo), hi = ld_cg(&t.lmeta[X].hi);
        const uint32_t nxt = ld_cg(&t.lmeta[X].next);
        const size_t xb = (size_t)X * LSTRIDE;
        const uint64_t okey = lane < FAN ? widen(ld_cg(t.lkeys + xb + lane)) : KEY_MAX;
        const uint64_t oval = lane < FAN ? widen(ld_cg(t.lvals + xb + lane)) : 0;
        if (k0 >= lo && k0 < hi) {
          uint32_t e2 = e;
          for (uint32_t base = b; base < e; base += 32) {
            const uint32_t j = base + lane;
            const uint32_t mk = __ballot_sync(FULL, j < e && C.wkey[j] >= hi);
            if (mk) {
              e2 = base + __ffs(mk) - 1;
              break;
            }
          }
          const uint32_t k = leaf_apply(C, X, b, e2, hi, nxt, okey, oval, C.eK[0], C.eC[0], ws);
          ws.runs += 1;
          if (k > 1) {
            bool rooted = false;
            if (ws.leaf_root && is_root(t, X, 0)) {
              build_root(C, 0, X, lo, hi, C.eK[0], C.eC[0], C.eK[1], C.eC[1], b, k - 1, ws);
              rooted = true;
            }
            unlock(vp, v + 2u);   // split: version + 1 step
            // parent hint: X was the located leaf (first try) and the inner levels are unchanged
            if (!rooted) acc_entries(C, acc, b, k - 1, X == hint0 ? C.wparent[b0] : NIL);
          } else {
            unlock(vp, v);
          }
          b = e2;
          hint = nxt;
          retry = 0;
          continue;
        }
        unlock(vp, v);   // key not in range(leaf): abort (Alg.1:40-43)
        if (lane == 0 && retry == 0) atomicAdd(&C.ctl->dbg[4], 1u);
      } else if (lane == 0 && retry == 0) {
        atomicAdd(&C.ctl->dbg[3], 1u);
      }
    }
    ++retry;
    ws.retries += 1;
    if (watchdog(C, ws, 1, b, e, X, retry)) return;
    backoff(retry);
  }
}


#ifndef UPD_BATCH_LAST
#define UPD_BATCH_LAST 1   // A/B: 0 = the chunk's last run always through process_run
#endif
#ifndef UPD_STRIPES
#define UPD_STRIPES 1   // level-0 chunk-claim counters (r4a: 8 striped counters: cfg4 update 508 -> 523 us)
#endif
constexpr uint32_t UPD_LSYNC_CH = 16;   // writes per level-0 chunk under a split storm (r3t: 32 slower on cfg1)
// Dynamic shared memory of batched_runs: per warp, the key + value blocks of up
// to UPD_LSYNC_CH locked leaves and the kept plan (upserts before each key)
constexpr size_t UPD_SMEM_PER_WARP = (size_t)UPD_LSYNC_CH * (2 * FAN * sizeof(uint64_t) + FAN);
#ifndef UPD_BATCH
#define UPD_BATCH 1   // A/B: 0 = every leaf run of a chunk through process_run, one after the other
#endif
// Split storms (level-synchronous mode): the leaf runs of one chunk that end
// inside it (head lanes `bm`, run of lane h = [base + h, eL_h), leaf lf_h,
// key order = lane order) applied TOGETHER, so the chunk pays each round trip
// of Alg.1:34-45 once instead of once per run: every leaf locked at once
// (test-and-set per lane), every locked leaf's fences and key/value block read
// at once (into shared memory), one allocation for all splits, one fence, all
// links and releases at once.  Each run holds <= 16 writes, so it leaves at
// most two leaves (k <= 2: one separator entry).  A run whose lock is busy or
// whose keys fall outside the leaf's fences (Alg.1:40-43) is released
// untouched and returned in the mask for process_run (retry / STM).  Per lane
// h of a split run: ek = the new leaf's first key, nid = its id.
__device__ uint32_t batched_runs(const Ctx& C, uint32_t base, uint32_t bm, uint32_t eL, uint32_t lf, WarpStats& ws,
                                 uint64_t& ek, uint32_t& nid, bool& split) {
  // [run head lane][key 0-15, value 0-15] of this warp (dynamic shared memory, UPD_SMEM_PER_WARP per warp)
  extern __shared__ __align__(16) unsigned char upd_smem[];
  const int lane = lane_id();
  const uint32_t wi = threadIdx.x >> 5;
  uint64_t (*s_lk)[2 * FAN] = reinterpret_cast<uint64_t (*)[2 * FAN]>(upd_smem + wi * UPD_SMEM_PER_WARP);
  uint8_t (*s_ub)[FAN] = reinterpret_cast<uint8_t (*)[FAN]>(upd_smem + wi * UPD_SMEM_PER_WARP +
                                                            (size_t)UPD_LSYNC_CH * 2 * FAN * sizeof(uint64_t));
  const Tree& t = C.t;
  const bool mine = ((bm >> lane) & 1u) && lf < t.leaf_cap;
  uint32_t* vp = &t.lmeta[mine ? lf : 0].version;
  uint32_t v = 0;
  bool got = false;
  if (mine) {   // TX_BEGIN for every run at once (eager ownership, Alg.1:37)
    v = atom_or_acquire(vp, 1u);
    got = !(v & 1u);
  }
  __syncwarp();
  uint64_t lo = 0, hi = 0, k0 = 0, kl = 0;
  uint32_t nxt = NIL;
  if (got) {   // leafvers / fences / link, and the run's first and last key (Alg.1:35-38)
    lo = ld_cg(&t.lmeta[lf].lo);
    hi = ld_cg(&t.lmeta[lf].hi);
    nxt = ld_cg(&t.lmeta[lf].next);
    k0 = C.wkey[base + lane];
    kl = C.wkey[eL - 1];
  }
  const uint32_t gm = __ballot_sync(FULL, got);
  for (uint32_t m = gm; m;) {   // the locked leaves' key + value blocks, four in flight per lane
    int r[4];
    uint64_t x[4];
#pragma unroll
    for (int u = 0; u < 4; ++u) {
      r[u] = m ? __ffs(m) - 1 : -1;
      if (m) m &= m - 1;
    }
#pragma unroll
    for (int u = 0; u < 4; ++u) {
      const uint32_t X = __shfl_sync(FULL, lf, r[u] < 0 ? 0 : r[u]);
      x[u] = r[u] >= 0 ? widen(ld_cg(t.lkeys + (size_t)X * LSTRIDE + lane)) : 0ull;   // (values follow the keys)
    }
#pragma unroll
    for (int u = 0; u < 4; ++u)
      if (r[u] >= 0) s_lk[r[u]][lane] = x[u];
  }
  __syncwarp();
  const bool ok = got && k0 >= lo && k0 < hi && kl < hi;   // key in range(leaf) (Alg.1:38)
  if (got && !ok) st_release(vp, v);                         // abort, untouched (Alg.1:40-43)
  const uint32_t om = __ballot_sync(FULL, ok);
  // plan: every run's size after the merge -> in place (0), one leaf (1) or two
  // (2); the plan is kept (lane r: c, mmask; smem: upserts before each leaf key)
  uint32_t tout_l = 0, k_l = 1, c_l = 0, mm_l = 0;
  for (uint32_t m = om; m; m &= m - 1) {
    const int r = __ffs(m) - 1;
    const uint32_t re = __shfl_sync(FULL, eL, r);
    const uint64_t okey = lane < FAN ? s_lk[r][lane] : KEY_MAX;
    const LeafPlan L = leaf_plan(C, base + r, re, okey);
    const uint32_t tout = L.c - __popc(L.mmask) + L.U;
    if (lane < FAN) s_ub[r][lane] = (uint8_t)L.ups_before;
    if (lane == r) {
      tout_l = tout;
      k_l = L.inplace ? 0u : (tout <= FAN ? 1u : 2u);
      c_l = L.c;
      mm_l = L.mmask;
    }
  }
  __syncwarp();
  const uint32_t sm = __ballot_sync(FULL, ok && k_l == 2);
  const uint32_t first = sm ? warp_alloc(&t.hdr->leaf_count, __popc(sm)) : 0u;   // one allocation for all splits
  nid = first + __popc(sm & lanemask_lt());
  for (uint32_t m = om; m; m &= m - 1) {   // the merges (stores only)
    const int r = __ffs(m) - 1;
    const uint32_t re = __shfl_sync(FULL, eL, r), X = __shfl_sync(FULL, lf, r);
    const uint32_t kr = __shfl_sync(FULL, k_l, r), tr = __shfl_sync(FULL, tout_l, r), idr = __shfl_sync(FULL, nid, r);
    const uint64_t okey = lane < FAN ? s_lk[r][lane] : KEY_MAX;
    if (kr == 0) {
      leaf_overwrite(C, X, base + r, re, okey);
      continue;
    }
    const uint64_t oval = lane < FAN ? s_lk[r][FAN + lane] : 0ull;
    LeafPlan L;
    L.c = __shfl_sync(FULL, c_l, r);
    L.mmask = __shfl_sync(FULL, mm_l, r);
    L.ups_before = lane < FAN ? s_ub[r][lane] : 0u;
    L.inplace = false;
    const uint64_t k1 = leaf_place(C, X, idr, base + r, re, okey, oval, L, tr, kr, nullptr, nullptr);
    if (lane == r) ek = k1;
  }
  split = (sm >> lane) & 1u;
  __syncwarp();
  if (split) {   // the fresh leaves' meta: unreachable until X links them below
    NodeMeta mt;
    mt.version = 0;
    mt.lo = ek;
    mt.hi = hi;
    mt.next = nxt;
    mt.count = tout_l / 2;
    mt.level = 0;
    t.lmeta[nid] = mt;
    t.lrf[nid] = t.lrf[lf];   // (inherits the RF, repaired lazily)
  }
  if (sm) __threadfence();    // one fence for every split of the chunk
  __syncwarp();
  if (ok) {
    if (split) {
      t.lmeta[lf].hi = ek;
      t.lmeta[lf].next = nid;
      t.lmeta[lf].count = tout_l - tout_l / 2;
    } else if (k_l == 1) {
      t.lmeta[lf].count = tout_l;
    }
  }
  __syncwarp();   // every lane's stores into the leaves happen-before the releases
  if (ok) st_release(vp, split ? v + 2u : v);   // a split: version + 1 step
  __syncwarp();
  ws.runs += __popc(om);
  ws.leaf_splits += __popc(sm);
  ws.new_leaves += __popc(sm);
  return bm & ~om;
}

// Level-0 entries of split runs (lanes in sm, one entry each: (ek, nid)) appended
// to the chunk's list in key (= lane) order; parent hint = the located leaf's parent.
__device__ __forceinline__ void append_entries(const Ctx& C, SepAcc& A, uint32_t base, uint32_t sm, uint64_t ek,
                                               uint32_t nid) {
  if (!sm) return;
  const int lane = lane_id();
  if (A.base == NIL) A.base = base + __ffs(sm) - 1;
  const uint32_t dst = A.base + A.n + __popc(sm & lanemask_lt());   // <= the run's own first write
  if ((sm >> lane) & 1u) {
    C.eK[0][dst] = ek;
    C.eC[0][dst] = nid;
    if (C.eparent) C.eparent[dst] = C.wparent[base + lane];
  }
  A.n += __popc(sm);
}

// ---------------------------------------------------------------- level-synchronous separators
// Under a split storm (cfg1: every leaf splits; cfg4) per-warp upward
// insertion makes every warp whose leaves share a parent queue on that
// parent's lock, and every split parent's warp queue on the grandparent's,
// up to the root.  When the batch can split (some issued upsert targets an
// absent key, ctl->nins), the kernel is a persistent grid and separators go
// up one level at a time instead (the regrouping of a4 applied to the inner
// levels):
//   level 0: every warp applies its leaf runs; each 32-write chunk leaves its
//            separators contiguous at [base, base+n) of entry buffer 0 and
//            records (base, n) in slots[0][chunk] -- chunk order = key order;
//   lookup : (grid barrier) every entry's parent at level L+1, by an
//            unprotected per-thread descent of the level-quiescent tree;
//   apply  : (grid barrier) the entries of one parent form one segment; the
//            warp whose unit range holds the segment's first entry owns it,
//            gathers it (in place, leftwards), locks the parent, validates its
//            fences (Alg.1:38) and merges the whole segment (inner_apply,
//            multi-way split); the next level's separators are recorded per
//            warp in slots[1 - x].  A root split builds the new root(s).
// Levels >= 1 (few entries, produced by owner warps): the producers' lists are
// first concatenated in key order into one flat list (per-CTA totals, a scan
// by CTA 0, every warp copies its list and looks its entries' parents up), so
// each parent's entries are contiguous; a warp owns the segments whose first
// entry falls in its slice of the flat list (no gather).
// Owners are unique per parent, so the locks are uncontended; a failed
// validation (not expected) falls back to insert_up's optimistic / STM retry.
__device__ int g_uprof = 0;   // diagnostic: print the phase times of the level-synchronous path
__device__ void grid_barrier(BatchCtl* ctl, uint32_t& gen) {
  const uint32_t bi = gen / gridDim.x;
  if (g_uprof && blockIdx.x == 0 && threadIdx.x == 0 && 2 * bi + 2 < 24) ctl->uprof[2 * bi + 1] = gtime_ns();
  __syncthreads();
  gen += gridDim.x;
  if (threadIdx.x == 0) {
    __threadfence();
    atomicAdd(&ctl->ubar, 1u);
    SpinGuard sg;
    while (ld_acquire(&ctl->ubar) < gen) {
      __nanosleep(64);
      if (sg.stuck(ctl)) break;
    }
    if (g_uprof && blockIdx.x == 0 && 2 * bi + 2 < 24) ctl->uprof[2 * bi + 2] = gtime_ns();
  }
  __syncthreads();
}

// Node at level `target` (>= 1) whose fences hold k: one thread, unprotected
// (the inner levels are quiescent during a lookup step), B-link move-right.
__device__ uint32_t descend_thread(const Tree& t, uint64_t k, uint32_t target) {
  const unsigned long long rw = ld_acquire64(&t.hdr->root_word);
  const uint32_t height = (uint32_t)(rw >> 32);
  uint32_t node = (uint32_t)rw;
  if (height == 0 || target + 1 > height) return NIL;
  uint32_t lvl = height - 1;
  for (int steps = 0; steps < 4096; ++steps) {
    const NodeMeta* m = t.imeta + node;
    const uint64_t hi = ld_cg(&m->hi);
    const uint32_t nxt = ld_cg(&m->next);
    if (k >= hi && nxt != NIL) {
      node = nxt;
      continue;
    }
    if (lvl == target) return node;
    const tkey_t* kl = t.ikeys + (size_t)node * FAN;
    uint32_t c = 0;
#pragma unroll
    for (int i = 0; i < FAN - 1; ++i) c += ld_cg(kl + i) <= k ? 1u : 0u;
    node = ld_cg(t.ichild + (size_t)node * FAN + c);
    --lvl;
  }
  return NIL;
}

// units [u0, u1) of a level's producer list, for this warp
__device__ __forceinline__ void unit_range(uint32_t U, uint32_t gw, uint32_t nwarps, uint32_t& u0, uint32_t& u1) {
  u0 = (uint32_t)(((unsigned long long)U * gw) / nwarps);
  u1 = (uint32_t)(((unsigned long long)U * (gw + 1)) / nwarps);
}

// Propagate the separators of level L (entries in buffer L&1, producer list
// slots[x] with U units) up to the root.
__device__ void levels_up(const Ctx& C, uint32_t U, uint32_t gw, uint32_t nwarps, uint32_t& gen, WarpStats& ws) {
  const int lane = lane_id();
  const Tree& t = C.t;
  for (uint32_t L = 0; L + 1 < MAX_LEVELS; ++L) {
    grid_barrier(C.ctl, gen);
    // (uniform: read after the barrier, by one thread per CTA -- every thread
    // loading the same word is an L2 same-address storm)
    __shared__ uint32_t s_lv;
    if (threadIdx.x == 0) s_lv = ld_cg(&C.ctl->lvl_ent[L]);
    __syncthreads();
    if (s_lv == 0) return;
    const uint2* sl = C.slots[L & 1];
    uint2* sn = C.slots[(L + 1) & 1];
    uint64_t* K = C.eK[L & 1];
    uint32_t* Ch = C.eC[L & 1];
    uint64_t* K2 = C.eK[(L + 1) & 1];
    uint32_t* Ch2 = C.eC[(L + 1) & 1];
    uint32_t u0, u1;
    unit_range(U, gw, nwarps, u0, u1);
    uint32_t ftotal = 0;   // L >= 1: entries of the flattened level
    if (L > 0) {
      // Upper levels: the producers are warps (one unit each, key order = warp
      // order) and a parent's entries come from many of them.  Concatenate the
      // units into one flat list (CTA 0 scans the counts, barrier, every warp
      // copies its unit), so every segment is contiguous and the apply step
      // walks 32-entry units instead of gathering unit by unit.
      // (1) per CTA: its warps' (= producers') counts and their offsets inside
      // the CTA; (2) CTA 0 scans the CTA totals; (3) every warp's offset
      __shared__ uint32_t s_woff[UPD_THREADS / 32], s_cta;
      if (threadIdx.x == 0) {
        uint32_t run = 0;
        for (uint32_t w = 0; w < (blockDim.x >> 5); ++w) {
          s_woff[w] = run;
          const uint32_t uw = blockIdx.x * (blockDim.x >> 5) + w;
          run += uw < U ? sl[uw].y : 0u;
        }
        C.flat_off[blockIdx.x] = run;   // this CTA's total (scanned by CTA 0 below)
      }
      grid_barrier(C.ctl, gen);
      if (blockIdx.x == 0) {
        __shared__ uint32_t s_part[UPD_THREADS];
        const uint32_t nc = gridDim.x, per = (nc + blockDim.x - 1) / blockDim.x;
        const uint32_t a0 = threadIdx.x * per, z0 = min(nc, a0 + per);
        uint32_t v[16];   // per <= 16 (<= 2048 CTAs)
        uint32_t sum = 0;
#pragma unroll
        for (int q = 0; q < 16; ++q) {
          v[q] = (a0 + q < z0) ? ld_cg(C.flat_off + a0 + q) : 0u;
          sum += v[q];
        }
        s_part[threadIdx.x] = sum;
        __syncthreads();
        if (threadIdx.x == 0) {
          uint32_t run = 0;
          for (uint32_t i = 0; i < blockDim.x; ++i) {
            const uint32_t c = s_part[i];
            s_part[i] = run;
            run += c;
          }
          C.ctl->flat_total = run;
        }
        __syncthreads();
        uint32_t run = s_part[threadIdx.x];
#pragma unroll
        for (int q = 0; q < 16; ++q) {
          if (a0 + q < z0) C.flat_off[a0 + q] = run;   // exclusive offset of CTA a0 + q
          run += v[q];
        }
      }
      grid_barrier(C.ctl, gen);
      // copy my unit into the flat list and look its entries' parents up (lanes over entries)
      __shared__ uint32_t s_ft;
      if (threadIdx.x == 0) {
        s_ft = ld_cg(&C.ctl->flat_total);
        s_cta = ld_cg(C.flat_off + blockIdx.x);
      }
      __syncthreads();
      ftotal = s_ft;
      for (uint32_t u = u0; u < u1; ++u) {   // (u == gw: my own unit)
        const uint2 su = sl[u];
        const uint32_t off = s_cta + s_woff[threadIdx.x >> 5];
        for (uint32_t x = lane; x < su.y; x += 32) {
          const uint64_t k = ld_cg(K + su.x + x);
          C.flat_key[off + x] = k;
          C.flat_child[off + x] = ld_cg(Ch + su.x + x);
          C.eparent[off + x] = descend_thread(t, k, L + 1);
        }
      }
    }
    // lookup step: parent of every entry (lanes over units, then over a unit's entries)
    if (L == 0) {   // many small units (chunks): lanes over units
      for (uint32_t ub = u0; ub < u1; ub += 32) {
        const uint32_t u = ub + lane;
        const uint2 su = u < u1 ? sl[u] : make_uint2(0, 0);
        for (uint32_t x = 0; x < su.y; ++x) {
          // level 0: entries carry their parent hint (acc_entries); look up the rest
          if (ld_cg(C.eparent + su.x + x) != NIL) continue;
          C.eparent[su.x + x] = descend_thread(t, ld_cg(K + su.x + x), L + 1);
        }
      }
    }
    grid_barrier(C.ctl, gen);
    // the apply step's units: L = 0 the chunks; L >= 1 32-entry slices of the flat list
    const uint32_t UA = L > 0 ? (ftotal + 31) / 32 : U;
    if (L > 0) {
      K = C.flat_key;
      Ch = C.flat_child;
      unit_range(UA, gw, nwarps, u0, u1);
    }
    auto unit = [&](uint32_t x) -> uint2 {
      return L > 0 ? make_uint2(32u * x, min(32u, ftotal - 32u * x)) : sl[x];
    };
    // apply step
    SepAcc nxt;
    // parent of the last entry before my range (the owner test of my first entry)
    uint32_t prevP = NIL;
    if (L > 0 && u0 > 0 && u0 <= UA) {   // flat units are all nonempty: the previous one is u0 - 1
      const uint2 su = unit(u0 - 1);
      prevP = ld_cg(C.eparent + su.x + su.y - 1);
    }
    for (uint32_t ue = L > 0 ? 0u : u0; ue > 0;) {   // level 0: nearest nonempty chunk before u0, 32 per step
      const uint32_t ub = ue > 32 ? ue - 32 : 0;
      const uint32_t uu = ub + lane;
      const uint2 su = uu < ue ? sl[uu] : make_uint2(0, 0);
      const uint32_t ne = __ballot_sync(FULL, su.y != 0);
      if (ne) {
        const int hl = 31 - __clz(ne);
        const uint32_t bx = __shfl_sync(FULL, su.x, hl), by = __shfl_sync(FULL, su.y, hl);
        prevP = ld_cg(C.eparent + bx + by - 1);
        break;
      }
      ue = ub;
    }
    // next unit >= from with entries (U if none), 32 units per step
    auto next_nonempty = [&](uint32_t from) -> uint32_t {
      if (L > 0) return from < UA ? from : UA;
      for (uint32_t ub = from; ub < U; ub += 32) {
        const uint32_t uu = ub + lane;
        const bool ne = uu < U && sl[uu].y != 0;
        const uint32_t bm = __ballot_sync(FULL, ne);
        if (bm) return ub + __ffs(bm) - 1;
      }
      return U;
    };
    // lock the parent P, validate its fences, merge the segment [hpos, hpos + m) of K / Ch
    auto apply_segment = [&](uint32_t P, uint32_t hpos, uint32_t m) {
      uint32_t* vp = &t.imeta[P].version;
      uint32_t v;
      bool done = false;
      if (P != NIL && try_lock(vp, &v)) {
        const size_t pb = (size_t)P * FAN;
        const uint64_t pk = lane < FAN ? widen(ld_cg(t.ikeys + pb + lane)) : KEY_MAX;
        const uint32_t pc = lane < FAN ? ld_cg(t.ichild + pb + lane) : NIL;
        const uint32_t cP = ld_cg(&t.imeta[P].count);
        const uint64_t plo = ld_cg(&t.imeta[P].lo), phi = ld_cg(&t.imeta[P].hi);
        const uint32_t pnext = ld_cg(&t.imeta[P].next);
        const uint64_t s0 = ld_cg(K + hpos), s1 = ld_cg(K + hpos + m - 1);
        if (s0 >= plo && s1 < phi) {
          uint32_t next_m = inner_apply(C, P, L + 1, pk, pc, cP, plo, phi, pnext, K, Ch, K2, Ch2, hpos, m, ws);
          if (next_m > 0 && is_root(t, P, L + 1)) {
            build_root(C, L + 1, P, plo, phi, K2, Ch2, K, Ch, hpos, next_m, ws);
            next_m = 0;
          }
          unlock(vp, v + 2u);
          if (next_m) acc_entries_buf(K2, Ch2, nxt, hpos, next_m);
          done = true;
        } else {
          unlock(vp, v);
        }
      }
      if (!done) {   // not expected: the generic optimistic / STM path, one level at a time upward
        ws.retries += 1;
        if (K != C.eK[L & 1]) {   // flat list: insert_up reads the level's own buffer (free by now)
          for (uint32_t q = lane; q < m; q += 32) {
            C.eK[L & 1][hpos + q] = ld_cg(K + hpos + q);
            C.eC[L & 1][hpos + q] = ld_cg(Ch + hpos + q);
          }
          __threadfence();
          __syncwarp();
        }
        insert_up(C, L, hpos, m, ws);
      }
    };
    if (L > 0) {
      // flat list: this warp owns the segments whose first entry lies in its
      // slice of the entries; a segment is contiguous, found by one ballot per 32
      const uint32_t e0 = (uint32_t)(((unsigned long long)ftotal * gw) / nwarps);
      const uint32_t e1 = (uint32_t)(((unsigned long long)ftotal * (gw + 1)) / nwarps);
      uint32_t prevE = e0 > 0 ? ld_cg(C.eparent + e0 - 1) : NIL;
      uint32_t e = e0;
      while (e < e1 && !ws.dead) {
        const uint32_t P = ld_cg(C.eparent + e);
        if (P == prevE) {   // continues a segment owned by an earlier warp
          ++e;
          continue;
        }
        uint32_t end = ftotal;
        for (uint32_t b0 = e + 1; b0 < ftotal; b0 += 32) {
          const uint32_t q = b0 + lane;
          const uint32_t bm = __ballot_sync(FULL, q < ftotal && ld_cg(C.eparent + q) != P);
          if (bm) {
            end = b0 + __ffs(bm) - 1;
            break;
          }
        }
        apply_segment(P, e, end - e);
        prevE = P;
        e = end;
      }
      u0 = u1 = 0;   // (the unit loop below has nothing left to do)
    }
    uint32_t u = u0, x = 0;   // cursor: entry x of unit u
    while (u < u1 && !ws.dead) {
      const uint2 su = unit(u);
      if (x >= su.y) {
        u = next_nonempty(u + 1);
        x = 0;
        continue;
      }
      const uint32_t hpos = su.x + x;
      const uint32_t P = ld_cg(C.eparent + hpos);
      if (P == prevP) {   // continues a segment owned by an earlier warp / segment
        ++x;
        continue;
      }
      // a segment head in my range: gather its entries to [hpos, hpos + m)
      uint32_t m = 0, cu = u, cx = x;
      for (;;) {
        if (cu >= UA) break;
        const uint2 sc = unit(cu);
        if (cx >= sc.y) {
          cu = next_nonempty(cu + 1);
          cx = 0;
          continue;
        }
        // entries cx.. of unit cu with parent P (lane-parallel, stops at the first other parent)
        const uint32_t avail = sc.y - cx;
        uint32_t take = 0;
        for (uint32_t b0 = 0; b0 < avail; b0 += 32) {
          const uint32_t q = b0 + lane;
          const bool same = q < avail && ld_cg(C.eparent + sc.x + cx + q) == P;
          const uint32_t bm = __ballot_sync(FULL, q < avail && !same);
          const uint32_t upto = bm ? (uint32_t)(__ffs(bm) - 1) : min(32u, avail - b0);
          // move [b0, b0 + upto) to [hpos + m + b0, ...) (leftwards or in place)
          uint64_t kk = 0;
          uint32_t cc = 0;
          if ((uint32_t)lane < upto) {
            kk = ld_cg(K + sc.x + cx + b0 + lane);
            cc = ld_cg(Ch + sc.x + cx + b0 + lane);
          }
          __syncwarp();
          if ((uint32_t)lane < upto) {
            K[hpos + m + b0 + lane] = kk;
            Ch[hpos + m + b0 + lane] = cc;
          }
          __syncwarp();
          take = b0 + upto;
          if (bm) break;
        }
        m += take;
        cx += take;
        if (cx < sc.y) break;   // another parent's entry: the segment ends here
      }
      __threadfence();
      __syncwarp();
      apply_segment(P, hpos, m);
      prevP = P;
      u = cu;
      x = cx;
      if (u >= u1) break;   // the segment ran past my range: the rest belongs to it
    }
    if (lane == 0) {
      sn[gw] = make_uint2(nxt.base == NIL ? 0u : nxt.base, nxt.n);
      if (nxt.n) atomicAdd(&C.ctl->lvl_ent[L + 1], nxt.n);
    }
    U = nwarps;
  }
}

#ifndef UPD_MINB
#if UPD_THREADS == 128
#define UPD_MINB 6   // resident CTAs per SM the register budget is fitted to (A/B builds: -DUPD_MINB=n;
                     // r1h: 6 (80 regs, no spills) vs 8 (64 regs, 432 B spills): cfg1 0.389 -> 0.404, cfg2 6.92 -> 7.04)
#else
#define UPD_MINB 1   // one CTA of UPD_THREADS per SM (the same 24 warps at 80 registers)
#endif
#endif
__device__ __forceinline__ void update_body(const Ctx& C);

// The batch's last kernel: the structural writes (Alg.1:23-46), then every
// CTA's share of the long-segment RESULT_CAL and the batch's BatchCtl
// (result_phase, eirene_internal.cuh) -- one launch for both.
__global__ void __launch_bounds__(UPD_THREADS, UPD_MINB) update_kernel(Ctx C, ResultArgs R) {
  pdl_wait();   // predecessor kernel complete, its writes visible (no-op without PDL)
  pdl_trigger();
  const BatchCtl* ctl = C.ctl;
  // What is left, read by ONE thread per CTA (every thread of every CTA
  // loading the same flags made a same-address load storm: r3v, a no-op update
  // kernel took 11 us with 3552 warps loading, 7.5 us with 592):
  //   0: nothing (no structural write, long segment or deferred hot key; the
  //      common case of a read-mostly batch): CTA 0 ends the batch at once, no
  //      arrival counting, the other CTAs just exit;
  //   1: the result phase only: a rejected batch, or every issued write was a
  //      value overwrite of a present key, all applied in place by the query
  //      kernel's locate (query.cu, retire) -- nothing structural is left;
  //   2: structural writes, then the result phase.
  // (Uniform: every CTA reads the same flags before any changes them.)
  __shared__ uint32_t s_mode;
  if (threadIdx.x == 0) {
    uint32_t m = 0;
    if (update_needed(ctl, R.A))
      m = (ctl->invalid || ctl->status != 0 || (ctl->nins == 0 && ctl->ndelp == 0)) ? 1u : 2u;
    s_mode = m;
  }
  __syncthreads();
  const uint32_t mode = s_mode;
  if (mode == 0) {
    if (blockIdx.x == 0) {
      if (threadIdx.x == 0) C.ctl->upd_ran = 1;
      publish_batch(C.ctl, R.A, R.hdr);
    }
    return;
  }
  if (blockIdx.x == 0 && threadIdx.x == 0) C.ctl->upd_ran = 1;
  if (mode == 2) update_body(C);
  result_phase(R);
}

__device__ __forceinline__ void update_body(const Ctx& C) {
  const BatchCtl* ctl = C.ctl;
  if (g_uprof && blockIdx.x == 0 && threadIdx.x == 0) C.ctl->uprof[0] = gtime_ns();
  const uint32_t nw = ctl->nw;
  const int lane = lane_id();
  const uint32_t gw = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const uint32_t nwarps = (gridDim.x * blockDim.x) >> 5;
  const Tree& t = C.t;
  WarpStats ws;
  ws.t0 = gtime_ns();
  ws.leaf_root = (uint32_t)(ld_acquire64(&t.hdr->root_word) >> 32) <= 1;   // (heights never shrink)
  SepAcc acc;
  // level-synchronous separators when the batch can split (launch: resident grid)
  const bool lsync = C.regroup && C.slots[0] != nullptr && ctl->nins > 0;
  // writes per chunk: a warp takes one chunk at a time and its leaf runs one
  // after the other; under a split storm (lsync) each run is a long dependent
  // chain, so chunks of 16 halve the runs a warp applies in a row
  const uint32_t CH = lsync ? (uint32_t)UPD_LSYNC_CH : 32u;
  const uint32_t nchunks = (nw + CH - 1) / CH;
  if (C.regroup) {
    // Under a split storm a chunk's cost varies with its leaf runs and splits:
    // chunks are handed out dynamically (a warp takes the next one when done) so
    // the level-0 phase ends at the average warp's time, not the unluckiest one's
    // (one chunk per claim: claiming 4 at a time, r3i, made cfg4's update 513 -> 532 us -- the
    // tail imbalance costs more than the claims' atomics on one address)
    const uint32_t G = 1u;
    uint32_t c_next = 0, c_end = 0;
#if UPD_STRIPES > 1
    // (and spread over UPD_STRIPES counters on their own lines: the chunks are
    // cut into that many contiguous stripes, a warp starts on stripe gw % S and
    // moves on when its stripe is exhausted -- the same dynamic balance with
    // 1/S of the same-address atomics per counter)
    (void)G;
    (void)c_end;
    const uint32_t NS = UPD_STRIPES, ssz = (nchunks + NS - 1) / NS;
    uint32_t stripe = gw % NS, tried = 0;
    auto next_chunk = [&]() -> uint32_t {
      while (tried < NS) {
        uint32_t c = 0;
        if (lane == 0) c = atomicAdd(&C.ctl->ustripe[stripe][0], 1u);
        c = __shfl_sync(FULL, c, 0);
        const uint32_t ch = stripe * ssz + c;
        if (c < ssz && ch < nchunks) return ch;
        stripe = (stripe + 1) % NS;
        ++tried;
      }
      return nchunks;   // (ends the loop: chunk * CH >= nw)
    };
#else
    auto next_chunk = [&]() -> uint32_t {
      if (c_next == c_end) {
        uint32_t c = 0;
        if (lane == 0) c = atomicAdd(&C.ctl->uchunk, G);
        c_next = __shfl_sync(FULL, c, 0);
        c_end = c_next + G;
      }
      return c_next++;
    };
#endif
    uint32_t lvl0 = 0;   // this warp's level-0 entries (one atomic per warp, not per chunk)
    for (uint32_t chunk = lsync ? next_chunk() : gw; chunk * CH < nw;
         chunk = lsync ? next_chunk() : chunk + nwarps) {
      const uint32_t base = chunk * CH;
      const uint32_t j = base + lane;
      const bool act = (uint32_t)lane < CH && j < nw;
      const uint32_t lf = act ? C.wleaf[j] : NIL;
      const uint32_t pv = (act && j > 0) ? C.wleaf[j - 1] : NIL;
      const bool head = act && (j == 0 || lf != pv);
      // Lane-parallel path for the common case: a run that lies inside this
      // chunk and whose writes all overwrite keys present in the leaf.  The run's
      // head lane is the run's "thread" of Alg.1:24: leafvers = version
      // (Alg.1:35); CAS(v -> v|1) (TX_BEGIN, eager ownership); every member
      // validates that its key still sits in the located slot (the range check
      // of Alg.1:38 specialised to an in-place write) and writes its value; the
      // head releases.  Any failure sends the run to the general path below
      // (value overwrites are idempotent, so redoing them there is harmless).
      const uint32_t nx = (act && j + 1 < nw) ? C.wleaf[j + 1] : NIL;
      const uint8_t sl = act ? C.wslot[j] : 255;
      const bool member = act && sl != 255 && C.wop[j] != OP_DELETE;
      const uint32_t allheads = __ballot_sync(FULL, head);
      const uint32_t tails = __ballot_sync(FULL, act && nx != lf);   // last write of its run
      const uint32_t nonmember = __ballot_sync(FULL, act && !member);
      // run of lane x: [head_x, tail_x]; fast iff it ends in this chunk and has no non-member
      const int hl = 31 - __clz(allheads & (lanemask_lt() | (1u << lane)));   // my run's head lane
      const uint32_t from_h = ~((1u << hl) - 1u);
      const uint32_t tail_after = tails & from_h;
      const int tl = tail_after ? __ffs(tail_after) - 1 : 32;
      const uint32_t span = tl < 32 ? (from_h & ((2u << tl) - 1u)) : 0u;
      bool fast = act && tl < 32 && (nonmember & span) == 0;
      uint32_t lk = 0;   // head: acquired?
      uint32_t v = 0;
      uint32_t* vp = &t.lmeta[act ? lf : 0].version;
      if (fast && lane == hl) {
        v = ld_relaxed(vp);
        lk = (!(v & 1u) && atom_cas_acquire(vp, v, v | 1u) == v) ? 1u : 0u;
      }
      const uint32_t got = __shfl_sync(FULL, lk, hl & 31);
      fast = fast && got;
      bool ok = true;
      if (fast) {
        const size_t at = (size_t)lf * LSTRIDE + sl;
        if (widen(ld_cg(t.lkeys + at)) == C.wkey[j]) {
          t.lvals[at] = C.wval[j];
        } else {
          ok = false;
        }
      }
      const uint32_t bad = __ballot_sync(FULL, fast && !ok);
      __syncwarp();
      if (lk) st_release(vp, v);
      fast = fast && (bad & span) == 0;
      const uint32_t fastm = __ballot_sync(FULL, fast);
      ws.runs += __popc(fastm & allheads);
      uint32_t heads = allheads & ~fastm;
#if UPD_BATCH
      // the runs ending inside the chunk, applied together (first attempts are
      // optimistic: not with FORCE_STM / THRESHOLD 0, whose first attempt is STM)
      if (lsync && !ws.leaf_root && !C.force_stm && C.threshold > 0) {
        const uint32_t later_l = allheads & ~((2u << lane) - 1u);
        bool cand = ((heads >> lane) & 1u) && later_l != 0;
        uint32_t eL = cand ? base + __ffs(later_l) - 1 : 0u;
#if UPD_BATCH_LAST
        // the chunk's last run (its end may lie in the next chunk, whose warp
        // skips it): its end found as process_run's caller would, then batched
        // too if short -- so a chunk is one batch, not a batch and a chain
        if (allheads) {
          const int hl = 31 - __clz(allheads);
          if ((heads >> hl) & 1u) {
            const uint32_t leaf = __shfl_sync(FULL, lf, hl);
            uint32_t e = nw;
            for (uint32_t s2 = base + CH; s2 < nw; s2 += 32) {
              const uint32_t jj = s2 + lane;
              const uint32_t mk = __ballot_sync(FULL, jj < nw && C.wleaf[jj] != leaf);
              if (mk) {
                e = s2 + __ffs(mk) - 1;
                break;
              }
            }
            if (lane == hl) {
              cand = true;
              eL = e;
            }
          }
        }
#endif
        cand = cand && eL - (base + lane) <= (uint32_t)FAN;   // <= 16 writes: at most two leaves (batched_runs)
        const uint32_t bm = __ballot_sync(FULL, cand);
        if (__popc(bm) >= 2) {
          uint64_t ek = 0;
          uint32_t nid = 0;
          bool split = false;
          const uint32_t fail = batched_runs(C, base, bm, eL, lf, ws, ek, nid, split);
          const uint32_t sm = __ballot_sync(FULL, split);
          if (!fail) {
            append_entries(C, acc, base, sm, ek, nid);
          } else {   // (rare) key order kept: failed runs through process_run in place
            for (uint32_t m = bm; m && !ws.dead; m &= m - 1) {
              const int r = __ffs(m) - 1;
              if ((fail >> r) & 1u) {
                process_run(C, base + r, __shfl_sync(FULL, eL, r), __shfl_sync(FULL, lf, r), ws, acc);
              } else {
                append_entries(C, acc, base, sm & (1u << r), ek, nid);
              }
            }
          }
          heads &= ~bm;
        }
      }
#endif
      while (heads) {
        const int h = __ffs(heads) - 1;
        heads &= heads - 1;
        const uint32_t b = base + h;
        const uint32_t leaf = shfl32(lf, h);
        const uint32_t later = allheads & ~((2u << h) - 1u);   // heads after h (fast ones included)
        uint32_t e;
        if (later) {
          e = base + __ffs(later) - 1;
        } else {
          e = nw;
          for (uint32_t s = base + CH; s < nw; s += 32) {
            const uint32_t jj = s + lane;
            const uint32_t mk = __ballot_sync(FULL, jj < nw && C.wleaf[jj] != leaf);
            if (mk) {
              e = s + __ffs(mk) - 1;
              break;
            }
            if (s + 32 >= nw) e = nw;
          }
        }
        process_run(C, b, e, leaf, ws, acc);
        if (ws.dead) break;
      }
      if (lsync) {
        if (lane == 0) {
          C.slots[0][chunk] = make_uint2(acc.base == NIL ? 0u : acc.base, acc.n);
          lvl0 += acc.n;
        }
      } else if (acc.n && !ws.dead) {
        insert_up(C, 0, acc.base, acc.n, ws);
      }
      acc = SepAcc{};
    }
    if (lsync) {
      if (lane == 0 && lvl0) atomicAdd(&C.ctl->lvl_ent[0], lvl0);   // (read after the grid barrier)
      uint32_t gen = 0;
      levels_up(C, nchunks, gw, nwarps, gen, ws);
    }
  } else {
    for (uint32_t j = gw; j < nw && !ws.dead; j += nwarps) {
      SepAcc one;
      process_run(C, j, j + 1, C.wleaf[j], ws, one);
      if (one.n && !ws.dead) insert_up(C, 0, one.base, one.n, ws);
    }
  }
  if (C.stats) {
    // reduce the counters per CTA first: one global atomic per CTA and counter
    // (same-address atomics serialise in L2)
    __shared__ unsigned long long red[7];
    if (threadIdx.x < 7) red[threadIdx.x] = 0;
    __syncthreads();
    if (lane == 0) {
      const unsigned long long v[7] = {ws.runs, ws.retries, ws.stm, ws.leaf_splits, ws.inner_splits,
                                       ws.new_leaves, ws.new_inner};
      for (int i = 0; i < 7; ++i)
        if (v[i]) atomicAdd(&red[i], v[i]);
    }
    __syncthreads();
    if (threadIdx.x < 7 && red[threadIdx.x]) {
      BatchCtl* c = C.ctl;
      unsigned long long* dst[7] = {&c->leaf_runs, &c->retries, &c->stm_fallbacks, &c->leaf_splits,
                                    &c->inner_splits, &c->new_leaves, &c->new_inner};
      atomicAdd(dst[threadIdx.x], red[threadIdx.x]);
    }
  }
}

}  // namespace

void launch_update(uint32_t n, const CombBufs& c, Tree t, BatchCtl* ctl, UpdParams p, const ResultArgs& r,
                   int num_sms, cudaStream_t st, int* launches) {
  Ctx C;
  C.t = t;
  C.wkey = c.wkey;
  C.wop = c.wop;
  C.wval = c.wval;
  C.wseg = c.wseg;
  C.wleaf = c.wleaf;
  C.wslot = c.wslot;
  C.wparent = c.wparent;
  C.old = c.old;
  C.eK[0] = p.entA_key;
  C.eC[0] = p.entA_child;
  C.eK[1] = p.entB_key;
  C.eC[1] = p.entB_child;
  C.threshold = (p.flags & EIRENE_F_FORCE_STM) ? 0u : p.threshold;
  C.force_stm = (p.flags & EIRENE_F_FORCE_STM) != 0 || p.threshold == 0;
  C.regroup = (p.flags & EIRENE_F_REGROUP) != 0;
  C.stats = (p.flags & EIRENE_F_STATS) != 0;
  C.ctl = ctl;
  C.slots[0] = p.slots[0];
  C.slots[1] = p.slots[1];
  C.eparent = p.eparent;
  C.flat_key = p.flat_key;
  C.flat_child = p.flat_child;
  C.flat_off = p.flat_off;
  const uint32_t warps_needed = C.regroup ? (n + 31) / 32 : n;
  constexpr uint32_t WPC = UPD_THREADS / 32;
  const size_t dsm = WPC * UPD_SMEM_PER_WARP;
  uint32_t blocks = (warps_needed + WPC - 1) / WPC;
  static int attr[MAX_DEVICES];
  per_device(attr, [dsm] {
    return (int)cudaFuncSetAttribute(update_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)dsm);
  });
  // the level-synchronous phases need every CTA resident (grid barriers)
  static int occ[MAX_DEVICES];
  const int per_sm = per_device(occ, [dsm] {
    int v = 0;
    return cudaOccupancyMaxActiveBlocksPerMultiprocessor(&v, update_kernel, UPD_THREADS, dsm) == cudaSuccess ? v : 0;
  });
  const uint32_t resident = (uint32_t)num_sms * (uint32_t)std::max(per_sm, 0);
  blocks = std::min<uint32_t>(blocks, resident ? resident : (uint32_t)num_sms * 4u);
#ifdef UPD_MAXCTAS   // diagnostic: launch-overhead floor of the update kernel
  blocks = std::min<uint32_t>(blocks, (uint32_t)UPD_MAXCTAS);
#endif
  if (blocks < 1) blocks = 1;
  static const bool no_lsync = std::getenv("EIRENE_NO_LSYNC") != nullptr;   // A/B: per-warp insertion only
  if (!resident || no_lsync) C.slots[0] = nullptr;   // no residency guarantee: per-warp insertion only
  static const char* serial = std::getenv("EIRENE_UPDATE_SERIAL");   // debug: one warp, no concurrency
  static int prof_set[MAX_DEVICES];
  per_device(prof_set, [] {
    const int on = std::getenv("EIRENE_UPDATE_PROF") != nullptr;
    return (int)cudaMemcpyToSymbol(g_uprof, &on, sizeof(int));
  });
  if (serial) {
    update_kernel<<<1, 32, dsm, st>>>(C, r);
  } else {
    if (C.slots[0]) {   // grid barriers: a resident-sized grid (cooperative only with EIRENE_COOP=1, launch_k)
      launch_k(update_kernel, dim3(blocks), dim3(UPD_THREADS), dsm, st, true, true, C, r);
    } else {
      launch_k(update_kernel, dim3(blocks), dim3(UPD_THREADS), dsm, st, true, false, C, r);
    }
  }
  ++*launches;
}

}  // namespace eirene
