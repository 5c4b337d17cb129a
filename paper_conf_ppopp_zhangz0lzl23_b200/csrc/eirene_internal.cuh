// eirene_internal.cuh -- device layout and helpers shared by the sm_100a kernels
// of the Eirene batched B+tree (never included by oracle/).
//
// Citations: P:N = /root/reference/PAPER.md line N; Alg.1:k = Algorithm 1 line k.
//
// Tree layout in HBM (SoA node pools):
//   leaves : one 256 B block per leaf: 16 u64 keys (a 128 B line) then 16 u64
//            values (the next line, same DRAM page), lmeta[cap] (32 B).
//            Unused key slots hold KEY_MAX (sorted to the end).
//   inner  : ikeys[cap][16] u64 separators (child i covers [key[i-1], key[i]),
//            key[c-1..15] = KEY_MAX), ichild[cap][16] u32, imeta[cap] (32 B).
//   The B+tree of P:327-330 / P:1622-1628, plus B-link right links and [lo, hi)
//   fences on every node (P:1363-1366 leaf links; "key in range(leaf)",
//   Alg.1:38) and a version word per node.
#pragma once
#include <algorithm>
#include <cstdint>
#include <utility>
#include <cuda_runtime.h>

#include "eirene.h"

namespace eirene {

constexpr int FAN = 16;
constexpr int LSTRIDE = 2 * FAN;   // tkey_t words per leaf block (keys, then values)
constexpr uint64_t KEY_MAX = ~0ull;
// Storage type of keys and values in the tree and in the caller's batch arrays
// (eirene_key_t: 64 bits, or 32 with -DEIRENE_KEY32 -- SURVEY §8(f) NEXT(4)).
// Kernels compute on 64-bit keys: a stored key is zero-extended on load (every
// valid key, and the padding TKEY_MAX above them, keep their order) and
// narrowed on store (KEY_MAX -> TKEY_MAX); widen() maps the padding / NOT_FOUND
// sentinel to KEY_MAX where a loaded word is compared with it.
typedef eirene_key_t tkey_t;
constexpr tkey_t TKEY_MAX = (tkey_t)~(tkey_t)0;
__host__ __device__ __forceinline__ uint64_t widen(tkey_t x) { return x == TKEY_MAX ? KEY_MAX : (uint64_t)x; }
constexpr uint32_t NIL = 0xFFFFFFFFu;
constexpr int MAX_LEVELS = 32;
constexpr uint32_t DONE_BIT = 0x80000000u;    // pinfo: an earlier write of the segment decides the result
constexpr uint32_t DEFER_BIT = 0x40000000u;   // pinfo (hot-key segments): that early result is written by
                                              // result phase from the nearest write's payload in kB
constexpr uint32_t SEG_MASK = 0x3FFFFFFFu;
constexpr uint32_t Q_SINGLE = 0x80000000u;    // qseg entry of a one-request query segment: Q_SINGLE | its timestamp
#ifndef EIRENE_RCHUNK
#define EIRENE_RCHUNK 512
#endif
constexpr uint32_t RCHUNK = EIRENE_RCHUNK;    // result phase work item: positions of one long segment
                                              // (4 per thread of the update kernel's 128-thread CTAs)
constexpr uint32_t FULL = 0xFFFFFFFFu;

enum { OP_QUERY = 0, OP_UPDATE = 1, OP_INSERT = 2, OP_DELETE = 3, OP_RANGE = 4 };

// Version word (D2, SURVEY §8(c) reading 18): bit 0 = lock (eager write
// ownership of the STM), bits 1.. = modification counter.
// Leaves: +2 on split only; inner nodes: +2 on every change.
struct NodeMeta {
  uint32_t version;
  uint32_t next;    // right sibling at the same level (B-link / leaf chain)
  uint64_t lo;      // fences: every key k below this node has lo <= k < hi
  uint64_t hi;
  uint32_t count;   // inner: number of children; leaf: informational
  uint32_t level;   // 0 = leaf
};
static_assert(sizeof(NodeMeta) == 32, "meta is 32 B");

// The allocation counters sit on lines of their own: under a split storm
// every split leaf's warp does an atomic on leaf_count, and the root word is
// read by every descent.  level_count[0] is not maintained by the update
// kernel (leaves are never freed: it equals leaf_count, which is what
// headroom_ok uses for level 0).
struct TreeHdr {
  unsigned long long root_word;          // (height << 32) | root id; height 1 = leaf root
  uint32_t pad0[30];
  uint32_t leaf_count;                   // leaf pool allocation counter
  uint32_t pad1[31];
  uint32_t inner_count;                  // inner pool allocation counter
  uint32_t level_count[MAX_LEVELS];      // nodes per level (EFULL bound; [0] see above)
};

// Per-batch device scalars; zeroed (cudaMemsetAsync) before every batch.
struct BatchCtl {
  int32_t status;
  uint32_t invalid;
  uint32_t tile_ctr[16];
  uint32_t nseg, nq, nw, height;
  uint32_t nlong, gbar;   // gbar: grid barrier of bsort_dist_kernel
  uint32_t nrange, nart;  // range queries in the batch; artificial queries resolved
  uint32_t hot_ctr;       // hot-key timestamp bitmaps claimed by oversized groups
  uint32_t hot_item;      // result phase: next (hot key, bitmap chunk) work item
  uint32_t nins;          // issued upserts of absent keys (query kernel): 0 -> no split is possible
  uint32_t ndelp;         // issued deletes of present keys (query kernel); nins == ndelp == 0 -> every
                          // issued write was a value overwrite, applied in place by the query kernel
  uint32_t fin_ctr;       // update kernel's result phase: residue classes finished (the last publishes the BatchCtl)
  uint32_t fin_sub[16];   // ... CTAs finished per residue class blockIdx % 16
  uint32_t qfin_ctr, qfin_sub[16];   // the same for the query kernel (graph mode: it may end the batch)
  uint32_t upd_ran;       // the update kernel ran (its conditional graph node was switched on)
  unsigned long long t_begin, t_end;   // %globaltimer (ns) at the batch's first / last kernel
  uint32_t ubar;          // grid barrier of the update kernel's level-synchronous phases
  uint32_t uchunk;        // update kernel: next 32-write chunk (dynamic, level-synchronous mode)
  uint32_t flat_total;    // update kernel: entries of the current upper level (flattened)
  uint32_t rg_vertical, rg_horizontal;   // EIRENE_F_ITERWARP: RGs traversed vertically / horizontally
  unsigned long long trav_steps;         // EIRENE_F_ITERWARP: traversal steps of the issued requests
  uint32_t lvl_ent[MAX_LEVELS];   // separator entries produced for level L+1 (update kernel)
  unsigned long long uprof[24];   // diagnostic (EIRENE_UPDATE_PROF): update-kernel phase timestamps
  unsigned long long leaf_runs, retries, stm_fallbacks, leaf_splits, inner_splits, new_leaves, new_inner;
  uint32_t dbg[8];   // watchdog diagnostics
  uint32_t ustripe[8][32];   // update kernel: level-0 chunk claims, one counter per stripe, each on its own line
};

// Device watchdog: spin / retry loops give up after this long and report
// EIRENE_EINTERNAL instead of hanging the GPU.
constexpr unsigned long long WATCHDOG_NS = 4000000000ull;
__device__ __forceinline__ unsigned long long gtime_ns() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}

// Decoupled look-back spin guard: a predecessor tile that never publishes is a
// bug; give up after the watchdog period instead of hanging.
struct SpinGuard {
  unsigned long long t0 = 0;
  __device__ __forceinline__ bool stuck(BatchCtl* ctl) {
    const unsigned long long now = gtime_ns();
    if (t0 == 0) {
      t0 = now;
      return false;
    }
    if (now - t0 > WATCHDOG_NS) {
      if (ctl) atomicExch(reinterpret_cast<int*>(&ctl->status), EIRENE_EINTERNAL);
      return true;
    }
    return false;
  }
};

// Per-batch caller pointers, written on the device by the first node of the
// batch graph so the captured pipeline can be replayed on new buffers by
// updating that single node (api.cu).
struct BatchArgs {
  const uint8_t* ops;
  const tkey_t* keys;
  const tkey_t* vals;        // values as read by the kernels after the distribution pass
  tkey_t* results;
  const tkey_t* vals_src;    // where the distribution pass reads the values of upserts
  tkey_t* vals_stage;        // non-null: it also copies them here (== vals); host path, zero-copy
  BatchCtl* ctl_out;    // device ring slot: the batch's final BatchCtl is copied here at the end
  tkey_t* rkeys;        // range-query output (eirene_submit_batch_range), else null: RANGE ops invalid
  tkey_t* rvals;
  uint32_t rcap;
  unsigned long long t0;   // %globaltimer when the batch's first kernel started (device batch time)
  uint32_t n;              // requests in the batch (launches are sized for the graph's size bucket >= n)
  unsigned long long* phase;   // diagnostic builds (-DEIRENE_PHASE_PROF): [kernel][CTA][phase] %globaltimer stamps
  uint32_t seq;                // the handle's batch sequence number (epoch of the result phase's look-back)
};

// Phase timestamps of the distribution / group kernels (diagnostic builds only:
// -DEIRENE_PHASE_PROF; read back with eirene_debug_phases).
constexpr int PROF_CTAS = 512, PROF_PHASES = 8;
#ifdef EIRENE_PHASE_PROF
#define EIRENE_PHASE(A, k, cta, i)                                                                   \
  do {                                                                                            \
    if (threadIdx.x == 0 && (A)->phase && (cta) < PROF_CTAS)                                       \
      (A)->phase[((size_t)(k) * PROF_CTAS + (cta)) * PROF_PHASES + (i)] = gtime_ns();             \
  } while (0)
#else
#define EIRENE_PHASE(A, k, cta, i) \
  do {                             \
  } while (0)
#endif

// tile counters
enum { TC_SORT0 = 0, TC_GROUP = 8, TC_GROUP2 = 9, TC_ROUTE = 10, TC_SCAN = 11, TC_HIST = 12 };

struct Tree {
  tkey_t* lkeys;     // leaf L: keys at lkeys[L * LSTRIDE + s]
  tkey_t* lvals;     // = lkeys + FAN: values at lvals[L * LSTRIDE + s]
  NodeMeta* lmeta;
  uint64_t* lrf;     // range field of every leaf (EIRENE_F_ITERWARP)
  tkey_t* ikeys;
  uint32_t* ichild;
  NodeMeta* imeta;
  TreeHdr* hdr;
  uint32_t leaf_cap, inner_cap;
};

// ------------------------------------------------------------ PTX helpers
__device__ __forceinline__ uint32_t lanemask_lt() {
  uint32_t m;
  asm volatile("mov.u32 %0, %%lanemask_lt;" : "=r"(m));
  return m;
}
__device__ __forceinline__ uint32_t lane_id() { return threadIdx.x & 31; }

// L2-coherent loads for data concurrently written by other SMs (the update kernel).
__device__ __forceinline__ uint64_t ld_cg(const uint64_t* p) {
  return __ldcg(reinterpret_cast<const unsigned long long*>(p));
}
__device__ __forceinline__ uint32_t ld_cg(const uint32_t* p) { return __ldcg(p); }
__device__ __forceinline__ uint32_t ld_acquire(const uint32_t* p) {
  uint32_t v;
  asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ unsigned long long ld_acquire64(const unsigned long long* p) {
  unsigned long long v;
  asm volatile("ld.acquire.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ uint32_t ld_relaxed(const uint32_t* p) {
  uint32_t v;
  asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
// CAS with acquire semantics: the lock acquisition of the STM's eager write ownership.
__device__ __forceinline__ uint32_t atom_cas_acquire(uint32_t* p, uint32_t cmp, uint32_t val) {
  uint32_t old;
  asm volatile("atom.acquire.gpu.global.cas.b32 %0, [%1], %2, %3;" : "=r"(old) : "l"(p), "r"(cmp), "r"(val) : "memory");
  return old;
}
__device__ __forceinline__ uint32_t atom_or_acquire(uint32_t* p, uint32_t val) {
  uint32_t old;
  asm volatile("atom.acquire.gpu.global.or.b32 %0, [%1], %2;" : "=r"(old) : "l"(p), "r"(val) : "memory");
  return old;
}
__device__ __forceinline__ void st_release(uint32_t* p, uint32_t v) {
  asm volatile("st.release.gpu.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ unsigned long long ld_relaxed64(const unsigned long long* p) {
  unsigned long long v;
  asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_relaxed64(unsigned long long* p, unsigned long long v) {
  asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}

// L2 eviction-priority policies (createpolicy) for per-load cache hints: the
// inner levels (<= 18 MB at 2^24 keys) are re-read by every batch and are
// loaded evict_last; leaf lines, values and streaming outputs are touched
// once per batch and are loaded / stored evict_first, so a batch's own
// streams do not push the inner levels out of L2.
__device__ __forceinline__ uint64_t pol_evict_last() {
  uint64_t p;
  asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(p));
  return p;
}
__device__ __forceinline__ uint64_t pol_evict_first() {
  uint64_t p;
  asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
  return p;
}
// read-only (nc) loads with an L2 policy; 256-bit loads skip L1 allocation.
// A/B (EIRENE_LEAF_PF=128): the leaf line loads with an explicit 128 B L2 fetch size
__device__ __forceinline__ ulonglong4 ldg256_pol(const uint64_t* p, uint64_t pol) {
  ulonglong4 v;
#if defined(EIRENE_LEAF_PF) && EIRENE_LEAF_PF == 128
  asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.L2::128B.v4.u64 {%0,%1,%2,%3}, [%4], %5;"
               : "=l"(v.x), "=l"(v.y), "=l"(v.z), "=l"(v.w) : "l"(p), "l"(pol));
#elif defined(EIRENE_LEAF_PF) && EIRENE_LEAF_PF == 64
  asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.L2::64B.v4.u64 {%0,%1,%2,%3}, [%4], %5;"
               : "=l"(v.x), "=l"(v.y), "=l"(v.z), "=l"(v.w) : "l"(p), "l"(pol));
#else
  asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.v4.u64 {%0,%1,%2,%3}, [%4], %5;"
               : "=l"(v.x), "=l"(v.y), "=l"(v.z), "=l"(v.w) : "l"(p), "l"(pol));
#endif
  return v;
}
// one value with an explicit 64 B L2 fetch size (A/B: EIRENE_VAL_LOAD=4)
__device__ __forceinline__ uint64_t ldg64_pol_64b(const uint64_t* p, uint64_t pol) {
  uint64_t v;
  asm volatile("ld.global.nc.L2::cache_hint.L2::64B.u64 %0, [%1], %2;" : "=l"(v) : "l"(p), "l"(pol));
  return v;
}
__device__ __forceinline__ uint64_t ldg64_pol_64b(const uint32_t* p, uint64_t pol) {
  uint32_t v;
  asm volatile("ld.global.nc.L2::cache_hint.L2::64B.u32 %0, [%1], %2;" : "=r"(v) : "l"(p), "l"(pol));
  return v;
}
// ... and without an eviction policy (data re-read later in the batch: the write values)
__device__ __forceinline__ uint64_t ldg64_64b(const uint64_t* p) {
  uint64_t v;
  asm volatile("ld.global.nc.L2::64B.u64 %0, [%1];" : "=l"(v) : "l"(p));
  return v;
}
__device__ __forceinline__ uint64_t ldg64_64b(const uint32_t* p) {
  uint32_t v;
  asm volatile("ld.global.nc.L2::64B.u32 %0, [%1];" : "=r"(v) : "l"(p));
  return v;
}
__device__ __forceinline__ uint64_t ldg64_pol(const uint64_t* p, uint64_t pol) {
  uint64_t v;
  asm volatile("ld.global.nc.L2::cache_hint.u64 %0, [%1], %2;" : "=l"(v) : "l"(p), "l"(pol));
  return v;
}
__device__ __forceinline__ uint64_t ldg64_pol(const uint32_t* p, uint64_t pol) {   // (32-bit keys: zero-extended)
  uint32_t v;
  asm volatile("ld.global.nc.L2::cache_hint.u32 %0, [%1], %2;" : "=r"(v) : "l"(p), "l"(pol));
  return v;
}
__device__ __forceinline__ uint32_t ldg32_pol(const uint32_t* p, uint64_t pol) {
  uint32_t v;
  asm volatile("ld.global.nc.L2::cache_hint.u32 %0, [%1], %2;" : "=r"(v) : "l"(p), "l"(pol));
  return v;
}
__device__ __forceinline__ void st64_pol(uint64_t* p, uint64_t v, uint64_t pol) {
  asm volatile("st.global.L2::cache_hint.u64 [%0], %1, %2;" ::"l"(p), "l"(v), "l"(pol) : "memory");
}
__device__ __forceinline__ void st64_pol(uint32_t* p, uint64_t v, uint64_t pol) {   // (32-bit keys: narrowed)
  asm volatile("st.global.L2::cache_hint.u32 [%0], %1, %2;" ::"l"(p), "r"((uint32_t)v), "l"(pol) : "memory");
}

// The 16 keys of a node line (a 128 B line of u64 keys, or 64 B of u32 keys)
// in registers, with 256-bit loads: Line16::at(s) = key s zero-extended.
struct Line16 {
  static constexpr int NW = FAN * (int)sizeof(tkey_t) / 32;   // 256-bit words: 4 (u64 keys) or 2 (u32)
  ulonglong4 w[NW];
  __device__ __forceinline__ void load(const tkey_t* p, uint64_t pol) {   // L1 no-allocate (leaves)
#pragma unroll
    for (int x = 0; x < NW; ++x) w[x] = ldg256_pol(reinterpret_cast<const uint64_t*>(p) + 4 * x, pol);
  }
  __device__ __forceinline__ void load_l1(const tkey_t* p, uint64_t pol) {   // L1-allocating (inner nodes)
#pragma unroll
    for (int x = 0; x < NW; ++x) {
      const uint64_t* q = reinterpret_cast<const uint64_t*>(p) + 4 * x;
      asm volatile("ld.global.nc.L2::cache_hint.v4.u64 {%0,%1,%2,%3}, [%4], %5;"
                   : "=l"(w[x].x), "=l"(w[x].y), "=l"(w[x].z), "=l"(w[x].w) : "l"(q), "l"(pol));
    }
  }
  __device__ __forceinline__ uint64_t at(uint32_t s) const {
    if constexpr (sizeof(tkey_t) == 8) {
      const ulonglong4 q = (s < 8) ? ((s < 4) ? w[0] : w[1]) : ((s < 12) ? w[2 % NW] : w[3 % NW]);
      const uint32_t r = s & 3;
      return r == 0 ? q.x : r == 1 ? q.y : r == 2 ? q.z : q.w;
    } else {
      const ulonglong4 q = (s < 8) ? w[0] : w[1];
      const uint32_t r = (s & 7) >> 1;
      const uint64_t x = r == 0 ? q.x : r == 1 ? q.y : r == 2 ? q.z : q.w;
      return (s & 1) ? (x >> 32) : (x & 0xFFFFFFFFull);
    }
  }
  // number of keys <= k (the child index of k in an inner node: padding is above every key)
  __device__ __forceinline__ uint32_t count_le(uint64_t k) const {
    uint32_t c = 0;
#pragma unroll
    for (int x = 0; x < NW; ++x) {
      const uint64_t q[4] = {w[x].x, w[x].y, w[x].z, w[x].w};
#pragma unroll
      for (int y = 0; y < 4; ++y) {
        if constexpr (sizeof(tkey_t) == 8) {
          c += q[y] <= k;
        } else {
          c += (q[y] & 0xFFFFFFFFull) <= k;
          c += (q[y] >> 32) <= k;
        }
      }
    }
    return c;
  }
  // slot of key k (a valid key: never the padding), -1 if absent
  __device__ __forceinline__ int find(uint64_t k) const {
    int s = -1;
#pragma unroll
    for (int x = 0; x < NW; ++x) {
      const uint64_t q[4] = {w[x].x, w[x].y, w[x].z, w[x].w};
#pragma unroll
      for (int y = 0; y < 4; ++y) {
        if constexpr (sizeof(tkey_t) == 8) {
          if (q[y] == k) s = 4 * x + y;
        } else {
          if ((q[y] & 0xFFFFFFFFull) == k) s = 8 * x + 2 * y;
          if ((q[y] >> 32) == k) s = 8 * x + 2 * y + 1;
        }
      }
    }
    return s;
  }
};

__device__ __forceinline__ uint64_t shfl64(uint64_t v, int src) {
  return __shfl_sync(FULL, (unsigned long long)v, src);
}

__host__ __device__ __forceinline__ bool is_write(uint32_t op) { return op != OP_QUERY; }

// ------------------------------------------------------------ per-device host state
// One-time host-side state (function attributes, occupancy) is per DEVICE:
// a process may hold handles on several GPUs.  Keyed by the current device
// (every ABI entry point makes the handle's device current).  0 = not yet
// computed; a benign race between threads computes the same value twice.
constexpr int MAX_DEVICES = 64;
inline int current_device() {
  int d = 0;
  cudaGetDevice(&d);
  return d;
}
template <class F>
inline int per_device(int (&cache)[MAX_DEVICES], F compute) {
  const int d = current_device();
  if (d < 0 || d >= MAX_DEVICES) return compute();
  if (cache[d] == 0) cache[d] = compute() + 1;
  return cache[d] - 1;
}

// Worst-case node demand of the update kernel (EFULL pre-check, SURVEY
// §8(b)), checked by the query kernel before anything changes (the front of a
// pipelined batch must not read the tree): new leaves <= issued writes; new inner nodes at level l+1 <=
// min(N_l, (I_l + N_l) / 8) because every node created by an even multi-way
// split keeps >= 8 children, plus root growth.
__device__ __forceinline__ bool headroom_ok(const Tree& t, uint32_t nw) {
  const TreeHdr* h = t.hdr;
  const uint32_t height = (uint32_t)(h->root_word >> 32);
  unsigned long long need_leaf = nw;
  unsigned long long N = nw, inner = 0;
  for (uint32_t l = 0; l + 1 < height && N > 0; ++l) {
    unsigned long long I = l == 0 ? h->leaf_count : h->level_count[l];
    unsigned long long Nn = min(N, (I + N) / 8 + 1);
    inner += Nn;
    N = Nn;
  }
  inner += 2 * (N + 1) + 64;   // new root levels
  return (unsigned long long)h->leaf_count + need_leaf <= t.leaf_cap &&
         (unsigned long long)h->inner_count + inner <= t.inner_cap;
}

// ------------------------------------------------------------ programmatic dependent launch
// Kernels 2.. of a batch are launched with programmatic stream serialization
// (PDL, EIRENE_PDL=1): a kernel may be scheduled while its predecessor drains,
// hiding the launch latency between the batch's kernels.  Every batch kernel
// starts with pdl_wait() (griddepcontrol.wait: returns once the predecessor
// grid has completed and its writes are visible; a no-op without PDL) before
// it touches anything, then pdl_trigger() lets its own successor be scheduled.
// All batch kernels are single-wave grids, so an early successor never takes
// SM slots a later wave of its predecessor would need.
__device__ __forceinline__ void pdl_wait() { asm volatile("griddepcontrol.wait;" ::: "memory"); }
__device__ __forceinline__ void pdl_trigger() { asm volatile("griddepcontrol.launch_dependents;" ::: "memory"); }
bool pdl_enabled();
bool coop_enabled();
template <typename... KArgs, typename... Args>
cudaError_t launch_k(void (*kern)(KArgs...), dim3 grid, dim3 block, size_t smem, cudaStream_t st, bool pdl,
                     bool coop, Args&&... args) {
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = grid;
  cfg.blockDim = block;
  cfg.dynamicSmemBytes = smem;
  cfg.stream = st;
  cudaLaunchAttribute at[2];
  unsigned na = 0;
  if (pdl && pdl_enabled()) {
    at[na].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    at[na].val.programmaticStreamSerializationAllowed = 1;
    ++na;
  }
  // The two grid-barrier kernels (distribution, update) run grids sized to the
  // occupancy calculator's co-resident capacity.  By default they are launched
  // WITHOUT the cooperative attribute (r3o: cfg2 9.03 -> 9.24 G req/s, the
  // cooperative launch cost ~2.5 us per batch): every CTA of such a grid fits
  // on the device at once, and no kernel that may share the device with it (the
  // library's own: a pipelined front, routing kernels, NCCL's -- stream-ordered
  // around it) waits on it, so every CTA is eventually scheduled and the
  // barrier completes.  A foreign kernel holding SMs indefinitely would make the
  // barrier wait; the device watchdog then ends the batch with EINTERNAL instead
  // of hanging.  EIRENE_COOP=1 restores cooperative launches (shared devices).
  if (coop && !coop_enabled()) coop = false;
  if (coop) {
    at[na].id = cudaLaunchAttributeCooperative;
    at[na].val.cooperative = 1;
    ++na;
  }
  cfg.attrs = at;
  cfg.numAttrs = na;
  return cudaLaunchKernelEx(&cfg, kern, std::forward<Args>(args)...);
}

// ------------------------------------------------------------ host-side launchers
// (defined in the .cu files; called from api.cu)
struct SortBufs {
  uint64_t* kA;
  uint32_t* pA;
  uint64_t* kB;
  uint32_t* pB;
  unsigned long long* lookback;   // [tiles * 256]
  uint32_t* ghist;                // [8 * 256]
};
constexpr int SORT_THREADS = 256;
constexpr int SORT_ITEMS = 16;
constexpr int SORT_TILE = SORT_THREADS * SORT_ITEMS;
constexpr int SORT_PASSES = 8;

// Sort (key, payload) pairs by key, stable.  If ops != nullptr the payload of
// element i is (i << 2) | ops[i] (logical timestamp + type),
// otherwise pay_in[i].  Returns (via *kout/*pout) which buffer holds the result.
// Also validates requests when ops != nullptr (sets ctl->invalid).
void launch_sort(const uint64_t* keys, const uint8_t* ops, const uint32_t* pay_in, const uint64_t* vals,
                 uint32_t n, uint64_t key_lo, uint64_t key_hi, const SortBufs& b, BatchCtl* ctl,
                 uint32_t epoch_base, cudaStream_t st, int* launches, uint64_t** kout, uint32_t** pout);

size_t sort_lookback_words(uint32_t max_n);

// Batch request sort (bsort.cu): bucket by the top bits, sort buckets in smem.
constexpr int BIN_BITS = 12;                  // bucket-sort bins = top bits of (key - key_lo) (fused path)
constexpr int NBINS = 1 << BIN_BITS;
constexpr int BIN_BITS_L = 14;                // bins of the two-kernel path (batches > 2^22 requests)
constexpr int NBINS_L = 1 << BIN_BITS_L;
constexpr int NBINS_MAX = NBINS_L;
// Bin of key k: the top `bits` bits of k - key_lo over the shard's range, so a
// shard of a multi-GPU tree (a fraction of the key space) still spreads its
// keys over all the bins.  Out-of-range keys (invalid requests, rejected
// later) are clamped.  shift = max(0, bits(key_hi - key_lo - 1) - bits).
__host__ __device__ __forceinline__ uint32_t bin_of(uint64_t k, uint64_t key_lo, uint32_t shift, uint32_t nbins) {
  const uint64_t d = k >= key_lo ? (k - key_lo) >> shift : 0ull;
  return d < nbins ? (uint32_t)d : nbins - 1u;
}
inline uint32_t bin_shift(uint64_t key_lo, uint64_t key_hi, int bits) {
  const uint64_t r = key_hi - key_lo - 1;   // key_hi > key_lo
  const int rb = r ? 64 - __builtin_clzll(r) : 0;
  return (uint32_t)(rb > bits ? rb - bits : 0);
}
struct BSortBufs {
  uint64_t* kA;      // [n] grouped (unordered inside a group)
  uint32_t* pA;
  uint64_t* kB;      // [n] scratch for oversized groups
  uint32_t* pB;      // [n] sorted payloads (output)
  uint32_t* bcount;  // [NBINS_MAX] zeroed per batch
  uint16_t* bin2grp; // [NBINS_MAX]
  uint32_t* gstart;  // [NBINS_MAX + 1] group starts
  uint32_t* cursor;  // [NBINS_MAX] group fill cursors (zeroed per batch)
};
uint32_t bsort_groups(uint32_t n, int num_sms);
bool bsort_fused(uint32_t n, int num_sms);         // the distribution path of an n-request batch
uint64_t bsort_fused_capacity(int num_sms);        // largest batch of the fused path
void launch_bucket_sort(const BatchArgs* A, uint32_t n, uint64_t key_lo, uint64_t key_hi, const BSortBufs& b,
                        BatchCtl* ctl, int num_sms, cudaStream_t st, int* launches);

struct CombBufs {
  uint32_t* pinfo;            // [n] seg | DONE
  unsigned long long* group_status;  // [GROUP_STATUS_WORDS] bucket look-back words (zeroed per batch)
  uint64_t* qkey;
  uint32_t* qseg;
  uint64_t* wkey;
  uint8_t* wop;
  uint64_t* wval;
  uint32_t* wseg;
  uint32_t* wleaf;
  uint8_t* wslot;             // [n] slot of the write's key in its leaf at locate time, 255 = absent
  uint32_t* wparent;          // [n] the write's leaf's parent (level-1 node) at locate time, NIL if the root is a leaf
  uint64_t* old;              // [n] old value per segment
  uint32_t* istart;           // [n+1] sorted position of each segment's first request (+ n at nseg)
  uint32_t* longseg;          // [n] segments longer than SHORT_SEG, finished by the result phase
  uint32_t* hot_bits;         // [HOT_SLOTS][3][hot_words] timestamp bitmaps of hot keys: present, op bit 0,
                              // op bit 1 (all zero between batches)
  uint32_t hot_words;         // >= max_batch / 32, a multiple of 4
  uint32_t* hot_seg;          // [HOT_SLOTS] segment of each hot key whose bitmap the result phase walks
  uint4* grec;                // [NBINS_MAX][3] per-group records of the two-phase group stage (multi-wave batches)
};
constexpr int HOT_SLOTS = 64;
#ifndef EIRENE_SHORT_SEG
#define EIRENE_SHORT_SEG 32   // A/B builds: -DEIRENE_SHORT_SEG=n
#endif
constexpr uint32_t SHORT_SEG = EIRENE_SHORT_SEG;
constexpr int GROUP_STATUS_WORDS = NBINS_MAX;   // >= bsort_groups(n) for every n

// bucket finish (sort in smem) + combine + partition, one CTA per bucket (group.cu)
// two_phase: a batch of more groups than are co-resident (several waves) and no
// range queries runs the group stage as two kernels -- sort + totals, then
// look-back + emit -- so that no CTA waits for a later wave's slow group
void launch_group(const BatchArgs* A, uint32_t n, const BSortBufs& b, const CombBufs& c, Tree t, BatchCtl* ctl,
                  int num_sms, bool two_phase, cudaStream_t st, int* launches);
bool group_two_phase(uint32_t n, int num_sms);   // the batch has more groups than one wave
// cond / use_cond: graph mode -- the query kernel's last CTA sets the
// conditional node around the update kernel (or ends the batch itself)
void launch_query(uint32_t n, const CombBufs& c, const uint32_t* spay, const BatchArgs* A, Tree t, BatchCtl* ctl,
                  int num_sms, uint32_t flags, uint32_t iter_rgs, cudaGraphConditionalHandle cond, int use_cond,
                  cudaStream_t st, int* launches);

struct UpdParams {
  uint32_t threshold;
  uint32_t flags;
  uint2* slots[2];      // per producer unit (base, n) of the level-synchronous separator lists
  uint32_t* eparent;    // [n] parent node of each entry position (lookup step)
  uint64_t* entA_key;
  uint32_t* entA_child;
  uint64_t* entB_key;
  uint32_t* entB_child;
  uint64_t* flat_key;   // [n] an upper level's entries, concatenated in producer (= key) order
  uint32_t* flat_child;
  uint32_t* flat_off;   // [producers] exclusive prefix of the producers' entry counts
};
struct ResultArgs;
// update kernel (Alg.1:23-46), then the result phase (long-segment RESULT_CAL, Alg.1:6, and the
// batch's final BatchCtl): the batch's last kernel
void launch_update(uint32_t n, const CombBufs& c, Tree t, BatchCtl* ctl, UpdParams p, const ResultArgs& r,
                   int num_sms, cudaStream_t st, int* launches);
// range queries R(l, u): between the query and the update kernel
void launch_range(uint32_t n, const CombBufs& c, const uint32_t* spay, const uint64_t* kB, const BatchArgs* A, Tree t,
                  BatchCtl* ctl, int num_sms, cudaStream_t st, int* launches);
void launch_result(const BatchCtl* ctl, int dbgprint, cudaStream_t st);   // diagnostics print only

// bulk build / scan
int build_tree(Tree t, const tkey_t* keys, const tkey_t* vals, uint64_t n, int per_leaf, uint64_t key_lo,
               uint64_t key_hi, cudaStream_t st, int* launches, uint32_t* height_out);
void launch_validate_bulk(const tkey_t* keys, const tkey_t* vals, uint64_t n, uint64_t key_lo, uint64_t key_hi,
                          uint32_t* flag, cudaStream_t st, int* launches);
int scan_tree(Tree t, uint32_t leaf_count, uint64_t lo, uint64_t hi, tkey_t* keys_out, tkey_t* vals_out,
              uint64_t cap, uint64_t* count, cudaStream_t st, int* launches);

// routing
// SoA outputs (sops/skeys/svals, counts[P]) or, with rec != null, 24 B records
// {key, value, op} and counts[2P] = (count, validity flag) per destination
void launch_route_partition(const uint8_t* ops, const uint64_t* keys, const uint64_t* vals, uint32_t n,
                            const uint64_t* splitters, int P, uint8_t* sops, uint64_t* skeys, uint64_t* svals,
                            uint64_t* rec, uint32_t* perm, uint32_t* counts, uint32_t cstride, uint32_t* invalid,
                            unsigned long long* lookback, uint32_t* tile_ctr, uint32_t epoch, cudaStream_t st,
                            int* launches, uint64_t* const* peer_rec = nullptr, uint32_t me = 0, uint32_t cap = 0);
// fused push over peer memory (NVLink): counts / arena compaction / results back
void launch_push_counts(const uint32_t* counts, const uint32_t* invalid, int P, uint32_t me, uint32_t* const* peer_cnt,
                        uint32_t epoch, cudaStream_t st, int* launches);
void launch_pull_unpack(const uint32_t* cnt, const uint64_t* rec, uint32_t cap, int P, uint32_t max_per_src,
                        uint8_t* ops, uint64_t* keys, uint64_t* vals, cudaStream_t st, int* launches);
void launch_push_results(const uint32_t* cnt, const uint64_t* res, int P, uint32_t max_per_src,
                         uint64_t* const* peer_res, cudaStream_t st, int* launches);
void launch_route_unpack(const uint64_t* rec, uint32_t n, uint8_t* ops, uint64_t* keys, uint64_t* vals,
                         cudaStream_t st, int* launches);
void launch_route_unpermute(const uint64_t* recv, const uint32_t* perm, uint32_t n, uint64_t* results,
                            cudaStream_t st, int* launches);

// RESULT_CAL is fused into the query kernel: every issued
// request scatters the value it retrieved to the pending positions of its own
// segment.  The segments longer than SHORT_SEG (hot keys) are queued instead
// and finished here, work items of RCHUNK positions spread over the CTAs, so a
// 56K-request Zipf key does not serialise one thread.
// True in exactly one CTA of the grid: the last to arrive (CTA-uniform; call
// with every thread).  Two levels -- 16 counters by blockIdx % 16, then one --
// so no address takes more than ~gridDim / 16 same-address atomics.
__device__ __forceinline__ bool last_cta(uint32_t* sub16, uint32_t* top) {
  __shared__ uint32_t s_last;
  __syncthreads();
  if (threadIdx.x == 0) {
    __threadfence();
    const uint32_t grp = blockIdx.x & 15u, gsize = (gridDim.x + 15u - grp) / 16u;   // CTAs with this residue
    bool last = false;
    if (atomicAdd(&sub16[grp], 1u) == gsize - 1) {   // the last of its residue class
      __threadfence();
      last = atomicAdd(top, 1u) == min(16u, gridDim.x) - 1;
    }
    s_last = last;
  }
  __syncthreads();
  const bool last = s_last;
  if (last) __threadfence();
  return last;
}

// End of a batch, by the last CTA of its last kernel: the device end time, the
// final status and height, and the whole BatchCtl copied to the batch's ring
// slot (one word per thread).
__device__ __forceinline__ void publish_batch(BatchCtl* ctl, const BatchArgs* A, const TreeHdr* hdr) {
  if (threadIdx.x == 0) {
    if (ld_cg(&ctl->invalid)) ctl->status = EIRENE_EINVAL;
    ctl->height = (uint32_t)(hdr->root_word >> 32);
    ctl->t_begin = A->t0;
    ctl->t_end = gtime_ns();
  }
  __syncthreads();
  static_assert(sizeof(BatchCtl) % 8 == 0, "BatchCtl is copied as u64 words");
  const unsigned long long* src = reinterpret_cast<const unsigned long long*>(ctl);
  unsigned long long* dst = reinterpret_cast<unsigned long long*>(A->ctl_out);
  for (uint32_t i = threadIdx.x; i < sizeof(BatchCtl) / 8; i += blockDim.x) dst[i] = __ldcg(src + i);
}

// Whether the update kernel has anything to do once the query kernel has run:
// structural writes, long segments, or deferred hot-key bitmaps (whose bits
// must be walked -- and cleared -- even when the batch failed after the group
// kernel).  Read by the query kernel's last CTA (graph conditional node).
__device__ __forceinline__ bool update_needed(const BatchCtl* ctl, const BatchArgs* A) {
  const uint32_t inv = ld_cg(&ctl->invalid), st = ld_cg(reinterpret_cast<const uint32_t*>(&ctl->status));
  const bool hot = A->rkeys == nullptr && ld_cg(&ctl->hot_ctr) > 0;
  return !inv && (hot || (st == 0 && (ld_cg(&ctl->nins) | ld_cg(&ctl->ndelp) | ld_cg(&ctl->nlong)) != 0));
}

struct ResultArgs {
  const uint32_t* spay;
  const uint64_t* kB;
  const uint32_t* pinfo;
  const uint32_t* istart;
  const uint32_t* longseg;
  const uint64_t* old;
  const BatchArgs* A;
  BatchCtl* ctl;
  const TreeHdr* hdr;
  uint32_t* hot_bits;             // deferred hot keys: bitmap slots [HOT_SLOTS][3][hot_words] (cleared here)
  uint32_t hot_words;
  const uint32_t* hot_seg;        // [HOT_SLOTS] their segments
  unsigned long long* hot_lb;     // [HOT_SLOTS][HOT_CHUNKS_MAX] epoch-tagged look-back words
  uint32_t hot_chunks;            // chunks per slot (hot_words / HOT_CHW, rounded up)
};
constexpr uint32_t HOT_CHW = 1024;   // bitmap words (32K timestamps) per result-phase work item
// Run by every CTA of the batch's last kernel (the update kernel), after its
// structural work: the long segments need only the query kernel's old values,
// so they need no grid barrier after the updates.
__device__ __forceinline__ void result_phase(const ResultArgs& R) {
  const uint32_t* __restrict__ spay = R.spay;
  const uint64_t* __restrict__ kB = R.kB;
  const uint32_t* __restrict__ pinfo = R.pinfo;
  const uint32_t* __restrict__ istart = R.istart;
  const uint32_t* __restrict__ longseg = R.longseg;
  const uint64_t* __restrict__ old = R.old;
  const BatchArgs* __restrict__ A = R.A;
  BatchCtl* __restrict__ ctl = R.ctl;
  const TreeHdr* hdr = R.hdr;
  __shared__ uint32_t s_hseg[HOT_SLOTS];
  __shared__ uint32_t s_item, s_red[32];
  // the batch's scalars, loaded together (independent loads: one round trip)
  // (plain loads: ctl was read at the kernel's start, written only by earlier kernels)
  const uint32_t c_invalid = ctl->invalid, c_status = (uint32_t)ctl->status;
  const uint32_t c_nlong = ctl->nlong, c_hot = ctl->hot_ctr;
  const bool c_range = A->rkeys != nullptr;
  const uint32_t njobs = min(c_hot, (uint32_t)HOT_SLOTS);
  // (a deferred hot key's segment is walked below, not through its positions)
#ifdef EIRENE_NO_HOTDEFER
  const uint32_t nhot = 0;
  (void)c_range;
  (void)njobs;
#else
  const uint32_t nhot = c_range ? 0u : njobs;
#endif
  if (nhot) {   // (uniform)
    for (uint32_t j = threadIdx.x; j < nhot; j += blockDim.x) s_hseg[j] = ld_cg(R.hot_seg + j);
    __syncthreads();
  }
  if (!(c_invalid || c_status != 0)) {
    tkey_t* __restrict__ results = A->results;
    const tkey_t* __restrict__ vals = A->vals;
    const uint32_t nl = c_nlong;
    for (uint32_t x = blockIdx.x; x < nl; x += gridDim.x) {
      const uint32_t s = longseg[2 * x], ch = longseg[2 * x + 1];
      bool hotseg = false;
      for (uint32_t j = 0; j < nhot; ++j) hotseg |= s_hseg[j] == s;
      if (hotseg) continue;   // (uniform in the CTA)
      const uint64_t v = old[s];
      const uint32_t b = istart[s] + ch * RCHUNK;
      const uint32_t e = min(istart[s + 1], b + RCHUNK);
      for (uint32_t p0 = b + threadIdx.x; p0 < e; p0 += 4 * blockDim.x) {   // 4 loads in flight
        uint32_t pi[4], py[4];
#pragma unroll
        for (int u = 0; u < 4; ++u) {
          const uint32_t p = p0 + u * blockDim.x;
          pi[u] = p < e ? pinfo[p] : DONE_BIT;
          py[u] = p < e ? spay[p] : 0u;
        }
#pragma unroll
        for (int u = 0; u < 4; ++u) {
          if (!(pi[u] & DONE_BIT)) {
            results[py[u] >> 2] = v;   // no earlier write in the segment: the issued request's value
          } else if (pi[u] & DEFER_BIT) {   // hot key: the nearest earlier write (its payload in kB)
            const uint32_t pw = (uint32_t)kB[p0 + u * blockDim.x];
            results[py[u] >> 2] = ((pw & 3) == OP_DELETE) ? KEY_MAX : vals[pw >> 2];
          }
        }
      }
    }
  }
  if (!c_invalid && nhot) {   // (the group kernel set the bits of any valid batch: walk them even if it failed later)
    tkey_t* __restrict__ results = A->results;
    const tkey_t* __restrict__ vals = A->vals;
    const bool ok = c_status == 0;
    // Deferred hot keys (SPLIT groups, group.cu): the bits of slot j are the key's
    // requests in timestamp order (present / op bit 0 / op bit 1 bitmaps over
    // [0, n)).  Work items (slot, chunk of HOT_CHW words) are taken in order; a
    // request's result is the value of the nearest earlier write of the key
    // (NOT_FOUND if a delete) or, with none, the pre-batch value old[seg]
    // (P:746-758); the nearest earlier write across chunks comes
    // from an epoch-tagged decoupled look-back (max of write payloads).
    const uint32_t C = R.hot_chunks, W = R.hot_words, items = nhot * C;
    const unsigned long long ep = (unsigned long long)(A->seq & 0x3FFFFFFFu) << 34;
    const uint32_t lane = threadIdx.x & 31, warp = threadIdx.x >> 5, nwarp = blockDim.x >> 5;
    for (; items;) {   // (no deferred hot key: no ticket atomics at all)
      __syncthreads();
      if (threadIdx.x == 0) s_item = atomicAdd(&ctl->hot_item, 1u);
      __syncthreads();
      const uint32_t item = s_item;
      if (item >= items) break;
      const uint32_t j = item / C, c = item - j * C;
      uint32_t* bits = R.hot_bits + (size_t)j * 3 * W;
      const uint32_t sH = s_hseg[j];
      const uint32_t w0 = c * HOT_CHW, w1 = min(W, w0 + HOT_CHW);
      const uint32_t PW = (HOT_CHW + blockDim.x - 1) / blockDim.x;
      const uint32_t tw0 = min(w1, w0 + threadIdx.x * PW), tw1 = min(w1, tw0 + PW);
      // pass 1: this thread's last write payload (0: none)
      uint32_t lw = 0;
      for (uint32_t x = tw0; x < tw1; ++x) {
        const uint32_t wm = __ldcg(bits + x) & (__ldcg(bits + W + x) | __ldcg(bits + 2 * W + x));
        if (wm) {
          const uint32_t tb = 31 - __clz(wm);
          lw = ((x * 32 + tb) << 2) | ((__ldcg(bits + W + x) >> tb) & 1u) | (((__ldcg(bits + 2 * W + x) >> tb) & 1u) << 1);
        }
      }
      // exclusive max-scan over the threads (ascending word ranges), chunk aggregate
      uint32_t inc = lw;
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        const uint32_t y = __shfl_up_sync(FULL, inc, o);
        if ((int)lane >= o) inc = max(inc, y);
      }
      if (lane == 31) s_red[warp] = inc;
      __syncthreads();
      uint32_t before = 0, agg = 0;
      for (uint32_t w = 0; w < nwarp; ++w) {
        if (w < warp) before = max(before, s_red[w]);
        agg = max(agg, s_red[w]);
      }
      const uint32_t excl = max(before, __shfl_up_sync(FULL, inc, 1) * (lane ? 1u : 0u));
      // look-back over the slot's earlier chunks: the nearest write before this chunk
      __shared__ uint32_t s_carry;
      if (threadIdx.x == 0) {
        unsigned long long* lb = R.hot_lb + (size_t)j * C;
        uint32_t carry = 0;
        if (c == 0) {
          st_relaxed64(lb, ep | (2ull << 32) | agg);
        } else {
          st_relaxed64(lb + c, ep | (1ull << 32) | agg);
          SpinGuard sg;
          for (int32_t pc = (int32_t)c - 1; pc >= 0;) {
            const unsigned long long wv = ld_relaxed64(lb + pc);
            const uint32_t fl = (uint32_t)(wv >> 32) & 3u;
            if ((wv & ~((1ull << 34) - 1)) != ep || fl == 0) {   // not yet published this batch
              if (sg.stuck(ctl)) break;
              continue;
            }
            carry = max(carry, (uint32_t)wv);
            if (fl == 2) break;
            --pc;
          }
          st_relaxed64(lb + c, ep | (2ull << 32) | max(carry, agg));
        }
        s_carry = carry;
      }
      __syncthreads();
      // pass 2: every request of the thread's words, in timestamp order
      uint32_t pv = max(s_carry, excl);
      const uint64_t vold = ok ? old[sH] : 0;
      for (uint32_t x = tw0; x < tw1; ++x) {
        const uint32_t pw = __ldcg(bits + x);
        if (!pw) continue;
        const uint32_t b0 = __ldcg(bits + W + x), b1 = __ldcg(bits + 2 * W + x);
        for (uint32_t m = pw; m; m &= m - 1) {
          const uint32_t tb = __ffs(m) - 1;
          const uint32_t op = ((b0 >> tb) & 1u) | (((b1 >> tb) & 1u) << 1);
          const uint32_t ts = x * 32 + tb;
          if (ok) results[ts] = pv ? (((pv & 3) == OP_DELETE) ? KEY_MAX : (uint64_t)vals[pv >> 2]) : vold;
          if (op) pv = (ts << 2) | op;
        }
        bits[x] = 0u;   // leave the slot clean for the next batch
        bits[W + x] = 0u;
        bits[2 * W + x] = 0u;
      }
    }
  }
  // End of the batch (the last kernel): the last CTA to finish publishes it
  if (last_cta(ctl->fin_sub, &ctl->fin_ctr)) publish_batch(ctl, A, hdr);
}


}  // namespace eirene
