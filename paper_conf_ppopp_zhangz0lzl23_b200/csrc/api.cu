// api.cu -- the C ABI (include/eirene.h): handle, pools, batch sequencing.
//
// A batch (Alg.1:1-7) is one CUDA graph replay of five kernels on the
// caller's stream:
//   set_args (zero the control region, publish the batch's pointers)
//   -> bsort_dist (key-range bucket distribution, Alg.1:10)
//   -> group (per-group smem sort + combine + partition, Alg.1:10-11, 3)
//   -> query (Alg.1:4, with the write locate and RESULT_CAL of short segments)
//   -> update (Alg.1:5, then the result phase: long segments, deferred hot
//      keys, the BatchCtl publish into a device ring slot).
// eirene_results() waits on the batch's event and fetches its BatchCtl off the
// pipeline.  No allocation and no host synchronisation happen inside submit.
// Graphs are captured per size bucket; pipelined handles (EIRENE_F_PIPELINE)
// split each batch into a front and a back graph on two streams (§7.2).
#include <algorithm>
#include <atomic>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <mutex>
#include <new>
#include <string>
#include <vector>

#include "eirene_internal.cuh"

using namespace eirene;

namespace {

constexpr int RING = 64;
constexpr int HOST_SLOTS = 3;   // host-path staging depth: H2D(b+1), kernels(b), D2H(b-1) in flight
constexpr int NSTAGE = 6;   // events: before sort, after sort / group / query / update / result

std::mutex g_err_mu;
std::string g_last_cuda_error = "no error";

int cuda_fail(cudaError_t e, const char* where) {
  std::lock_guard<std::mutex> lk(g_err_mu);
  g_last_cuda_error = std::string(where) + ": " + cudaGetErrorString(e);
  return EIRENE_ECUDA;
}

// Makes the handle's device current for the duration of an ABI call and
// restores the caller's current device on return (the caller's CUDA state is
// not changed behind its back).
struct DeviceGuard {
  int prev = -1;
  cudaError_t err = cudaSuccess;
  explicit DeviceGuard(int dev) {
    if (cudaGetDevice(&prev) != cudaSuccess) prev = -1;
    if (prev != dev) err = cudaSetDevice(dev);
  }
  ~DeviceGuard() {
    int cur = -1;
    if (prev >= 0 && cudaGetDevice(&cur) == cudaSuccess && cur != prev) cudaSetDevice(prev);
  }
};

#define CK(expr)                                    \
  do {                                              \
    cudaError_t _e = (expr);                        \
    if (_e != cudaSuccess) return cuda_fail(_e, #expr); \
  } while (0)

__global__ void init_empty_kernel(Tree t, uint64_t key_lo, uint64_t key_hi) {
  const int i = threadIdx.x;
  if (i < FAN) {
    t.lkeys[i] = KEY_MAX;
    t.lvals[i] = 0;
  }
  if (i == 0) {
    NodeMeta m;
    m.version = 0;
    m.next = NIL;
    m.lo = key_lo;
    m.hi = key_hi;
    m.count = 0;
    m.level = 0;
    t.lmeta[0] = m;
    t.lrf[0] = KEY_MAX;   // no leaf `height` links to the right
    TreeHdr* h = t.hdr;
    h->root_word = (1ull << 32) | 0ull;
    h->leaf_count = 1;
    h->inner_count = 0;
    for (int l = 0; l < MAX_LEVELS; ++l) h->level_count[l] = 0;
    h->level_count[0] = 1;
  }
}

// First node of the batch graph: zero the per-batch control region (BatchCtl,
// bin counts, group look-back words) and publish the batch's pointers.
__global__ void __launch_bounds__(1024) set_args_kernel(BatchArgs* dst, const uint8_t* ops, const tkey_t* keys,
                                                        const tkey_t* vals_src, tkey_t* vals_stage,
                                                        tkey_t* results, BatchCtl* ctl_out, uint4* zero,
                                                        uint32_t zero_n16, uint4* zero2, uint32_t zero2_n16,
                                                        tkey_t* rkeys, tkey_t* rvals, uint32_t rcap,
                                                        uint32_t n, unsigned long long* phase, uint32_t seq) {
  for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < zero_n16; i += gridDim.x * blockDim.x)
    zero[i] = make_uint4(0, 0, 0, 0);
  for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < zero2_n16; i += gridDim.x * blockDim.x)
    zero2[i] = make_uint4(0, 0, 0, 0);
  if (blockIdx.x == 0 && threadIdx.x == 0) {
    dst->t0 = gtime_ns();
    dst->ops = ops;
    dst->keys = keys;
    dst->vals = vals_stage ? vals_stage : vals_src;
    dst->vals_src = vals_src;
    dst->vals_stage = vals_stage;
    dst->results = results;
    dst->ctl_out = ctl_out;
    dst->rkeys = rkeys;
    dst->rvals = rvals;
    dst->rcap = rcap;
    dst->n = n;
    dst->phase = phase;
    dst->seq = seq;
  }
}

// kernels in one batch graph: set_args, 1-2 sort, group, query, (range), update + result phase
constexpr int SET_ARGS_CTAS = 4;
constexpr int MAX_GRAPHS = 8;

struct GraphEntry {
  uint32_t n = 0;
  bool range = false;               // batch graph with the range kernel
  cudaGraph_t graph = nullptr;      // kept alive: args_node belongs to it
  cudaGraphExec_t exec = nullptr;
  cudaGraphNode_t args_node = nullptr;
  int launches = 0;                 // kernels in the graph
  bool cond = false;                // the update kernel is a conditional node (may not run)
};

// One set of the buffers a batch's front (distribution + group: sort, combine,
// partition) hands to its back (query, range, update, RESULT_CAL), plus the
// per-batch control region.  Lane 0 always exists; with EIRENE_F_PIPELINE a
// second lane lets the front of batch b+1 run while the back of batch b runs
// (§8(f) NEXT(3)): the front never reads the tree, only the back does, and
// backs stay in submission order (query(b+1) after update(b)).
struct Lane {
  BSortBufs bs{}, bsL{};
  CombBufs cb{}, cbL{};
  BatchArgs* dargs = nullptr;
  BatchCtl* ctl = nullptr;
  unsigned char* zero_region = nullptr;
  unsigned char* zero_large = nullptr;
  GraphEntry fg[MAX_GRAPHS], bg[MAX_GRAPHS];   // pipelined mode: front / back graphs per size bucket
  uint32_t next_fg = 0, next_bg = 0;
  cudaEvent_t front_done = nullptr, back_done = nullptr;
  bool used = false;
};

struct Rec {
  uint64_t ticket = 0;
  bool used = false;
  bool timing = false;
  bool cond = false;      // its graph's update kernel is conditional
  uint32_t n = 0;
  int launches = 0;
  cudaEvent_t done = nullptr;
  cudaEvent_t st[NSTAGE] = {};
};

}  // namespace

struct eirene_tree {
  eirene_config cfg{};
  int num_sms = 148;
  Tree t{};
  SortBufs sb{};
  BSortBufs bs{};
  BatchArgs* dargs = nullptr;
  unsigned long long* phase = nullptr;   // diagnostic phase stamps (filled by -DEIRENE_PHASE_PROF builds)
  cudaStream_t cap_stream = nullptr;
  cudaStream_t cap_stream2 = nullptr;   // captures the body of the update kernel's conditional node
  // EIRENE_COND=1: the update kernel as a conditional graph node (measured r2: device batch time -2 us but the
  // gap between graph launches +8 us on cfg2 -- off by default)
  bool use_cond = std::getenv("EIRENE_COND") != nullptr;
  GraphEntry graphs[MAX_GRAPHS];
  Lane lanes[2];
  int nlanes = 1;
  uint32_t lane_seq = 0;
  cudaStream_t back_stream = nullptr;   // pipelined mode: the backs of all batches, in order
  cudaEvent_t last_done = nullptr;      // pipelined mode: the last submitted batch's end
  uint32_t next_graph = 0;
  bool use_graphs = std::getenv("EIRENE_NO_GRAPHS") == nullptr;
  CombBufs cb{};
  UpdParams up{};
  unsigned char* zero_region = nullptr;
  size_t zero_bytes = 0;
  // the two-kernel bucket sort of batches > 2^22 requests (16384 bins): its
  // bin counts, group cursors and group look-back words, zeroed only for them
  unsigned char* zero_large = nullptr;
  size_t zero_large_bytes = 0;
  BSortBufs bsL{};
  CombBufs cbL{};
  BatchCtl* ctl = nullptr;
  BatchCtl* host_ctl = nullptr;   // pinned [RING]: landing buffer of eirene_results
  BatchCtl* ctl_ring = nullptr;   // device [RING]: each batch's final BatchCtl (written by the update kernel's result phase)
  cudaStream_t res_stream = nullptr;
  cudaStream_t h2d_stream = nullptr, d2h_stream = nullptr;
  cudaEvent_t h2d_done[HOST_SLOTS] = {}, comp_ev[HOST_SLOTS] = {}, comp_done[HOST_SLOTS] = {};
  bool slot_used[HOST_SLOTS] = {};
  uint32_t host_slot = 0;
  uint8_t* st_ops = nullptr;
  tkey_t* st_keys = nullptr;
  tkey_t* st_vals = nullptr;
  tkey_t* st_res = nullptr;
  unsigned long long* route_lb = nullptr;
  unsigned long long* hot_lb = nullptr;   // result phase's look-back over the deferred hot keys' chunks
  uint32_t hot_chunks = 0;
  uint32_t* route_ctr = nullptr;
  uint32_t route_epoch = 0;
  Rec ring[RING];
  uint64_t next_ticket = 1;
  uint32_t batch_seq = 0;
  bool loaded = false;
  bool modified = false;
  uint64_t launches = 0;
  size_t device_bytes = 0;
  std::vector<void*> allocs;
  bool counted_pipelined = false;   // counted in g_pipelined_handles (cooperative grid launches while > 0)
  // fused routing (eirene_route_arena_*): this rank's receive arena, the P
  // peers' arenas (IPC-mapped or, in one process, plain device pointers)
  struct Arena {
    void* base = nullptr;
    uint32_t P = 0, me = 0, cap = 0, epoch = 0;
    uint32_t* cnt = nullptr;        // [P] uint4 {count, invalid, start, epoch} written by the sources
    uint64_t* res = nullptr;        // [cap] results pushed back by the shards (this rank's partition order)
    uint64_t* rec = nullptr;        // [P][cap][3] records pushed by the sources
    uint32_t* lcnt = nullptr;       // [64] local per-destination counts of the push
    uint32_t* linv = nullptr;       // validity flag of the push
    uint64_t** d_prec = nullptr;    // device tables [P]: peers' rec / res / cnt
    uint64_t** d_pres = nullptr;
    uint32_t** d_pcnt = nullptr;
    uint32_t* h_cnt = nullptr;      // pinned [P * 4]
    uint32_t pushed_n = 0;          // largest per-source count of the last pull (grid sizing)
    bool connected = false;
    std::vector<void*> opened;      // IPC mappings to close
  } ar;

  template <class T>
  cudaError_t dalloc(T** p, size_t count) {
    size_t bytes = sizeof(T) * (count ? count : 1);
    cudaError_t e = cudaMalloc(reinterpret_cast<void**>(p), bytes);
    if (e == cudaSuccess) {
      allocs.push_back(*p);
      device_bytes += bytes;
    }
    return e;
  }
};

namespace eirene {
// EIRENE_PDL=0/1 (read once per process): programmatic dependent launch of the
// batch's kernels 2.. (eirene_internal.cuh)
bool pdl_enabled() {
  static const bool on = [] {
    const char* e = std::getenv("EIRENE_PDL");
    return e ? std::atoi(e) != 0 : false;
  }();
  return on;
}
// EIRENE_COOP=0/1 (read once per process): cooperative launches of the
// grid-barrier kernels (default off: eirene_internal.cuh, launch_k)
// (also on while any pipelined handle exists in the process: its front's
// distribution kernel and its back's update kernel run concurrently on two
// streams, and two plain grid-barrier kernels could each hold the SMs the
// other needs)
std::atomic<int> g_pipelined_handles{0};
bool coop_enabled() {
  static const bool on = [] {
    const char* e = std::getenv("EIRENE_COOP");
    return e ? std::atoi(e) != 0 : false;
  }();
  return on || g_pipelined_handles.load(std::memory_order_relaxed) > 0;
}
}  // namespace eirene

extern "C" {

void eirene_default_config(eirene_config* c) {
  if (!c) return;
  std::memset(c, 0, sizeof(*c));
  c->device = 0;
  c->fanout = 16;
  c->max_keys = 1ull << 24;
  c->max_batch = 1u << 20;
  c->retry_threshold = 4;
  c->flags = EIRENE_F_REGROUP | EIRENE_F_STATS;
  c->key_lo = 0;
  c->key_hi = UINT64_MAX;
}

const char* eirene_strerror(int code) {
  switch (code) {
    case EIRENE_OK: return "ok";
    case EIRENE_EINVAL: return "invalid argument or invalid request";
    case EIRENE_ENOMEM: return "device allocation failed";
    case EIRENE_EFULL: return "node pools lack headroom for the batch";
    case EIRENE_ESTATE: return "call not valid in this state (or stale ticket)";
    case EIRENE_ECUDA: return "CUDA error (see eirene_last_cuda_error)";
    case EIRENE_EINTERNAL: return "internal error: the device watchdog fired (no forward progress; discard the tree) or a peer's routed push never arrived";
    default: return "unknown error";
  }
}

const char* eirene_last_cuda_error(void) {
  std::lock_guard<std::mutex> lk(g_err_mu);
  static thread_local std::string copy;
  copy = g_last_cuda_error;
  return copy.c_str();
}

int eirene_destroy(eirene_handle h);

int eirene_create(const eirene_config* cfg, eirene_handle* out) {
  if (!cfg || !out) return EIRENE_EINVAL;
  *out = nullptr;
  if (cfg->fanout != 16 || cfg->max_batch == 0 || cfg->max_batch > (1u << 29) || cfg->key_lo >= cfg->key_hi ||
      cfg->max_keys == 0)
    return EIRENE_EINVAL;
  if (sizeof(tkey_t) == 4 && cfg->key_lo >= 0xFFFFFFFFull) return EIRENE_EINVAL;   // (32-bit keys: empty range)
  DeviceGuard dg_(cfg->device);
  CK(dg_.err);
  eirene_tree* h = new (std::nothrow) eirene_tree();
  if (!h) return EIRENE_ENOMEM;
  h->cfg = *cfg;
  cudaDeviceGetAttribute(&h->num_sms, cudaDevAttrMultiProcessorCount, cfg->device);
  const uint64_t nb = cfg->max_batch;
  // Pools: leaves for max_keys at >= half fill plus one batch of worst-case
  // splits; inner nodes: a 1/4 of that (every inner node keeps >= 8 children
  // after a split) plus a batch of root growth.
  uint64_t leaf_cap = cfg->max_keys / 8 + 2 * nb + 1024;
  uint64_t inner_cap = leaf_cap / 4 + nb + 1024;
  if (leaf_cap > 0x7FFFFFF0ull || inner_cap > 0x7FFFFFF0ull) {
    delete h;
    return EIRENE_EINVAL;
  }
  cudaError_t e = cudaSuccess;
  Tree& t = h->t;
  t.leaf_cap = (uint32_t)leaf_cap;
  t.inner_cap = (uint32_t)inner_cap;
  const size_t sort_tiles = (nb + SORT_TILE - 1) / SORT_TILE;
#define AL(p, n)                                 \
  if (e == cudaSuccess) e = h->dalloc(&(p), (n));
  AL(t.lkeys, leaf_cap * LSTRIDE);   // keys and values of a leaf share one 256 B block
  if (e == cudaSuccess) t.lvals = t.lkeys + FAN;
  AL(t.lmeta, leaf_cap);
  AL(t.lrf, leaf_cap);
  AL(t.ikeys, inner_cap * FAN);
  AL(t.ichild, inner_cap * FAN);
  AL(t.imeta, inner_cap);
  AL(t.hdr, 1);
  AL(h->sb.kA, nb);
  AL(h->sb.kB, nb);
  AL(h->sb.pA, nb);
  AL(h->sb.pB, nb);
  AL(h->sb.lookback, sort_tiles * 256);
  AL(h->cb.pinfo, nb);
  AL(h->cb.qkey, nb);
  AL(h->cb.qseg, nb);
  AL(h->cb.wkey, nb);
  AL(h->cb.wop, nb);
  AL(h->cb.wval, nb);
  AL(h->cb.wseg, nb);
  AL(h->cb.wleaf, nb);
  AL(h->cb.wslot, nb);
  AL(h->cb.wparent, nb);
  AL(h->cb.old, nb);
  AL(h->cb.istart, nb + 1);
  AL(h->cb.longseg, nb + 64);   // (segment, chunk) pairs of the long segments
  h->cb.hot_words = (uint32_t)(((nb + 127) / 128) * 4);   // multiple of 4 (uint4 access)
  AL(h->cb.hot_bits, (size_t)HOT_SLOTS * 3 * h->cb.hot_words);
  AL(h->cb.hot_seg, HOT_SLOTS);
  AL(h->cb.grec, (size_t)NBINS_MAX * 4);   // GroupRec per group (the two-phase group stage)
  h->hot_chunks = (h->cb.hot_words + HOT_CHW - 1) / HOT_CHW;
  AL(h->hot_lb, (size_t)HOT_SLOTS * h->hot_chunks);   // epoch-tagged: never needs zeroing between batches
  AL(h->up.entA_key, nb + 64);
  AL(h->up.entA_child, nb + 64);
  AL(h->up.entB_key, nb + 64);
  AL(h->up.entB_child, nb + 64);
  AL(h->up.slots[0], nb / 16 + 32768);   // level-0 chunks of 16 writes
  AL(h->up.slots[1], nb / 32 + 32768);
  AL(h->up.eparent, nb + 64);
  AL(h->up.flat_key, nb + 64);
  AL(h->up.flat_child, nb + 64);
  AL(h->up.flat_off, nb / 32 + 32768);
  AL(h->st_ops, HOST_SLOTS * nb);
  AL(h->st_keys, HOST_SLOTS * nb);
  AL(h->st_vals, HOST_SLOTS * nb);
  AL(h->st_res, HOST_SLOTS * nb);
  if (e == cudaSuccess) e = cudaStreamCreateWithFlags(&h->h2d_stream, cudaStreamNonBlocking);
  if (e == cudaSuccess) e = cudaStreamCreateWithFlags(&h->d2h_stream, cudaStreamNonBlocking);
  for (int s = 0; s < HOST_SLOTS && e == cudaSuccess; ++s) {
    e = cudaEventCreateWithFlags(&h->h2d_done[s], cudaEventDisableTiming);
    if (e == cudaSuccess) e = cudaEventCreateWithFlags(&h->comp_done[s], cudaEventDisableTiming);
    if (e == cudaSuccess) e = cudaEventCreateWithFlags(&h->comp_ev[s], cudaEventDisableTiming);
  }
  AL(h->route_lb, ((nb + 2047) / 2048) * 64);
  AL(h->route_ctr, 2);   // [0] scatter tile counter, [1] validity flag of the packed partition
  AL(h->bs.gstart, NBINS_MAX + 1);
  AL(h->bs.bin2grp, NBINS_MAX);
  AL(h->dargs, 1);
  AL(h->phase, 2 * PROF_CTAS * PROF_PHASES);
  AL(h->ctl_ring, RING);
  if (e == cudaSuccess) e = cudaStreamCreateWithFlags(&h->cap_stream, cudaStreamNonBlocking);
  if (e == cudaSuccess) e = cudaStreamCreateWithFlags(&h->cap_stream2, cudaStreamNonBlocking);
  // one contiguous region zeroed before every batch: BatchCtl | ghist | comb/part status
  {
    size_t off = 0;
    auto bump = [&](size_t bytes) {
      size_t o = off;
      off += (bytes + 255) & ~size_t(255);
      return o;
    };
    const size_t o_ctl = bump(sizeof(BatchCtl));
    const size_t o_gh = bump(sizeof(uint32_t) * 8 * 256);
    const size_t o_bc = bump(sizeof(uint32_t) * NBINS);
    const size_t o_cu = bump(sizeof(uint32_t) * NBINS);
    const size_t o_gs = bump(sizeof(unsigned long long) * NBINS);
    h->zero_bytes = off;
    AL(h->zero_region, off);
    off = 0;
    const size_t l_bc = bump(sizeof(uint32_t) * NBINS_L);
    const size_t l_cu = bump(sizeof(uint32_t) * NBINS_L);
    const size_t l_gs = bump(sizeof(unsigned long long) * NBINS_L);
    h->zero_large_bytes = off;
    if (nb > bsort_fused_capacity(h->num_sms)) AL(h->zero_large, off);   // the two-kernel path's region
    if (e == cudaSuccess) {
      h->ctl = reinterpret_cast<BatchCtl*>(h->zero_region + o_ctl);
      h->sb.ghist = reinterpret_cast<uint32_t*>(h->zero_region + o_gh);
      h->bs.bcount = reinterpret_cast<uint32_t*>(h->zero_region + o_bc);
      h->bs.cursor = reinterpret_cast<uint32_t*>(h->zero_region + o_cu);
      h->bs.kA = h->sb.kA;
      h->bs.pA = h->sb.pA;
      h->bs.kB = h->sb.kB;
      h->bs.pB = h->sb.pB;
      h->cb.group_status = reinterpret_cast<unsigned long long*>(h->zero_region + o_gs);
      h->bsL = h->bs;
      h->cbL = h->cb;
      if (h->zero_large) {
        h->bsL.bcount = reinterpret_cast<uint32_t*>(h->zero_large + l_bc);
        h->bsL.cursor = reinterpret_cast<uint32_t*>(h->zero_large + l_cu);
        h->cbL.group_status = reinterpret_cast<unsigned long long*>(h->zero_large + l_gs);
      }
    }
  }
  // lane 0 = the buffers above; lane 1 (EIRENE_F_PIPELINE) = its own copy of
  // every buffer a front hands to its back and of the control regions
  if (e == cudaSuccess) {
    Lane& L0 = h->lanes[0];
    L0.bs = h->bs;
    L0.bsL = h->bsL;
    L0.cb = h->cb;
    L0.cbL = h->cbL;
    L0.dargs = h->dargs;
    L0.ctl = h->ctl;
    L0.zero_region = h->zero_region;
    L0.zero_large = h->zero_large;
  }
  if (e == cudaSuccess && (cfg->flags & EIRENE_F_PIPELINE)) {
    Lane& L1 = h->lanes[1];
    L1 = h->lanes[0];
    uint64_t *kB = nullptr, *qkey = nullptr, *wkey = nullptr, *wval = nullptr;
    uint32_t *pB = nullptr, *pinfo = nullptr, *istart = nullptr, *qseg = nullptr, *wseg = nullptr;
    uint8_t* wop = nullptr;
    AL(kB, nb);
    AL(pB, nb);
    AL(pinfo, nb);
    AL(istart, nb + 1);
    AL(qkey, nb);
    AL(qseg, nb);
    AL(wkey, nb);
    AL(wop, nb);
    AL(wval, nb);
    AL(wseg, nb);
    uint32_t *hbits = nullptr, *hseg = nullptr;   // hot-key bitmaps: set by the front, walked by the back
    AL(hbits, (size_t)HOT_SLOTS * 3 * h->cb.hot_words);
    AL(hseg, HOT_SLOTS);
    AL(L1.dargs, 1);
    AL(L1.zero_region, h->zero_bytes);
    if (h->zero_large) AL(L1.zero_large, h->zero_large_bytes);
    if (e == cudaSuccess) {
      const ptrdiff_t dz = L1.zero_region - h->zero_region;
      const ptrdiff_t dl = h->zero_large ? L1.zero_large - h->zero_large : 0;
      auto rz = [&](auto* p) { return reinterpret_cast<decltype(p)>(reinterpret_cast<unsigned char*>(p) + dz); };
      auto rl = [&](auto* p) { return reinterpret_cast<decltype(p)>(reinterpret_cast<unsigned char*>(p) + dl); };
      L1.ctl = rz(h->ctl);
      for (BSortBufs* b : {&L1.bs, &L1.bsL}) {
        b->kB = kB;
        b->pB = pB;
      }
      L1.bs.bcount = rz(h->bs.bcount);
      L1.bs.cursor = rz(h->bs.cursor);
      if (h->zero_large) {
        L1.bsL.bcount = rl(h->bsL.bcount);
        L1.bsL.cursor = rl(h->bsL.cursor);
      }
      for (CombBufs* c : {&L1.cb, &L1.cbL}) {
        c->pinfo = pinfo;
        c->istart = istart;
        c->qkey = qkey;
        c->qseg = qseg;
        c->wkey = wkey;
        c->wop = wop;
        c->wval = wval;
        c->wseg = wseg;
        c->hot_bits = hbits;
        c->hot_seg = hseg;
      }
      L1.cb.group_status = rz(h->cb.group_status);
      if (h->zero_large) L1.cbL.group_status = rl(h->cbL.group_status);
      h->nlanes = 2;
      e = cudaMemset(L1.zero_region, 0, h->zero_bytes);
      if (e == cudaSuccess) e = cudaMemset(hbits, 0, sizeof(uint32_t) * HOT_SLOTS * 3 * h->cb.hot_words);
      if (e == cudaSuccess && L1.zero_large) e = cudaMemset(L1.zero_large, 0, h->zero_large_bytes);
      if (e == cudaSuccess) e = cudaStreamCreateWithFlags(&h->back_stream, cudaStreamNonBlocking);
    }
  }
  for (int l = 0; l < h->nlanes && e == cudaSuccess; ++l) {
    e = cudaEventCreateWithFlags(&h->lanes[l].front_done, cudaEventDisableTiming);
    if (e == cudaSuccess) e = cudaEventCreateWithFlags(&h->lanes[l].back_done, cudaEventDisableTiming);
  }
#undef AL
  if (e == cudaSuccess) e = cudaMallocHost(reinterpret_cast<void**>(&h->host_ctl), sizeof(BatchCtl) * RING);
  if (e == cudaSuccess) e = cudaStreamCreateWithFlags(&h->res_stream, cudaStreamNonBlocking);
  for (int i = 0; i < RING && e == cudaSuccess; ++i) {
    e = cudaEventCreateWithFlags(&h->ring[i].done, cudaEventDisableTiming);
    for (int s = 0; s < NSTAGE && e == cudaSuccess; ++s) e = cudaEventCreate(&h->ring[i].st[s]);
  }
  if (e == cudaSuccess) e = cudaMemset(h->cb.hot_bits, 0, sizeof(uint32_t) * HOT_SLOTS * 3 * h->cb.hot_words);
  if (e == cudaSuccess) e = cudaMemset(h->hot_lb, 0, sizeof(unsigned long long) * HOT_SLOTS * h->hot_chunks);
  if (e == cudaSuccess) e = cudaMemset(h->sb.lookback, 0, sizeof(unsigned long long) * sort_tiles * 256);
  if (e == cudaSuccess) e = cudaMemset(h->route_lb, 0, sizeof(unsigned long long) * ((nb + 2047) / 2048) * 64);
  if (e == cudaSuccess) {
    init_empty_kernel<<<1, 32>>>(t, cfg->key_lo, cfg->key_hi);
    e = cudaGetLastError();
    if (e == cudaSuccess) e = cudaDeviceSynchronize();
  }
  if (e != cudaSuccess) {
    int rc = (e == cudaErrorMemoryAllocation) ? EIRENE_ENOMEM : cuda_fail(e, "eirene_create");
    eirene_destroy(h);
    return rc;
  }
  h->up.threshold = cfg->retry_threshold;
  h->up.flags = cfg->flags;
  if (cfg->flags & EIRENE_F_PIPELINE) {
    eirene::g_pipelined_handles.fetch_add(1);
    h->counted_pipelined = true;
  }
  *out = h;
  return EIRENE_OK;
}

int eirene_destroy(eirene_handle h) {
  if (!h) return EIRENE_EINVAL;
  DeviceGuard dg_(h->cfg.device);
  cudaDeviceSynchronize();
  for (int i = 0; i < RING; ++i) {
    if (h->ring[i].done) cudaEventDestroy(h->ring[i].done);
    for (int s = 0; s < NSTAGE; ++s)
      if (h->ring[i].st[s]) cudaEventDestroy(h->ring[i].st[s]);
  }
  for (auto& g : h->graphs) {
    if (g.exec) cudaGraphExecDestroy(g.exec);
    if (g.graph) cudaGraphDestroy(g.graph);
  }
  if (h->cap_stream) cudaStreamDestroy(h->cap_stream);
  if (h->cap_stream2) cudaStreamDestroy(h->cap_stream2);
  for (auto& L : h->lanes) {
    for (GraphEntry* ge : {L.fg, L.bg})
      for (int i = 0; i < MAX_GRAPHS; ++i) {
        if (ge[i].exec) cudaGraphExecDestroy(ge[i].exec);
        if (ge[i].graph) cudaGraphDestroy(ge[i].graph);
      }
    if (L.front_done) cudaEventDestroy(L.front_done);
    if (L.back_done) cudaEventDestroy(L.back_done);
  }
  if (h->back_stream) cudaStreamDestroy(h->back_stream);
  if (h->h2d_stream) cudaStreamDestroy(h->h2d_stream);
  if (h->d2h_stream) cudaStreamDestroy(h->d2h_stream);
  for (int s = 0; s < HOST_SLOTS; ++s) {
    if (h->h2d_done[s]) cudaEventDestroy(h->h2d_done[s]);
    if (h->comp_done[s]) cudaEventDestroy(h->comp_done[s]);
    if (h->comp_ev[s]) cudaEventDestroy(h->comp_ev[s]);
  }
  if (h->counted_pipelined) eirene::g_pipelined_handles.fetch_sub(1);
  for (void* p : h->ar.opened) cudaIpcCloseMemHandle(p);
  if (h->ar.h_cnt) cudaFreeHost(h->ar.h_cnt);
  for (void* p : h->allocs) cudaFree(p);
  if (h->host_ctl) cudaFreeHost(h->host_ctl);
  if (h->res_stream) cudaStreamDestroy(h->res_stream);
  delete h;
  return EIRENE_OK;
}

int eirene_bulk_load(eirene_handle h, const tkey_t* keys, const tkey_t* vals, uint64_t n, float leaf_fill,
                     eirene_stream_t stream) {
  if (!h) return EIRENE_EINVAL;
  if (h->loaded || h->modified) return EIRENE_ESTATE;
  if (n == 0) return EIRENE_OK;
  if (!keys || !vals || !(leaf_fill > 0.f) || leaf_fill > 1.f) return EIRENE_EINVAL;
  DeviceGuard dg_(h->cfg.device);
  CK(dg_.err);
  cudaStream_t st = reinterpret_cast<cudaStream_t>(stream);
  int per = (int)(16.f * leaf_fill + 0.5f);
  if (per < 1) per = 1;
  if (per > 16) per = 16;
  if ((n + per - 1) / per > h->t.leaf_cap) return EIRENE_EFULL;
  int launches = 0;
  uint32_t* flag = &h->ctl->invalid;
  CK(cudaMemsetAsync(h->zero_region, 0, h->zero_bytes, st));
  if (h->zero_large) CK(cudaMemsetAsync(h->zero_large, 0, h->zero_large_bytes, st));
  launch_validate_bulk(keys, vals, n, h->cfg.key_lo, h->cfg.key_hi, flag, st, &launches);
  uint32_t bad = 0;
  CK(cudaMemcpyAsync(&bad, flag, sizeof(uint32_t), cudaMemcpyDeviceToHost, st));
  CK(cudaStreamSynchronize(st));
  if (bad) return EIRENE_EINVAL;
  uint32_t height = 0;
  int rc = build_tree(h->t, keys, vals, n, per, h->cfg.key_lo, h->cfg.key_hi, st, &launches, &height);
  h->launches += launches;
  CK(cudaGetLastError());
  if (rc == EIRENE_OK) h->loaded = true;
  return rc;
}

// Size bucket of an n-request batch: exact up to 256, else n rounded up to
// 1/8 of its power of two (<= 12.5% padding, 8 buckets per octave), at most
// max_batch.
static uint32_t size_bucket(uint32_t n, uint32_t max_batch) {
  if (n <= 256) return n;
  const int k = 31 - __builtin_clz(n);
  const uint32_t step = 1u << (k - 3);
  const uint64_t b = ((uint64_t)n + step - 1) / step * step;
  return (uint32_t)std::min<uint64_t>(b, max_batch);
}

static cudaError_t capture_node(cudaStream_t s, cudaGraphNode_t* out) {
  cudaStreamCaptureStatus cs;
  const cudaGraphNode_t* deps = nullptr;
  size_t nd = 0;
  cudaError_t e = cudaStreamGetCaptureInfo(s, &cs, nullptr, nullptr, &deps, &nd);
  if (e != cudaSuccess) return e;
  if (nd != 1) return cudaErrorStreamCaptureInvalidated;
  *out = deps[0];
  return cudaSuccess;
}

}  // extern "C"

// The graph of `table` for (size bucket, range), captured from `enqueue` on
// first use (kept: up to MAX_GRAPHS per table).
template <class F>
static int get_graph(eirene_handle h, GraphEntry* table, uint32_t& next, uint32_t nk, bool range, bool want_args,
                     F&& enqueue, GraphEntry** out) {
  for (int i = 0; i < MAX_GRAPHS; ++i)
    if (table[i].exec && table[i].n == nk && table[i].range == range) {
      *out = &table[i];
      return EIRENE_OK;
    }
  GraphEntry& e = table[next++ % MAX_GRAPHS];
  if (e.exec) cudaGraphExecDestroy(e.exec);
  if (e.graph) cudaGraphDestroy(e.graph);
  e = GraphEntry{};
  int launches = 0;
  CK(cudaStreamBeginCapture(h->cap_stream, cudaStreamCaptureModeRelaxed));
  cudaError_t ce = enqueue(h->cap_stream, want_args ? &e.args_node : nullptr, &launches);
  cudaError_t ee = cudaStreamEndCapture(h->cap_stream, &e.graph);
  if (ce != cudaSuccess) return cuda_fail(ce, "capture");
  CK(ee);
  // A/B (EIRENE_L2WIN=MB): an L2 persisting access-policy window over the
  // first MB of the inner nodes' separator lines on every kernel node
  static const int l2win = std::getenv("EIRENE_L2WIN") ? std::atoi(std::getenv("EIRENE_L2WIN")) : 0;
  if (l2win > 0) {
    int maxp = 0, maxw = 0;
    cudaDeviceGetAttribute(&maxp, cudaDevAttrMaxPersistingL2CacheSize, h->cfg.device);
    cudaDeviceGetAttribute(&maxw, cudaDevAttrMaxAccessPolicyWindowSize, h->cfg.device);
    const size_t want = std::min<size_t>({(size_t)l2win << 20, (size_t)maxp, (size_t)maxw,
                                          (size_t)h->t.inner_cap * FAN * sizeof(tkey_t)});
    cudaDeviceSetLimit(cudaLimitPersistingL2CacheSize, want);
    cudaLaunchAttributeValue v{};
    v.accessPolicyWindow.base_ptr = h->t.ikeys;
    v.accessPolicyWindow.num_bytes = want;
    v.accessPolicyWindow.hitRatio = 1.0f;
    v.accessPolicyWindow.hitProp = cudaAccessPropertyPersisting;
    v.accessPolicyWindow.missProp = cudaAccessPropertyStreaming;
    size_t nn = 0;
    CK(cudaGraphGetNodes(e.graph, nullptr, &nn));
    std::vector<cudaGraphNode_t> nodes(nn);
    CK(cudaGraphGetNodes(e.graph, nodes.data(), &nn));
    for (cudaGraphNode_t nd : nodes) {
      cudaGraphNodeType ty;
      if (cudaGraphNodeGetType(nd, &ty) == cudaSuccess && ty == cudaGraphNodeTypeKernel)
        CK(cudaGraphKernelNodeSetAttribute(nd, cudaLaunchAttributeAccessPolicyWindow, &v));
    }
  }
  CK(cudaGraphInstantiate(&e.exec, e.graph, 0));
  e.n = nk;
  e.range = range;
  e.launches = launches;
  *out = &e;
  return EIRENE_OK;
}

extern "C" {

static int submit_impl(eirene_handle h, const uint8_t* ops, const tkey_t* keys, const tkey_t* vals, uint32_t n,
                       tkey_t* results, cudaStream_t st, tkey_t* vals_stage, uint64_t* ticket,
                       tkey_t* rkeys = nullptr, tkey_t* rvals = nullptr, uint32_t rcap = 0,
                       bool prepare_only = false, bool prepare_range = false, cudaStream_t* end_stream = nullptr) {
  const bool range = rkeys != nullptr || prepare_range;
  DeviceGuard dg_(h->cfg.device);
  CK(dg_.err);
  if (prepare_only && (!h->use_graphs || (h->cfg.flags & EIRENE_F_TIMING))) return EIRENE_OK;
  static const bool dbg = std::getenv("EIRENE_DEBUG_SYNC") != nullptr;
  const bool timing = (h->cfg.flags & EIRENE_F_TIMING) != 0;
  // cross-batch pipelining (EIRENE_F_PIPELINE): graph replays only
  const bool pipe = h->nlanes == 2 && h->use_graphs && !timing && !dbg;
  const uint64_t tk = prepare_only ? 0 : h->next_ticket++;
  Rec scratch_rec;
  Rec& r = prepare_only ? scratch_rec : h->ring[tk % RING];
  if (!prepare_only) {
    r.ticket = tk;
    r.used = true;
  }
  r.n = n;
  // Launches (grids, group count, distribution path) and the captured graphs
  // are sized for n's size bucket; the kernels read the batch's own n from
  // BatchArgs.  Batches of varying size (the shards of a multi-GPU batch)
  // then replay a handful of graphs instead of capturing one per size.
  const uint32_t nk = size_bucket(n, h->cfg.max_batch);
  r.timing = timing;
  const uint32_t seq = ++h->batch_seq;
  auto stage = [&](const char* name, cudaStream_t s) {
    if (!dbg) return;
    cudaError_t e = cudaStreamSynchronize(s);
    std::fprintf(stderr, "[eirene] batch %u stage %s done: %s\n", seq, name, cudaGetErrorString(e));
  };
  auto rec = [&](int i, cudaStream_t s) { cudaEventRecord(r.st[i], s); };
  bool cond_captured = false;   // set by `back` when it captured a conditional update node
  bool* cond_out = &cond_captured;
  BatchCtl* ctl_slot = h->ctl_ring + tk % RING;
  const bool large = !bsort_fused(nk, h->num_sms);   // two-kernel bucket sort with 16384 bins (bsort.cu)
  // The front of a batch: a tiny node publishing its pointers to the lane's
  // device-side BatchArgs (and zeroing the lane's control region), then the
  // distribution and group kernels (sort Alg.1:10, combine Alg.1:11, partition
  // Alg.1:3).  Nothing in it reads the tree.
  auto front = [&](Lane& L, cudaStream_t s, cudaGraphNode_t* args_node, int* nl) -> cudaError_t {
    uint4* zero16 = reinterpret_cast<uint4*>(L.zero_region);
    const uint32_t zero_n16 = (uint32_t)(h->zero_bytes / 16);
    uint4* zero2 = reinterpret_cast<uint4*>(large ? L.zero_large : L.zero_region);
    const uint32_t zero2_n16 = large ? (uint32_t)(h->zero_large_bytes / 16) : 0u;
    set_args_kernel<<<SET_ARGS_CTAS, 1024, 0, s>>>(L.dargs, ops, keys, vals, vals_stage, results, ctl_slot, zero16,
                                                   zero_n16, zero2, zero2_n16, rkeys, rvals, rcap, n, h->phase, seq);
    ++*nl;
    if (args_node) {
      cudaError_t e = capture_node(s, args_node);
      if (e != cudaSuccess) return e;
    }
    if (timing) rec(0, s);
    // (32-bit keys: the bins span [key_lo, min(key_hi, 2^32)), not the 64-bit range)
    const uint64_t bin_hi = sizeof(tkey_t) == 4 ? std::min<uint64_t>(h->cfg.key_hi, 1ull << 32) : h->cfg.key_hi;
    launch_bucket_sort(L.dargs, nk, h->cfg.key_lo, bin_hi, large ? L.bsL : L.bs, L.ctl, h->num_sms, s, nl);
    stage("sort", s);
    if (timing) rec(1, s);
    // (range batches keep the one-kernel stage: their hot keys are walked by the group kernel)
    launch_group(L.dargs, nk, large ? L.bsL : L.bs, large ? L.cbL : L.cb, h->t, L.ctl, h->num_sms,
                 !range && group_two_phase(nk, h->num_sms), s, nl);
    stage("group", s);
    return cudaGetLastError();
  };
  // The back: query (Alg.1:15-21; it checks the pool headroom first), range,
  // update (Alg.1:23-46), RESULT_CAL (Alg.1:6) -- the kernels that read or
  // change the tree.
  // capture: the update kernel becomes the body of a conditional graph node
  // that the query kernel's last CTA switches on only when there is anything
  // left for it (structural writes, long segments, deferred hot keys); else
  // the query kernel ends the batch (query_end, query.cu).  Not for range
  // batches (their range kernel sits between the two).
  auto back = [&](Lane& L, cudaStream_t s, int* nl, bool capture) -> cudaError_t {
    const uint32_t* spay = L.bs.pB;
    const bool cond_mode = capture && !range && h->use_cond;
    cudaGraphConditionalHandle cond = 0;
    cudaGraph_t cg = nullptr;
    if (cond_mode) {
      cudaStreamCaptureStatus cs;
      cudaError_t e = cudaStreamGetCaptureInfo(s, &cs, nullptr, &cg, nullptr, nullptr);
      if (e == cudaSuccess) e = cudaGraphConditionalHandleCreate(&cond, cg, 0, cudaGraphCondAssignDefault);
      if (e != cudaSuccess) return e;
    }
    if (timing) rec(2, s);
    launch_query(nk, L.cb, spay, L.dargs, h->t, L.ctl, h->num_sms, h->cfg.flags, h->cfg.iter_rgs, cond,
                 cond_mode ? 1 : 0, s, nl);
    if (range) launch_range(nk, L.cb, spay, L.bs.kB, L.dargs, h->t, L.ctl, h->num_sms, s, nl);
    stage("query", s);
    if (timing) rec(3, s);
    const ResultArgs ra{spay,          L.bs.kB,  L.cb.pinfo,       L.cb.istart,    L.cb.longseg,
                        L.cb.old,      L.dargs,  L.ctl,            h->t.hdr,       L.cb.hot_bits,
                        L.cb.hot_words, L.cb.hot_seg, h->hot_lb,   h->hot_chunks};
    cudaStream_t us = s;
    if (cond_mode) {
      cudaStreamCaptureStatus cs;
      const cudaGraphNode_t* deps = nullptr;
      size_t nd = 0;
      cudaError_t e = cudaStreamGetCaptureInfo(s, &cs, nullptr, &cg, &deps, &nd);
      cudaGraphNodeParams cp{};
      cp.type = cudaGraphNodeTypeConditional;
      cp.conditional.handle = cond;
      cp.conditional.type = cudaGraphCondTypeIf;
      cp.conditional.size = 1;
      cudaGraphNode_t cn = nullptr;
      if (e == cudaSuccess) e = cudaGraphAddNode(&cn, cg, deps, nd, &cp);
      if (e == cudaSuccess) e = cudaStreamUpdateCaptureDependencies(s, &cn, 1, cudaStreamSetCaptureDependencies);
      if (e == cudaSuccess)
        e = cudaStreamBeginCaptureToGraph(h->cap_stream2, cp.conditional.phGraph_out[0], nullptr, nullptr, 0,
                                          cudaStreamCaptureModeRelaxed);
      if (e != cudaSuccess) return e;
      us = h->cap_stream2;
    }
    launch_update(nk, L.cb, h->t, L.ctl, h->up, ra, h->num_sms, us, nl);
    if (cond_mode) {
      cudaGraph_t body = nullptr;
      cudaError_t e = cudaStreamEndCapture(h->cap_stream2, &body);
      if (e != cudaSuccess) return e;
      *cond_out = true;
    }
    stage("update", s);
    if (timing) rec(4, s);
    if (dbg) launch_result(L.ctl, 1, s);
    else launch_result(L.ctl, 0, s);
    stage("result", s);
    if (timing) rec(5, s);
    return cudaGetLastError();
  };
  auto set_args_params = [&](GraphEntry* g, Lane& L) -> int {
    uint4* zero16 = reinterpret_cast<uint4*>(L.zero_region);
    uint32_t zero_n16 = (uint32_t)(h->zero_bytes / 16);
    uint4* zero2 = reinterpret_cast<uint4*>(large ? L.zero_large : L.zero_region);
    uint32_t zero2_n16 = large ? (uint32_t)(h->zero_large_bytes / 16) : 0u;
    void* params[] = {&L.dargs, const_cast<uint8_t**>(&ops), const_cast<tkey_t**>(&keys),
                      const_cast<tkey_t**>(&vals), &vals_stage, &results, &ctl_slot, &zero16, &zero_n16,
                      &zero2, &zero2_n16, &rkeys, &rvals, &rcap, &n, &h->phase, const_cast<uint32_t*>(&seq)};
    cudaKernelNodeParams p{};
    p.func = reinterpret_cast<void*>(set_args_kernel);
    p.gridDim = dim3(SET_ARGS_CTAS);
    p.blockDim = dim3(1024);
    p.sharedMemBytes = 0;
    p.kernelParams = params;
    p.extra = nullptr;
    CK(cudaGraphExecKernelNodeSetParams(g->exec, g->args_node, &p));
    return EIRENE_OK;
  };
  int launches = 0;
  cudaStream_t end = st;
  if (pipe) {
    // front of this batch on the caller's stream, back on the handle's back stream
    auto fq = [&](cudaStream_t s, cudaGraphNode_t* an, int* nl) { return front(h->lanes[0], s, an, nl); };
    if (prepare_only) {
      for (int l = 0; l < 2; ++l) {
        Lane& L = h->lanes[l];
        GraphEntry *gf, *gb;
        int rc = get_graph(h, L.fg, L.next_fg, nk, range, true,
                           [&](cudaStream_t s, cudaGraphNode_t* an, int* nl) { return front(L, s, an, nl); }, &gf);
        if (rc != EIRENE_OK) return rc;
        rc = get_graph(h, L.bg, L.next_bg, nk, range, false,
                       [&](cudaStream_t s, cudaGraphNode_t*, int* nl) { return back(L, s, nl, true); }, &gb);
        if (rc != EIRENE_OK) return rc;
        if (cond_captured) gb->cond = true;
        cond_captured = false;
      }
      (void)fq;
      return EIRENE_OK;
    }
    Lane& L = h->lanes[h->lane_seq++ & 1];
    GraphEntry *gf, *gb;
    int rc = get_graph(h, L.fg, L.next_fg, nk, range, true,
                       [&](cudaStream_t s, cudaGraphNode_t* an, int* nl) { return front(L, s, an, nl); }, &gf);
    if (rc != EIRENE_OK) return rc;
    rc = get_graph(h, L.bg, L.next_bg, nk, range, false,
                   [&](cudaStream_t s, cudaGraphNode_t*, int* nl) { return back(L, s, nl, true); }, &gb);
    if (rc != EIRENE_OK) return rc;
    if (cond_captured) gb->cond = true;
    if (L.used) CK(cudaStreamWaitEvent(st, L.back_done, 0));   // the back of batch b-2 released this lane
    rc = set_args_params(gf, L);
    if (rc != EIRENE_OK) return rc;
    CK(cudaGraphLaunch(gf->exec, st));
    CK(cudaEventRecord(L.front_done, st));
    CK(cudaStreamWaitEvent(h->back_stream, L.front_done, 0));
    CK(cudaGraphLaunch(gb->exec, h->back_stream));
    CK(cudaEventRecord(L.back_done, h->back_stream));
    L.used = true;
    launches = gf->launches + gb->launches;
    r.cond = gb->cond;
    end = h->back_stream;
  } else {
    Lane& L = h->lanes[0];
    if (h->nlanes == 2 && h->last_done) CK(cudaStreamWaitEvent(st, h->last_done, 0));   // pipelined batches first
    auto whole = [&](cudaStream_t s, cudaGraphNode_t* an, int* nl) -> cudaError_t {
      cudaError_t e = front(L, s, an, nl);
      return e != cudaSuccess ? e : back(L, s, nl, an != nullptr);
    };
    if (dbg || timing || !h->use_graphs) {   // per-stage events: direct launches
      CK(whole(st, nullptr, &launches));
    } else {
      // one captured graph per batch size bucket; a replay updates only the args node
      GraphEntry* g = nullptr;
      int rc = get_graph(h, h->graphs, h->next_graph, nk, range, true, whole, &g);
      if (rc != EIRENE_OK) return rc;
      if (cond_captured) g->cond = true;
      if (prepare_only) return EIRENE_OK;   // graph captured and instantiated, nothing launched
      rc = set_args_params(g, L);
      if (rc != EIRENE_OK) return rc;
      CK(cudaGraphLaunch(g->exec, st));
      launches = g->launches;
      r.cond = g->cond;
    }
  }
  CK(cudaEventRecord(r.done, end));
  if (h->nlanes == 2) h->last_done = r.done;
  if (end_stream) *end_stream = end;
  r.launches = launches;
  h->launches += launches;
  h->modified = true;
  *ticket = tk;
  return EIRENE_OK;
}

int eirene_submit_batch(eirene_handle h, const uint8_t* ops, const tkey_t* keys, const tkey_t* vals, uint32_t n,
                        tkey_t* results, eirene_stream_t stream, uint64_t* ticket) {
  if (!h || !ops || !keys || !vals || !results || !ticket) return EIRENE_EINVAL;
  if (n == 0 || n > h->cfg.max_batch) return EIRENE_EINVAL;
  return submit_impl(h, ops, keys, vals, n, results, reinterpret_cast<cudaStream_t>(stream), nullptr, ticket);
}

int eirene_prepare_batch(eirene_handle h, uint32_t n, int with_ranges) {
  if (!h || n == 0 || n > h->cfg.max_batch) return EIRENE_EINVAL;
  uint64_t tk = 0;
  return submit_impl(h, nullptr, nullptr, nullptr, n, nullptr, nullptr, nullptr, &tk, nullptr, nullptr, 0, true,
                     with_ranges != 0);
}

int eirene_submit_batch_range(eirene_handle h, const uint8_t* ops, const tkey_t* keys, const tkey_t* vals,
                              uint32_t n, tkey_t* results, uint32_t cap, tkey_t* range_keys,
                              tkey_t* range_vals, eirene_stream_t stream, uint64_t* ticket) {
  if (!h || !ops || !keys || !vals || !results || !ticket || !range_keys || !range_vals) return EIRENE_EINVAL;
  if (n == 0 || n > h->cfg.max_batch || cap == 0 || cap > 4096) return EIRENE_EINVAL;
  return submit_impl(h, ops, keys, vals, n, results, reinterpret_cast<cudaStream_t>(stream), nullptr, ticket,
                     range_keys, range_vals, cap);
}

int eirene_submit_batch_host(eirene_handle h, const uint8_t* ops, const tkey_t* keys, const tkey_t* vals,
                             uint32_t n, tkey_t* results, eirene_stream_t stream, uint64_t* ticket) {
  if (!h || !ops || !keys || !vals || !results || !ticket) return EIRENE_EINVAL;
  if (n == 0 || n > h->cfg.max_batch) return EIRENE_EINVAL;
  cudaStream_t st = reinterpret_cast<cudaStream_t>(stream);
  DeviceGuard dg_(h->cfg.device);
  CK(dg_.err);
  // Triple-buffered staging (HOST_SLOTS), three streams: the H2D of this batch (copy
  // stream) overlaps the previous batch's kernels (`st`) and the D2H of its
  // results (d2h stream).  A slot is reused only after the D2H of the batch
  // that last used it.  Values are not copied when the host buffer is pinned:
  // the distribution kernel reads the values of the batch's upserts (the only
  // ones any kernel reads) straight from host memory and stages them, so a
  // read-mostly batch ships 9 of its 17 B/request.
  const int s = (int)(h->host_slot++ % HOST_SLOTS);
  const size_t off = (size_t)s * h->cfg.max_batch;
  if (h->slot_used[s]) CK(cudaStreamWaitEvent(h->h2d_stream, h->comp_done[s], 0));
  CK(cudaMemcpyAsync(h->st_ops + off, ops, n, cudaMemcpyHostToDevice, h->h2d_stream));
  CK(cudaMemcpyAsync(h->st_keys + off, keys, sizeof(tkey_t) * n, cudaMemcpyHostToDevice, h->h2d_stream));
  cudaPointerAttributes pa{};
  static const bool vals_copy = std::getenv("EIRENE_VALS_COPY") != nullptr;   // A/B: always copy the values
  const bool pinned = !vals_copy && cudaPointerGetAttributes(&pa, vals) == cudaSuccess &&
                      pa.type == cudaMemoryTypeHost && pa.devicePointer != nullptr;
  cudaGetLastError();   // (clear a pageable-pointer query error, if any)
  const tkey_t* vsrc;
  tkey_t* vstage = nullptr;
  if (pinned) {
    vsrc = static_cast<const tkey_t*>(pa.devicePointer);
    vstage = h->st_vals + off;
  } else {
    CK(cudaMemcpyAsync(h->st_vals + off, vals, sizeof(tkey_t) * n, cudaMemcpyHostToDevice, h->h2d_stream));
    vsrc = h->st_vals + off;
  }
  CK(cudaEventRecord(h->h2d_done[s], h->h2d_stream));
  CK(cudaStreamWaitEvent(st, h->h2d_done[s], 0));
  uint64_t tk = 0;
  cudaStream_t end = st;   // (the handle's back stream when pipelined)
  int rc = submit_impl(h, h->st_ops + off, h->st_keys + off, vsrc, n, h->st_res + off, st, vstage, &tk, nullptr,
                       nullptr, 0, false, false, &end);
  if (rc != EIRENE_OK) return rc;
  CK(cudaEventRecord(h->comp_ev[s], end));
  CK(cudaStreamWaitEvent(h->d2h_stream, h->comp_ev[s], 0));
  CK(cudaMemcpyAsync(results, h->st_res + off, sizeof(tkey_t) * n, cudaMemcpyDeviceToHost, h->d2h_stream));
  CK(cudaEventRecord(h->comp_done[s], h->d2h_stream));
  CK(cudaEventRecord(h->ring[tk % RING].done, h->d2h_stream));   // eirene_results waits for the D2H too
  h->slot_used[s] = true;
  *ticket = tk;
  return EIRENE_OK;
}

int eirene_results(eirene_handle h, uint64_t ticket, eirene_batch_stats* stats) {
  if (!h) return EIRENE_EINVAL;
  DeviceGuard dg_(h->cfg.device);
  CK(dg_.err);
  Rec& r = h->ring[ticket % RING];
  if (!r.used || r.ticket != ticket) return EIRENE_ESTATE;
  CK(cudaEventSynchronize(r.done));
  // the batch's BatchCtl stays on the device (no copy on the batch's stream);
  // fetched here, off the GPU pipeline
  CK(cudaMemcpyAsync(&h->host_ctl[ticket % RING], h->ctl_ring + ticket % RING, sizeof(BatchCtl),
                     cudaMemcpyDeviceToHost, h->res_stream));
  CK(cudaStreamSynchronize(h->res_stream));
  const BatchCtl& c = h->host_ctl[ticket % RING];
  if (stats) {
    std::memset(stats, 0, sizeof(*stats));
    stats->status = c.status;
    stats->n = r.n;
    stats->distinct = c.nseg;
    stats->issued_q = c.nq;
    stats->issued_w = c.nw;
    stats->leaf_runs = c.leaf_runs;
    stats->retries = c.retries;
    stats->stm_fallbacks = c.stm_fallbacks;
    stats->leaf_splits = c.leaf_splits;
    stats->inner_splits = c.inner_splits;
    stats->new_leaves = c.new_leaves;
    stats->new_inner = c.new_inner;
    stats->height = c.height;
    // (a conditional update kernel that did not run is not counted)
    stats->launches = (uint32_t)r.launches - ((r.cond && !c.upd_ran) ? 1u : 0u);
    stats->ranges = c.nrange;
    stats->artificial = c.nart;
    stats->trav_steps = c.trav_steps;
    stats->rg_vertical = c.rg_vertical;
    stats->rg_horizontal = c.rg_horizontal;
    stats->device_ns = c.t_end > c.t_begin ? c.t_end - c.t_begin : 0;
    stats->t_begin_ns = c.t_begin;
    stats->t_end_ns = c.t_end;
    stats->nins = c.nins;
    stats->ndelp = c.ndelp;
    if (r.timing) {
      for (int s = 0; s + 1 < NSTAGE; ++s) cudaEventElapsedTime(&stats->stage_ms[s], r.st[s], r.st[s + 1]);
      cudaEventElapsedTime(&stats->stage_ms[7], r.st[0], r.st[NSTAGE - 1]);
    }
  }
  return c.status;
}

int eirene_scan(eirene_handle h, uint64_t lo, uint64_t hi, tkey_t* keys_out, tkey_t* vals_out, uint64_t cap,
                uint64_t* count, eirene_stream_t stream) {
  if (!h || !count) return EIRENE_EINVAL;
  if (cap > 0 && !keys_out && !vals_out) return EIRENE_EINVAL;
  DeviceGuard dg_(h->cfg.device);
  CK(dg_.err);
  cudaStream_t st = reinterpret_cast<cudaStream_t>(stream);
  if (h->nlanes == 2 && h->last_done) CK(cudaStreamWaitEvent(st, h->last_done, 0));   // pipelined batches first
  TreeHdr hdr;
  CK(cudaMemcpyAsync(&hdr, h->t.hdr, sizeof(hdr), cudaMemcpyDeviceToHost, st));
  CK(cudaStreamSynchronize(st));
  int launches = 0;
  int rc = scan_tree(h->t, hdr.leaf_count, lo, hi, keys_out, vals_out, cap, count, st, &launches);
  h->launches += launches;
  if (rc == EIRENE_ECUDA) return cuda_fail(cudaGetLastError(), "eirene_scan");
  return rc;
}

int eirene_debug_phases(eirene_handle h, uint64_t* out, uint32_t n_words) {
  if (!h || !out) return EIRENE_EINVAL;
  DeviceGuard dg_(h->cfg.device);
  CK(dg_.err);
  CK(cudaDeviceSynchronize());
  const uint32_t m = std::min<uint32_t>(n_words, 2 * PROF_CTAS * PROF_PHASES);
  CK(cudaMemcpy(out, h->phase, sizeof(uint64_t) * m, cudaMemcpyDeviceToHost));
  return EIRENE_OK;
}

int eirene_set_flags(eirene_handle h, uint32_t flags) {
  if (!h) return EIRENE_EINVAL;
  h->cfg.flags = flags;
  h->up.flags = flags;
  // captured graphs bake the update kernel's flags in: drop them
  for (auto& g : h->graphs) {
    if (g.exec) cudaGraphExecDestroy(g.exec);
    if (g.graph) cudaGraphDestroy(g.graph);
    g = GraphEntry{};
  }
  for (auto& L : h->lanes)
    for (GraphEntry* ge : {L.fg, L.bg})
      for (int i = 0; i < MAX_GRAPHS; ++i) {
        if (ge[i].exec) cudaGraphExecDestroy(ge[i].exec);
        if (ge[i].graph) cudaGraphDestroy(ge[i].graph);
        ge[i] = GraphEntry{};
      }
  return EIRENE_OK;
}

int eirene_stream_wait_batch(eirene_handle h, uint64_t ticket, eirene_stream_t stream) {
  if (!h) return EIRENE_EINVAL;
  const Rec& r = h->ring[ticket % RING];
  if (!r.used || r.ticket != ticket) return EIRENE_ESTATE;
  DeviceGuard dg_(h->cfg.device);
  CK(dg_.err);
  CK(cudaStreamWaitEvent(reinterpret_cast<cudaStream_t>(stream), r.done, 0));
  return EIRENE_OK;
}

int eirene_get_info(eirene_handle h, eirene_tree_info* info) {
  if (!h || !info) return EIRENE_EINVAL;
  DeviceGuard dg_(h->cfg.device);
  CK(dg_.err);
  TreeHdr hdr;
  if (h->back_stream) CK(cudaStreamSynchronize(h->back_stream));
  CK(cudaMemcpy(&hdr, h->t.hdr, sizeof(hdr), cudaMemcpyDeviceToHost));
  info->height = (uint32_t)(hdr.root_word >> 32);
  info->root = (uint32_t)hdr.root_word;
  info->leaves = hdr.leaf_count;
  info->inner = hdr.inner_count;
  info->leaf_cap = h->t.leaf_cap;
  info->inner_cap = h->t.inner_cap;
  info->launches = h->launches;
  info->device_bytes = h->device_bytes;
  return EIRENE_OK;
}

// ---------------------------------------------------------------- invariants
// Host-side structural check of a quiescent tree (debug utility).
int eirene_check_invariants(eirene_handle h, uint64_t* n_keys) {
  if (!h) return EIRENE_EINVAL;
  DeviceGuard dg_(h->cfg.device);
  CK(dg_.err);
  CK(cudaDeviceSynchronize());
  TreeHdr hdr;
  CK(cudaMemcpy(&hdr, h->t.hdr, sizeof(hdr), cudaMemcpyDeviceToHost));
  const uint32_t L = hdr.leaf_count, I = hdr.inner_count;
  std::vector<tkey_t> lk((size_t)L * FAN), ik((size_t)I * FAN);
  std::vector<uint32_t> ic((size_t)I * FAN);
  std::vector<NodeMeta> lm(L), im(I);
  CK(cudaMemcpy2D(lk.data(), FAN * sizeof(tkey_t), h->t.lkeys, LSTRIDE * sizeof(tkey_t), FAN * sizeof(tkey_t), L,
                   cudaMemcpyDeviceToHost));
  CK(cudaMemcpy(lm.data(), h->t.lmeta, lm.size() * sizeof(NodeMeta), cudaMemcpyDeviceToHost));
  if (I) {
    CK(cudaMemcpy(ik.data(), h->t.ikeys, ik.size() * sizeof(tkey_t), cudaMemcpyDeviceToHost));
    CK(cudaMemcpy(ic.data(), h->t.ichild, ic.size() * 4, cudaMemcpyDeviceToHost));
    CK(cudaMemcpy(im.data(), h->t.imeta, im.size() * sizeof(NodeMeta), cudaMemcpyDeviceToHost));
  }
  const uint32_t height = (uint32_t)(hdr.root_word >> 32), root = (uint32_t)hdr.root_word;
  if (height == 0 || height > MAX_LEVELS) return 10;
  std::vector<uint32_t> inorder;
  uint64_t total = 0;
  // iterative DFS: (node, level, lo, hi)
  struct Fr { uint32_t node, level; uint64_t lo, hi; };
  std::vector<Fr> stack{{root, height - 1, h->cfg.key_lo, h->cfg.key_hi}};
  std::vector<uint8_t> seen_leaf(L, 0);
  while (!stack.empty()) {
    Fr f = stack.back();
    stack.pop_back();
    if (f.level == 0) {
      if (f.node >= L) return 11;
      if (seen_leaf[f.node]++) return 12;
      const NodeMeta& m = lm[f.node];
      if (m.version & 1u) return 13;
      if (m.lo != f.lo || m.hi != f.hi) return 14;
      uint64_t prev = 0;
      bool first = true, ended = false;
      for (int s = 0; s < FAN; ++s) {
        const uint64_t k = widen(lk[(size_t)f.node * FAN + s]);
        if (k == KEY_MAX) { ended = true; continue; }
        if (ended) return 15;               // key after padding
        if (!first && !(prev < k)) return 16;   // strictly increasing
        if (k < m.lo || k >= m.hi) return 17;   // inside fences
        prev = k;
        first = false;
        ++total;
      }
      inorder.push_back(f.node);
      continue;
    }
    if (f.node >= I) return 18;
    const NodeMeta& m = im[f.node];
    if (m.version & 1u) return 13;
    if (m.level != f.level) return 19;
    if (m.lo != f.lo || m.hi != f.hi) return 14;
    const uint32_t c = m.count;
    if (c < 1 || c > FAN) return 20;
    const tkey_t* Kr = &ik[(size_t)f.node * FAN];
    auto K = [&](uint32_t i) { return widen(Kr[i]); };
    const uint32_t* Cc = &ic[(size_t)f.node * FAN];
    for (uint32_t i = 0; i + 1 < c; ++i) {
      if (K(i) == KEY_MAX) return 21;
      if (i > 0 && !(K(i - 1) < K(i))) return 16;
      if (K(i) <= f.lo || K(i) >= f.hi) return 17;
    }
    for (uint32_t i = c - 1; i < FAN; ++i)
      if (K(i) != KEY_MAX) return 21;
    // push children right-to-left so the leftmost is visited first
    for (int i = (int)c - 1; i >= 0; --i) {
      const uint64_t clo = i == 0 ? f.lo : K(i - 1);
      const uint64_t chi = (uint32_t)i + 1 < c ? K(i) : f.hi;
      stack.push_back({Cc[i], f.level - 1, clo, chi});
    }
  }
  // leaf chain == in-order leaves; every allocated leaf is reachable
  if (inorder.size() != L) return 22;
  for (size_t i = 0; i < inorder.size(); ++i) {
    const uint32_t want = i + 1 < inorder.size() ? inorder[i + 1] : NIL;
    if (lm[inorder[i]].next != want) return 23;
  }
  if (n_keys) *n_keys = total;
  return 0;
}

// ---------------------------------------------------------------- routing
int eirene_route_partition(eirene_handle h, const uint8_t* ops, const uint64_t* keys, const uint64_t* vals, uint32_t n,
                           const uint64_t* splitters, int P, uint8_t* sops, uint64_t* skeys, uint64_t* svals,
                           uint32_t* perm, uint32_t* counts, uint32_t* invalid, eirene_stream_t stream) {
  if (!h || P < 1 || P > 64 || !counts) return EIRENE_EINVAL;
  if (n > h->cfg.max_batch) return EIRENE_EINVAL;
  if (n > 0 && (!ops || !keys || !vals || !sops || !skeys || !svals || !perm)) return EIRENE_EINVAL;
  if (P > 1 && !splitters) return EIRENE_EINVAL;
  DeviceGuard dg_(h->cfg.device);
  CK(dg_.err);
  int launches = 0;
  launch_route_partition(ops, keys, vals, n, splitters, P, sops, skeys, svals, nullptr, perm, counts, 1, invalid,
                         h->route_lb, h->route_ctr, ++h->route_epoch, reinterpret_cast<cudaStream_t>(stream),
                         &launches);
  h->launches += launches;
  CK(cudaGetLastError());
  return EIRENE_OK;
}

int eirene_route_partition_packed(eirene_handle h, const uint8_t* ops, const uint64_t* keys, const uint64_t* vals,
                                  uint32_t n, const uint64_t* splitters, int P, uint64_t* send_rec, uint32_t* perm,
                                  uint32_t* counts2, eirene_stream_t stream) {
  if (!h || P < 1 || P > 64 || !counts2) return EIRENE_EINVAL;
  if (n > h->cfg.max_batch) return EIRENE_EINVAL;
  if (n > 0 && (!ops || !keys || !vals || !send_rec || !perm)) return EIRENE_EINVAL;
  if (P > 1 && !splitters) return EIRENE_EINVAL;
  DeviceGuard dg_(h->cfg.device);
  CK(dg_.err);
  cudaStream_t st = reinterpret_cast<cudaStream_t>(stream);
  int launches = 0;
  CK(cudaMemsetAsync(h->route_ctr + 1, 0, sizeof(uint32_t), st));
  launch_route_partition(ops, keys, vals, n, splitters, P, nullptr, nullptr, nullptr, send_rec, perm, counts2, 2,
                         h->route_ctr + 1, h->route_lb, h->route_ctr, ++h->route_epoch, st, &launches);
  h->launches += launches;
  CK(cudaGetLastError());
  return EIRENE_OK;
}

int eirene_route_unpack(eirene_handle h, const uint64_t* recv_rec, uint32_t n, uint8_t* ops_out, uint64_t* keys_out,
                        uint64_t* vals_out, eirene_stream_t stream) {
  if (!h) return EIRENE_EINVAL;
  if (n > 0 && (!recv_rec || !ops_out || !keys_out || !vals_out)) return EIRENE_EINVAL;
  DeviceGuard dg_(h->cfg.device);
  CK(dg_.err);
  int launches = 0;
  launch_route_unpack(recv_rec, n, ops_out, keys_out, vals_out, reinterpret_cast<cudaStream_t>(stream), &launches);
  h->launches += launches;
  CK(cudaGetLastError());
  return EIRENE_OK;
}

int eirene_batch_status_async(eirene_handle h, uint64_t ticket, int32_t* status_dev, eirene_stream_t stream) {
  if (!h || !status_dev) return EIRENE_EINVAL;
  const Rec& r = h->ring[ticket % RING];
  if (!r.used || r.ticket != ticket) return EIRENE_ESTATE;
  DeviceGuard dg_(h->cfg.device);
  CK(dg_.err);
  CK(cudaStreamWaitEvent(reinterpret_cast<cudaStream_t>(stream), r.done, 0));   // (pipelined: ends elsewhere)
  CK(cudaMemcpyAsync(status_dev, &h->ctl_ring[ticket % RING].status, sizeof(int32_t), cudaMemcpyDeviceToDevice,
                     reinterpret_cast<cudaStream_t>(stream)));
  return EIRENE_OK;
}

int eirene_route_unpermute(eirene_handle h, const uint64_t* recv, const uint32_t* perm, uint32_t n, uint64_t* results,
                           eirene_stream_t stream) {
  if (!h) return EIRENE_EINVAL;
  if (n > 0 && (!recv || !perm || !results)) return EIRENE_EINVAL;
  DeviceGuard dg_(h->cfg.device);
  CK(dg_.err);
  int launches = 0;
  launch_route_unpermute(recv, perm, n, results, reinterpret_cast<cudaStream_t>(stream), &launches);
  h->launches += launches;
  CK(cudaGetLastError());
  return EIRENE_OK;
}

// ---------------------------------------------------------------- fused routing over peer memory
// Arena layout (identical on every rank): [0, 1024) the P source slots
// {count, invalid, start, epoch}; [1024, ..) res[cap]; then rec[P][cap][3].
static size_t arena_res_off() { return 1024; }
static size_t arena_rec_off(uint32_t cap) { return 1024 + (((size_t)cap * 8 + 255) / 256) * 256; }
static size_t arena_bytes(uint32_t P, uint32_t cap) { return arena_rec_off(cap) + (size_t)P * cap * 24; }

int eirene_route_arena_create(eirene_handle h, int P, int rank, uint32_t cap, void** arena_dev_out,
                              void* ipc_handle_out) {
  if (!h || P < 1 || P > 64 || rank < 0 || rank >= P || cap == 0 || !arena_dev_out) return EIRENE_EINVAL;
  if (h->ar.base) return EIRENE_ESTATE;
  DeviceGuard dg_(h->cfg.device);
  CK(dg_.err);
  auto& A = h->ar;
  unsigned char* base = nullptr;
  CK(h->dalloc(&base, arena_bytes((uint32_t)P, cap)));
  CK(cudaMemset(base, 0, 1024));
  A.base = base;
  A.P = (uint32_t)P;
  A.me = (uint32_t)rank;
  A.cap = cap;
  A.cnt = reinterpret_cast<uint32_t*>(base);
  A.res = reinterpret_cast<uint64_t*>(base + arena_res_off());
  A.rec = reinterpret_cast<uint64_t*>(base + arena_rec_off(cap));
  CK(h->dalloc(&A.lcnt, 64));
  CK(h->dalloc(&A.linv, 1));
  CK(h->dalloc(&A.d_prec, 64));
  CK(h->dalloc(&A.d_pres, 64));
  CK(h->dalloc(&A.d_pcnt, 64));
  CK(cudaMallocHost(reinterpret_cast<void**>(&A.h_cnt), sizeof(uint32_t) * 4 * 64));
  *arena_dev_out = base;
  if (ipc_handle_out) {
    cudaIpcMemHandle_t ih;
    CK(cudaIpcGetMemHandle(&ih, base));
    std::memcpy(ipc_handle_out, &ih, sizeof(ih));
  }
  return EIRENE_OK;
}

int eirene_route_arena_open_ipc(eirene_handle h, const void* ipc_handle, void** arena_dev_out) {
  if (!h || !ipc_handle || !arena_dev_out) return EIRENE_EINVAL;
  DeviceGuard dg_(h->cfg.device);
  CK(dg_.err);
  cudaIpcMemHandle_t ih;
  std::memcpy(&ih, ipc_handle, sizeof(ih));
  void* p = nullptr;
  CK(cudaIpcOpenMemHandle(&p, ih, cudaIpcMemLazyEnablePeerAccess));
  h->ar.opened.push_back(p);
  *arena_dev_out = p;
  return EIRENE_OK;
}

int eirene_route_arena_connect(eirene_handle h, void* const* peer_arenas) {
  if (!h || !peer_arenas) return EIRENE_EINVAL;
  auto& A = h->ar;
  if (!A.base) return EIRENE_ESTATE;
  DeviceGuard dg_(h->cfg.device);
  CK(dg_.err);
  uint64_t* prec[64];
  uint64_t* pres[64];
  uint32_t* pcnt[64];
  for (uint32_t d = 0; d < A.P; ++d) {
    unsigned char* b = static_cast<unsigned char*>(peer_arenas[d]);
    if (!b) return EIRENE_EINVAL;
    prec[d] = reinterpret_cast<uint64_t*>(b + arena_rec_off(A.cap));
    pres[d] = reinterpret_cast<uint64_t*>(b + arena_res_off());
    pcnt[d] = reinterpret_cast<uint32_t*>(b);
  }
  CK(cudaMemcpy(A.d_prec, prec, sizeof(void*) * A.P, cudaMemcpyHostToDevice));
  CK(cudaMemcpy(A.d_pres, pres, sizeof(void*) * A.P, cudaMemcpyHostToDevice));
  CK(cudaMemcpy(A.d_pcnt, pcnt, sizeof(void*) * A.P, cudaMemcpyHostToDevice));
  A.connected = true;
  return EIRENE_OK;
}

int eirene_route_push(eirene_handle h, const uint8_t* ops, const uint64_t* keys, const uint64_t* vals, uint32_t n,
                      const uint64_t* splitters, uint32_t* perm, eirene_stream_t stream) {
  if (!h) return EIRENE_EINVAL;
  auto& A = h->ar;
  if (!A.connected) return EIRENE_ESTATE;
  if (n > A.cap || n > h->cfg.max_batch) return EIRENE_EINVAL;
  if (n > 0 && (!ops || !keys || !vals || !perm)) return EIRENE_EINVAL;
  if (A.P > 1 && !splitters) return EIRENE_EINVAL;
  DeviceGuard dg_(h->cfg.device);
  CK(dg_.err);
  cudaStream_t st = reinterpret_cast<cudaStream_t>(stream);
  int launches = 0;
  CK(cudaMemsetAsync(A.linv, 0, sizeof(uint32_t), st));
  launch_route_partition(ops, keys, vals, n, splitters, (int)A.P, nullptr, nullptr, nullptr, nullptr, perm, A.lcnt, 1,
                         A.linv, h->route_lb, h->route_ctr, ++h->route_epoch, st, &launches, A.d_prec, A.me, A.cap);
  launch_push_counts(A.lcnt, A.linv, (int)A.P, A.me, A.d_pcnt, ++A.epoch, st, &launches);
  h->launches += launches;
  CK(cudaGetLastError());
  return EIRENE_OK;
}

int eirene_route_pull(eirene_handle h, uint8_t* ops_out, uint64_t* keys_out, uint64_t* vals_out, uint32_t n_cap,
                      uint32_t* n_out, uint32_t* invalid_out, eirene_stream_t stream) {
  if (!h || !n_out || !invalid_out) return EIRENE_EINVAL;
  auto& A = h->ar;
  if (!A.connected) return EIRENE_ESTATE;
  DeviceGuard dg_(h->cfg.device);
  CK(dg_.err);
  cudaStream_t st = reinterpret_cast<cudaStream_t>(stream);
  CK(cudaMemcpyAsync(A.h_cnt, A.cnt, sizeof(uint32_t) * 4 * A.P, cudaMemcpyDeviceToHost, st));
  CK(cudaStreamSynchronize(st));   // the one host synchronisation of a fused-routing batch
  uint64_t n = 0;
  uint32_t inv = 0, mx = 0;
  for (uint32_t s = 0; s < A.P; ++s) {
    const uint32_t* e = A.h_cnt + 4 * s;
    if (e[3] != A.epoch) return EIRENE_EINTERNAL;   // a source's push of this batch never arrived
    n += e[0];
    inv |= e[1];
    mx = std::max(mx, e[0]);
  }
  *invalid_out = inv;
  *n_out = (uint32_t)std::min<uint64_t>(n, 0xFFFFFFFFull);
  A.pushed_n = 0;
  if (inv) return EIRENE_OK;
  if (n > n_cap || n > h->cfg.max_batch) return EIRENE_EINVAL;
  if (n > 0 && (!ops_out || !keys_out || !vals_out)) return EIRENE_EINVAL;
  int launches = 0;
  launch_pull_unpack(A.cnt, A.rec, A.cap, (int)A.P, mx, ops_out, keys_out, vals_out, st, &launches);
  A.pushed_n = mx;
  h->launches += launches;
  CK(cudaGetLastError());
  return EIRENE_OK;
}

int eirene_route_push_results(eirene_handle h, const uint64_t* results, eirene_stream_t stream) {
  if (!h) return EIRENE_EINVAL;
  auto& A = h->ar;
  if (!A.connected) return EIRENE_ESTATE;
  if (A.pushed_n > 0 && !results) return EIRENE_EINVAL;
  DeviceGuard dg_(h->cfg.device);
  CK(dg_.err);
  int launches = 0;
  launch_push_results(A.cnt, results, (int)A.P, A.pushed_n, A.d_pres, reinterpret_cast<cudaStream_t>(stream),
                      &launches);
  A.pushed_n = 0;
  h->launches += launches;
  CK(cudaGetLastError());
  return EIRENE_OK;
}

int eirene_route_unpermute_arena(eirene_handle h, const uint32_t* perm, uint32_t n, uint64_t* results,
                                 eirene_stream_t stream) {
  if (!h) return EIRENE_EINVAL;
  auto& A = h->ar;
  if (!A.connected) return EIRENE_ESTATE;
  if (n > A.cap || (n > 0 && (!perm || !results))) return EIRENE_EINVAL;
  DeviceGuard dg_(h->cfg.device);
  CK(dg_.err);
  int launches = 0;
  launch_route_unpermute(A.res, perm, n, results, reinterpret_cast<cudaStream_t>(stream), &launches);
  h->launches += launches;
  CK(cudaGetLastError());
  return EIRENE_OK;
}

}  // extern "C"
