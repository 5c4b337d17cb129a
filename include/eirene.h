/*
 * eirene.h -- C ABI of the B200-native Eirene batched B+tree.
 *
 * The library processes batches of Query / Update / Insert / Delete requests
 * on a B+tree resident in GPU global memory and returns linearizable results
 * (PAPER.md, Zhang et al., PPoPP'23).  Citations: P:N = /root/reference/PAPER.md
 * line N, Alg.1:k = line k of Algorithm 1, SURVEY §x = SURVEY.md.
 *
 * Problem statement the calls follow:
 *   - requests are buffered by the host and shipped to the GPU in batches
 *     (P:167-171);
 *   - each request carries a key, a value and a type: query, or one of the
 *     update requests update / insertion / deletion;
 *   - the logical timestamp of a request is its position in the buffer
 *     (P:718-722); batches are linearized in submission order;
 *   - results are linearizable: result[i] is the value the key
 *     held immediately before request i in timestamp order, or
 *     EIRENE_NOT_FOUND if it was absent.  Writes return the prior value too
 *     (SURVEY §8(c) reading 1).  UPDATE and INSERT are both blind upserts,
 *     DELETE erases (no-op on an absent key) (§8(c) readings 2-3).
 *
 * Conventions: pointers named *_dev are CUDA device pointers, *_host are host
 * pointers (pinned memory recommended).  All calls return EIRENE_OK (0) or a
 * negative error code; eirene_strerror() names it.  A handle is bound to one
 * device, is single-stream and is NOT thread-safe.  No call allocates device
 * memory after eirene_create except eirene_scan / eirene_check_invariants
 * (quiescent utilities).
 */
#ifndef EIRENE_H
#define EIRENE_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct CUstream_st* eirene_stream_t;   /* == cudaStream_t; NULL = legacy default stream */

/* Key / value width.  libeirene.so: 64-bit keys and values (BASELINE configs).
 * Built with -DEIRENE_KEY32 (libeirene32.so): 32-bit keys
 * and values, the paper's record width -- the leaves and inner nodes
 * hold 32-bit keys, so a leaf key line is 64 B and a value sector 8 values.
 * Every key / value / result pointer of the single-GPU API below is
 * eirene_key_t; the multi-GPU routing calls are 64-bit only.
 * Result sentinel (null): the all-ones value of the width.  It is
 * also reserved as a key and as a written value; requests using it are
 * rejected with EIRENE_EINVAL. */
#ifdef EIRENE_KEY32
typedef uint32_t eirene_key_t;
#define EIRENE_NOT_FOUND UINT32_MAX
#else
typedef uint64_t eirene_key_t;
#define EIRENE_NOT_FOUND UINT64_MAX
#endif

enum {
  EIRENE_OK = 0,
  EIRENE_EINVAL = -1,   /* bad argument or invalid request in a batch          */
  EIRENE_ENOMEM = -2,   /* device allocation failed in create                  */
  EIRENE_EFULL = -3,    /* node pools lack headroom for the batch's worst case */
  EIRENE_ESTATE = -4,   /* call not valid in the handle's state / stale ticket */
  EIRENE_ECUDA = -5,    /* a CUDA runtime error; eirene_last_cuda_error()      */
  EIRENE_EINTERNAL = -6 /* device watchdog fired (a bug: no forward progress); the
                           tree must be discarded                              */
};

/* Request types; EIRENE_RANGE = range query R(l, u),
 * accepted only by eirene_submit_batch_range. */
enum { EIRENE_QUERY = 0, EIRENE_UPDATE = 1, EIRENE_INSERT = 2, EIRENE_DELETE = 3, EIRENE_RANGE = 4 };

/* eirene_config.flags */
enum {
  EIRENE_F_REGROUP = 1u << 0,   /* leaf-bucketed warp regrouping in the update kernel;
                                   off = one warp per issued write (ablation, exercises retries) */
  EIRENE_F_STATS = 1u << 1,     /* count retries / STM fallbacks / splits on the device           */
  EIRENE_F_FORCE_STM = 1u << 2, /* every traversal in the update kernel is STM-protected
                                   (equivalent to retry_threshold = 0, Alg.1:28-33)               */
  EIRENE_F_TIMING = 1u << 3,    /* record per-stage CUDA events (eirene_batch_stats.stage_ms)     */
  EIRENE_F_ITERWARP = 1u << 4,  /* query kernel: the paper's iteration warps with a per-leaf range
                                   field (RF) choosing vertical (root-to-leaf) or horizontal
                                   (leaf-link) traversal per request group (Fig.6);
                                   off = one key-sorted request per thread with path sharing (the
                                   default).  Results are identical either way;
                                   with EIRENE_F_STATS the batch stats report the decisions      */
  EIRENE_F_PIPELINE = 1u << 5   /* (at create) cross-batch pipelining, §8(f) NEXT(3): the front
                                   of batch b+1 (distribution, group sort, combine, partition --
                                   nothing that reads the tree) runs on the caller's stream while
                                   the back of batch b (query, update, RESULT_CAL) runs on the
                                   handle's back stream; backs stay in submission order, so
                                   query(b+1) follows update(b).  Double-buffers the
                                   front->back scratch.  A batch's results are then NOT ordered on
                                   the caller's stream: use eirene_results or
                                   eirene_stream_wait_batch before consuming them there        */
};

typedef struct {
  int device;                 /* CUDA device ordinal                                           */
  uint32_t fanout;            /* node capacity; must be 16 (SURVEY §8(c) reading 12)           */
  uint64_t max_keys;          /* sizes the node pools (keys the tree may hold)                 */
  uint32_t max_batch;         /* largest n accepted by submit (sizes all scratch), <= 2^30     */
  uint32_t retry_threshold;   /* THRESHOLD of Alg.1:28; attempts before the STM fallback       */
  uint32_t flags;             /* EIRENE_F_*                                                    */
  uint64_t key_lo, key_hi;    /* key range owned by this tree (shard), [key_lo, key_hi);
                                 0 .. UINT64_MAX for a single GPU                              */
  uint32_t iter_rgs;          /* EIRENE_F_ITERWARP: request groups (32 issued requests each) per
                                 iteration warp; 0 = spread the RGs evenly over the resident
                                 warps                                           */
} eirene_config;

/* Fills *cfg with the defaults: device 0, fanout 16, max_keys 2^24,
 * max_batch 2^20, retry_threshold 4, flags REGROUP|STATS, range [0, UINT64_MAX), iter_rgs 0. */
void eirene_default_config(eirene_config* cfg);

typedef struct eirene_tree* eirene_handle;

typedef struct {
  int32_t status;             /* EIRENE_OK, EIRENE_EINVAL (invalid request: tree untouched),
                                 EIRENE_EFULL (no headroom: tree untouched)                    */
  uint32_t n;                 /* requests in the batch                                         */
  uint64_t distinct;          /* distinct keys == issued requests                  */
  uint64_t issued_q;          /* issued queries  (query kernel, Alg.1:4)                       */
  uint64_t issued_w;          /* issued writes   (update kernel, Alg.1:5)                      */
  uint64_t leaf_runs;         /* leaf runs processed by the update kernel (regrouping)         */
  uint64_t retries;           /* failed optimistic / transactional attempts (Alg.1:41)         */
  uint64_t stm_fallbacks;     /* attempts made with STM-protected traversal (Alg.1:30-33)      */
  uint64_t leaf_splits;       /* leaves split                                    */
  uint64_t inner_splits;      /* inner nodes split                                             */
  uint64_t new_leaves, new_inner;
  uint32_t height;            /* tree height after the batch (1 = root is a leaf)              */
  uint32_t launches;          /* kernels launched for this batch                               */
  float stage_ms[8];          /* EIRENE_F_TIMING: [0] sort (bucket scatter), [1] group (bucket
                                 sort + combine + partition), [2] query, [3] update, [4] result,
                                 [5], [6] unused, [7] total                                    */
  uint64_t ranges;            /* range queries in the batch (eirene_submit_batch_range)         */
  uint64_t artificial;        /* artificial queries resolved for them               */
  uint64_t trav_steps;        /* EIRENE_F_ITERWARP|STATS: nodes visited by the issued requests'
                                 traversals (vertical: height; horizontal: 1 + links followed;
                                 Fig.10 "traversal steps"); 0 otherwise            */
  uint64_t rg_vertical;       /* EIRENE_F_ITERWARP|STATS: request groups traversed from the root */
  uint64_t rg_horizontal;     /* ... and along the leaf links from the iteration warp's buffer  */
  uint64_t device_ns;         /* batch response time on the device: %globaltimer at the start of
                                 the batch's first kernel to the end of its last one (ns); the
                                 paper's per-batch time without host
                                 launch jitter                                                  */
  uint64_t t_begin_ns, t_end_ns;   /* the two %globaltimer stamps of device_ns (gaps between batches) */
  uint64_t nins, ndelp;       /* issued inserts of absent keys / deletes of present keys: the
                                 structural writes left to the update kernel (value overwrites
                                 of present keys are applied in place by the query kernel)      */
} eirene_batch_stats;

/* Creates a tree (one empty leaf) on cfg->device and allocates every pool and
 * scratch buffer up front.  Errors: EINVAL (null / fanout != 16 / sizes),
 * ENOMEM, ECUDA. */
int eirene_create(const eirene_config* cfg, eirene_handle* out);

/* Builds the tree bottom-up from n key/value pairs in device memory (the RF /
 * tree construction step).  keys_dev must be strictly increasing,
 * inside [key_lo, key_hi) and != UINT64_MAX; vals_dev != UINT64_MAX.  leaf_fill
 * in (0, 1] sets the initial keys per leaf (round(16*fill)); it changes shape
 * and speed only (§8(c) reading 13).  Valid only on a freshly created tree
 * (ESTATE otherwise).  Synchronous with respect to `stream`; EINVAL if the
 * device check of the keys fails (tree left empty). */
int eirene_bulk_load(eirene_handle h, const eirene_key_t* keys_dev, const eirene_key_t* vals_dev,
                     uint64_t n, float leaf_fill, eirene_stream_t stream);

/* Submits one batch of n requests (Alg.1:1-7): ops_dev[n] (u8, EIRENE_*),
 * keys_dev[n], vals_dev[n] (ignored for queries and deletes) and writes
 * results_dev[n] (u64, timestamp = index order).  Asynchronous on `stream`;
 * the caller keeps every buffer alive until eirene_results(ticket) returns.
 * Pipeline: sort by (key, timestamp) (Alg.1:10) as a distribution into
 * balanced key-range groups + a per-group sort fused with combine/resolve
 * (Alg.1:11) and partition (Alg.1:3), query kernel (Alg.1:15-21),
 * update kernel with optimistic retry and STM fallback (Alg.1:23-46),
 * RESULT_CAL (Alg.1:6).
 * Synchronous errors: EINVAL (null pointers, n == 0 or n > max_batch), ESTATE.
 * Invalid requests (op > 3, key == UINT64_MAX or outside [key_lo, key_hi),
 * upsert value == UINT64_MAX) are detected on the device: the batch then
 * leaves the tree untouched and eirene_results reports EINVAL. */
int eirene_submit_batch(eirene_handle h, const uint8_t* ops_dev, const eirene_key_t* keys_dev,
                        const eirene_key_t* vals_dev, uint32_t n, eirene_key_t* results_dev,
                        eirene_stream_t stream, uint64_t* ticket);

/* Same batch from HOST buffers.  ops and keys are copied host->device into
 * handle-owned triple-buffered staging on the handle's copy stream (which
 * overlaps the previous batch's kernels); the pipeline runs on `stream`; the
 * results are copied device->host on the handle's d2h stream.  If vals_host is
 * pinned (page-locked, device-mapped under UVA) it is not copied: the
 * distribution kernel reads the values of the batch's upserts -- the only
 * values any kernel reads -- from host memory and stages them; pageable
 * values are copied.  The copies run at full speed only from pinned memory.
 * Results are valid after eirene_results(ticket); keep every buffer alive
 * until then. */
int eirene_submit_batch_host(eirene_handle h, const uint8_t* ops_host, const eirene_key_t* keys_host,
                             const eirene_key_t* vals_host, uint32_t n, eirene_key_t* results_host,
                             eirene_stream_t stream, uint64_t* ticket);

/* Same as eirene_submit_batch, and the batch may also hold range queries
 * (§4.1.2): ops_dev[i] == EIRENE_RANGE with
 * keys_dev[i] = l and vals_dev[i] = u asks for the pairs with l <= key <= u
 * (inclusive, any u64 bounds; l > u is empty) of the state visible
 * immediately before request i (linearizable), in ascending key
 * order, limited to the first `cap` pairs (reading R1).  They go to
 * range_keys_dev[i*cap + j] / range_vals_dev[i*cap + j] (caller-owned device
 * buffers of n*cap u64 each; rows of other requests are not touched) and
 * results_dev[i] = the number of pairs written (<= cap).  1 <= cap <= 4096.
 * Point requests behave exactly as in eirene_submit_batch.
 * Mechanism: range queries do not enter the sort; they read the pre-batch
 * tree in a range kernel between the query and update kernels (P:1066-1074:
 * range queries run in the query kernel's phase), and every key in [l, u]
 * that has update requests in the batch takes the result of an "artificial
 * query" at the range's timestamp, resolved by a binary search of
 * that key's timestamp-sorted segment.  Not accepted by the multi-GPU
 * routing (EINVAL there).  Errors as eirene_submit_batch, plus EINVAL for
 * cap == 0, cap > 4096 or null range buffers. */
int eirene_submit_batch_range(eirene_handle h, const uint8_t* ops_dev, const eirene_key_t* keys_dev,
                              const eirene_key_t* vals_dev, uint32_t n, eirene_key_t* results_dev,
                              uint32_t cap, eirene_key_t* range_keys_dev, eirene_key_t* range_vals_dev,
                              eirene_stream_t stream, uint64_t* ticket);

/* Optional warm-up: captures and instantiates the CUDA graph that batches of
 * exactly n requests (with_ranges != 0: submitted by eirene_submit_batch_range)
 * replay, without launching anything and without touching the tree, so that
 * the first such batch does not pay the capture.  A handle keeps graphs for a
 * few distinct sizes.  Errors: EINVAL (n == 0 or n > max_batch), ECUDA. */
int eirene_prepare_batch(eirene_handle h, uint32_t n, int with_ranges);

/* Makes `stream` wait (on the device, no host synchronisation) until batch
 * `ticket` has finished, so work enqueued on `stream` afterwards may consume
 * its results.  Needed with EIRENE_F_PIPELINE, where a batch ends on the
 * handle's back stream; a no-op ordering otherwise.  ESTATE for an unknown or
 * too old ticket. */
int eirene_stream_wait_batch(eirene_handle h, uint64_t ticket, eirene_stream_t stream);

/* Waits for batch `ticket` and returns its status (EIRENE_OK, EINVAL, EFULL);
 * fills *stats if non-NULL.  ESTATE if the ticket is unknown or too old (the
 * handle remembers the last 64 batches). */
int eirene_results(eirene_handle h, uint64_t ticket, eirene_batch_stats* stats);

/* In-order scan of the quiescent tree: pairs with lo <= key <= hi (inclusive,
 * §8(c) reading 23) in ascending key order.  Writes min(count, cap) pairs to
 * keys_out_dev / vals_out_dev (either may be NULL when cap == 0) and the total
 * to *count.  Synchronous with respect to `stream`.  Used for parity and as
 * the save half of save/restore (bulk_load is the restore half). */
int eirene_scan(eirene_handle h, uint64_t lo, uint64_t hi, eirene_key_t* keys_out_dev,
                eirene_key_t* vals_out_dev, uint64_t cap, uint64_t* count, eirene_stream_t stream);

/* Debug: copies the node pools to the host and checks the structural
 * invariants of the quiescent tree: keys strictly increasing in every node,
 * counts <= 16, children inside their parent's fences, uniform leaf depth,
 * leaf chain == in-order leaves, fences contiguous, no node locked.  Returns
 * 0 when they hold, else a positive code; *n_keys = keys in the tree. */
int eirene_check_invariants(eirene_handle h, uint64_t* n_keys);

typedef struct {
  uint32_t height;            /* 1 = the root is a leaf */
  uint32_t root;
  uint64_t leaves, inner;     /* allocated nodes */
  uint64_t leaf_cap, inner_cap;
  uint64_t launches;          /* kernels launched by this handle so far */
  uint64_t device_bytes;      /* device memory owned by the handle */
} eirene_tree_info;

/* Synchronous snapshot of the tree's size counters. */
int eirene_get_info(eirene_handle h, eirene_tree_info* info);

/* Replaces cfg.flags (EIRENE_F_*) for the batches submitted from now on, e.g.
 * to turn per-stage timing on for a diagnostic run.  Batches are normally
 * replayed from a captured CUDA graph; with EIRENE_F_TIMING the kernels are
 * launched directly so that stage events can be recorded between them. */
int eirene_set_flags(eirene_handle h, uint32_t flags);

/* Measurement helper (not part of the request path): launches one random-access
 * probe on `stream` over the caller's device buffer pool_dev[pool_bytes]
 * (256 B aligned, a power of two bytes): n accesses, kind 0 = uniformly random
 * 128 B line reads, 1 = random 32 B sector reads (a value sector), 2 = random
 * 32 B sector writes (an in-place value update), 3 = the query kernel's leaf
 * access: the 128 B key line of a 256 B leaf block then, dependent on it, one
 * 32 B sector of the block's value line, at a key-sorted batch's order and
 * density (access i visits block ~ i * blocks / n, ascending).  The caller
 * times it with events on `stream`; accesses/s are the denominators of the
 * random-access roofline of SURVEY §8(d) (BASELINE north_star).  Kind 2
 * overwrites pool contents.  EINVAL for a null / misaligned / non-power-of-two
 * pool or an unknown kind; ECUDA if the launch fails. */
int eirene_probe_gather(void* pool_dev, uint64_t pool_bytes, uint32_t n, int kind, uint64_t seed,
                        eirene_stream_t stream);

/* Diagnostic: copies min(n_words, 2*512*8) u64 %globaltimer stamps of the
 * last batch's distribution (kernel 0) and group (kernel 1) kernels,
 * [kernel][CTA][phase], to host memory `out` (synchronises the device).  Only
 * builds compiled with -DEIRENE_PHASE_PROF write them (tools/phase_prof.py);
 * otherwise the buffer stays zero. */
int eirene_debug_phases(eirene_handle h, uint64_t* out, uint32_t n_words);

/* Frees every device and host resource of the handle (waits for pending work). */
int eirene_destroy(eirene_handle h);

const char* eirene_strerror(int code);
/* Text of the last CUDA error seen by any handle in this process. */
const char* eirene_last_cuda_error(void);

/* ---- multi-GPU key-range routing; the collective itself is
 * torch.distributed all_to_all_single (NCCL) issued by the caller ----------- */

/* Stable partition of n requests by destination shard,
 * dest(k) = #{ s in splitters[0..P-2] : s <= k } (upper_bound), so shard r
 * owns [splitters[r-1], splitters[r]).  splitters_dev holds P-1 increasing
 * keys (device), 1 <= P <= 64.  Writes send_ops/keys/vals_dev[n] grouped by
 * destination in input (timestamp) order, perm_dev[n] (perm[j] = input index
 * of send slot j) and counts_dev[P] (u32).  If invalid_dev != NULL, the
 * request validation of eirene_submit_batch runs here too and sets
 * *invalid_dev = 1 (never clears it) when any request is invalid, so all
 * ranks can agree to reject the whole global batch before any shard applies
 * its part.  `h` provides scratch only.  Asynchronous on `stream`. */
int eirene_route_partition(eirene_handle h, const uint8_t* ops_dev, const uint64_t* keys_dev,
                           const uint64_t* vals_dev, uint32_t n, const uint64_t* splitters_dev,
                           int P, uint8_t* send_ops_dev, uint64_t* send_keys_dev,
                           uint64_t* send_vals_dev, uint32_t* perm_dev, uint32_t* counts_dev,
                           uint32_t* invalid_dev, eirene_stream_t stream);

/* The same partition for ONE payload exchange: each request becomes a 24 B
 * record {key, value, op} (three u64 words) in send_rec_dev[3n], grouped by
 * destination in timestamp order; perm_dev[n] as above; counts2_dev[2P] (u32)
 * holds, per destination d, counts2[2d] = requests for shard d and
 * counts2[2d+1] = 1 if ANY request of this slice is invalid (the validation
 * of eirene_submit_batch, always on), else 0 -- so a single all-to-all of
 * [P][2] words gives every rank the receive counts and every rank's validity
 * flag (the whole global batch is rejected if one is set; SURVEY §8(b),
 * §8(e)).  `h` provides scratch only.  Asynchronous on `stream`. */
int eirene_route_partition_packed(eirene_handle h, const uint8_t* ops_dev, const uint64_t* keys_dev,
                                  const uint64_t* vals_dev, uint32_t n, const uint64_t* splitters_dev,
                                  int P, uint64_t* send_rec_dev, uint32_t* perm_dev, uint32_t* counts2_dev,
                                  eirene_stream_t stream);

/* Receiver side of the packed exchange: splits n records recv_rec_dev[3n]
 * (the source ranks' segments concatenated in rank order = timestamp order)
 * into ops_out_dev[n], keys_out_dev[n], vals_out_dev[n] for
 * eirene_submit_batch.  Asynchronous on `stream`. */
int eirene_route_unpack(eirene_handle h, const uint64_t* recv_rec_dev, uint32_t n, uint8_t* ops_out_dev,
                        uint64_t* keys_out_dev, uint64_t* vals_out_dev, eirene_stream_t stream);

/* Enqueues on `stream` a copy of batch `ticket`'s final status (the value
 * eirene_results would return) into status_dev (one int32 in device memory),
 * without a host synchronisation: the multi-GPU layer all-reduces it so that
 * every rank agrees on the global batch's outcome (EFULL / EINTERNAL on one
 * shard fails the batch everywhere).  `stream` must be ordered after the
 * batch's stream.  ESTATE for an unknown or too old ticket. */
int eirene_batch_status_async(eirene_handle h, uint64_t ticket, int32_t* status_dev, eirene_stream_t stream);

/* Inverse of the partition for the returned results:
 * results_dev[perm_dev[j]] = recv_results_dev[j] for j < n.  Asynchronous. */
int eirene_route_unpermute(eirene_handle h, const uint64_t* recv_results_dev,
                           const uint32_t* perm_dev, uint32_t n, uint64_t* results_dev,
                           eirene_stream_t stream);

/* ---- fused routing over peer memory (one-shot NVLink
 * push fusing route_partition with the exchange; §8(e) steps 2-8).  Each rank
 * owns a receive ARENA in device memory: P source slots {count, invalid flag,
 * start, epoch} (u32 x4), cap result words (this rank's slice, partition
 * order) and P x cap 24 B records.  The partition kernel stores every request
 * directly into its destination's arena (peer memory over NVLink 5 /
 * NVSwitch, mapped by CUDA IPC; in one process, any device pointers), so no
 * payload collective runs: the caller only orders the ranks with a barrier
 * (e.g. a one-word NCCL all_reduce on the same stream) after eirene_route_push
 * and after eirene_route_push_results.  Every rank calls every function for
 * every global batch in the same order, with the same P and cap. ---------- */
#define EIRENE_IPC_HANDLE_BYTES 64

/* Allocates this rank's arena for P ranks (1 <= P <= 64), rank `rank`, at
 * most `cap` requests per rank slice (the source's n of eirene_route_push).
 * *arena_dev_out = its device address; if ipc_handle_out != NULL it receives
 * EIRENE_IPC_HANDLE_BYTES of CUDA IPC handle for the other processes.  Freed
 * by eirene_destroy.  ESTATE if the handle already has an arena. */
int eirene_route_arena_create(eirene_handle h, int P, int rank, uint32_t cap, void** arena_dev_out,
                              void* ipc_handle_out);
/* Maps a peer process's arena (its IPC handle) into this process:
 * *arena_dev_out = the address to pass to eirene_route_arena_connect.
 * Unmapped by eirene_destroy. */
int eirene_route_arena_open_ipc(eirene_handle h, const void* ipc_handle, void** arena_dev_out);
/* peer_arenas (host array of P device addresses; entry `rank` = this rank's own
 * arena): the destinations of the pushes.  Synchronous. */
int eirene_route_arena_connect(eirene_handle h, void* const* peer_arenas);
/* Source side (steps 2+4 fused): the stable partition of eirene_route_partition
 * (dest = upper_bound(splitters, key), perm_dev[n] as there, validation of
 * eirene_submit_batch) whose scatter stores each request as a {key, value, op}
 * record into arena(dest).rec[rank][j], j its index among this slice's
 * requests for dest (timestamp order); then every destination's slot [rank]
 * gets {count, invalid, start of dest's segment in perm order, epoch}.
 * n <= cap.  Asynchronous on `stream`; the pushes are complete (system-scope
 * fenced) when the stream reaches its end. */
int eirene_route_push(eirene_handle h, const uint8_t* ops_dev, const uint64_t* keys_dev, const uint64_t* vals_dev,
                      uint32_t n, const uint64_t* splitters_dev, uint32_t* perm_dev, eirene_stream_t stream);
/* Receiver side, after the barrier that follows every rank's push: reads the
 * P slots (ONE host synchronisation of `stream`), sets *n_out = requests
 * received and *invalid_out = 1 if any source's slice holds an invalid request
 * (then nothing is written: every rank sees the same flags, so all reject the
 * global batch), else compacts the records in source-rank order (= timestamp
 * order) into ops/keys/vals_out[*n_out] (n_cap entries
 * available) for eirene_submit_batch.  EINTERNAL if a source's slot does not
 * carry this batch's epoch (its push never arrived). */
int eirene_route_pull(eirene_handle h, uint8_t* ops_out_dev, uint64_t* keys_out_dev, uint64_t* vals_out_dev,
                      uint32_t n_cap, uint32_t* n_out, uint32_t* invalid_out, eirene_stream_t stream);
/* Receiver side: the shard's results_dev[*n_out of the last pull] (pulled
 * order) stored back into every source's arena at its partition positions
 * (step 7).  Asynchronous; the caller's barrier must follow it. */
int eirene_route_push_results(eirene_handle h, const uint64_t* results_dev, eirene_stream_t stream);
/* Source side, after that barrier: results_dev[perm_dev[j]] = arena.res[j] for
 * j < n (step 8).  Asynchronous. */
int eirene_route_unpermute_arena(eirene_handle h, const uint32_t* perm_dev, uint32_t n, uint64_t* results_dev,
                                 eirene_stream_t stream);

#ifdef __cplusplus
}
#endif
#endif /* EIRENE_H */
