/*
 * eirene_oracle.h -- CPU oracle for the Eirene batched B+tree path.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and
 * bench.py's cpu_baseline / --impl reference legs may load this library.
 * It shares no code, header, table or helper with the CUDA path
 * (paper_conf_ppopp_zhangz0lzl23_b200/csrc, include/eirene.h).
 *
 * Citations: P:N = /root/reference/PAPER.md line N; Alg.1:k = line k of
 * Algorithm 1; SURVEY §8(c) = the readings taken where the
 * paper is silent.
 *
 * Three engines, all applying a batch of requests (op, key, val) whose
 * logical timestamp is the index in the batch:
 *
 *  (i)   orc_map_*  : the PLAIN DEFINITION: a std::map applied
 *                     sequentially in timestamp order; every request returns
 *                     the value visible immediately before it, NOT_FOUND if
 *                     absent.  UPDATE == INSERT == blind upsert, DELETE == erase.
 *                     Linearizability per P:505-517 and the proof sketch
 *                     P:1527-1577 make this the result the method must reach.
 *  (ii)  orc_bt_*   : a textbook sequential B+tree (fanout F, split on
 *                     overflow, borrow/merge on underflow) applying the same
 *                     definition; checked against (i) and by invariants.
 *                     This is the timed CPU baseline.
 *  (iii) orc_comb_* : the method itself, step by step in Algorithm 1's order
 *                     (sort, combine, partition, query, update, result_cal,
 *                     P:1117-1194 with the issue rule of P:724-758) on top of
 *                     engine (i); exposes the intermediates (issued set per
 *                     segment) the GPU path's combine step must reproduce.
 *
 * Parity status: (i) pinned by the Fig.3 worked example,
 * special cases that reduce to library routines (query-only == lower_bound
 * over the loaded arrays; distinct upserts == merge-with-overwrite) and
 * metamorphic invariants; (ii) pinned against (i) + invariants; (iii)
 * pinned against (i) and the Fig.3 issued set.  Throughput numbers are
 * parity-unpinned vs the paper (different hardware and record width).
 */
#ifndef EIRENE_ORACLE_H
#define EIRENE_ORACLE_H
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define ORC_NOT_FOUND UINT64_MAX
enum { ORC_QUERY = 0, ORC_UPDATE = 1, ORC_INSERT = 2, ORC_DELETE = 3, ORC_RANGE = 4 };

/* ---- engine (i): std::map definition ---- */
void*    orc_map_new(void);
void     orc_map_free(void* h);
/* keys strictly increasing; returns 0 or -1 on bad input */
int      orc_map_load(void* h, const uint64_t* keys, const uint64_t* vals, uint64_t n);
/* results[i] = value visible just before request i (NOT_FOUND if absent) */
int      orc_map_apply(void* h, const uint8_t* ops, const uint64_t* keys,
                       const uint64_t* vals, uint64_t n, uint64_t* results);
uint64_t orc_map_size(void* h);
/* inclusive [lo, hi], ascending; writes min(count, cap) pairs, returns count */
uint64_t orc_map_scan(void* h, uint64_t lo, uint64_t hi, uint64_t* keys_out,
                      uint64_t* vals_out, uint64_t cap);

/* ---- engine (ii): sequential B+tree, fanout 3..64 ---- */
void*    orc_bt_new(int fanout);
void     orc_bt_free(void* h);
int      orc_bt_load(void* h, const uint64_t* keys, const uint64_t* vals, uint64_t n);
int      orc_bt_apply(void* h, const uint8_t* ops, const uint64_t* keys,
                      const uint64_t* vals, uint64_t n, uint64_t* results);
uint64_t orc_bt_size(void* h);
uint64_t orc_bt_scan(void* h, uint64_t lo, uint64_t hi, uint64_t* keys_out,
                     uint64_t* vals_out, uint64_t cap);
/* 0 if every invariant holds, else a positive code naming the first violation */
int      orc_bt_check(void* h);
int      orc_bt_height(void* h);
/* test hook: corrupt the tree in a way `kind` names, so the checker can be pinned */
int      orc_bt_corrupt(void* h, int kind);

/* ---- engine (iii): Algorithm 1 step by step, state in engine (i) ----
 * Outputs (all optional, may be NULL):
 *   sorted_ts[n]      : the stable sort of timestamps by key (Alg.1:10)
 *   seg_of_sorted[n]  : segment (distinct-key) index of each sorted position
 *   issued_key/op/val[m], m = number of segments: the request issued for each
 *                       segment (all-query -> last query; any
 *                       write -> last write); val is NOT_FOUND for queries and deletes
 *   n_issued          : m
 *   n_issued_w        : number of issued writes
 */
int      orc_comb_apply(void* map_h, const uint8_t* ops, const uint64_t* keys,
                        const uint64_t* vals, uint64_t n, uint64_t* results,
                        uint32_t* sorted_ts, uint32_t* seg_of_sorted,
                        uint64_t* issued_key, uint8_t* issued_op, uint64_t* issued_val,
                        uint64_t* n_issued, uint64_t* n_issued_w);

/* ---- range queries R(l, u) ----
 * A batch may hold ORC_RANGE requests: key = lower bound l, val = upper
 * bound u, both inclusive (§8(c) reading 23).  The result of range request i
 * is the set of pairs (k, v) of the state visible immediately before i
 * (linearizability) with l <= k <= u, in ascending key order,
 * limited to its first `cap` pairs (reading R1): results[i] = the
 * number of pairs written, the pairs go to rkeys[i*cap + j], rvals[i*cap + j].
 * l > u is an empty range.  Point requests are as in *_apply.
 *   orc_map_apply_range  : engine (i), the plain definition.
 *   orc_bt_apply_range   : engine (ii), leaf-chain walk of the B+tree.
 *   orc_comb_apply_range : engine (iii), the paper's mechanism step by step:
 *     sort with range queries placed by their lower bound; scan;
 *     an artificial query Qr(k)@t for every key k in [l, u] that has update
 *     requests in the batch, inserted into k's sequence by timestamp
 *     (P:925-935); combine / partition / query / update / RESULT_CAL as
 *     Alg.1 with the range query in the query kernel reading the tree "in
 *     the original manner"; then every key with an artificial query
 *     takes that query's result (NOT_FOUND removes it, a value
 *     adds or replaces it).  *n_artificial = artificial queries generated. */
int      orc_map_apply_range(void* h, const uint8_t* ops, const uint64_t* keys,
                             const uint64_t* vals, uint64_t n, uint64_t* results,
                             uint32_t cap, uint64_t* rkeys, uint64_t* rvals);
int      orc_bt_apply_range(void* h, const uint8_t* ops, const uint64_t* keys,
                            const uint64_t* vals, uint64_t n, uint64_t* results,
                            uint32_t cap, uint64_t* rkeys, uint64_t* rvals);
int      orc_comb_apply_range(void* map_h, const uint8_t* ops, const uint64_t* keys,
                              const uint64_t* vals, uint64_t n, uint64_t* results,
                              uint32_t cap, uint64_t* rkeys, uint64_t* rvals,
                              uint64_t* n_artificial);

#ifdef __cplusplus
}
#endif
#endif
