// route.cu -- key-range routing for the multi-GPU mode.
//
// Each rank owns the contiguous timestamp slice r of the global batch; a request
// goes to shard dest(k) = #{splitters <= k}.  The stable partition keeps each
// destination's requests in timestamp order, so after the all-to-all (NCCL,
// issued by the caller) the receiver's concatenation in source-rank order is
// timestamp-ordered and the per-shard stable sort preserves linearizability
// (§8(c) reading 7; per-key locality of linearizability, P:2487-2492 / [17]).
// Same single-pass-per-digit design as sort.cu with <= 64 destinations.
#include "eirene_internal.cuh"

namespace eirene {

namespace {

constexpr int RT_THREADS = 256;
constexpr int RT_ITEMS = 8;
constexpr int RT_TILE = RT_THREADS * RT_ITEMS;
constexpr int RT_MAXP = 64;
constexpr int RT_WARPS = RT_THREADS / 32;
constexpr unsigned long long LB_AGG = 1ull << 30;
constexpr unsigned long long LB_INC = 2ull << 30;
constexpr unsigned long long LB_VAL = (1ull << 30) - 1;

__device__ __forceinline__ uint32_t dest_of(uint64_t k, const uint64_t* sp, int P) {
  uint32_t d = 0;
  for (int i = 0; i < P - 1; ++i) d += (sp[i] <= k) ? 1u : 0u;
  return d;
}

__global__ void __launch_bounds__(RT_THREADS) route_count_kernel(const uint64_t* __restrict__ keys,
                                                                 const uint8_t* __restrict__ ops,
                                                                 const uint64_t* __restrict__ vals, uint32_t n,
                                                                 const uint64_t* __restrict__ splitters, int P,
                                                                 uint32_t* __restrict__ counts, uint32_t cstride,
                                                                 uint32_t* __restrict__ invalid) {
  __shared__ uint64_t sp[RT_MAXP];
  __shared__ uint32_t h[RT_MAXP];
  const int tid = threadIdx.x;
  if (tid < RT_MAXP) {
    sp[tid] = tid < P - 1 ? splitters[tid] : KEY_MAX;
    h[tid] = 0;
  }
  __syncthreads();
  bool bad = false;
  for (uint32_t i = blockIdx.x * RT_THREADS + tid; i < n; i += gridDim.x * RT_THREADS) {
    const uint64_t k = keys[i];
    atomicAdd(&h[dest_of(k, sp, P)], 1u);
    if (invalid) {
      const uint32_t o = ops[i];
      const bool up = (o == OP_UPDATE || o == OP_INSERT);
      bad |= o > OP_DELETE || k == KEY_MAX || (up && vals[i] == KEY_MAX);
    }
  }
  if (__any_sync(FULL, bad) && (tid & 31) == 0) atomicOr(invalid, 1u);
  __syncthreads();
  if (tid < P && h[tid]) atomicAdd(&counts[tid * cstride], h[tid]);
}

struct RtSmem {
  uint64_t keys[RT_TILE];
  uint64_t vals[RT_TILE];
  uint32_t idx[RT_TILE];
  uint8_t ops[RT_TILE];
  uint64_t sp[RT_MAXP];
  uint32_t wh[RT_WARPS][RT_MAXP];
  uint32_t tile_off[RT_MAXP];
  uint32_t cnt[RT_MAXP];
  uint32_t bin_base[RT_MAXP];
  uint32_t bin_start[RT_MAXP];
  uint64_t* prec[RT_MAXP];   // fused push: destination d's receive arena records (peer memory)
  uint32_t tile_id;
};

__global__ void __launch_bounds__(RT_THREADS) route_scatter_kernel(
    const uint8_t* __restrict__ ops, const uint64_t* __restrict__ keys, const uint64_t* __restrict__ vals, uint32_t n,
    const uint64_t* __restrict__ splitters, int P, uint32_t* __restrict__ counts, uint32_t cstride,
    const uint32_t* __restrict__ invalid, uint8_t* __restrict__ sops, uint64_t* __restrict__ skeys,
    uint64_t* __restrict__ svals, uint64_t* __restrict__ rec, uint32_t* __restrict__ perm,
    unsigned long long* __restrict__ lookback, uint32_t epoch, uint32_t* __restrict__ tile_ctr,
    uint64_t* const* __restrict__ peer_rec, uint32_t me, uint32_t cap) {
  extern __shared__ __align__(16) unsigned char smem_raw[];
  RtSmem& S = *reinterpret_cast<RtSmem*>(smem_raw);
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  if (tid == 0) {
    S.tile_id = atomicAdd(tile_ctr, 1u);
    uint32_t run = 0;
    for (int d = 0; d < P; ++d) {
      S.bin_start[d] = run;
      run += counts[d * cstride];
    }
  }
  for (int i = tid; i < RT_WARPS * RT_MAXP; i += RT_THREADS) (&S.wh[0][0])[i] = 0;
  if (tid < RT_MAXP) S.sp[tid] = tid < P - 1 ? splitters[tid] : KEY_MAX;
  if (peer_rec && tid < P) S.prec[tid] = peer_rec[tid];
  __syncthreads();
  const uint32_t tile = S.tile_id, base = tile * RT_TILE;
  // packed mode: every destination's count word is followed by the batch's
  // validity flag (final: route_count_kernel ran before this kernel), so ONE
  // exchange of [P][2] words tells every rank the counts and whether the
  // global batch is rejected
  if (cstride == 2 && tile == 0 && tid < P) counts[2 * tid + 1] = invalid ? *invalid : 0u;
  const uint32_t wbase = base + warp * (RT_ITEMS * 32);
  uint64_t k[RT_ITEMS];
  uint32_t d[RT_ITEMS], r[RT_ITEMS];
#pragma unroll
  for (int j = 0; j < RT_ITEMS; ++j) {
    const uint32_t i = wbase + j * 32 + lane;
    const bool act = i < n;
    k[j] = act ? keys[i] : 0;
    d[j] = act ? dest_of(k[j], S.sp, P) : RT_MAXP;
    const uint32_t peers = __match_any_sync(FULL, d[j]);
    const uint32_t before = act ? S.wh[warp][d[j]] : 0;
    r[j] = before + __popc(peers & lanemask_lt());
    __syncwarp();
    if (act && lane == 31 - __clz(peers)) S.wh[warp][d[j]] = before + __popc(peers);
    __syncwarp();
  }
  __syncthreads();
  if (tid < RT_MAXP) {
    uint32_t run = 0;
    for (int w = 0; w < RT_WARPS; ++w) {
      const uint32_t c = S.wh[w][tid];
      S.wh[w][tid] = run;
      run += c;
    }
    S.cnt[tid] = run;
  }
  __syncthreads();
  if (tid == 0) {
    uint32_t run = 0;
    for (int dd = 0; dd < RT_MAXP; ++dd) {
      S.tile_off[dd] = run;
      run += S.cnt[dd];
    }
  }
  __syncthreads();
  if (tid < P) {
    const uint32_t cnt_ok = S.cnt[tid];
    unsigned long long* my = lookback + (size_t)tile * RT_MAXP + tid;
    const unsigned long long ep = (unsigned long long)epoch << 32;
    uint32_t excl = 0;
    if (tile == 0) {
      st_relaxed64(my, ep | LB_INC | cnt_ok);
    } else {
      st_relaxed64(my, ep | LB_AGG | cnt_ok);
      SpinGuard sg;
      int32_t pt = (int32_t)tile - 1;
      while (pt >= 0) {
        const unsigned long long w = ld_relaxed64(lookback + (size_t)pt * RT_MAXP + tid);
        if ((w >> 32) != epoch || (w & (3ull << 30)) == 0) {
          if (sg.stuck(nullptr)) break;
          continue;
        }
        excl += (uint32_t)(w & LB_VAL);
        if (w & LB_INC) break;
        --pt;
      }
      st_relaxed64(my, ep | LB_INC | (excl + cnt_ok));
    }
    S.bin_base[tid] = S.bin_start[tid] + excl - S.tile_off[tid];
  }
  __syncthreads();
#pragma unroll
  for (int j = 0; j < RT_ITEMS; ++j) {
    const uint32_t i = wbase + j * 32 + lane;
    if (i < n) {
      const uint32_t pos = S.tile_off[d[j]] + S.wh[warp][d[j]] + r[j];
      S.keys[pos] = k[j];
      S.vals[pos] = vals[i];
      S.ops[pos] = ops[i];
      S.idx[pos] = i;
    }
  }
  __syncthreads();
  const uint32_t tile_n = min((uint32_t)RT_TILE, n - base);
  for (uint32_t i = tid; i < tile_n; i += RT_THREADS) {
    const uint64_t key = S.keys[i];
    const uint32_t d = dest_of(key, S.sp, P);
    const uint32_t o = S.bin_base[d] + i;
    if (peer_rec) {   // fused push: straight into destination d's arena, region of source `me`
      uint64_t* dst = S.prec[d] + 3 * ((size_t)me * cap + (o - S.bin_start[d]));
      dst[0] = key;
      dst[1] = S.vals[i];
      dst[2] = S.ops[i];
    } else if (rec) {   // one 24 B record {key, value, op} per request: one payload exchange
      rec[3 * (size_t)o] = key;
      rec[3 * (size_t)o + 1] = S.vals[i];
      rec[3 * (size_t)o + 2] = S.ops[i];
    } else {
      skeys[o] = key;
      svals[o] = S.vals[i];
      sops[o] = S.ops[i];
    }
    perm[o] = S.idx[i];
  }
  // (the records must be visible to the peer once this kernel is complete: the
  // caller's barrier -- an NCCL collective on the same stream -- follows it)
  if (peer_rec) __threadfence_system();
}

// Fused push, after the scatter: source `me` tells every destination d how
// many records it pushed, whether its slice holds an invalid request, where
// d's segment starts in its own partition order (the results come back
// there) and the batch epoch, in d's arena slot [me]: {count, invalid,
// start, epoch}.  Written for every d (also count 0), so a receiver always
// hears from every source.
__global__ void push_counts_kernel(const uint32_t* __restrict__ counts, const uint32_t* __restrict__ invalid, int P,
                                   uint32_t me, uint32_t* const* __restrict__ peer_cnt, uint32_t epoch) {
  const int d = threadIdx.x;
  if (d < P) {
    uint32_t start = 0;
    for (int x = 0; x < d; ++x) start += counts[x];
    uint4* dst = reinterpret_cast<uint4*>(peer_cnt[d]) + me;
    *dst = make_uint4(counts[d], invalid ? *invalid : 0u, start, epoch);
    __threadfence_system();
  }
}

// Receiver: the P sources' records in its arena, rx_rec[src][0, cnt_src),
// compacted in source-rank (= timestamp) order into the shard's SoA batch.
__global__ void pull_unpack_kernel(const uint4* __restrict__ cnt, const uint64_t* __restrict__ rec, uint32_t cap,
                                   uint8_t* __restrict__ ops, uint64_t* __restrict__ keys,
                                   uint64_t* __restrict__ vals) {
  const uint32_t src = blockIdx.y;
  uint32_t off = 0;
  for (uint32_t x = 0; x < src; ++x) off += cnt[x].x;
  const uint32_t c = cnt[src].x;
  const uint64_t* r = rec + 3 * (size_t)src * cap;
  for (uint32_t j = blockIdx.x * blockDim.x + threadIdx.x; j < c; j += gridDim.x * blockDim.x) {
    keys[off + j] = r[3 * (size_t)j];
    vals[off + j] = r[3 * (size_t)j + 1];
    ops[off + j] = (uint8_t)r[3 * (size_t)j + 2];
  }
}

// Receiver: the shard's results (source-rank order) pushed back into every
// source's arena at the position its partition gave them (start_src + j).
__global__ void push_results_kernel(const uint4* __restrict__ cnt, const uint64_t* __restrict__ res,
                                    uint64_t* const* __restrict__ peer_res) {
  const uint32_t src = blockIdx.y;
  uint32_t off = 0;
  for (uint32_t x = 0; x < src; ++x) off += cnt[x].x;
  const uint4 e = cnt[src];
  uint64_t* dst = peer_res[src] + e.z;
  for (uint32_t j = blockIdx.x * blockDim.x + threadIdx.x; j < e.x; j += gridDim.x * blockDim.x)
    dst[j] = res[off + j];
  __threadfence_system();
}

__global__ void unpermute_kernel(const uint64_t* __restrict__ recv, const uint32_t* __restrict__ perm, uint32_t n,
                                 uint64_t* __restrict__ out) {
  for (uint32_t j = blockIdx.x * blockDim.x + threadIdx.x; j < n; j += gridDim.x * blockDim.x) out[perm[j]] = recv[j];
}

__global__ void unpack_kernel(const uint64_t* __restrict__ rec, uint32_t n, uint8_t* __restrict__ ops,
                              uint64_t* __restrict__ keys, uint64_t* __restrict__ vals) {
  for (uint32_t j = blockIdx.x * blockDim.x + threadIdx.x; j < n; j += gridDim.x * blockDim.x) {
    keys[j] = rec[3 * (size_t)j];
    vals[j] = rec[3 * (size_t)j + 1];
    ops[j] = (uint8_t)rec[3 * (size_t)j + 2];
  }
}

}  // namespace

void launch_route_unpack(const uint64_t* rec, uint32_t n, uint8_t* ops, uint64_t* keys, uint64_t* vals,
                         cudaStream_t st, int* launches) {
  if (n == 0) return;
  int blocks = (int)std::min<uint32_t>((n + 255) / 256, 148u * 8u);
  unpack_kernel<<<blocks, 256, 0, st>>>(rec, n, ops, keys, vals);
  ++*launches;
}

void launch_route_partition(const uint8_t* ops, const uint64_t* keys, const uint64_t* vals, uint32_t n,
                            const uint64_t* splitters, int P, uint8_t* sops, uint64_t* skeys, uint64_t* svals,
                            uint64_t* rec, uint32_t* perm, uint32_t* counts, uint32_t cstride, uint32_t* invalid,
                            unsigned long long* lookback, uint32_t* tile_ctr, uint32_t epoch, cudaStream_t st,
                            int* launches, uint64_t* const* peer_rec, uint32_t me, uint32_t cap) {
  static int attr[MAX_DEVICES];
  per_device(attr, [] {
    return (int)cudaFuncSetAttribute(route_scatter_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                     (int)sizeof(RtSmem));
  });
  cudaMemsetAsync(counts, 0, sizeof(uint32_t) * P * cstride, st);
  cudaMemsetAsync(tile_ctr, 0, sizeof(uint32_t), st);
  if (n == 0) return;
  int blocks = (int)std::min<uint32_t>((n + RT_THREADS * 8 - 1) / (RT_THREADS * 8), 148u * 4u);
  route_count_kernel<<<blocks, RT_THREADS, 0, st>>>(keys, ops, vals, n, splitters, P, counts, cstride, invalid);
  const uint32_t tiles = (n + RT_TILE - 1) / RT_TILE;
  route_scatter_kernel<<<tiles, RT_THREADS, sizeof(RtSmem), st>>>(ops, keys, vals, n, splitters, P, counts, cstride,
                                                                  invalid, sops, skeys, svals, rec, perm, lookback,
                                                                  epoch, tile_ctr, peer_rec, me, cap);
  *launches += 2;
}

void launch_push_counts(const uint32_t* counts, const uint32_t* invalid, int P, uint32_t me, uint32_t* const* peer_cnt,
                        uint32_t epoch, cudaStream_t st, int* launches) {
  push_counts_kernel<<<1, 64, 0, st>>>(counts, invalid, P, me, peer_cnt, epoch);
  ++*launches;
}

void launch_pull_unpack(const uint32_t* cnt, const uint64_t* rec, uint32_t cap, int P, uint32_t max_per_src,
                        uint8_t* ops, uint64_t* keys, uint64_t* vals, cudaStream_t st, int* launches) {
  if (max_per_src == 0) return;
  const dim3 grid(std::max(1u, std::min<uint32_t>((max_per_src + 255) / 256, 148u * 8u / (uint32_t)P)), P);
  pull_unpack_kernel<<<grid, 256, 0, st>>>(reinterpret_cast<const uint4*>(cnt), rec, cap, ops, keys, vals);
  ++*launches;
}

void launch_push_results(const uint32_t* cnt, const uint64_t* res, int P, uint32_t max_per_src,
                         uint64_t* const* peer_res, cudaStream_t st, int* launches) {
  if (max_per_src == 0) return;
  const dim3 grid(std::max(1u, std::min<uint32_t>((max_per_src + 255) / 256, 148u * 8u / (uint32_t)P)), P);
  push_results_kernel<<<grid, 256, 0, st>>>(reinterpret_cast<const uint4*>(cnt), res, peer_res);
  ++*launches;
}

void launch_route_unpermute(const uint64_t* recv, const uint32_t* perm, uint32_t n, uint64_t* results,
                            cudaStream_t st, int* launches) {
  if (n == 0) return;
  int blocks = (int)std::min<uint32_t>((n + 255) / 256, 148u * 8u);
  unpermute_kernel<<<blocks, 256, 0, st>>>(recv, perm, n, results);
  ++*launches;
}

}  // namespace eirene
