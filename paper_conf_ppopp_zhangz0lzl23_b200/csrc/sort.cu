// sort.cu -- stable one-key LSD radix sort of (u64 key, u32 payload), sm_100a.
//
// Alg.1:10 / P:706-716: requests are sorted by target key and, within a key,
// by logical timestamp.  Requests arrive in timestamp order, so a
// STABLE sort on the key alone produces the (key, timestamp) order (SURVEY
// §8(c) reading 8).  The payload carries ts<<2 | op.
//
// Design (B200): "onesweep"-style single-pass-per-digit LSD
// sort, 8 passes of 8 bits.  Each pass kernel takes a 4096-element tile
// (dynamic tile id, so predecessor tiles are always resident), ranks the tile
// stably with warp __match_any_sync, publishes per-digit tile counts for a
// decoupled look-back across tiles, stages the tile in shared memory in digit
// order and writes it out with coalesced runs.  The global digit histogram the
// pass needs is accumulated by the PREVIOUS pass (digit p+1 counted while the
// keys of pass p are in registers), so only digit 0 needs a separate upsweep,
// fused with request validation.  At n = 2^20 the 12 MiB of (key, payload)
// ping-pong traffic stays L2-resident (126 MB L2).
#include "eirene_internal.cuh"

namespace eirene {

namespace {

constexpr int RADIX = 256;
constexpr int NWARPS = SORT_THREADS / 32;
constexpr unsigned long long LB_AGG = 1ull << 30;
constexpr unsigned long long LB_INC = 2ull << 30;
constexpr unsigned long long LB_VAL = (1ull << 30) - 1;

__device__ __forceinline__ uint32_t digit_of(uint64_t k, int shift) { return (uint32_t)(k >> shift) & 0xFF; }

// Histogram of digit 0 (+ request validation, SURVEY §8(b) "Errors").
__global__ void __launch_bounds__(SORT_THREADS) sort_upsweep_kernel(const uint64_t* __restrict__ keys,
                                                                   const uint8_t* __restrict__ ops,
                                                                   const uint64_t* __restrict__ vals, uint32_t n,
                                                                   uint64_t key_lo, uint64_t key_hi,
                                                                   uint32_t* __restrict__ ghist0,
                                                                   BatchCtl* __restrict__ ctl) {
  __shared__ uint32_t wh[NWARPS][RADIX];
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  for (int i = tid; i < NWARPS * RADIX; i += SORT_THREADS) (&wh[0][0])[i] = 0;
  __syncthreads();
  bool bad = false;
  const uint32_t stride = gridDim.x * SORT_THREADS;
  for (uint32_t base = blockIdx.x * SORT_THREADS; base < n; base += stride) {
    uint32_t i = base + tid;
    bool act = i < n;
    uint64_t k = act ? keys[i] : 0;
    uint32_t d = act ? digit_of(k, 0) : RADIX;  // inactive lanes form their own group
    uint32_t peers = __match_any_sync(FULL, d);
    if (act && lane == 31 - __clz(peers)) wh[warp][d] += __popc(peers);
    __syncwarp();
    if (act && ops) {
      uint32_t o = ops[i];
      bool up = (o == OP_UPDATE || o == OP_INSERT);
      bad |= o > OP_DELETE || k == KEY_MAX || k < key_lo || k >= key_hi || (up && vals[i] == KEY_MAX);
    }
  }
  if (__any_sync(FULL, bad) && lane == 0) atomicOr(&ctl->invalid, 1u);
  __syncthreads();
  for (int d = tid; d < RADIX; d += SORT_THREADS) {
    uint32_t s = 0;
    for (int w = 0; w < NWARPS; ++w) s += wh[w][d];
    if (s) atomicAdd(&ghist0[d], s);
  }
}

struct PassSmem {
  uint64_t keys[SORT_TILE];
  uint32_t pay[SORT_TILE];
  uint32_t wh[NWARPS][RADIX];    // ranking digit: per-warp counts -> per-warp exclusive offsets
  uint32_t wh2[NWARPS][RADIX];   // next digit: per-warp counts
  uint32_t tile_off[RADIX];      // exclusive offset of each digit inside the tile
  uint32_t bin_base[RADIX];      // global position of tile-local sorted index 0 for each digit
  uint32_t bin_start[RADIX];     // exclusive scan of the global digit histogram
  uint32_t tile_id;
  uint32_t scan_tmp[NWARPS];
};

// 256-thread exclusive scan of one value per thread.
__device__ __forceinline__ uint32_t block_excl_scan(uint32_t v, uint32_t* tmp, uint32_t* total) {
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
  for (int w = 0; w < NWARPS; ++w) {
    uint32_t t = tmp[w];
    if (w < warp) wpre += t;
    tot += t;
  }
  __syncthreads();
  *total = tot;
  return wpre + x - v;
}

__global__ void __launch_bounds__(SORT_THREADS) sort_pass_kernel(
    const uint64_t* __restrict__ kin, const uint32_t* __restrict__ pin, const uint8_t* __restrict__ ops0,
    uint64_t* __restrict__ kout, uint32_t* __restrict__ pout, uint32_t n, int shift, int next_shift,
    const uint32_t* __restrict__ ghist, uint32_t* __restrict__ ghist_next, unsigned long long* __restrict__ lookback,
    uint32_t epoch, uint32_t* __restrict__ tile_ctr, BatchCtl* __restrict__ ctl) {
  extern __shared__ __align__(16) unsigned char smem_raw[];
  PassSmem& S = *reinterpret_cast<PassSmem*>(smem_raw);
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  if (ctl && ctl->invalid) return;

  if (tid == 0) S.tile_id = atomicAdd(tile_ctr, 1u);
  for (int i = tid; i < NWARPS * RADIX; i += SORT_THREADS) {
    (&S.wh[0][0])[i] = 0;
    (&S.wh2[0][0])[i] = 0;
  }
  // global bin starts for this digit
  {
    uint32_t tot;
    uint32_t ex = block_excl_scan(ghist[tid], S.scan_tmp, &tot);
    S.bin_start[tid] = ex;
  }
  __syncthreads();
  const uint32_t tile = S.tile_id;
  const uint32_t base = tile * SORT_TILE;
  const uint32_t wbase = base + warp * (SORT_ITEMS * 32);

  uint64_t k[SORT_ITEMS];
  uint32_t p[SORT_ITEMS];
  uint32_t r[SORT_ITEMS];
#pragma unroll
  for (int j = 0; j < SORT_ITEMS; ++j) {
    uint32_t idx = wbase + j * 32 + lane;
    bool act = idx < n;
    k[j] = act ? kin[idx] : KEY_MAX;
    if (ops0)
      p[j] = act ? ((idx << 2) | (uint32_t)ops0[idx]) : 0;
    else
      p[j] = act ? pin[idx] : 0;
  }
  // stable warp-local ranking (items in index order: j-major, lane-minor)
#pragma unroll
  for (int j = 0; j < SORT_ITEMS; ++j) {
    uint32_t idx = wbase + j * 32 + lane;
    bool act = idx < n;
    uint32_t d = act ? digit_of(k[j], shift) : RADIX;
    uint32_t peers = __match_any_sync(FULL, d);
    uint32_t before = act ? S.wh[warp][d] : 0;
    r[j] = before + __popc(peers & lanemask_lt());
    __syncwarp();
    if (act && lane == 31 - __clz(peers)) S.wh[warp][d] = before + __popc(peers);
    if (ghist_next) {
      uint32_t d2 = act ? digit_of(k[j], next_shift) : RADIX;
      uint32_t peers2 = __match_any_sync(FULL, d2);
      if (act && lane == 31 - __clz(peers2)) S.wh2[warp][d2] += __popc(peers2);
    }
    __syncwarp();
  }
  __syncthreads();
  // per digit (thread tid == digit): warp exclusive offsets, tile count
  uint32_t cnt = 0;
  {
    const int d = tid;
    uint32_t run = 0;
#pragma unroll
    for (int w = 0; w < NWARPS; ++w) {
      uint32_t c = S.wh[w][d];
      S.wh[w][d] = run;
      run += c;
    }
    cnt = run;
    if (ghist_next) {
      uint32_t s2 = 0;
#pragma unroll
      for (int w = 0; w < NWARPS; ++w) s2 += S.wh2[w][d];
      if (s2) atomicAdd(&ghist_next[d], s2);
    }
  }
  // decoupled look-back, one chain per digit
  unsigned long long* my = lookback + (size_t)tile * RADIX + tid;
  const unsigned long long ep = (unsigned long long)epoch << 32;
  uint32_t excl = 0;
  if (tile == 0) {
    st_relaxed64(my, ep | LB_INC | cnt);
  } else {
    st_relaxed64(my, ep | LB_AGG | cnt);
    SpinGuard sg;
    int32_t pt = (int32_t)tile - 1;
    while (pt >= 0) {
      unsigned long long w = ld_relaxed64(lookback + (size_t)pt * RADIX + tid);
      if ((w >> 32) != epoch || (w & (3ull << 30)) == 0) {  // not yet published
        if (sg.stuck(ctl)) break;
        continue;
      }
      excl += (uint32_t)(w & LB_VAL);
      if (w & LB_INC) break;
      --pt;
    }
    st_relaxed64(my, ep | LB_INC | (excl + cnt));
  }
  {
    uint32_t tot;
    uint32_t off = block_excl_scan(cnt, S.scan_tmp, &tot);
    S.tile_off[tid] = off;
    S.bin_base[tid] = S.bin_start[tid] + excl - off;
  }
  __syncthreads();
  // stage in smem in tile-local sorted order
#pragma unroll
  for (int j = 0; j < SORT_ITEMS; ++j) {
    uint32_t idx = wbase + j * 32 + lane;
    if (idx < n) {
      uint32_t d = digit_of(k[j], shift);
      uint32_t pos = S.tile_off[d] + S.wh[warp][d] + r[j];
      S.keys[pos] = k[j];
      S.pay[pos] = p[j];
    }
  }
  __syncthreads();
  const uint32_t tile_n = min((uint32_t)SORT_TILE, n - base);
  for (uint32_t i = tid; i < tile_n; i += SORT_THREADS) {
    uint64_t key = S.keys[i];
    uint32_t d = digit_of(key, shift);
    uint32_t o = S.bin_base[d] + i;
    kout[o] = key;
    pout[o] = S.pay[i];
  }
}

}  // namespace

size_t sort_lookback_words(uint32_t max_n) {
  size_t tiles = (max_n + SORT_TILE - 1) / SORT_TILE;
  return tiles * RADIX;
}

void launch_sort(const uint64_t* keys, const uint8_t* ops, const uint32_t* pay_in, const uint64_t* vals, uint32_t n,
                 uint64_t key_lo, uint64_t key_hi, const SortBufs& b, BatchCtl* ctl, uint32_t epoch_base,
                 cudaStream_t st, int* launches, uint64_t** kout, uint32_t** pout) {
  static int attr[MAX_DEVICES];
  per_device(attr, [] {
    return (int)cudaFuncSetAttribute(sort_pass_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                     (int)sizeof(PassSmem));
  });
  const uint32_t tiles = (n + SORT_TILE - 1) / SORT_TILE;
  int up_blocks = (int)std::min<uint32_t>((n + SORT_THREADS * 8 - 1) / (SORT_THREADS * 8), 148u * 4u);
  if (up_blocks < 1) up_blocks = 1;
  sort_upsweep_kernel<<<up_blocks, SORT_THREADS, 0, st>>>(keys, ops, vals, n, key_lo, key_hi, b.ghist, ctl);
  ++*launches;
  const uint64_t* ki = keys;
  const uint32_t* pi = pay_in;
  uint64_t* kbuf[2] = {b.kA, b.kB};
  uint32_t* pbuf[2] = {b.pA, b.pB};
  for (int pass = 0; pass < SORT_PASSES; ++pass) {
    uint64_t* ko = kbuf[pass & 1];
    uint32_t* po = pbuf[pass & 1];
    const bool last = pass == SORT_PASSES - 1;
    sort_pass_kernel<<<tiles, SORT_THREADS, sizeof(PassSmem), st>>>(
        ki, pi, pass == 0 ? ops : nullptr, ko, po, n, pass * 8, (pass + 1) * 8, b.ghist + pass * RADIX,
        last ? nullptr : b.ghist + (pass + 1) * RADIX, b.lookback, epoch_base + pass, &ctl->tile_ctr[TC_SORT0 + pass],
        ctl);
    ++*launches;
    ki = ko;
    pi = po;
  }
  *kout = const_cast<uint64_t*>(ki);
  *pout = const_cast<uint32_t*>(pi);
}

}  // namespace eirene
