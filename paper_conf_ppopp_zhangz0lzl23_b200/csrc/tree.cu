// tree.cu -- tree construction (bulk load, "initialized when the
// tree is constructed") and the quiescent in-order scan, sm_100a.
#include <vector>

#include "eirene_internal.cuh"

namespace eirene {

namespace {

__global__ void validate_bulk_kernel(const tkey_t* __restrict__ keys, const tkey_t* __restrict__ vals, uint64_t n,
                                     uint64_t key_lo, uint64_t key_hi, uint32_t* flag) {
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  bool bad = false;
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += stride) {
    const uint64_t k = widen(keys[i]);
    bad |= k == KEY_MAX || k < key_lo || k >= key_hi || widen(vals[i]) == KEY_MAX || (i > 0 && !(keys[i - 1] < k));
  }
  if (__any_sync(FULL, bad) && (threadIdx.x & 31) == 0) atomicOr(flag, 1u);
}

// Leaves: leaf q holds keys [q*per, min((q+1)*per, n)); fences from the keys.
__global__ void build_leaves_kernel(const tkey_t* __restrict__ keys, const tkey_t* __restrict__ vals, uint64_t n,
                                    uint32_t per, uint32_t L, uint64_t key_lo, uint64_t key_hi, Tree t) {
  const uint64_t gid = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  const uint64_t leaf = gid / FAN;
  const uint32_t s = (uint32_t)(gid % FAN);
  if (leaf >= L) return;
  const uint64_t idx = leaf * per + s;
  const bool valid = s < per && idx < n;
  t.lkeys[leaf * LSTRIDE + s] = valid ? keys[idx] : KEY_MAX;
  t.lvals[leaf * LSTRIDE + s] = valid ? vals[idx] : 0;
  if (s == 0) {
    NodeMeta m;
    m.version = 0;
    m.next = leaf + 1 < L ? (uint32_t)(leaf + 1) : NIL;
    m.lo = leaf == 0 ? key_lo : keys[leaf * per];
    m.hi = leaf + 1 < L ? keys[(leaf + 1) * per] : key_hi;
    m.count = (uint32_t)std::min<uint64_t>(per, n - leaf * per);
    m.level = 0;
    t.lmeta[leaf] = m;
  }
}

// Range field of every bulk-loaded leaf (reading 22): the min
// key (= lo fence) of the leaf `height` links to the right, KEY_MAX past the
// end of the chain.  Bulk-loaded leaf ids are their chain positions.
__global__ void build_rf_kernel(Tree t, uint32_t L, uint32_t height) {
  const uint32_t i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i < L) t.lrf[i] = (uint64_t)i + height < L ? t.lmeta[i + height].lo : KEY_MAX;
}

// One inner level over nc children with consecutive ids [cbase, cbase+nc)
// (leaves when child_level == 0), nn = ceil(nc/16) nodes, even distribution.
__global__ void build_inner_kernel(Tree t, uint32_t child_level, uint32_t cbase, uint32_t nc, uint32_t nbase,
                                   uint32_t nn) {
  const uint64_t gid = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  const uint32_t q = (uint32_t)(gid / FAN), i = (uint32_t)(gid % FAN);
  if (q >= nn) return;
  const uint32_t bs = nc / nn, rem = nc % nn;
  const uint32_t size = bs + (q < rem ? 1u : 0u);
  const uint32_t start = q * bs + min(q, rem);
  const NodeMeta* cm = child_level == 0 ? t.lmeta : t.imeta;
  const uint32_t id = nbase + q;
  t.ichild[(size_t)id * FAN + i] = i < size ? cbase + start + i : NIL;
  t.ikeys[(size_t)id * FAN + i] = (i + 1 < size) ? cm[cbase + start + i + 1].lo : KEY_MAX;
  if (i == 0) {
    NodeMeta m;
    m.version = 0;
    m.next = q + 1 < nn ? id + 1 : NIL;
    m.lo = cm[cbase + start].lo;
    m.hi = cm[cbase + start + size - 1].hi;
    m.count = size;
    m.level = child_level + 1;
    t.imeta[id] = m;
  }
}

// ---------------------------------------------------------------- scan
__global__ void leaf_lo_kernel(Tree t, uint32_t lc, uint64_t* __restrict__ lo_out, uint32_t* __restrict__ id_out) {
  const uint32_t i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= lc) return;
  lo_out[i] = t.lmeta[i].lo;
  id_out[i] = i;
}

__global__ void leaf_count_kernel(Tree t, const uint32_t* __restrict__ order, uint32_t lc, uint64_t lo, uint64_t hi,
                                  uint64_t* __restrict__ cnt) {
  const uint32_t i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= lc) return;
  const uint32_t leaf = order[i];
  uint64_t c = 0;
  for (int s = 0; s < FAN; ++s) {
    const uint64_t k = widen(t.lkeys[(size_t)leaf * LSTRIDE + s]);
    c += (k != KEY_MAX && k >= lo && k <= hi) ? 1 : 0;
  }
  cnt[i] = c;
}

// exclusive scan of u64 counts, single block of 1024 threads, sequential chunks
__global__ void __launch_bounds__(1024) excl_scan_u64_kernel(uint64_t* __restrict__ a, uint64_t n,
                                                             uint64_t* __restrict__ total) {
  __shared__ uint64_t wsum[32];
  __shared__ uint64_t carry;
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  if (tid == 0) carry = 0;
  __syncthreads();
  for (uint64_t base = 0; base < n; base += 1024) {
    const uint64_t i = base + tid;
    const uint64_t v = i < n ? a[i] : 0;
    uint64_t x = v;
    for (int o = 1; o < 32; o <<= 1) {
      const uint64_t y = __shfl_up_sync(FULL, x, o);
      if (lane >= o) x += y;
    }
    if (lane == 31) wsum[warp] = x;
    __syncthreads();
    uint64_t wp = 0, tot = 0;
    for (int w = 0; w < 32; ++w) {
      if (w < warp) wp += wsum[w];
      tot += wsum[w];
    }
    const uint64_t c = carry;
    if (i < n) a[i] = c + wp + x - v;
    __syncthreads();
    if (tid == 0) carry = c + tot;
    __syncthreads();
  }
  if (tid == 0) *total = carry;
}

__global__ void leaf_emit_kernel(Tree t, const uint32_t* __restrict__ order, const uint64_t* __restrict__ off,
                                 uint32_t lc, uint64_t lo, uint64_t hi, tkey_t* __restrict__ ko,
                                 tkey_t* __restrict__ vo, uint64_t cap) {
  const uint32_t i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= lc) return;
  const uint32_t leaf = order[i];
  uint64_t o = off[i];
  for (int s = 0; s < FAN; ++s) {
    const uint64_t k = widen(t.lkeys[(size_t)leaf * LSTRIDE + s]);
    if (k != KEY_MAX && k >= lo && k <= hi) {
      if (o < cap) {
        if (ko) ko[o] = k;
        if (vo) vo[o] = t.lvals[(size_t)leaf * LSTRIDE + s];
      }
      ++o;
    }
  }
}

}  // namespace

int build_tree(Tree t, const tkey_t* keys, const tkey_t* vals, uint64_t n, int per, uint64_t key_lo,
               uint64_t key_hi, cudaStream_t st, int* launches, uint32_t* height_out) {
  // caller has validated and zeroed; per in [1, 16]
  const uint64_t L64 = (n + per - 1) / per;
  if (L64 > t.leaf_cap) return EIRENE_EFULL;
  const uint32_t L = (uint32_t)L64;
  TreeHdr hdr{};
  {
    const uint64_t threads = (uint64_t)L * FAN;
    build_leaves_kernel<<<(unsigned)((threads + 255) / 256), 256, 0, st>>>(keys, vals, n, per, L, key_lo, key_hi, t);
    ++*launches;
  }
  hdr.leaf_count = L;
  hdr.level_count[0] = L;
  uint32_t level = 0, cbase = 0, nc = L, nbase = 0;
  while (nc > 1) {
    const uint32_t nn = (nc + FAN - 1) / FAN;
    if ((uint64_t)nbase + nn > t.inner_cap) return EIRENE_EFULL;
    const uint64_t threads = (uint64_t)nn * FAN;
    build_inner_kernel<<<(unsigned)((threads + 255) / 256), 256, 0, st>>>(t, level, cbase, nc, nbase, nn);
    ++*launches;
    hdr.level_count[level + 1] = nn;
    cbase = nbase;
    nbase += nn;
    nc = nn;
    ++level;
  }
  hdr.inner_count = nbase;
  hdr.root_word = ((unsigned long long)(level + 1) << 32) | cbase;
  *height_out = level + 1;
  build_rf_kernel<<<(L + 255) / 256, 256, 0, st>>>(t, L, level + 1);
  ++*launches;
  cudaMemcpyAsync(t.hdr, &hdr, sizeof(hdr), cudaMemcpyHostToDevice, st);
  cudaStreamSynchronize(st);
  return EIRENE_OK;
}

void launch_validate_bulk(const tkey_t* keys, const tkey_t* vals, uint64_t n, uint64_t key_lo, uint64_t key_hi,
                          uint32_t* flag, cudaStream_t st, int* launches) {
  unsigned blocks = (unsigned)std::min<uint64_t>((n + 255) / 256, 148ull * 16ull);
  if (blocks < 1) blocks = 1;
  validate_bulk_kernel<<<blocks, 256, 0, st>>>(keys, vals, n, key_lo, key_hi, flag);
  ++*launches;
}

int scan_tree(Tree t, uint32_t lc, uint64_t lo, uint64_t hi, tkey_t* ko, tkey_t* vo, uint64_t cap,
              uint64_t* count, cudaStream_t st, int* launches) {
  *count = 0;
  if (lc == 0 || lo > hi) return EIRENE_OK;
  // leaves ordered by their lo fence == the leaf chain order
  uint64_t *lo_a = nullptr, *cnt = nullptr, *tot = nullptr;
  uint32_t* id_a = nullptr;
  SortBufs sb{};
  BatchCtl* ctl = nullptr;
  const size_t lbw = sort_lookback_words(lc);
  cudaError_t e = cudaSuccess;
  e = cudaMalloc(&lo_a, sizeof(uint64_t) * lc);
  if (e == cudaSuccess) e = cudaMalloc(&id_a, sizeof(uint32_t) * lc);
  if (e == cudaSuccess) e = cudaMalloc(&cnt, sizeof(uint64_t) * lc);
  if (e == cudaSuccess) e = cudaMalloc(&tot, sizeof(uint64_t));
  if (e == cudaSuccess) e = cudaMalloc(&sb.kA, sizeof(uint64_t) * lc);
  if (e == cudaSuccess) e = cudaMalloc(&sb.kB, sizeof(uint64_t) * lc);
  if (e == cudaSuccess) e = cudaMalloc(&sb.pA, sizeof(uint32_t) * lc);
  if (e == cudaSuccess) e = cudaMalloc(&sb.pB, sizeof(uint32_t) * lc);
  if (e == cudaSuccess) e = cudaMalloc(&sb.lookback, sizeof(unsigned long long) * lbw);
  if (e == cudaSuccess) e = cudaMalloc(&sb.ghist, sizeof(uint32_t) * 8 * 256);
  if (e == cudaSuccess) e = cudaMalloc(&ctl, sizeof(BatchCtl));
  int rc = EIRENE_OK;
  if (e != cudaSuccess) {
    rc = EIRENE_ECUDA;
  } else {
    cudaMemsetAsync(sb.lookback, 0, sizeof(unsigned long long) * lbw, st);
    cudaMemsetAsync(sb.ghist, 0, sizeof(uint32_t) * 8 * 256, st);
    cudaMemsetAsync(ctl, 0, sizeof(BatchCtl), st);
    leaf_lo_kernel<<<(lc + 255) / 256, 256, 0, st>>>(t, lc, lo_a, id_a);
    ++*launches;
    uint64_t* sk;
    uint32_t* sp;
    launch_sort(lo_a, nullptr, id_a, nullptr, lc, 0, KEY_MAX, sb, ctl, 1, st, launches, &sk, &sp);
    leaf_count_kernel<<<(lc + 255) / 256, 256, 0, st>>>(t, sp, lc, lo, hi, cnt);
    excl_scan_u64_kernel<<<1, 1024, 0, st>>>(cnt, lc, tot);
    leaf_emit_kernel<<<(lc + 255) / 256, 256, 0, st>>>(t, sp, cnt, lc, lo, hi, ko, vo, cap);
    *launches += 3;
    cudaMemcpyAsync(count, tot, sizeof(uint64_t), cudaMemcpyDeviceToHost, st);
    if (cudaStreamSynchronize(st) != cudaSuccess) rc = EIRENE_ECUDA;
  }
  cudaFree(lo_a);
  cudaFree(id_a);
  cudaFree(cnt);
  cudaFree(tot);
  cudaFree(sb.kA);
  cudaFree(sb.kB);
  cudaFree(sb.pA);
  cudaFree(sb.pB);
  cudaFree(sb.lookback);
  cudaFree(sb.ghist);
  cudaFree(ctl);
  return rc;
}

}  // namespace eirene
