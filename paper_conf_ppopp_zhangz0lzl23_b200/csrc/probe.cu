// probe.cu -- random-access probes of the GPU's HBM, the denominators of the
// random-access roofline of SURVEY §8(d) (BASELINE north_star: "the fraction
// of the HBM random-access roofline").  The hot path touches the leaves at
// random: one 128 B key line and one 32 B value sector per issued request,
// and one 32 B value sector written per issued write.  These kernels measure
// how many such accesses per second the memory system sustains on this GPU:
// uniformly random lines / sectors of a pool much larger than L2, the same
// load instructions as the query kernel (256-bit, L1 no-allocate).
#include "eirene_internal.cuh"

namespace eirene {
namespace {

__device__ __forceinline__ uint64_t mix64(uint64_t x) {
  x += 0x9e3779b97f4a7c15ull;
  x = (x ^ (x >> 30)) * 0xbf58476d1ce4e5b9ull;
  x = (x ^ (x >> 27)) * 0x94d049bb133111ebull;
  return x ^ (x >> 31);
}

// Pool sizes are powers of two here (masks, not 64-bit modulo).
// kind 0: uniformly random 128 B line reads (4 x 256-bit); 1: random 32 B
// sector reads; 2: random 32 B sector writes; 3: the query kernel's leaf
// access -- the 128 B key line of a 256 B leaf block, then (dependent) one
// 32 B sector of its value line -- at the batch's density and order: access i
// of n goes to block floor(i * nblk / n) + a random offset below nblk / n,
// so consecutive threads touch ascending, nearby blocks as a key-sorted batch
// does (kind 3 counts one access per leaf block visited).
__global__ void __launch_bounds__(256) probe_kernel(uint64_t* __restrict__ pool, uint64_t nsect, uint32_t n, int kind,
                                                    uint64_t seed, uint64_t* __restrict__ sink) {
  const uint64_t pf = pol_evict_first();
  const uint64_t smask = nsect - 1, lmask = nsect / 4 - 1, nblk = nsect / 8;
  uint64_t acc = 0;
  for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x) {
    const uint64_t h = mix64(seed ^ i);
    if (kind == 0) {
      const uint64_t* p = pool + ((h & lmask) * 16);   // 128 B aligned line
#pragma unroll
      for (int x = 0; x < 4; ++x) {
        const ulonglong4 v = ldg256_pol(p + 4 * x, pf);
        acc ^= v.x ^ v.y ^ v.z ^ v.w;
      }
    } else if (kind == 1) {
      const ulonglong4 v = ldg256_pol(pool + (h & smask) * 4, pf);
      acc ^= v.x ^ v.y ^ v.z ^ v.w;
    } else if (kind == 2) {
      uint64_t* p = pool + (h & smask) * 4;
      asm volatile("st.global.L2::cache_hint.v4.u64 [%0], {%1,%2,%3,%4}, %5;" ::"l"(p), "l"(h), "l"(h), "l"(h),
                   "l"(h), "l"(pf)
                   : "memory");
    } else {
      const uint64_t span = nblk > n ? nblk / n : 1;   // blocks per access (>= 1)
      const uint64_t blk = ((uint64_t)i * nblk) / n + (((h & 0xFFFFFFFFull) * span) >> 32);   // (span < 2^32)
      const uint64_t* p = pool + (blk < nblk ? blk : nblk - 1) * 32;   // 256 B leaf block
      uint64_t k = 0;
#pragma unroll
      for (int x = 0; x < 4; ++x) {
        const ulonglong4 v = ldg256_pol(p + 4 * x, pf);
        k ^= v.x ^ v.y ^ v.z ^ v.w;
      }
      // the value sector depends on the key line (as the slot found in it does)
      const ulonglong4 v = ldg256_pol(p + 16 + 4 * ((k ^ h) & 3), pf);
      acc ^= v.x ^ v.y ^ v.z ^ v.w;
    }
  }
  if (acc == 0x123456789ull) sink[0] = acc;   // keeps the loads
}

}  // namespace
}  // namespace eirene

extern "C" int eirene_probe_gather(void* pool_dev, uint64_t pool_bytes, uint32_t n, int kind, uint64_t seed,
                                   eirene_stream_t stream) {
  using namespace eirene;
  if (!pool_dev || pool_bytes < 4096 || (pool_bytes & (pool_bytes - 1)) || kind < 0 || kind > 3 ||
      (reinterpret_cast<uintptr_t>(pool_dev) & 255))
    return EIRENE_EINVAL;
  int dev = 0, sms = 148;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  const uint64_t nsect = pool_bytes / 32;
  probe_kernel<<<sms * 8, 256, 0, reinterpret_cast<cudaStream_t>(stream)>>>(
      static_cast<uint64_t*>(pool_dev), nsect, n, kind, seed, static_cast<uint64_t*>(pool_dev));
  const cudaError_t e = cudaGetLastError();
  return e == cudaSuccess ? EIRENE_OK : EIRENE_ECUDA;
}
