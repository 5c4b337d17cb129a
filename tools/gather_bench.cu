// gather_bench.cu -- microbenchmark of random-gather bandwidth on the GPU the
// query kernel runs on (diagnostic for the roofline discussion in DESIGN.md).
// Models the leaf stage of QUERY_KERNEL: n random 128 B lines out of a pool of
// `pool_mb`, with and without a dependent 32 B value read.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/gb tools/gather_bench.cu
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ ulonglong4 ldg256(const uint64_t* p) {
  ulonglong4 v;
  asm volatile("ld.global.nc.v4.u64 {%0,%1,%2,%3}, [%4];" : "=l"(v.x), "=l"(v.y), "=l"(v.z), "=l"(v.w) : "l"(p));
  return v;
}
__device__ __forceinline__ uint64_t hash(uint64_t x) {
  x += 0x9e3779b97f4a7c15ull;
  x = (x ^ (x >> 30)) * 0xbf58476d1ce4e5b9ull;
  x = (x ^ (x >> 27)) * 0x94d049bb133111ebull;
  return x ^ (x >> 31);
}

// mode 0: per-thread line (4 x 256-bit); 1: 4 lanes per line (1 x 256-bit each)
// 2: per-thread 32 B sector; 3: mode 0 + dependent 32 B from a second pool
// 4: sorted indices, per-thread line (like sorted queries: index = i*stride)
__global__ void gather(const uint64_t* __restrict__ pool, const uint64_t* __restrict__ pool2, uint64_t nlines,
                       uint32_t n, int mode, uint64_t seed, uint64_t* out) {
  const uint32_t stride = gridDim.x * blockDim.x;
  uint64_t acc = 0;
  for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += stride) {
    if (mode == 1) {
      const uint32_t q = i >> 2, part = i & 3;
      const uint64_t line = hash(q ^ seed) % nlines;
      ulonglong4 v = ldg256(pool + line * 16 + part * 4);
      acc += v.x ^ v.y ^ v.z ^ v.w;
      continue;
    }
    uint64_t line = mode == 4 ? (uint64_t)i * (nlines / n) : hash(i ^ seed) % nlines;
    if (mode == 6 || mode == 7) line &= ~1ull;
    if (mode == 2) {
      ulonglong4 v = ldg256(pool + line * 16 + (i & 3) * 4);
      acc += v.x ^ v.y ^ v.z ^ v.w;
      continue;
    }
    ulonglong4 v[4];
#pragma unroll
    for (int x = 0; x < 4; ++x) v[x] = ldg256(pool + line * 16 + 4 * x);
    uint64_t s = 0;
#pragma unroll
    for (int x = 0; x < 4; ++x) s += v[x].x ^ v[x].y ^ v[x].z ^ v[x].w;
    if (mode == 3) s += __ldg(pool2 + line * 16 + (s & 15));
    if (mode == 5 || mode == 6) {   // 5: value line (second pool) loaded in parallel; 6: interleaved 256 B leaf
      const uint64_t* vl = mode == 5 ? pool2 + line * 16 : pool + (line & ~1ull) * 16 + 16;
      ulonglong4 w[4];
#pragma unroll
      for (int x = 0; x < 4; ++x) w[x] = ldg256(vl + 4 * x);
      const int sl = (int)(s & 15);
      uint64_t r = 0;
#pragma unroll
      for (int x = 0; x < 4; ++x) {
        r = sl == 4 * x ? w[x].x : r;
        r = sl == 4 * x + 1 ? w[x].y : r;
        r = sl == 4 * x + 2 ? w[x].z : r;
        r = sl == 4 * x + 3 ? w[x].w : r;
      }
      s += r;
    }
    if (mode == 7) s += __ldg(pool + (line & ~1ull) * 16 + 16 + (s & 15));   // interleaved, dependent 8 B
    acc += s;
  }
  if (acc == 0x12345) out[0] = acc;
}

__global__ void flush(uint64_t* p, size_t n, int wr) {
  uint64_t acc = 0;
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x) {
    if (wr) p[i] += 1; else acc += __ldcg(p + i);
  }
  if (acc == 0x777) p[0] = acc;
}

int main() {
  const size_t pool_bytes = 256ull << 20;
  const uint64_t nlines = pool_bytes / 128;
  uint64_t *pool, *pool2, *out, *fl;
  cudaMalloc(&pool, pool_bytes);
  cudaMalloc(&pool2, pool_bytes);
  cudaMalloc(&out, 64);
  const size_t fl_n = (512ull << 20) / 8;
  cudaMalloc(&fl, fl_n * 8);
  cudaMemset(pool, 1, pool_bytes);
  cudaMemset(pool2, 2, pool_bytes);
  cudaMemset(fl, 0, fl_n * 8);
  int sms;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  const char* names[] = {"line/thread 4x256b", "line/4 lanes 1x256b", "32B sector/thread", "line+dep 32B",
                         "sorted line/thread", "key+val lines par", "interleaved 256B par", "interleaved dep 8B"};
  const double bytes_per[] = {128, 32, 32, 160, 128, 256, 256, 160};
  for (int wr : {1, 0})
  for (uint32_t n : {1u << 20, 1u << 22}) {
    for (int mode = 0; mode < 8; ++mode) {
      for (int bpsm : {8, 32}) {
        const uint32_t units = mode == 1 ? n * 4 : n;
        float best = 1e9f;
        for (int r = 0; r < 5; ++r) {
          flush<<<sms * 4, 1024>>>(fl, fl_n, wr);
          cudaEventRecord(a);
          gather<<<sms * bpsm, 256>>>(pool, pool2, nlines, units, mode, r * 7919 + 1, out);
          cudaEventRecord(b);
          cudaEventSynchronize(b);
          float ms;
          cudaEventElapsedTime(&ms, a, b);
          if (ms < best) best = ms;
        }
        const double gbs = (double)units * bytes_per[mode] / (best * 1e-3) / 1e9;
        printf("wr=%d n=%u %-22s blocks/sm=%2d  %8.2f us  %7.0f GB/s  %.3f Gq/s\n", wr, n, names[mode], bpsm, best * 1e3, gbs,
               (double)n / (best * 1e-3) / 1e9);
      }
    }
  }
  cudaError_t e = cudaGetLastError();
  printf("status %s\n", cudaGetErrorString(e));
  return 0;
}
