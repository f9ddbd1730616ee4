// Measurement helper (not product code): the L2 and HBM read bandwidth peaks used by the
// bench's roofline (SURVEY §8(d) asks for BW_L2 beside BW_HBM).  Prints one JSON line.
//   L2 read: 128-bit ld.global.cg (L1 bypassed) sweeps over an L2-resident buffer, every SM.
//   HBM read: 128-bit streaming loads over a 4 GiB buffer; HBM copy: read + write.
// nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o tools/bin/peaks tools/peaks.cu
#include <cstdio>
#include <cstdint>
#include <algorithm>
#include <cmath>
#include <cuda_runtime.h>

__global__ void k_fill(uint4* p, size_t n) {
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x)
    p[i] = make_uint4((uint32_t)i, 1, 2, 3);
}

__device__ __forceinline__ uint4 ld_cg(const uint4* p) {
  uint4 v;
  asm volatile("ld.global.cg.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(p));
  return v;
}
__device__ __forceinline__ uint4 ld_cs(const uint4* p) {
  uint4 v;
  asm volatile("ld.global.cs.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(p));
  return v;
}

// every CTA sweeps the whole buffer `reps` times starting at a CTA-dependent offset
template <bool kL2>
__global__ void __launch_bounds__(512) k_read(const uint4* __restrict__ p, size_t n, int reps, uint32_t* sink) {
  uint32_t acc = 0;
  const size_t stride = (size_t)gridDim.x * blockDim.x;
  for (int r = 0; r < reps; ++r) {
    size_t i = (blockIdx.x * (size_t)blockDim.x + threadIdx.x + (size_t)r * 4099 * blockDim.x) % n;
    for (size_t k = 0; k < n; k += 4 * stride) {
      uint4 v[4];
#pragma unroll
      for (int u = 0; u < 4; ++u) {
        size_t j = i + u * stride;
        j = j >= n ? j - n : j;
        v[u] = kL2 ? ld_cg(p + j) : ld_cs(p + j);
      }
#pragma unroll
      for (int u = 0; u < 4; ++u) acc ^= v[u].x ^ v[u].y ^ v[u].z ^ v[u].w;
      i += 4 * stride;
      i = i >= n ? i % n : i;
    }
  }
  if (acc == 0x12345678u) *sink = acc;
}

__global__ void k_copy(const uint4* __restrict__ a, uint4* __restrict__ b, size_t n) {
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x)
    b[i] = ld_cs(a + i);
}

template <class F>
float best_ms(F f, int it = 7) {
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  float best = 1e30f;
  for (int k = 0; k < it; ++k) {
    cudaEventRecord(a);
    f();
    cudaEventRecord(b);
    cudaEventSynchronize(b);
    float ms;
    cudaEventElapsedTime(&ms, a, b);
    if (k > 0) best = std::min(best, ms);
  }
  return best;
}

int main() {
  int dev = 0, sm = 0, l2 = 0;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sm, cudaDevAttrMultiProcessorCount, dev);
  cudaDeviceGetAttribute(&l2, cudaDevAttrL2CacheSize, dev);
  uint32_t* sink;
  cudaMalloc(&sink, 4);
  printf("{\"sm_count\": %d, \"l2_bytes\": %d", sm, l2);
  // L2: buffers well inside the 126 MB (both dies' halves hold the lines)
  for (size_t mib : {16, 32, 48}) {
    const size_t n = mib * (1 << 20) / 16;
    uint4* p;
    cudaMalloc(&p, n * 16);
    k_fill<<<sm * 4, 512>>>(p, n);
    const int reps = 64;
    const int grid = sm * 4;
    float ms = best_ms([&] { k_read<true><<<grid, 512>>>(p, n, reps, sink); });
    // total loads: every thread issues ceil(n / (4*stride)) * 4 loads per rep
    const double stride = (double)grid * 512;
    const double per_thread = 4.0 * std::ceil((double)n / (4 * stride));
    const double tot = per_thread * stride * 16.0 * reps;
    printf(", \"l2_read_gbs_%zumib\": %.1f", mib, tot / ms / 1e6);
    cudaFree(p);
  }
  {
    const size_t n = (size_t)4 << 30 >> 4;  // 4 GiB
    uint4 *a, *b;
    cudaMalloc(&a, n * 16);
    cudaMalloc(&b, n * 16);
    k_fill<<<sm * 4, 512>>>(a, n);
    const int grid = sm * 4;
    float ms = best_ms([&] { k_read<false><<<grid, 512>>>(a, n, 1, sink); }, 5);
    const double stride = (double)grid * 512;
    const double tot = 4.0 * std::ceil((double)n / (4 * stride)) * stride * 16.0;
    printf(", \"hbm_read_gbs\": %.1f", tot / ms / 1e6);
    float mc = best_ms([&] { k_copy<<<sm * 8, 512>>>(a, b, n); }, 5);
    printf(", \"hbm_copy_gbs\": %.1f", 2.0 * n * 16 / mc / 1e6);
    cudaFree(a);
    cudaFree(b);
  }
  cudaError_t e = cudaDeviceSynchronize();
  printf(", \"status\": \"%s\"}\n", cudaGetErrorString(e));
  return 0;
}
