// Measurement helper (not product code): cost of a one-pass wide MSD partition with
// per-CTA shared-memory bin cursors (hist -> scan -> scatter) and of its inverse gather,
// at Q = 2^26 u64 queries, against a plain copy.  nvcc -O3 -arch=sm_100a exp_segscatter.cu
#include <cstdio>
#include <cstdint>
#include <vector>
#include <cuda_runtime.h>

#define CK(x) do { cudaError_t e_ = (x); if (e_ != cudaSuccess) { printf("%s:%d %s\n", __FILE__, __LINE__, cudaGetErrorString(e_)); return 1; } } while (0)

__device__ __forceinline__ uint64_t sm64(uint64_t x) {
  x += 0x9E3779B97F4A7C15ull;
  uint64_t z = (x ^ (x >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}
__global__ void k_gen(uint64_t* q, size_t n) {
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x) q[i] = sm64(i);
}
__global__ void k_copy(const uint4* a, uint4* b, size_t n) {
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x) b[i] = a[i];
}

// K1: per-CTA histogram of the top BITS bits; CTA c owns [c*per, (c+1)*per)
template <int BITS>
__global__ void __launch_bounds__(1024) k_hist(const uint64_t* __restrict__ q, size_t n, uint32_t* __restrict__ gh) {
  extern __shared__ uint32_t h[];
  const int nb = 1 << BITS;
  for (int i = threadIdx.x; i < nb; i += blockDim.x) h[i] = 0;
  __syncthreads();
  const size_t per = (n + gridDim.x - 1) / gridDim.x;
  const size_t lo = blockIdx.x * per, hi = min(n, lo + per);
  const uint4* q4 = reinterpret_cast<const uint4*>(q);
  for (size_t i = lo / 2 + threadIdx.x; i < hi / 2; i += blockDim.x * 4) {
    uint4 v[4];
#pragma unroll
    for (int u = 0; u < 4; ++u) { size_t j = i + u * blockDim.x; v[u] = j < hi / 2 ? __ldcs(q4 + j) : make_uint4(0, 0, 0, 0); }
#pragma unroll
    for (int u = 0; u < 4; ++u) {
      size_t j = i + u * blockDim.x;
      if (j < hi / 2) {
        atomicAdd(&h[v[u].y >> (32 - BITS)], 1u);
        atomicAdd(&h[v[u].w >> (32 - BITS)], 1u);
      }
    }
  }
  __syncthreads();
  for (int b = threadIdx.x; b < nb; b += blockDim.x) gh[(size_t)b * gridDim.x + blockIdx.x] = h[b];
}

// simple scan (one block per 1024-chunk + serial carry, measurement only)
__global__ void k_scan_serial(uint32_t* a, size_t n) {
  __shared__ uint32_t s[1024];
  __shared__ uint32_t carry;
  if (threadIdx.x == 0) carry = 0;
  __syncthreads();
  for (size_t base = 0; base < n; base += 1024) {
    uint32_t v = base + threadIdx.x < n ? a[base + threadIdx.x] : 0;
    s[threadIdx.x] = v;
    __syncthreads();
    for (int d = 1; d < 1024; d <<= 1) {
      uint32_t y = threadIdx.x >= d ? s[threadIdx.x - d] : 0;
      __syncthreads();
      s[threadIdx.x] += y;
      __syncthreads();
    }
    if (base + threadIdx.x < n) a[base + threadIdx.x] = carry + s[threadIdx.x] - v;
    __syncthreads();
    if (threadIdx.x == 1023) carry += s[1023];
    __syncthreads();
  }
}

// K3: scatter with per-CTA shared cursors
template <int BITS>
__global__ void __launch_bounds__(1024) k_scatter(const uint64_t* __restrict__ q, size_t n, const uint32_t* __restrict__ off,
                                                  uint64_t* __restrict__ sq, uint32_t* __restrict__ dest) {
  extern __shared__ uint32_t cur[];
  const int nb = 1 << BITS;
  for (int b = threadIdx.x; b < nb; b += blockDim.x) cur[b] = off[(size_t)b * gridDim.x + blockIdx.x];
  __syncthreads();
  const size_t per = (n + gridDim.x - 1) / gridDim.x;
  const size_t lo = blockIdx.x * per, hi = min(n, lo + per);
  const uint4* q4 = reinterpret_cast<const uint4*>(q);
  uint2* d2 = reinterpret_cast<uint2*>(dest);
  for (size_t i = lo / 2 + threadIdx.x; i < hi / 2; i += blockDim.x * 4) {
    uint4 v[4];
#pragma unroll
    for (int u = 0; u < 4; ++u) { size_t j = i + u * blockDim.x; v[u] = j < hi / 2 ? __ldcs(q4 + j) : make_uint4(0, 0, 0, 0); }
#pragma unroll
    for (int u = 0; u < 4; ++u) {
      size_t j = i + u * blockDim.x;
      if (j < hi / 2) {
        uint32_t s0 = atomicAdd(&cur[v[u].y >> (32 - BITS)], 1u);
        uint32_t s1 = atomicAdd(&cur[v[u].w >> (32 - BITS)], 1u);
        sq[s0] = ((uint64_t)v[u].y << 32) | v[u].x;
        sq[s1] = ((uint64_t)v[u].w << 32) | v[u].z;
        __stcs(d2 + j, make_uint2(s0, s1));
      }
    }
  }
}

// K6: out[i] = res[dest[i]]
__global__ void __launch_bounds__(1024) k_gather(const uint64_t* __restrict__ res, const uint32_t* __restrict__ dest, size_t n,
                                                 uint64_t* __restrict__ out) {
  const size_t per = (n + gridDim.x - 1) / gridDim.x;
  const size_t lo = blockIdx.x * per, hi = min(n, lo + per);
  const uint4* d4 = reinterpret_cast<const uint4*>(dest);
  uint4* o4 = reinterpret_cast<uint4*>(out);
  for (size_t i = lo / 4 + threadIdx.x; i < hi / 4; i += blockDim.x * 2) {
    uint4 d[2];
#pragma unroll
    for (int u = 0; u < 2; ++u) { size_t j = i + u * blockDim.x; d[u] = j < hi / 4 ? __ldcs(d4 + j) : make_uint4(0, 0, 0, 0); }
    uint64_t r[8];
#pragma unroll
    for (int u = 0; u < 2; ++u) {
      size_t j = i + u * blockDim.x;
      if (j < hi / 4) { r[4*u] = res[d[u].x]; r[4*u+1] = res[d[u].y]; r[4*u+2] = res[d[u].z]; r[4*u+3] = res[d[u].w]; }
    }
#pragma unroll
    for (int u = 0; u < 2; ++u) {
      size_t j = i + u * blockDim.x;
      if (j < hi / 4) {
        __stcs(o4 + 2 * j, make_uint4((uint32_t)r[4*u], (uint32_t)(r[4*u] >> 32), (uint32_t)r[4*u+1], (uint32_t)(r[4*u+1] >> 32)));
        __stcs(o4 + 2 * j + 1, make_uint4((uint32_t)r[4*u+2], (uint32_t)(r[4*u+2] >> 32), (uint32_t)r[4*u+3], (uint32_t)(r[4*u+3] >> 32)));
      }
    }
  }
}

template <int BITS>
int run(uint64_t* q, uint64_t* sq, uint32_t* dest, uint64_t* out, size_t n, int nct) {
  uint32_t* gh;
  size_t nh = (size_t)nct << BITS;
  CK(cudaMalloc(&gh, nh * 4));
  size_t smem = (size_t)4 << BITS;
  CK(cudaFuncSetAttribute(k_hist<BITS>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
  CK(cudaFuncSetAttribute(k_scatter<BITS>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
  cudaEvent_t e[5];
  for (auto& x : e) cudaEventCreate(&x);
  float best[4] = {1e9, 1e9, 1e9, 1e9};
  for (int it = 0; it < 6; ++it) {
    cudaEventRecord(e[0]);
    k_hist<BITS><<<nct, 1024, smem>>>(q, n, gh);
    cudaEventRecord(e[1]);
    k_scan_serial<<<1, 1024>>>(gh, nh);
    cudaEventRecord(e[2]);
    k_scatter<BITS><<<nct, 1024, smem>>>(q, n, gh, sq, dest);
    cudaEventRecord(e[3]);
    k_gather<<<nct, 1024>>>(sq, dest, n, out);
    cudaEventRecord(e[4]);
    CK(cudaEventSynchronize(e[4]));
    for (int k = 0; k < 4; ++k) { float ms; cudaEventElapsedTime(&ms, e[k], e[k + 1]); if (it > 0 && ms < best[k]) best[k] = ms; }
  }
  CK(cudaGetLastError());
  // check: out == q and sq bucket-sorted
  std::vector<uint64_t> h(n), hs(n);
  CK(cudaMemcpy(h.data(), out, n * 8, cudaMemcpyDeviceToHost));
  CK(cudaMemcpy(hs.data(), sq, n * 8, cudaMemcpyDeviceToHost));
  size_t bad = 0, unsorted = 0;
  for (size_t i = 0; i < n; ++i) {
    uint64_t x = i + 0x9E3779B97F4A7C15ull;
    uint64_t z = (x ^ (x >> 30)) * 0xBF58476D1CE4E5B9ull; z = (z ^ (z >> 27)) * 0x94D049BB133111EBull; z ^= z >> 31;
    bad += h[i] != z;
    if (i && (hs[i] >> (64 - BITS)) < (hs[i - 1] >> (64 - BITS))) ++unsorted;
  }
  printf("bits=%d ctas=%d hist %.3f scan %.3f scatter %.3f gather %.3f ms  bad=%zu unsorted=%zu\n", BITS, nct, best[0], best[1],
         best[2], best[3], bad, unsorted);
  cudaFree(gh);
  return 0;
}

int main() {
  const size_t n = (size_t)1 << 26;
  uint64_t *q, *sq, *out;
  uint32_t* dest;
  CK(cudaMalloc(&q, n * 8)); CK(cudaMalloc(&sq, n * 8)); CK(cudaMalloc(&out, n * 8)); CK(cudaMalloc(&dest, n * 4));
  k_gen<<<1184, 256>>>(q, n);
  CK(cudaDeviceSynchronize());
  cudaEvent_t a, b;
  cudaEventCreate(&a); cudaEventCreate(&b);
  float bc = 1e9;
  for (int it = 0; it < 5; ++it) {
    cudaEventRecord(a);
    k_copy<<<148 * 8, 512>>>((const uint4*)q, (uint4*)out, n / 2);
    cudaEventRecord(b);
    cudaEventSynchronize(b);
    float ms; cudaEventElapsedTime(&ms, a, b); if (ms < bc) bc = ms;
  }
  printf("copy 512 MiB: %.3f ms (%.0f GB/s)\n", bc, 2.0 * n * 8 / bc / 1e6);
  for (int nct : {148, 296}) {
    run<11>(q, sq, dest, out, n, nct);
    run<12>(q, sq, dest, out, n, nct);
    run<13>(q, sq, dest, out, n, nct);
    if (nct == 148) run<14>(q, sq, dest, out, n, nct);
  }
  return 0;
}
