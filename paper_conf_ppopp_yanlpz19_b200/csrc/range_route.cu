// Range queries over a key-range partitioned tree: a range
// [lo, hi] is cut at every splitter it crosses; each piece is answered by the shard that owns
// it and the pieces are concatenated in shard order, which is key order (C-A10: ascending
// records, true total count).
//
//   harmonia_range_split_count  pieces per range and per destination shard (one pass)
//   harmonia_range_split_emit   pieces written destination-major: (plo, phi) + piece id
//   (caller) exchange the pieces, harmonia_range_batch on each shard, exchange the answers
//   harmonia_range_assemble     per range, its pieces' records in shard order, cut at cap,
//                               counts summed
//
// Shard p owns [sigma_p, sigma_{p+1}) (sigma_0 = 0, sigma_P = 2^64): a piece of [lo, hi] on
// shard d is [max(lo, sigma_d), min(hi, sigma_{d+1} - 1)].  lo > hi gives one empty piece on
// dest(lo) (count 0).  Pieces of range i are numbered pbase[i] .. pbase[i+1]-1 in shard order.
#include <cub/cub.cuh>

#include <algorithm>

#include "common.cuh"

namespace hm {
namespace {

constexpr int kRT = 256;
constexpr uint32_t kMaxShards = 256;

__device__ __forceinline__ void piece_span(const BucketSplit& f, uint64_t lo, uint64_t hi, uint32_t* d0,
                                           uint32_t* np) {
  const uint32_t a = f(lo);
  *d0 = a;
  *np = lo > hi ? 1u : f(hi) - a + 1;
}

__global__ void __launch_bounds__(kRT) k_split_count(BucketSplit f, uint32_t P, const uint64_t* __restrict__ lo,
                                                     const uint64_t* __restrict__ hi, uint64_t n,
                                                     uint32_t* __restrict__ npieces, uint32_t* __restrict__ dcount) {
  __shared__ uint32_t c[kMaxShards];
  for (uint32_t d = threadIdx.x; d < P; d += kRT) c[d] = 0;
  __syncthreads();
  for (uint64_t i = blockIdx.x * (uint64_t)kRT + threadIdx.x; i < n; i += (uint64_t)gridDim.x * kRT) {
    uint32_t d0, np;
    piece_span(f, lo[i], hi[i], &d0, &np);
    npieces[i] = np;
    for (uint32_t j = 0; j < np; ++j) atomicAdd(&c[d0 + j], 1u);
  }
  __syncthreads();
  for (uint32_t d = threadIdx.x; d < P; d += kRT)
    if (c[d]) atomicAdd(dcount + d, c[d]);
}

// dest-major slots: cursor[d] starts at the exclusive prefix of dcount; order inside a run is
// unspecified (each piece carries its id)
__global__ void __launch_bounds__(kRT) k_split_emit(BucketSplit f, uint32_t P, const uint64_t* __restrict__ lo,
                                                    const uint64_t* __restrict__ hi, uint64_t n,
                                                    const uint32_t* __restrict__ pbase,
                                                    uint32_t* __restrict__ cursor, uint64_t* __restrict__ plo,
                                                    uint64_t* __restrict__ phi, uint32_t* __restrict__ pid) {
  for (uint64_t i = blockIdx.x * (uint64_t)kRT + threadIdx.x; i < n; i += (uint64_t)gridDim.x * kRT) {
    const uint64_t l = lo[i], h = hi[i];
    uint32_t d0, np;
    piece_span(f, l, h, &d0, &np);
    for (uint32_t j = 0; j < np; ++j) {
      const uint32_t d = d0 + j;
      const uint32_t slot = atomicAdd(cursor + d, 1u);
      uint64_t a = l, b = h;
      if (l <= h) {
        if (j > 0) a = f.split[d - 1];                // sigma_d
        if (j + 1 < np) b = f.split[d] - 1;           // sigma_{d+1} - 1 (splitter keys go up)
      }
      plo[slot] = a;
      phi[slot] = b;
      pid[slot] = pbase[i] + j;
    }
  }
}

__global__ void k_excl_cursor(const uint32_t* __restrict__ dcount, uint32_t P, uint32_t* __restrict__ cursor) {
  if (threadIdx.x == 0 && blockIdx.x == 0) {
    uint32_t s = 0;
    for (uint32_t d = 0; d < P; ++d) {
      cursor[d] = s;
      s += dcount[d];
    }
  }
}

// answers arrive in routed (dest-major) order: row_of[pid[r]] = r
__global__ void k_piece_rows(const uint32_t* __restrict__ pid, uint64_t m, uint32_t* __restrict__ row_of) {
  for (uint64_t r = blockIdx.x * (uint64_t)kRT + threadIdx.x; r < m; r += (uint64_t)gridDim.x * kRT)
    row_of[pid[r]] = (uint32_t)r;
}

// one warp per range: walk its pieces in shard order, copy records until cap, sum counts
__global__ void __launch_bounds__(kRT) k_assemble(uint64_t n, uint32_t cap, const uint32_t* __restrict__ pbase,
                                                  const uint32_t* __restrict__ row_of,
                                                  const uint32_t* __restrict__ cnt, const uint64_t* __restrict__ rk,
                                                  const uint64_t* __restrict__ rv, uint64_t* __restrict__ ko,
                                                  uint64_t* __restrict__ vo, uint64_t* __restrict__ total) {
  const unsigned lane = threadIdx.x & 31;
  const uint64_t warps = (uint64_t)gridDim.x * (kRT / 32);
  for (uint64_t i = (blockIdx.x * (uint64_t)kRT + threadIdx.x) >> 5; i < n; i += warps) {
    uint64_t filled = 0, tot = 0;
    for (uint32_t p = pbase[i]; p < pbase[i + 1]; ++p) {
      const uint32_t r = row_of[p];
      const uint64_t c = cnt[r];
      tot += c;
      const uint64_t take = filled < cap ? std::min<uint64_t>(c, cap - filled) : 0;
      for (uint64_t t = lane; t < take; t += 32) {
        ko[i * cap + filled + t] = rk[(uint64_t)r * cap + t];
        vo[i * cap + filled + t] = rv[(uint64_t)r * cap + t];
      }
      filled += take;
    }
    if (lane == 0) total[i] = tot;
  }
}

int grid_for(uint64_t n) {
  int dev = 0, sm = 148;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sm, cudaDevAttrMultiProcessorCount, dev);
  return (int)std::max<uint64_t>(1, std::min<uint64_t>(ceil_div(n, kRT), (uint64_t)sm * 8));
}

size_t scan_bytes(uint64_t n) {
  size_t b = 0;
  cub::DeviceScan::ExclusiveSum(nullptr, b, (const uint32_t*)nullptr, (uint32_t*)nullptr,
                                (int)std::max<uint64_t>(n + 1, 1));
  return b;
}

}  // namespace
}  // namespace hm

using namespace hm;

extern "C" size_t harmonia_range_split_workspace_bytes(uint64_t n) {
  return round_up(scan_bytes(n), 256) + 2 * kMaxShards * 4 + 256;
}

extern "C" harmonia_status harmonia_range_split_count(const uint64_t* d_split, uint32_t P, const uint64_t* d_lo,
                                                      const uint64_t* d_hi, uint64_t n, uint32_t* d_npieces,
                                                      uint32_t* d_pbase, uint64_t* h_counts, uint64_t* h_total,
                                                      void* ws, size_t ws_bytes, void* stream) {
  if (P == 0 || P > kMaxShards || (P > 1 && !d_split) || !h_counts || !h_total || n >= (1ull << 31))
    return HARMONIA_ERR_INVALID_ARG;
  for (uint32_t d = 0; d < P; ++d) h_counts[d] = 0;
  *h_total = 0;
  if (n == 0) return HARMONIA_OK;
  if (!d_lo || !d_hi || !d_npieces || !d_pbase || !ws || ws_bytes < harmonia_range_split_workspace_bytes(n))
    return HARMONIA_ERR_INVALID_ARG;
  cudaStream_t st = (cudaStream_t)stream;
  char* base = (char*)ws;
  if ((uintptr_t)base & 255) base += 256 - ((uintptr_t)base & 255);
  uint32_t* dcount = (uint32_t*)base;
  char* cubt = base + 2 * kMaxShards * 4;
  const BucketSplit f{d_split, P - 1};
  HM_CUDA(cudaMemsetAsync(dcount, 0, P * 4, st));
  HM_CUDA(cudaMemsetAsync(d_npieces + n, 0, 4, st));
  k_split_count<<<grid_for(n), kRT, 0, st>>>(f, P, d_lo, d_hi, n, d_npieces, dcount);
  HM_LAUNCHED();
  size_t cb = scan_bytes(n);
  HM_CUDA(cub::DeviceScan::ExclusiveSum(cubt, cb, d_npieces, d_pbase, (int)(n + 1), st));
  count_launch(2);
  uint32_t hc[kMaxShards], tot = 0;
  HM_CUDA(cudaMemcpyAsync(hc, dcount, P * 4, cudaMemcpyDeviceToHost, st));
  HM_CUDA(cudaMemcpyAsync(&tot, d_pbase + n, 4, cudaMemcpyDeviceToHost, st));
  HM_CUDA(cudaStreamSynchronize(st));
  for (uint32_t d = 0; d < P; ++d) h_counts[d] = hc[d];
  *h_total = tot;
  return HARMONIA_OK;
}

extern "C" harmonia_status harmonia_range_split_emit(const uint64_t* d_split, uint32_t P, const uint64_t* d_lo,
                                                     const uint64_t* d_hi, uint64_t n, const uint32_t* d_pbase,
                                                     uint64_t* d_plo, uint64_t* d_phi, uint32_t* d_pid, void* ws,
                                                     size_t ws_bytes, void* stream) {
  if (P == 0 || P > kMaxShards || (P > 1 && !d_split) || n >= (1ull << 31)) return HARMONIA_ERR_INVALID_ARG;
  if (n == 0) return HARMONIA_OK;
  if (!d_lo || !d_hi || !d_pbase || !d_plo || !d_phi || !d_pid || !ws ||
      ws_bytes < harmonia_range_split_workspace_bytes(n))
    return HARMONIA_ERR_INVALID_ARG;
  cudaStream_t st = (cudaStream_t)stream;
  char* base = (char*)ws;
  if ((uintptr_t)base & 255) base += 256 - ((uintptr_t)base & 255);
  uint32_t* dcount = (uint32_t*)base;  // from harmonia_range_split_count on this workspace
  uint32_t* cursor = dcount + kMaxShards;
  k_excl_cursor<<<1, 32, 0, st>>>(dcount, P, cursor);
  HM_LAUNCHED();
  k_split_emit<<<grid_for(n), kRT, 0, st>>>(BucketSplit{d_split, P - 1}, P, d_lo, d_hi, n, d_pbase, cursor, d_plo,
                                           d_phi, d_pid);
  HM_LAUNCHED();
  return HARMONIA_OK;
}

extern "C" harmonia_status harmonia_range_assemble(uint64_t n, uint32_t cap, const uint32_t* d_pbase,
                                                   const uint32_t* d_pid, uint64_t m, const uint32_t* d_counts,
                                                   const uint64_t* d_keys, const uint64_t* d_values,
                                                   uint32_t* d_row_scratch, uint64_t* d_keys_out,
                                                   uint64_t* d_values_out, uint64_t* d_total_out, void* stream) {
  if (n == 0) return HARMONIA_OK;
  if (!d_pbase || !d_total_out || (m && (!d_pid || !d_counts || !d_row_scratch)) ||
      (cap && m && (!d_keys || !d_values)) || (cap && (!d_keys_out || !d_values_out)) || m >= (1ull << 32))
    return HARMONIA_ERR_INVALID_ARG;
  cudaStream_t st = (cudaStream_t)stream;
  if (m) {
    k_piece_rows<<<grid_for(m), kRT, 0, st>>>(d_pid, m, d_row_scratch);
    HM_LAUNCHED();
  }
  k_assemble<<<grid_for(n * 32), kRT, 0, st>>>(n, cap, d_pbase, d_row_scratch, d_counts, d_keys, d_values,
                                                d_keys_out, d_values_out, d_total_out);
  HM_LAUNCHED();
  return HARMONIA_OK;
}
