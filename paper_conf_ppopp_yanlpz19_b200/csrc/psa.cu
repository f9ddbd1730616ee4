// Partially-sorted aggregation (PSA, §4.1) on sm_100a.
//
// "the queries will be sorted based on their most significant N bits"; Eq 2 picks
// N = log2(T/K).  The sort is a one-pass MSB bucket partition of a query
// window (the paper's "time window"):
//   psa_histogram   counts per bucket (warp-aggregated with match.any, then one global
//                   atomic per distinct bucket per warp)
//   psa_scan        exclusive scan of the counts (reduce pass + apply pass)
//   psa_scatter     sorted_q[dst] = q, idx[dst] = original position; dst = bucket offset +
//                   rank among the warp's equal-bucket lanes (one atomic per warp-bucket)
// Order inside a bucket is not specified (C-A12): results do not depend on it because each
// query carries its original position and the search kernel writes out[idx] directly.
// The same partition with a splitter-based bucket routes queries to shards (multi-GPU).
#include <algorithm>

#include "common.cuh"

namespace hm {

namespace {

__device__ __forceinline__ unsigned lanemask_lt() {
  unsigned m;
  asm("mov.u32 %0, %%lanemask_lt;" : "=r"(m));
  return m;
}

template <class Bucket>
__global__ void __launch_bounds__(kBlock) k_psa_histogram(const uint64_t* __restrict__ q, uint64_t n,
                                                          Bucket f, uint32_t* __restrict__ counts) {
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  const uint64_t n_round = round_up_dev(n);
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n_round; i += stride) {
    const bool act = i < n;
    const uint32_t b = act ? f(__ldg(q + i)) : 0xFFFFFFFFu;
    const unsigned peers = __match_any_sync(kFull, b);
    if (act && (threadIdx.x & 31) == (unsigned)(__ffs(peers) - 1)) atomicAdd(counts + b, __popc(peers));
  }
}

template <class Bucket>
__global__ void __launch_bounds__(kBlock) k_psa_scatter(const uint64_t* __restrict__ q, uint64_t n,
                                                        Bucket f, uint32_t* __restrict__ offs,
                                                        uint64_t* __restrict__ sorted_q,
                                                        uint32_t* __restrict__ idx) {
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  const uint64_t n_round = round_up_dev(n);
  const unsigned lane = threadIdx.x & 31;
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n_round; i += stride) {
    const bool act = i < n;
    const uint64_t qv = act ? __ldg(q + i) : 0;
    const uint32_t b = act ? f(qv) : 0xFFFFFFFFu;
    const unsigned peers = __match_any_sync(kFull, b);
    const int leader = __ffs(peers) - 1;
    uint32_t base = 0;
    if (act && lane == (unsigned)leader) base = atomicAdd(offs + b, __popc(peers));
    base = __shfl_sync(kFull, base, leader);
    if (act) {
      const uint32_t dst = base + __popc(peers & lanemask_lt());
      sorted_q[dst] = qv;
      idx[dst] = (uint32_t)i;
    }
  }
}

// exclusive scan over nbins counters, tiles of kScanTile = 4096 (1024 threads x 4)
__global__ void __launch_bounds__(1024) k_scan_reduce(const uint32_t* __restrict__ counts, uint32_t nbins,
                                                      uint32_t* __restrict__ tile_sums) {
  __shared__ uint32_t warp_sums[32];
  const uint32_t base = blockIdx.x * kScanTile + threadIdx.x * 4;
  uint32_t s = 0;
#pragma unroll
  for (int k = 0; k < 4; ++k) s += (base + k < nbins) ? counts[base + k] : 0;
  s = __reduce_add_sync(kFull, s);
  if ((threadIdx.x & 31) == 0) warp_sums[threadIdx.x >> 5] = s;
  __syncthreads();
  if (threadIdx.x < 32) {
    uint32_t w = warp_sums[threadIdx.x];
    w = __reduce_add_sync(kFull, w);
    if (threadIdx.x == 0) tile_sums[blockIdx.x] = w;
  }
}

__global__ void __launch_bounds__(1024) k_scan_apply(uint32_t* __restrict__ counts, uint32_t nbins,
                                                     const uint32_t* __restrict__ tile_sums) {
  __shared__ uint32_t warp_sums[32];
  __shared__ uint32_t tile_prefix;
  const unsigned lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  // prefix of the tiles before this one
  uint32_t p = 0;
  for (uint32_t t = threadIdx.x; t < blockIdx.x; t += blockDim.x) p += tile_sums[t];
  p = __reduce_add_sync(kFull, p);
  if (lane == 0) warp_sums[warp] = p;
  __syncthreads();
  if (threadIdx.x < 32) {
    uint32_t w = __reduce_add_sync(kFull, warp_sums[threadIdx.x]);
    if (threadIdx.x == 0) tile_prefix = w;
  }
  __syncthreads();
  const uint32_t base = blockIdx.x * kScanTile + threadIdx.x * 4;
  uint32_t v[4];
  uint32_t s = 0;
#pragma unroll
  for (int k = 0; k < 4; ++k) {
    v[k] = (base + k < nbins) ? counts[base + k] : 0;
    s += v[k];
  }
  // inclusive warp scan of the per-thread sums
  uint32_t inc = s;
#pragma unroll
  for (int d = 1; d < 32; d <<= 1) {
    uint32_t y = __shfl_up_sync(kFull, inc, d);
    if (lane >= (unsigned)d) inc += y;
  }
  __syncthreads();  // warp_sums reuse
  if (lane == 31) warp_sums[warp] = inc;
  __syncthreads();
  if (warp == 0) {
    uint32_t w = warp_sums[lane];
    uint32_t wi = w;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
      uint32_t y = __shfl_up_sync(kFull, wi, d);
      if (lane >= (unsigned)d) wi += y;
    }
    warp_sums[lane] = wi - w;  // exclusive prefix of warps
  }
  __syncthreads();
  uint32_t run = tile_prefix + warp_sums[warp] + (inc - s);
#pragma unroll
  for (int k = 0; k < 4; ++k) {
    if (base + k < nbins) counts[base + k] = run;
    run += v[k];
  }
}

__global__ void __launch_bounds__(kBlock) k_gather(const uint64_t* __restrict__ sorted_out,
                                                   const uint32_t* __restrict__ idx, uint64_t n,
                                                   uint64_t* __restrict__ out) {
  // out[idx[j]] = sorted_out[j] expressed as a scatter of the window (L2-resident)
  for (uint64_t j = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; j < n;
       j += (uint64_t)gridDim.x * blockDim.x)
    out[__ldg(idx + j)] = __ldg(sorted_out + j);
}

__global__ void __launch_bounds__(kBlock) k_scatter_back(const uint64_t* __restrict__ vals,
                                                         const uint32_t* __restrict__ pos, uint64_t n,
                                                         uint64_t* __restrict__ out) {
  for (uint64_t j = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; j < n;
       j += (uint64_t)gridDim.x * blockDim.x)
    out[__ldg(pos + j)] = __ldg(vals + j);
}

int stream_grid(uint64_t n, int sm) {
  uint64_t g = ceil_div(std::max<uint64_t>(n, 1), kBlock);
  return (int)std::min<uint64_t>(g, (uint64_t)sm * 8);
}

}  // namespace

size_t psa_ws_bytes(const Plan& p) {
  if (!p.psa) return 0;
  size_t b = round_up((size_t)std::max<uint32_t>(p.nbins, 512) * 4, 256);
  b += round_up(ceil_div(p.nbins, kScanTile) * 4, 256);
  b += round_up(p.window * 8, 256);
  b += round_up(p.window * 4, 256);
  if (p.gather || p.ret) b += round_up(p.window * 8, 256);
  b += round_up(p.window * 4, 256);                        // packed digit/rank
  b += round_up(l1_rows_bytes(p.window), 256);        // per-tile counts
  b += 2 * kL1CtaRows * 4;                             // per-CTA counts and bases
  if (p.psa_levels == 2) b += l2_ws_bytes(p.window, p.chunk);
  if (p.ret) b += round_up(cbounds_entries(p.window) * 8, 256);
  return b;
}

PsaWs psa_ws_carve(const Plan& p, void* base) {
  char* c = (char*)base;
  PsaWs w{};
  w.counts = (uint32_t*)c;
  c += round_up((size_t)std::max<uint32_t>(p.nbins, 512) * 4, 256);
  w.tile_sums = (uint32_t*)c;
  c += round_up(ceil_div(p.nbins, kScanTile) * 4, 256);
  w.sorted_q = (uint64_t*)c;
  c += round_up(p.window * 8, 256);
  w.idx = (uint32_t*)c;
  c += round_up(p.window * 4, 256);
  w.sorted_out = (p.gather || p.ret) ? (uint64_t*)c : nullptr;
  if (p.gather || p.ret) c += round_up(p.window * 8, 256);
  w.packed = (uint32_t*)c;
  c += round_up(p.window * 4, 256);
  w.tile_counts = (uint32_t*)c;
  c += round_up(l1_rows_bytes(p.window), 256);
  w.cta_counts = (uint32_t*)c;
  c += kL1CtaRows * 4;
  w.cta_base = (uint32_t*)c;
  c += kL1CtaRows * 4;
  if (p.ret) {
    w.cbounds = (uint2*)c;
    c += round_up(cbounds_entries(p.window) * 8, 256);
  }
  if (p.psa_levels == 2) {
    const L2Sizes z = l2_sizes(p.window, p.chunk);
    w.seg = (uint32_t*)c;
    c += round_up((2 * 257 + 3 * 64) * 4, 256);  // + the layout's CTA totals
    w.l2_scratch = (uint32_t*)c;
    c += round_up(3 * kL2Buckets * 4, 256);
    w.packed2 = (uint32_t*)c;
    c += round_up(p.window * 4, 256);
    w.tile_counts2 = (uint32_t*)c;
    c += round_up(z.tiles * 256 * 4, 256);
    w.tile_base2 = (uint32_t*)c;
    c += round_up(z.tiles * 256 * 4, 256);
    w.comp_cnt = (uint32_t*)c;
    c += round_up(kL2Buckets * 4, 256);
    w.comp_start = (uint32_t*)c;
    c += round_up((kL2Buckets + 1) * 4, 256);
    w.chunks = (uint2*)c;
    c += round_up(z.chunks * 8, 256);
    w.chunk_pos = (uint32_t*)c;
    c += round_up(z.chunks * 4, 256);
    w.nchunks = (uint32_t*)c;
    c += 256;
    w.sorted2 = (uint64_t*)c;
    c += round_up(z.padded * 8, 256);
    w.res2 = (uint64_t*)c;
    c += round_up(z.padded * 8, 256);
    w.idx = (uint32_t*)c;  // chunk-local offsets (uint16) at level-2 positions
  }
  return w;
}

template <class Bucket>
harmonia_status psa_partition(const uint64_t* q, uint64_t n, const Bucket& f, uint32_t nbins,
                              const PsaWs& ws, int sm, cudaStream_t st, uint64_t* h_counts) {
  HM_CUDA(cudaMemsetAsync(ws.counts, 0, (size_t)nbins * 4, st));
  const int g = stream_grid(n, sm);
  {
    ProfScope ps_(HARMONIA_PROF_PSA_HIST, st);
    k_psa_histogram<Bucket><<<g, kBlock, 0, st>>>(q, n, f, ws.counts);
  }
  HM_LAUNCHED();
  if (h_counts) {
    // small destination histogram for the multi-GPU router: read it back synchronously
    uint32_t tmp[1024];
    if (nbins > 1024) return HARMONIA_ERR_INVALID_ARG;
    HM_CUDA(cudaMemcpyAsync(tmp, ws.counts, nbins * 4, cudaMemcpyDeviceToHost, st));
    HM_CUDA(cudaStreamSynchronize(st));
    for (uint32_t b = 0; b < nbins; ++b) h_counts[b] = tmp[b];
  }
  const uint32_t tiles = (uint32_t)ceil_div(nbins, kScanTile);
  {
    ProfScope ps_(HARMONIA_PROF_PSA_SCAN, st);
    k_scan_reduce<<<tiles, 1024, 0, st>>>(ws.counts, nbins, ws.tile_sums);
    count_launch();
    k_scan_apply<<<tiles, 1024, 0, st>>>(ws.counts, nbins, ws.tile_sums);
  }
  HM_LAUNCHED();
  {
    ProfScope ps_(HARMONIA_PROF_PSA_SCATTER, st);
    k_psa_scatter<Bucket><<<g, kBlock, 0, st>>>(q, n, f, ws.counts, ws.sorted_q, ws.idx);
  }
  HM_LAUNCHED();
  return HARMONIA_OK;
}

template harmonia_status psa_partition<BucketBits>(const uint64_t*, uint64_t, const BucketBits&,
                                                   uint32_t, const PsaWs&, int, cudaStream_t,
                                                   uint64_t*);
template harmonia_status psa_partition<BucketSplit>(const uint64_t*, uint64_t, const BucketSplit&,
                                                    uint32_t, const PsaWs&, int, cudaStream_t,
                                                    uint64_t*);

harmonia_status launch_gather(const uint64_t* sorted_out, const uint32_t* idx, uint64_t n,
                              uint64_t* out, int sm, cudaStream_t st) {
  if (n == 0) return HARMONIA_OK;
  ProfScope ps_(HARMONIA_PROF_RETURN, st);
  k_gather<<<stream_grid(n, sm), kBlock, 0, st>>>(sorted_out, idx, n, out);
  HM_LAUNCHED();
  return HARMONIA_OK;
}

harmonia_status launch_scatter_back(const uint64_t* vals, const uint32_t* pos, uint64_t n,
                                    uint64_t* out, int sm, cudaStream_t st) {
  if (n == 0) return HARMONIA_OK;
  ProfScope ps_(HARMONIA_PROF_RETURN, st);
  k_scatter_back<<<stream_grid(n, sm), kBlock, 0, st>>>(vals, pos, n, out);
  HM_LAUNCHED();
  return HARMONIA_OK;
}

}  // namespace hm
