// Two-level partially-sorted aggregation (default PSA path).
//
// "the queries will be sorted based on their most significant N bits", N from
// Eq 2.  On sm_100a a one-pass partition over 2^N buckets costs one global atomic per query
// and shared-memory atomics cost ~2 cycles per lane, so the N-bit order is built in two
// atomic-free levels:
//   level 1  coarse MSB partition of the PSA window on the top kCoarseBits bits of the
//            N-bit bucket: warp multisplit by ballots (rank = popc(peers & lanemask_lt)),
//            per-warp counters, one global atomic per (tile, bin), tile staged in shared
//            memory so that every bin's run is written with consecutive lanes;
//   level 2  every kChunk-sized chunk of that order is sorted by its full N-bit bucket
//            (offset by the chunk minimum, capped at kLocalBits bits) with two stable LSD
//            passes of the same ballot multisplit, entirely in shared memory.
// The result orders each chunk by the top-N bits and the chunks by the top-8 bits, which is
// the paper's partial sort at chunk granularity; order inside a bucket is free (C-A12).
#include <algorithm>

#include "common.cuh"

namespace hm {

namespace {

constexpr int kCoarseBits = 8, kCoarseBins = 1 << kCoarseBits;
constexpr int kWarps = kBlock / 32;                      // 8 warps per 256-thread CTA
constexpr int kBatches = 8;                              // 32-query batches per warp per tile
constexpr int kCoarseTile = kBlock * kBatches;           // 2048 queries per scatter tile
#ifndef HM_SORT_THREADS
#define HM_SORT_THREADS 512
#endif
constexpr int kSortThreads = HM_SORT_THREADS, kSortWarps = kSortThreads / 32;
constexpr int kChunk = kSortThreads * kBatches;          // 4096 queries per local-sort chunk
constexpr int kLocalBits = 11, kLoBits = 6, kHiBits = kLocalBits - kLoBits;
constexpr size_t kSortSmem = (size_t)kChunk * (8 + 4 + 2);  // keys, positions, local digits

__device__ __forceinline__ unsigned lane_lt() {
  unsigned m;
  asm("mov.u32 %0, %%lanemask_lt;" : "=r"(m));
  return m;
}

// lanes of the warp whose digit equals mine (BITS-bit digits), restricted to `valid`
template <int BITS>
__device__ __forceinline__ unsigned peers_of(uint32_t d, unsigned valid) {
#ifndef HARMONIA_MATCH_ANY  // measured: BITS ballots beat one MATCH.ANY on sm_100a
  unsigned m = valid;
#pragma unroll
  for (int b = 0; b < BITS; ++b) {
    const bool bit = (d >> b) & 1u;
    const unsigned bb = __ballot_sync(kFull, bit);
    m &= bit ? bb : ~bb;
  }
  return m;
#else
  return __match_any_sync(kFull, d) & valid;  // one MATCH.ANY instead of BITS ballots
#endif
}

// exclusive scan of one value per thread (NT threads); `tmp` needs NT/32 + 1 words
template <int NT>
__device__ __forceinline__ uint32_t block_scan(uint32_t v, uint32_t* tmp, uint32_t* total) {
  const unsigned lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  uint32_t inc = v;
#pragma unroll
  for (int d = 1; d < 32; d <<= 1) {
    const uint32_t y = __shfl_up_sync(kFull, inc, d);
    if (lane >= (unsigned)d) inc += y;
  }
  if (lane == 31) tmp[warp] = inc;
  __syncthreads();
  if (warp == 0) {
    const uint32_t w = lane < NT / 32 ? tmp[lane] : 0;
    uint32_t wi = w;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
      const uint32_t y = __shfl_up_sync(kFull, wi, d);
      if (lane >= (unsigned)d) wi += y;
    }
    if (lane < NT / 32) tmp[lane] = wi - w;
    if (lane == 31) tmp[NT / 32] = wi;
  }
  __syncthreads();
  const uint32_t r = tmp[warp] + inc - v;
  if (total) *total = tmp[NT / 32];
  __syncthreads();
  return r;
}

// coarse digit of the PSA bucket (top kCoarseBits of the Nb-bit bucket)
struct CoarseDigit {
  BucketBits f;
  uint32_t shift;
  __device__ __forceinline__ uint32_t operator()(uint64_t q) const { return f(q) >> shift; }
};

// ---- level 1: histogram of the coarse digit ------------------------------------------
// Digit: any functor mapping a query to [0, kCoarseBins) (PSA coarse digit, or the
// destination shard of the partitioned multi-GPU mode).
template <class Digit>
__global__ void __launch_bounds__(kBlock) k_psa2_hist(const uint64_t* __restrict__ q, uint64_t n, Digit dg,
                                                      uint32_t* __restrict__ counts) {
  __shared__ uint32_t wh[kWarps][kCoarseBins];
  const unsigned lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  for (int i = threadIdx.x; i < kWarps * kCoarseBins; i += kBlock) (&wh[0][0])[i] = 0;
  __syncthreads();
  // tiles of kBatches x 32 queries per warp, all loads issued before the multisplit so that
  // each thread keeps kBatches loads in flight
  const uint64_t per_warp_tile = 32 * kBatches;
  const uint64_t gw = (blockIdx.x * (uint64_t)kBlock + threadIdx.x) >> 5;
  const uint64_t nw = ((uint64_t)gridDim.x * kBlock) >> 5;
  for (uint64_t t0 = gw * per_warp_tile; t0 < n; t0 += nw * per_warp_tile) {
    uint64_t v[kBatches];
#pragma unroll
    for (int k = 0; k < kBatches; ++k) {
      const uint64_t i = t0 + k * 32 + lane;
      v[k] = i < n ? __ldg(q + i) : 0;
    }
#pragma unroll
    for (int k = 0; k < kBatches; ++k) {
      const bool valid = t0 + k * 32 + lane < n;
      const uint32_t d = valid ? dg(v[k]) : 0u;
      const unsigned peers = peers_of<kCoarseBits>(d, __ballot_sync(kFull, valid));
      if (valid && lane == (unsigned)(__ffs(peers) - 1)) wh[warp][d] += __popc(peers);
      __syncwarp();
    }
  }
  __syncthreads();
  uint32_t c = 0;
#pragma unroll
  for (int w = 0; w < kWarps; ++w) c += wh[w][threadIdx.x];
  if (c) atomicAdd(counts + threadIdx.x, c);
}

// ---- level 1: coarse scatter ------------------------------------------------------------
template <class Digit>
__global__ void __launch_bounds__(kBlock) k_psa2_scatter(const uint64_t* __restrict__ q, uint64_t n, Digit dg,
                                                         const uint32_t* __restrict__ counts,
                                                         uint32_t* __restrict__ cursor, uint64_t* __restrict__ sorted_q,
                                                         uint32_t* __restrict__ idx) {
  __shared__ uint32_t wcnt[kWarps][kCoarseBins];
  __shared__ uint32_t prefix[kCoarseBins], bin_start[kCoarseBins], gbase[kCoarseBins], tmp[kWarps + 1];
  __shared__ uint64_t st_q[kCoarseTile];
  __shared__ uint32_t st_i[kCoarseTile];
  __shared__ uint8_t st_d[kCoarseTile];
  const unsigned lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  prefix[threadIdx.x] = block_scan<kBlock>(counts[threadIdx.x], tmp, nullptr);
  for (uint64_t t0 = (uint64_t)blockIdx.x * kCoarseTile; t0 < n; t0 += (uint64_t)gridDim.x * kCoarseTile) {
    for (int i = threadIdx.x; i < kWarps * kCoarseBins; i += kBlock) (&wcnt[0][0])[i] = 0;
    __syncthreads();
    uint64_t v[kBatches];
    uint32_t d[kBatches], pos[kBatches];
#pragma unroll
    for (int k = 0; k < kBatches; ++k) {  // all loads first (kBatches in flight per thread)
      const uint64_t e = t0 + warp * (32 * kBatches) + k * 32 + lane;
      v[k] = e < n ? __ldg(q + e) : 0;
    }
#pragma unroll
    for (int k = 0; k < kBatches; ++k) {
      const uint64_t e = t0 + warp * (32 * kBatches) + k * 32 + lane;
      const bool valid = e < n;
      d[k] = valid ? dg(v[k]) : 0u;
      const unsigned peers = peers_of<kCoarseBits>(d[k], __ballot_sync(kFull, valid));
      const uint32_t run = valid ? wcnt[warp][d[k]] : 0u;
      __syncwarp();
      if (valid && lane == (unsigned)(__ffs(peers) - 1)) wcnt[warp][d[k]] = run + __popc(peers);
      __syncwarp();
      pos[k] = run + __popc(peers & lane_lt());
    }
    __syncthreads();
    // per bin: offsets of each warp's run, tile total, tile-local start, global reservation
    uint32_t acc = 0;
#pragma unroll
    for (int w = 0; w < kWarps; ++w) {
      const uint32_t c = wcnt[w][threadIdx.x];
      wcnt[w][threadIdx.x] = acc;
      acc += c;
    }
    const uint32_t tile_n = (uint32_t)std::min<uint64_t>(kCoarseTile, n - t0);
    bin_start[threadIdx.x] = block_scan<kBlock>(acc, tmp, nullptr);
    if (acc) gbase[threadIdx.x] = prefix[threadIdx.x] + atomicAdd(cursor + threadIdx.x, acc);
    __syncthreads();
#pragma unroll
    for (int k = 0; k < kBatches; ++k) {
      const uint64_t e = t0 + warp * (32 * kBatches) + k * 32 + lane;
      if (e < n) {
        const uint32_t lp = bin_start[d[k]] + wcnt[warp][d[k]] + pos[k];
        st_q[lp] = v[k];
        st_i[lp] = (uint32_t)e;
        st_d[lp] = (uint8_t)d[k];
      }
    }
    __syncthreads();
    for (uint32_t i = threadIdx.x; i < tile_n; i += kBlock) {  // runs written by consecutive lanes
      const uint32_t dd = st_d[i];
      const uint32_t dst = gbase[dd] + (i - bin_start[dd]);
      sorted_q[dst] = st_q[i];
      idx[dst] = st_i[i];
    }
    __syncthreads();
  }
}

// ---- level 2: chunk-local sort by the N-bit bucket (two stable LSD passes) ---------------
template <int BITS, int SHIFT>
__device__ __forceinline__ void lsd_pass(uint64_t (&v)[kBatches], uint32_t (&ix)[kBatches], uint32_t (&lk)[kBatches],
                                         uint32_t m, uint32_t (*wcnt)[1 << kLoBits], uint32_t* bin_start, uint32_t* tmp,
                                         uint64_t* s_q, uint32_t* s_i, uint16_t* s_k) {
  constexpr int NB = 1 << BITS;
  const unsigned lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  for (int i = threadIdx.x; i < kSortWarps * NB; i += kSortThreads) wcnt[i / NB][i % NB] = 0;
  __syncthreads();
  uint32_t pos[kBatches], dg[kBatches];
#pragma unroll
  for (int k = 0; k < kBatches; ++k) {  // element order = (warp, batch, lane): stable ranks
    const uint32_t e = warp * (32 * kBatches) + k * 32 + lane;
    const bool valid = e < m;
    dg[k] = (lk[k] >> SHIFT) & (NB - 1);
    const unsigned peers = peers_of<BITS>(dg[k], __ballot_sync(kFull, valid));
    const uint32_t run = valid ? wcnt[warp][dg[k]] : 0u;
    __syncwarp();
    if (valid && lane == (unsigned)(__ffs(peers) - 1)) wcnt[warp][dg[k]] = run + __popc(peers);
    __syncwarp();
    pos[k] = run + __popc(peers & lane_lt());
  }
  __syncthreads();
  uint32_t acc = 0;
  if (threadIdx.x < NB) {
#pragma unroll
    for (int w = 0; w < kSortWarps; ++w) {
      const uint32_t c = wcnt[w][threadIdx.x];
      wcnt[w][threadIdx.x] = acc;
      acc += c;
    }
  }
  const uint32_t bs = block_scan<kSortThreads>(threadIdx.x < NB ? acc : 0u, tmp, nullptr);
  if (threadIdx.x < NB) bin_start[threadIdx.x] = bs;
  __syncthreads();
#pragma unroll
  for (int k = 0; k < kBatches; ++k) {
    const uint32_t e = warp * (32 * kBatches) + k * 32 + lane;
    if (e < m) {
      const uint32_t dst = bin_start[dg[k]] + wcnt[warp][dg[k]] + pos[k];
      s_q[dst] = v[k];
      s_i[dst] = ix[k];
      s_k[dst] = (uint16_t)lk[k];
    }
  }
  __syncthreads();
#pragma unroll
  for (int k = 0; k < kBatches; ++k) {  // reload in the new order for the next pass
    const uint32_t e = warp * (32 * kBatches) + k * 32 + lane;
    if (e < m) {
      v[k] = s_q[e];
      ix[k] = s_i[e];
      lk[k] = s_k[e];
    }
  }
  __syncthreads();
}

__global__ void __launch_bounds__(kSortThreads, 2) k_psa2_local_sort(uint64_t* __restrict__ sorted_q,
                                                                  uint32_t* __restrict__ idx, uint64_t n, BucketBits f) {
  extern __shared__ __align__(16) unsigned char sm[];
  uint64_t* s_q = reinterpret_cast<uint64_t*>(sm);
  uint32_t* s_i = reinterpret_cast<uint32_t*>(sm + kChunk * 8);
  uint16_t* s_k = reinterpret_cast<uint16_t*>(sm + kChunk * 12);
  __shared__ uint32_t wcnt[kSortWarps][1 << kLoBits];
  __shared__ uint32_t bin_start[1 << kLoBits], tmp[kSortWarps + 1], s_mm[2][kSortWarps];
  const unsigned lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  for (uint64_t c0 = (uint64_t)blockIdx.x * kChunk; c0 < n; c0 += (uint64_t)gridDim.x * kChunk) {
    const uint32_t m = (uint32_t)std::min<uint64_t>(kChunk, n - c0);
    uint64_t v[kBatches];
    uint32_t ix[kBatches], lk[kBatches];
    uint32_t bmin = 0xFFFFFFFFu, bmax = 0;
#pragma unroll
    for (int k = 0; k < kBatches; ++k) {
      const uint32_t e = warp * (32 * kBatches) + k * 32 + lane;
      if (e < m) {
        v[k] = sorted_q[c0 + e];
        ix[k] = idx[c0 + e];
        lk[k] = f(v[k]);
        bmin = min(bmin, lk[k]);
        bmax = max(bmax, lk[k]);
      } else {
        v[k] = 0;
        ix[k] = 0;
        lk[k] = 0;
      }
    }
    bmin = __reduce_min_sync(kFull, bmin);
    bmax = __reduce_max_sync(kFull, bmax);
    if (lane == 0) {
      s_mm[0][warp] = bmin;
      s_mm[1][warp] = bmax;
    }
    __syncthreads();
#pragma unroll
    for (int w = 0; w < kSortWarps; ++w) {
      bmin = min(bmin, s_mm[0][w]);
      bmax = max(bmax, s_mm[1][w]);
    }
    uint32_t sh = 0;
    while (((bmax - bmin) >> sh) >= (1u << kLocalBits)) ++sh;
#pragma unroll
    for (int k = 0; k < kBatches; ++k) lk[k] = (lk[k] - bmin) >> sh;
    lsd_pass<kLoBits, 0>(v, ix, lk, m, wcnt, bin_start, tmp, s_q, s_i, s_k);
    lsd_pass<kHiBits, kLoBits>(v, ix, lk, m, wcnt, bin_start, tmp, s_q, s_i, s_k);
#pragma unroll
    for (int k = 0; k < kBatches; ++k) {  // write back (coalesced)
      const uint32_t e = warp * (32 * kBatches) + k * 32 + lane;
      if (e < m) {
        sorted_q[c0 + e] = v[k];
        idx[c0 + e] = ix[k];
      }
    }
  }
}

constexpr int kLocalBins = 1 << kLocalBits;
constexpr size_t kCountSortSmem = (size_t)kLocalBins * 4 + (size_t)kChunk * 12;
#include "psa2_count_sort.inc"

// level-1 partition by any <= 256-bin digit: histogram, then the staged scatter.
// h_counts (optional) receives the first `nbins` bin counts synchronously.
template <class Digit>
harmonia_status coarse_partition(const uint64_t* q, uint64_t n, const Digit& dg, uint32_t* counts,
                                 uint64_t* sorted_q, uint32_t* idx, int sm, cudaStream_t st, uint64_t* h_counts,
                                 uint32_t nbins) {
  HM_CUDA(cudaMemsetAsync(counts, 0, 2 * kCoarseBins * 4, st));
  {
    ProfScope ps_(HARMONIA_PROF_PSA_HIST, st);
    const int g = (int)std::min<uint64_t>(ceil_div(n, kBlock * 8), (uint64_t)sm * 8);
    k_psa2_hist<Digit><<<std::max(g, 1), kBlock, 0, st>>>(q, n, dg, counts);
  }
  HM_LAUNCHED();
  if (h_counts) {
    uint32_t tmp[kCoarseBins];
    HM_CUDA(cudaMemcpyAsync(tmp, counts, nbins * 4, cudaMemcpyDeviceToHost, st));
    HM_CUDA(cudaStreamSynchronize(st));
    for (uint32_t b = 0; b < nbins; ++b) h_counts[b] = tmp[b];
  }
  {
    ProfScope ps_(HARMONIA_PROF_PSA_SCATTER, st);
    const int g = (int)std::min<uint64_t>(ceil_div(n, kCoarseTile), (uint64_t)sm * 4);
    k_psa2_scatter<Digit><<<std::max(g, 1), kBlock, 0, st>>>(q, n, dg, counts, counts + kCoarseBins, sorted_q, idx);
  }
  HM_LAUNCHED();
  return HARMONIA_OK;
}

}  // namespace

// multi-GPU router: destination-major grouping by splitters (P <= 256 shards)
harmonia_status route_partition2(const uint64_t* q, uint64_t n, const BucketSplit& f, uint32_t P, uint32_t* counts,
                                 uint64_t* routed, uint32_t* pos, int sm, cudaStream_t st, uint64_t* h_counts) {
  if (P > (uint32_t)kCoarseBins) return HARMONIA_ERR_INVALID_ARG;
  return coarse_partition(q, n, f, counts, routed, pos, sm, st, h_counts, P);
}

harmonia_status psa_partition2(const uint64_t* q, uint64_t n, const BucketBits& f, int nb, const PsaWs& ws, int sm,
                               cudaStream_t st, int level2) {
  const uint32_t b1 = (uint32_t)std::min(nb, kCoarseBits);
  const uint32_t shift1 = (uint32_t)nb - b1;
  harmonia_status s = coarse_partition(q, n, CoarseDigit{f, shift1}, ws.counts, ws.sorted_q, ws.idx, sm, st, nullptr, 0);
  if (s != HARMONIA_OK) return s;
  if (level2 == 2) return HARMONIA_OK;  // coarse partition only (ablation)
  {
    ProfScope ps_(HARMONIA_PROF_PSA_SCAN, st);  // reported in the "scan" class: level-2 sort
    static bool configured = false;
    if (!configured) {
      HM_CUDA(cudaFuncSetAttribute(k_psa2_local_sort, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kSortSmem));
      HM_CUDA(cudaFuncSetAttribute(k_psa2_count_sort, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                   (int)kCountSortSmem));
      configured = true;
    }
    const int g = (int)std::min<uint64_t>(ceil_div(n, kChunk), (uint64_t)sm * 4);
    if (level2 == 1)  // two stable LSD passes of ballot multisplit (ablation)
      k_psa2_local_sort<<<std::max(g, 1), kSortThreads, kSortSmem, st>>>(ws.sorted_q, ws.idx, n, f);
    else              // one counting pass with shared-memory atomics (default, measured faster)
      k_psa2_count_sort<<<std::max(g, 1), kSortThreads, kCountSortSmem, st>>>(ws.sorted_q, ws.idx, n, f);
  }
  HM_LAUNCHED();
  return HARMONIA_OK;
}

}  // namespace hm
