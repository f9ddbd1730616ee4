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

#include <type_traits>

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
static_assert(kCoarseTile == (int)kPsaTile && kChunk == (int)kPsaChunk, "tile sizes shared with search.cu");
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

// ---- level 1, pass 1: per-tile digit ranks ---------------------------------------------
// Tiles of kCoarseTile consecutive queries. Each query's coarse digit d and its rank among the
// tile's queries with digit d are taken once, with a shared-memory atomic, and stored packed
// (d | rank << 8) so that the move pass below needs no multisplit. Per-tile bin counts go to
// tile_counts[tile][256]; bin totals to counts[256] (one global atomic per tile and bin).
// Digit: any functor mapping a query to [0, kCoarseBins) (the PSA coarse digit, or the
// destination shard of the partitioned multi-GPU mode).
template <class Digit>
__global__ void __launch_bounds__(kBlock) k_psa2_rank(const uint64_t* __restrict__ q, uint64_t n, Digit dg,
                                                      uint32_t* __restrict__ counts,
                                                      uint32_t* __restrict__ tile_counts,
                                                      uint32_t* __restrict__ packed) {
#ifndef HARMONIA_RANK_BALLOT
  __shared__ uint32_t cnt[kCoarseBins];
  uint64_t v[kBatches];
#pragma unroll
  for (int k = 0; k < kBatches; ++k) {  // all loads first (kBatches in flight per thread)
    const uint64_t e = (uint64_t)blockIdx.x * kCoarseTile + k * kBlock + threadIdx.x;
    v[k] = e < n ? __ldg(q + e) : 0;
  }
  for (uint64_t tile = blockIdx.x; tile * kCoarseTile < n; tile += gridDim.x) {
    const uint64_t t0 = tile * kCoarseTile;
    cnt[threadIdx.x] = 0;
    __syncthreads();
#pragma unroll
    for (int k = 0; k < kBatches; ++k) {
      const uint64_t e = t0 + k * kBlock + threadIdx.x;
      if (e < n) {
        const uint32_t d = dg(v[k]);
        packed[e] = d | (atomicAdd(&cnt[d], 1u) << kCoarseBits);
      }
    }
    __syncthreads();
    const uint32_t c = cnt[threadIdx.x];
    tile_counts[tile * kCoarseBins + threadIdx.x] = c;
    if (c) atomicAdd(counts + threadIdx.x, c);
    __syncthreads();
#pragma unroll
    for (int k = 0; k < kBatches; ++k) {
      const uint64_t e = t0 + (uint64_t)gridDim.x * kCoarseTile + k * kBlock + threadIdx.x;
      v[k] = e < n ? __ldg(q + e) : 0;
    }
  }
#else  // ballot multisplit ranks (per-warp runs, then warp offsets per bin)
  __shared__ uint32_t wcnt[kWarps][kCoarseBins];
  const unsigned lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  for (uint64_t tile = blockIdx.x; tile * kCoarseTile < n; tile += gridDim.x) {
    const uint64_t t0 = tile * kCoarseTile;
    for (int i = threadIdx.x; i < kWarps * kCoarseBins; i += kBlock) (&wcnt[0][0])[i] = 0;
    __syncthreads();
    uint64_t v[kBatches];
    uint32_t d[kBatches], pos[kBatches];
#pragma unroll
    for (int k = 0; k < kBatches; ++k) {
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
    uint32_t acc = 0;
#pragma unroll
    for (int w = 0; w < kWarps; ++w) {
      const uint32_t c = wcnt[w][threadIdx.x];
      wcnt[w][threadIdx.x] = acc;
      acc += c;
    }
    tile_counts[tile * kCoarseBins + threadIdx.x] = acc;
    if (acc) atomicAdd(counts + threadIdx.x, acc);
    __syncthreads();
#pragma unroll
    for (int k = 0; k < kBatches; ++k) {
      const uint64_t e = t0 + warp * (32 * kBatches) + k * 32 + lane;
      if (e < n) packed[e] = d[k] | ((wcnt[warp][d[k]] + pos[k]) << kCoarseBits);
    }
    __syncthreads();
  }
#endif
}

// ---- level 1, pass 2: move ----------------------------------------------------------------
// Global position of query e = exclusive-prefix(counts)[d] + this tile's reservation in bin d
// (one atomic per tile and bin on cursor[d]) + rank. Staged through shared memory in bin order
// so that each bin's run is written by consecutive lanes. The scattered shared-memory stores
// are the kernel's limiter (ncu: shared-store wavefronts), so only the query is staged when the
// digit is cheap to recompute (the PSA coarse digit) and the position only when idx is wanted.
template <class Digit>
__global__ void __launch_bounds__(kBlock) k_psa2_move(const uint64_t* __restrict__ q, uint64_t n, Digit dg,
                                                      const uint32_t* __restrict__ counts,
                                                      uint32_t* __restrict__ cursor,
                                                      const uint32_t* __restrict__ tile_counts,
                                                      const uint32_t* __restrict__ packed,
                                                      uint64_t* __restrict__ sorted_q, uint32_t* __restrict__ idx,
                                                      uint32_t* __restrict__ tile_base) {
  constexpr bool kRecompute = std::is_same<Digit, CoarseDigit>::value;
  __shared__ uint32_t prefix[kCoarseBins], bin_start[kCoarseBins], gbase[kCoarseBins], tmp[kWarps + 1];
  __shared__ uint64_t st_q[kCoarseTile];
  __shared__ uint32_t st_i[kCoarseTile];
  __shared__ uint8_t st_d[kRecompute ? 1 : kCoarseTile];
  prefix[threadIdx.x] = block_scan<kBlock>(counts[threadIdx.x], tmp, nullptr);
  for (uint64_t tile = blockIdx.x; tile * kCoarseTile < n; tile += gridDim.x) {
    const uint64_t t0 = tile * kCoarseTile;
    uint64_t v[kBatches];
    uint32_t pk[kBatches];
#pragma unroll
    for (int k = 0; k < kBatches; ++k) {
      const uint64_t e = t0 + k * kBlock + threadIdx.x;
      v[k] = e < n ? __ldg(q + e) : 0;
      pk[k] = e < n ? __ldg(packed + e) : 0;
    }
    const uint32_t c = tile_counts[tile * kCoarseBins + threadIdx.x];
    bin_start[threadIdx.x] = block_scan<kBlock>(c, tmp, nullptr);
    const uint32_t gb = c ? prefix[threadIdx.x] + atomicAdd(cursor + threadIdx.x, c) : 0u;
    gbase[threadIdx.x] = gb;
    if (tile_base) tile_base[tile * kCoarseBins + threadIdx.x] = gb;  // for the staged return
    __syncthreads();
#pragma unroll
    for (int k = 0; k < kBatches; ++k) {
      const uint64_t e = t0 + k * kBlock + threadIdx.x;
      if (e < n) {
        const uint32_t d = pk[k] & (kCoarseBins - 1);
        const uint32_t lp = bin_start[d] + (pk[k] >> kCoarseBits);
        st_q[lp] = v[k];
        if (idx) st_i[lp] = (uint32_t)e;
        if constexpr (!kRecompute) st_d[lp] = (uint8_t)d;
      }
    }
    __syncthreads();
    const uint32_t tile_n = (uint32_t)std::min<uint64_t>(kCoarseTile, n - t0);
    for (uint32_t i = threadIdx.x; i < tile_n; i += kBlock) {  // runs written by consecutive lanes
      const uint64_t x = st_q[i];
      uint32_t dd;
      if constexpr (kRecompute) dd = dg(x);
      else dd = st_d[i];
      const uint32_t dst = gbase[dd] + (i - bin_start[dd]);
      sorted_q[dst] = x;
      if (idx) idx[dst] = st_i[i];
    }
    __syncthreads();
  }
}

// ---- staged return: inverse of the move -------------------------------------------------
// res1 holds the results in level-1 order. For the tile of original positions [t0, t0+2048)
// the slots of its (bin, rank) pairs are restaged exactly as in k_psa2_move; slot i of the
// tile's bin order sits at level-1 position tile_base[d] + (i - bin_start[d]), so res1 is read
// in runs and out[] written contiguously -- no scattered global access on either side.
__global__ void __launch_bounds__(kBlock) k_psa2_unmove(const uint32_t* __restrict__ tile_counts,
                                                        const uint32_t* __restrict__ tile_base,
                                                        const uint32_t* __restrict__ packed,
                                                        const uint64_t* __restrict__ res1, uint64_t n,
                                                        uint64_t* __restrict__ out) {
  __shared__ uint32_t bin_start[kCoarseBins], gbase[kCoarseBins], tmp[kWarps + 1];
  __shared__ uint64_t st_r[kCoarseTile];
  __shared__ uint32_t st_od[kCoarseTile];  // tile offset | bin << 16
  for (uint64_t tile = blockIdx.x; tile * kCoarseTile < n; tile += gridDim.x) {
    const uint64_t t0 = tile * kCoarseTile;
    uint32_t pk[kBatches];
#pragma unroll
    for (int k = 0; k < kBatches; ++k) {
      const uint64_t e = t0 + k * kBlock + threadIdx.x;
      pk[k] = e < n ? __ldg(packed + e) : 0;
    }
    bin_start[threadIdx.x] = block_scan<kBlock>(tile_counts[tile * kCoarseBins + threadIdx.x], tmp, nullptr);
    gbase[threadIdx.x] = tile_base[tile * kCoarseBins + threadIdx.x];
    __syncthreads();
#pragma unroll
    for (int k = 0; k < kBatches; ++k) {
      const uint64_t e = t0 + k * kBlock + threadIdx.x;
      if (e < n) {
        const uint32_t d = pk[k] & (kCoarseBins - 1);
        const uint32_t lp = bin_start[d] + (pk[k] >> kCoarseBits);
        st_od[lp] = (uint32_t)(k * kBlock + threadIdx.x) | (d << 16);
      }
    }
    __syncthreads();
    const uint32_t tile_n = (uint32_t)std::min<uint64_t>(kCoarseTile, n - t0);
    uint64_t rv[kBatches];
    uint32_t oo[kBatches];
#pragma unroll
    for (int k = 0; k < kBatches; ++k) {  // all kBatches loads in flight before the stores
      const uint32_t i = k * kBlock + threadIdx.x;
      if (i < tile_n) {
        const uint32_t od = st_od[i], dd = od >> 16;
        oo[k] = od & 0xFFFFu;
        rv[k] = __ldg(res1 + gbase[dd] + (i - bin_start[dd]));
      }
    }
#pragma unroll
    for (int k = 0; k < kBatches; ++k)
      if (k * kBlock + threadIdx.x < tile_n) st_r[oo[k]] = rv[k];
    __syncthreads();
    for (uint32_t i = threadIdx.x; i < tile_n; i += kBlock) out[t0 + i] = st_r[i];
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

// level-1 partition by any <= 256-bin digit: rank pass, then the staged move.
// h_counts (optional) receives the first `nbins` bin counts synchronously.
template <class Digit>
harmonia_status coarse_partition(const uint64_t* q, uint64_t n, const Digit& dg, const PsaWs& ws,
                                 uint64_t* sorted_q, uint32_t* idx, int sm, cudaStream_t st, uint64_t* h_counts,
                                 uint32_t nbins, uint32_t* tile_base = nullptr) {
  HM_CUDA(cudaMemsetAsync(ws.counts, 0, 2 * kCoarseBins * 4, st));
  // one tile per CTA (measured faster than persistent grid-stride CTAs: the phases of
  // different CTAs overlap)
  const int g = (int)std::min<uint64_t>(ceil_div(n, kCoarseTile), 1u << 30);
  {
    ProfScope ps_(HARMONIA_PROF_PSA_HIST, st);
    k_psa2_rank<Digit><<<std::max(g, 1), kBlock, 0, st>>>(q, n, dg, ws.counts, ws.tile_counts, ws.packed);
  }
  HM_LAUNCHED();
  if (h_counts) {
    uint32_t tmp[kCoarseBins];
    HM_CUDA(cudaMemcpyAsync(tmp, ws.counts, nbins * 4, cudaMemcpyDeviceToHost, st));
    HM_CUDA(cudaStreamSynchronize(st));
    for (uint32_t b = 0; b < nbins; ++b) h_counts[b] = tmp[b];
  }
  {
    ProfScope ps_(HARMONIA_PROF_PSA_SCATTER, st);
        k_psa2_move<Digit><<<std::max(g, 1), kBlock, 0, st>>>(q, n, dg, ws.counts, ws.counts + kCoarseBins, ws.tile_counts,
                                                   ws.packed, sorted_q, idx, tile_base);
  }
  HM_LAUNCHED();
  return HARMONIA_OK;
}

}  // namespace

// multi-GPU router: destination-major grouping by splitters (P <= 256 shards)
harmonia_status route_partition2(const uint64_t* q, uint64_t n, const BucketSplit& f, uint32_t P, const PsaWs& ws,
                                 int sm, cudaStream_t st, uint64_t* h_counts) {
  if (P > (uint32_t)kCoarseBins) return HARMONIA_ERR_INVALID_ARG;
  return coarse_partition(q, n, f, ws, ws.sorted_q, ws.idx, sm, st, h_counts, P);
}

harmonia_status psa_partition2(const uint64_t* q, uint64_t n, const BucketBits& f, int nb, const PsaWs& ws, int sm,
                               cudaStream_t st, int level2, bool local) {
  const uint32_t b1 = (uint32_t)std::min(nb, kCoarseBits);
  const uint32_t shift1 = (uint32_t)nb - b1;
  harmonia_status s = coarse_partition(q, n, CoarseDigit{f, shift1}, ws, ws.sorted_q, local ? nullptr : ws.idx, sm,
                                       st, nullptr, 0, local ? ws.tile_base : nullptr);
  if (s != HARMONIA_OK) return s;
  if (level2 == 2) return HARMONIA_OK;  // coarse partition only (ablation)
  {
    ProfScope ps_(HARMONIA_PROF_PSA_SCAN, st);  // reported in the "scan" class: level-2 sort
    static bool configured = false;
    if (!configured) {
      HM_CUDA(cudaFuncSetAttribute(k_psa2_local_sort, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kSortSmem));
      HM_CUDA(cudaFuncSetAttribute(k_psa2_count_sort<false>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                   (int)kCountSortSmem));
      HM_CUDA(cudaFuncSetAttribute(k_psa2_count_sort<true>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                   (int)kCountSortSmem));
      configured = true;
    }
    const int g = (int)std::min<uint64_t>(ceil_div(n, kChunk), (uint64_t)sm * 4);
    if (level2 == 1)  // two stable LSD passes of ballot multisplit (ablation)
      k_psa2_local_sort<<<std::max(g, 1), kSortThreads, kSortSmem, st>>>(ws.sorted_q, ws.idx, n, f);
    else if (local)   // one counting pass with shared-memory atomics (default, measured faster)
      k_psa2_count_sort<true><<<std::max(g, 1), kSortThreads, kCountSortSmem, st>>>(ws.sorted_q, ws.idx, n, f);
    else
      k_psa2_count_sort<false><<<std::max(g, 1), kSortThreads, kCountSortSmem, st>>>(ws.sorted_q, ws.idx, n, f);
  }
  HM_LAUNCHED();
  return HARMONIA_OK;
}

harmonia_status psa_unpartition2(const PsaWs& ws, const uint64_t* res1, uint64_t n, uint64_t* out, cudaStream_t st) {
  if (n == 0) return HARMONIA_OK;
  {
    ProfScope ps_(HARMONIA_PROF_RETURN, st);
    const int g = (int)std::min<uint64_t>(ceil_div(n, kCoarseTile), 1u << 30);
    k_psa2_unmove<<<g, kBlock, 0, st>>>(ws.tile_counts, ws.tile_base, ws.packed, res1, n, out);
  }
  HM_LAUNCHED();
  return HARMONIA_OK;
}

}  // namespace hm
