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

#ifndef HM_UNMOVE_TMA_STORE
#define HM_UNMOVE_TMA_STORE 1
#endif
#ifndef HM_MOVE_MINB
#define HM_MOVE_MINB 4
#endif
#ifndef HM_UNMOVE_MINB
#define HM_UNMOVE_MINB 4
#endif
#ifndef HM_L1_WAVES
#define HM_L1_WAVES 6
#endif
#ifndef HM_L1_WAVES_MV
#define HM_L1_WAVES_MV 16
#endif

namespace {

constexpr int kBatches = 8;                              // 32-query batches per warp per tile
constexpr int kCoarseTile = kBlock * kBatches;           // 2048 queries per scatter tile
#ifndef HM_SORT_THREADS
#define HM_SORT_THREADS 512
#endif
constexpr int kSortThreads = HM_SORT_THREADS, kSortWarps = kSortThreads / 32;
constexpr int kChunk = (int)kPsaChunk;                   // queries per LSD local-sort chunk (4096)
constexpr int kSortBatches = kChunk / kSortThreads;      // 32-query batches per warp per chunk
static_assert(kChunk == kSortThreads * kSortBatches, "chunk = threads x batches");
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

// ---- level-1 configurations -------------------------------------------------------------
// BITS-bit coarse digit, TILE queries per tile, NT threads per CTA (PER = TILE / NT queries
// per thread).  Narrow: 256 bins -- the multi-GPU router and the non-staged PSA modes.  Wide:
// 2048 bins -- the default staged-return PSA: a 4096-query level-2 chunk then spans ~2
// coarse bins instead of 1/8 of one, so the search sees ~8x denser key ranges per warp.
template <int BITS_, int TILE_, int NT_>
struct L1Cfg {
  static constexpr int BITS = BITS_, BINS = 1 << BITS_, TILE = TILE_, NT = NT_, PER = TILE_ / NT_;
  static constexpr int BPT = BINS / NT_;  // bins per thread in scans
  static constexpr int MINB = 1024 / NT_;  // >= 1024 resident threads per SM (<= 64 registers)
  static constexpr int TILE_SHIFT = (TILE_ == 2048 ? 11 : TILE_ == 4096 ? 12 : 13);
  static_assert(BINS % NT_ == 0 && TILE_ % NT_ == 0 && (1 << TILE_SHIFT) == TILE_, "L1Cfg");
  static_assert(BITS_ + TILE_SHIFT <= 32 && BITS_ + TILE_SHIFT + 0 <= 32, "packed digit|rank");
};
#ifndef HM_NARROW_TILE
#define HM_NARROW_TILE 2048
#endif
#ifndef HM_NARROW_NT
#define HM_NARROW_NT 256
#endif
using Narrow = L1Cfg<8, HM_NARROW_TILE, HM_NARROW_NT>;
#ifndef HM_WIDE_TILE
#define HM_WIDE_TILE 4096
#endif
using Wide = L1Cfg<11, HM_WIDE_TILE, 512>;

// exclusive scan over C::BINS values held BPT per thread (thread t owns [t*BPT, t*BPT+BPT))
template <class C>
__device__ __forceinline__ void scan_bins(const uint32_t (&v)[C::BPT], uint32_t (&ex)[C::BPT], uint32_t* tmp) {
  uint32_t s = 0;
#pragma unroll
  for (int k = 0; k < C::BPT; ++k) {
    ex[k] = s;
    s += v[k];
  }
  const uint32_t base = block_scan<C::NT>(s, tmp, nullptr);
#pragma unroll
  for (int k = 0; k < C::BPT; ++k) ex[k] += base;
}

// Level-1 CTAs are persistent: CTA c owns the contiguous tile range [c*T/G, (c+1)*T/G) in all
// three passes (rank, move, unmove), so bin space is reserved once per (CTA, bin) -- one
// global atomic each -- instead of once per (tile, bin), and the inverse move recomputes
// every tile's run starts from the CTA base and the tile counts.
__device__ __forceinline__ void l1_tile_range(uint64_t n, uint32_t tile, uint64_t* tb, uint64_t* te) {
  const uint64_t T = (n + tile - 1) / tile;
  *tb = (uint64_t)blockIdx.x * T / gridDim.x;
  *te = (uint64_t)(blockIdx.x + 1) * T / gridDim.x;
}

// ---- tile prefetch: every level-1 CTA walks a contiguous tile range, so the next tile's
// inputs stream into shared memory by TMA bulk copies (one thread) while the current tile is
// processed -- the per-tile load latency was exposed (ncu: long-scoreboard stalls).
#ifndef HM_L1_PREFETCH
#define HM_L1_PREFETCH 0  // measured: neutral to -2 % (the level-1 passes are bound by shared-store conflicts)
#endif
template <class C>
__device__ __forceinline__ uint32_t tile_bytes(uint64_t tile, uint64_t n, uint32_t elem) {
  const uint64_t m = std::min<uint64_t>(C::TILE, n - tile * C::TILE);
  return (uint32_t)((m * elem + 15) & ~15ull);  // the tail rounds up inside its 16-byte block
}

// ---- level 1, pass 1: per-tile digit ranks ---------------------------------------------
// Each query's coarse digit d and its rank among the tile's queries with digit d are taken
// once, with a shared-memory atomic, and stored packed (d | rank << BITS) so that the move
// pass needs no multisplit (the ballot multisplit was measured slower: DESIGN.md §8).
// Per-tile bin counts go to tile_counts[tile][BINS], the CTA's totals to cta_counts[c][BINS]
// and the bin totals to counts[BINS].  Digit: any functor mapping a query to [0, BINS) (the
// PSA coarse digit, or the destination shard of the partitioned multi-GPU mode).
template <class Digit, class C>
__global__ void __launch_bounds__(C::NT, C::MINB) k_psa2_rank(const uint64_t* __restrict__ q, uint64_t n, Digit dg,
                                                              uint32_t* __restrict__ counts,
                                                              uint32_t* __restrict__ tile_counts,
                                                              uint32_t* __restrict__ packed,
                                                              uint32_t* __restrict__ cta_counts) {
  __shared__ uint32_t cnt[C::BINS];
  __shared__ __align__(16) uint64_t sq[HM_L1_PREFETCH ? C::TILE : 2];
  __shared__ __align__(8) uint64_t bar;
  uint64_t tb, te;
  l1_tile_range(n, C::TILE, &tb, &te);
  const bool pf = HM_L1_PREFETCH && ((uintptr_t)q & 15) == 0;
  if (pf && threadIdx.x == 0) {
    mbar_init(&bar, 1);
    if (tb < te) bulk_load(sq, q + tb * C::TILE, tile_bytes<C>(tb, n, 8), &bar);
  }
  __syncthreads();
  uint32_t phase = 0;
  uint32_t acc[C::BPT];
#pragma unroll
  for (int k = 0; k < C::BPT; ++k) acc[k] = 0;
  for (uint64_t tile = tb; tile < te; ++tile) {
    const uint64_t t0 = tile * C::TILE;
    uint64_t v[C::PER];
    if (pf) {
      mbar_wait(&bar, phase);
      phase ^= 1;
    }
#pragma unroll
    for (int k = 0; k < C::PER; ++k) {  // all loads first (PER in flight per thread)
      const uint64_t e = t0 + k * C::NT + threadIdx.x;
      v[k] = e < n ? (pf ? sq[k * C::NT + threadIdx.x] : __ldg(q + e)) : 0;
    }
#pragma unroll
    for (int k = 0; k < C::BPT; ++k) cnt[k * C::NT + threadIdx.x] = 0;
    __syncthreads();
    if (pf && threadIdx.x == 0 && tile + 1 < te)
      bulk_load(sq, q + (tile + 1) * C::TILE, tile_bytes<C>(tile + 1, n, 8), &bar);
    // Router digits (few destinations): warp-aggregated ranks -- one shared atomic per distinct
    // digit per warp (lanes with equal digits found by MATCH.ANY); with P <= 8 shards a warp
    // otherwise serialises up to 32 atomics on one counter.  The PSA coarse digit (256 bins,
    // ~30 distinct per warp) keeps one atomic per query.
    constexpr bool kAgg = !std::is_same<Digit, CoarseDigit>::value;
#pragma unroll
    for (int k = 0; k < C::PER; ++k) {
      const uint64_t e = t0 + k * C::NT + threadIdx.x;
      if constexpr (kAgg) {
        const bool in = e < n;  // every lane takes part in the match (tile tails)
        const uint32_t d = in ? dg(v[k]) : 0xFFFFFFFFu;
        const unsigned peers = __match_any_sync(kFull, d);
        const unsigned lane = threadIdx.x & 31, leader = __ffs(peers) - 1;
        uint32_t base = 0;
        if (in && lane == leader) base = atomicAdd(&cnt[d], (uint32_t)__popc(peers));
        base = __shfl_sync(kFull, base, leader);
        if (in) packed[e] = d | ((base + __popc(peers & ((1u << lane) - 1))) << C::BITS);
      } else if (e < n) {
        const uint32_t d = dg(v[k]);
        packed[e] = d | (atomicAdd(&cnt[d], 1u) << C::BITS);
      }
    }
    __syncthreads();
#pragma unroll
    for (int k = 0; k < C::BPT; ++k) {
      const uint32_t c = cnt[k * C::NT + threadIdx.x];
      tile_counts[tile * C::BINS + k * C::NT + threadIdx.x] = c;
      acc[k] += c;
    }
    __syncthreads();
  }
#pragma unroll
  for (int k = 0; k < C::BPT; ++k) {
    const uint32_t b = k * C::NT + threadIdx.x;
    cta_counts[(uint64_t)blockIdx.x * C::BINS + b] = acc[k];
    if (acc[k]) atomicAdd(counts + b, acc[k]);
  }
}

// ---- level 1, pass 2: move ----------------------------------------------------------------
// Global position of query e = exclusive-prefix(counts)[d] + the CTA's reservation in bin d
// (one atomic per CTA and non-empty bin on cursor[d]) + the earlier tiles of the CTA + rank.
// Staged through shared memory in bin order so that each bin's run is written by consecutive
// lanes.  The scattered shared-memory stores are the limiter (ncu: shared-store wavefronts),
// so only the query is staged when the digit is cheap to recompute (the PSA coarse digit) and
// the position only when idx is wanted (kIdx).
//
// kPush (partitioned multi-GPU mode, fused routing): the run of destination d is written
// straight into the receive buffer of rank d (a peer-mapped device pointer, NVLink stores),
// push_dst[d] = address of this rank's segment there; nothing is written locally.
template <class Digit, class C, bool kIdx, bool kPush = false>
__global__ void __launch_bounds__(C::NT, (C::BINS == 256 ? HM_MOVE_MINB : C::MINB)) k_psa2_move(const uint64_t* __restrict__ q, uint64_t n, Digit dg,
                                                              const uint32_t* __restrict__ counts,
                                                              uint32_t* __restrict__ cursor,
                                                              const uint32_t* __restrict__ tile_counts,
                                                              const uint32_t* __restrict__ packed,
                                                              const uint32_t* __restrict__ cta_counts,
                                                              uint32_t* __restrict__ cta_base,
                                                              uint64_t* __restrict__ sorted_q,
                                                              uint32_t* __restrict__ idx,
                                                              const uint64_t* __restrict__ push_dst = nullptr) {
  constexpr bool kRecompute = std::is_same<Digit, CoarseDigit>::value;
  constexpr bool kCtaSums = HM_L1_WAVES_MV != HM_L1_WAVES;
  __shared__ uint64_t s_push[kPush ? C::BINS : 1];  // push_dst[d] - 8 * (first global slot of bin d)
  extern __shared__ __align__(16) unsigned char l1_smem[];
  uint64_t* st_q = reinterpret_cast<uint64_t*>(l1_smem);
  uint32_t* bin_start = reinterpret_cast<uint32_t*>(l1_smem + C::TILE * 8);
  uint32_t* gbase = bin_start + C::BINS;
  uint32_t* st_i = gbase + C::BINS;                                       // kIdx
  uint8_t* st_d = reinterpret_cast<uint8_t*>(st_i + (kIdx ? C::TILE : 0));  // !kRecompute
  // prefetch stage (16-byte aligned): next tile's queries and packed ranks
  uint64_t* pq = reinterpret_cast<uint64_t*>(l1_smem + ((C::TILE * 8 + 2 * C::BINS * 4 + (kIdx ? C::TILE * 4 : 0) +
                                                          (kRecompute ? 0 : C::TILE) + 15) & ~15));
  uint32_t* pp = reinterpret_cast<uint32_t*>(pq + C::TILE);
  __shared__ uint32_t tmp[C::NT / 32 + 1];
  __shared__ __align__(8) uint64_t bar;
  uint64_t tb, te;
  l1_tile_range(n, C::TILE, &tb, &te);
  const bool pf = HM_L1_PREFETCH && ((uintptr_t)q & 15) == 0;
  if (pf && threadIdx.x == 0) {
    mbar_init(&bar, 1);
    if (tb < te) {
      bulk_expect(&bar, tile_bytes<C>(tb, n, 8) + tile_bytes<C>(tb, n, 4));
      bulk_copy(pq, q + tb * C::TILE, tile_bytes<C>(tb, n, 8), &bar);
      bulk_copy(pp, packed + tb * C::TILE, tile_bytes<C>(tb, n, 4), &bar);
    }
  }
  uint32_t phase = 0;
  uint32_t run[C::BPT];  // next free global slot of bins threadIdx.x * BPT + k for this CTA
  {
    uint32_t cv[C::BPT];
#pragma unroll
    for (int k = 0; k < C::BPT; ++k) cv[k] = counts[threadIdx.x * C::BPT + k];
    scan_bins<C>(cv, run, tmp);
#pragma unroll
    for (int k = 0; k < C::BPT; ++k) {
      const uint64_t b = threadIdx.x * C::BPT + k;
      if constexpr (kPush) s_push[b] = push_dst[b] - 8ull * run[k];  // run[k] = bin start here
      // this CTA's total in bin b, from the per-tile counts of its own tile range: the move
      // grid need not equal the rank grid (cta_counts is only read when it does)
      uint32_t cc = 0;
      if (kCtaSums) {
        for (uint64_t tt = tb; tt < te; ++tt) cc += tile_counts[tt * C::BINS + b];
      } else {
        cc = cta_counts[(uint64_t)blockIdx.x * C::BINS + b];
      }
      run[k] = cc ? run[k] + atomicAdd(cursor + b, cc) : 0u;
      cta_base[(uint64_t)blockIdx.x * C::BINS + b] = run[k];  // for the staged return
    }
  }
  for (uint64_t tile = tb; tile < te; ++tile) {
    const uint64_t t0 = tile * C::TILE;
    uint64_t v[C::PER];
    uint32_t pk[C::PER];
    if (pf) {
      mbar_wait(&bar, phase);
      phase ^= 1;
    }
#pragma unroll
    for (int k = 0; k < C::PER; ++k) {
      const uint64_t e = t0 + k * C::NT + threadIdx.x;
      v[k] = e < n ? (pf ? pq[k * C::NT + threadIdx.x] : __ldg(q + e)) : 0;
      pk[k] = e < n ? (pf ? pp[k * C::NT + threadIdx.x] : __ldg(packed + e)) : 0;
    }
    {
      uint32_t cv[C::BPT], ex[C::BPT];
#pragma unroll
      for (int k = 0; k < C::BPT; ++k) cv[k] = tile_counts[tile * C::BINS + threadIdx.x * C::BPT + k];
      scan_bins<C>(cv, ex, tmp);
#pragma unroll
      for (int k = 0; k < C::BPT; ++k) {
        bin_start[threadIdx.x * C::BPT + k] = ex[k];
        gbase[threadIdx.x * C::BPT + k] = run[k];
        run[k] += cv[k];
      }
    }
    __syncthreads();
    if (pf && threadIdx.x == 0 && tile + 1 < te) {  // every thread has read the stage
      bulk_expect(&bar, tile_bytes<C>(tile + 1, n, 8) + tile_bytes<C>(tile + 1, n, 4));
      bulk_copy(pq, q + (tile + 1) * C::TILE, tile_bytes<C>(tile + 1, n, 8), &bar);
      bulk_copy(pp, packed + (tile + 1) * C::TILE, tile_bytes<C>(tile + 1, n, 4), &bar);
    }
#pragma unroll
    for (int k = 0; k < C::PER; ++k) {
      const uint64_t e = t0 + k * C::NT + threadIdx.x;
      if (e < n) {
        const uint32_t d = pk[k] & (C::BINS - 1);
        const uint32_t lp = bin_start[d] + (pk[k] >> C::BITS);
        st_q[lp] = v[k];
        if constexpr (kIdx) st_i[lp] = (uint32_t)e;
        if constexpr (!kRecompute) st_d[lp] = (uint8_t)d;
      }
    }
    __syncthreads();
    const uint32_t tile_n = (uint32_t)std::min<uint64_t>(C::TILE, n - t0);
    for (uint32_t i = threadIdx.x; i < tile_n; i += C::NT) {  // runs written by consecutive lanes
      const uint64_t x = st_q[i];
      uint32_t dd;
      if constexpr (kRecompute) dd = dg(x);
      else dd = st_d[i];
      const uint32_t dst = gbase[dd] + (i - bin_start[dd]);
      if constexpr (kPush) {
        *reinterpret_cast<uint64_t*>(s_push[dd] + 8ull * dst) = x;
      } else {
        sorted_q[dst] = x;
      }
      if constexpr (kIdx) idx[dst] = st_i[i];
    }
    __syncthreads();
  }
}
template <class C, bool kIdx, bool kRecompute>
constexpr size_t move_smem() {
  return (((size_t)C::TILE * 8 + 2 * C::BINS * 4 + (kIdx ? C::TILE * 4 : 0) + (kRecompute ? 0 : C::TILE) + 15) & ~15) +
         (HM_L1_PREFETCH ? (size_t)C::TILE * 12 : 0);
}

// ---- staged return: inverse of the move -------------------------------------------------
// res1 holds the results in level-1 order.  For the tile of original positions
// [t0, t0 + TILE) the slots of its (bin, rank) pairs are restaged exactly as in k_psa2_move;
// slot i of the tile's bin order sits at level-1 position gbase[d] + (i - bin_start[d]) with
// gbase rebuilt from the CTA base, so res1 is read in runs and out[] written contiguously --
// no scattered global access on either side.
template <class C>
__global__ void __launch_bounds__(C::NT, (C::BINS == 256 ? HM_UNMOVE_MINB : C::MINB)) k_psa2_unmove(const uint32_t* __restrict__ tile_counts,
                                                                const uint32_t* __restrict__ cta_base,
                                                                const uint32_t* __restrict__ packed,
                                                                const uint64_t* __restrict__ res1, uint64_t n,
                                                                uint64_t* __restrict__ out) {
  extern __shared__ __align__(16) unsigned char l1_smem[];
  uint64_t* st_r = reinterpret_cast<uint64_t*>(l1_smem);
  uint32_t* st_od = reinterpret_cast<uint32_t*>(l1_smem + C::TILE * 8);  // offset | bin << TILE_SHIFT
  uint32_t* bin_start = st_od + C::TILE;
  uint32_t* gbase = bin_start + C::BINS;
  uint32_t* pp = gbase + C::BINS;  // prefetch stage: the next tile's packed ranks
  __shared__ uint32_t tmp[C::NT / 32 + 1];
  __shared__ __align__(8) uint64_t bar;
  uint64_t tb, te;
  l1_tile_range(n, C::TILE, &tb, &te);
  const bool pf = HM_L1_PREFETCH;
  if (pf && threadIdx.x == 0) {
    mbar_init(&bar, 1);
    if (tb < te) bulk_load(pp, packed + tb * C::TILE, tile_bytes<C>(tb, n, 4), &bar);
  }
  __syncthreads();  // barrier initialised before anyone waits on it
  uint32_t phase = 0;
  uint32_t run[C::BPT];
#pragma unroll
  for (int k = 0; k < C::BPT; ++k) run[k] = cta_base[(uint64_t)blockIdx.x * C::BINS + threadIdx.x * C::BPT + k];
  for (uint64_t tile = tb; tile < te; ++tile) {
    const uint64_t t0 = tile * C::TILE;
    uint32_t pk[C::PER];
    if (pf) {
      mbar_wait(&bar, phase);
      phase ^= 1;
    }
#pragma unroll
    for (int k = 0; k < C::PER; ++k) {
      const uint64_t e = t0 + k * C::NT + threadIdx.x;
      pk[k] = e < n ? (pf ? pp[k * C::NT + threadIdx.x] : __ldg(packed + e)) : 0;
    }
    {
      uint32_t cv[C::BPT], ex[C::BPT];
#pragma unroll
      for (int k = 0; k < C::BPT; ++k) cv[k] = tile_counts[tile * C::BINS + threadIdx.x * C::BPT + k];
      scan_bins<C>(cv, ex, tmp);
#pragma unroll
      for (int k = 0; k < C::BPT; ++k) {
        bin_start[threadIdx.x * C::BPT + k] = ex[k];
        gbase[threadIdx.x * C::BPT + k] = run[k];
        run[k] += cv[k];
      }
    }
    __syncthreads();
    if (pf && threadIdx.x == 0 && tile + 1 < te)
      bulk_load(pp, packed + (tile + 1) * C::TILE, tile_bytes<C>(tile + 1, n, 4), &bar);
#pragma unroll
    for (int k = 0; k < C::PER; ++k) {
      const uint64_t e = t0 + k * C::NT + threadIdx.x;
      if (e < n) {
        const uint32_t d = pk[k] & (C::BINS - 1);
        const uint32_t lp = bin_start[d] + (pk[k] >> C::BITS);
        st_od[lp] = (uint32_t)(k * C::NT + threadIdx.x) | (d << C::TILE_SHIFT);
      }
    }
    if (HM_UNMOVE_TMA_STORE && threadIdx.x == 0) bulk_store_wait_read();  // st_r free again
    __syncthreads();
    const uint32_t tile_n = (uint32_t)std::min<uint64_t>(C::TILE, n - t0);
    uint64_t rv[C::PER];
    uint32_t oo[C::PER];
#pragma unroll
    for (int k = 0; k < C::PER; ++k) {  // all loads in flight before the stores
      const uint32_t i = k * C::NT + threadIdx.x;
      if (i < tile_n) {
        const uint32_t od = st_od[i], dd = od >> C::TILE_SHIFT;
        oo[k] = od & (C::TILE - 1);
        rv[k] = __ldg(res1 + gbase[dd] + (i - bin_start[dd]));
      }
    }
#pragma unroll
    for (int k = 0; k < C::PER; ++k)
      if (k * C::NT + threadIdx.x < tile_n) st_r[oo[k]] = rv[k];
    // TMA store of a full tile (one thread, async); the next tile's st_r writes wait above
    const bool tma = HM_UNMOVE_TMA_STORE && tile_n == (uint32_t)C::TILE && ((uintptr_t)(out + t0) & 15) == 0;
    if (tma) fence_proxy_async_smem();
    __syncthreads();
    if (tma) {
      if (threadIdx.x == 0) {
        bulk_store(out + t0, st_r, C::TILE * 8);
        bulk_store_commit();
      }
    } else {
      for (uint32_t i = threadIdx.x; i < tile_n; i += C::NT) out[t0 + i] = st_r[i];
      __syncthreads();
    }
  }
  if (HM_UNMOVE_TMA_STORE && threadIdx.x == 0) bulk_store_wait_all();
}
template <class C>
constexpr size_t unmove_smem() {
  return (size_t)C::TILE * 12 + 2 * C::BINS * 4 + (HM_L1_PREFETCH ? (size_t)C::TILE * 4 : 0);
}

// ---- level 2: chunk-local sort by the N-bit bucket (two stable LSD passes) ---------------
template <int BITS, int SHIFT>
__device__ __forceinline__ void lsd_pass(uint64_t (&v)[kSortBatches], uint32_t (&ix)[kSortBatches], uint32_t (&lk)[kSortBatches],
                                         uint32_t m, uint32_t (*wcnt)[1 << kLoBits], uint32_t* bin_start, uint32_t* tmp,
                                         uint64_t* s_q, uint32_t* s_i, uint16_t* s_k) {
  constexpr int NB = 1 << BITS;
  const unsigned lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  for (int i = threadIdx.x; i < kSortWarps * NB; i += kSortThreads) wcnt[i / NB][i % NB] = 0;
  __syncthreads();
  uint32_t pos[kSortBatches], dg[kSortBatches];
#pragma unroll
  for (int k = 0; k < kSortBatches; ++k) {  // element order = (warp, batch, lane): stable ranks
    const uint32_t e = warp * (32 * kSortBatches) + k * 32 + lane;
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
  for (int k = 0; k < kSortBatches; ++k) {
    const uint32_t e = warp * (32 * kSortBatches) + k * 32 + lane;
    if (e < m) {
      const uint32_t dst = bin_start[dg[k]] + wcnt[warp][dg[k]] + pos[k];
      s_q[dst] = v[k];
      s_i[dst] = ix[k];
      s_k[dst] = (uint16_t)lk[k];
    }
  }
  __syncthreads();
#pragma unroll
  for (int k = 0; k < kSortBatches; ++k) {  // reload in the new order for the next pass
    const uint32_t e = warp * (32 * kSortBatches) + k * 32 + lane;
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
    uint64_t v[kSortBatches];
    uint32_t ix[kSortBatches], lk[kSortBatches];
    uint32_t bmin = 0xFFFFFFFFu, bmax = 0;
#pragma unroll
    for (int k = 0; k < kSortBatches; ++k) {
      const uint32_t e = warp * (32 * kSortBatches) + k * 32 + lane;
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
    for (int k = 0; k < kSortBatches; ++k) lk[k] = (lk[k] - bmin) >> sh;
    lsd_pass<kLoBits, 0>(v, ix, lk, m, wcnt, bin_start, tmp, s_q, s_i, s_k);
    lsd_pass<kHiBits, kLoBits>(v, ix, lk, m, wcnt, bin_start, tmp, s_q, s_i, s_k);
#pragma unroll
    for (int k = 0; k < kSortBatches; ++k) {  // write back (coalesced)
      const uint32_t e = warp * (32 * kSortBatches) + k * 32 + lane;
      if (e < m) {
        sorted_q[c0 + e] = v[k];
        idx[c0 + e] = ix[k];
      }
    }
  }
}

constexpr int kLocalBins = 1 << kLocalBits;
// local histogram, sorted keys + positions, and (prefetch) the next chunk's staged queries
template <int kCh>
constexpr size_t count_sort_smem();
#include "psa2_count_sort.inc"
template <int kCh>
constexpr size_t count_sort_smem() {
  return (size_t)kLocalBins * 4 + (size_t)kCh * 12 + (sort_prefetch<kCh>() ? (size_t)kCh * 8 : 0);
}

// level-1 grids: CTAs own contiguous tile ranges, ~2048 resident threads per SM, waves x the
// resident CTAs.  The rank pass and the move/unmove pair may use different wave counts (the
// move then sums its CTA's per-tile counts itself): measured best 6 for the rank pass (4-8 within 4 %), 16 for
// the move and its inverse.
template <class C>
int l1_grid(uint64_t n, int sm, int waves = HM_L1_WAVES) {
  const uint64_t g = std::min<uint64_t>((uint64_t)sm * (2048 / C::NT) * waves, kL1CtaRows / C::BINS);
  return (int)std::max<uint64_t>(1, std::min<uint64_t>(ceil_div(n, C::TILE), g));
}
template <class C>
int l1_grid_mv(uint64_t n, int sm) {
  return l1_grid<C>(n, sm, HM_L1_WAVES_MV);
}

// level-1 partition by a C::BITS-bit digit: rank pass, then the staged move.
// h_counts (optional) receives the first `nbins` bin counts synchronously.
template <class C, class Digit>
harmonia_status coarse_partition(const uint64_t* q, uint64_t n, const Digit& dg, const PsaWs& ws,
                                 uint64_t* sorted_q, uint32_t* idx, int sm, cudaStream_t st, uint64_t* h_counts,
                                 uint32_t nbins) {
  constexpr bool kRecompute = std::is_same<Digit, CoarseDigit>::value;
  HM_CUDA(cudaMemsetAsync(ws.counts, 0, 2 * C::BINS * 4, st));
  const int g = l1_grid<C>(n, sm), gm = l1_grid_mv<C>(n, sm);
  {
    ProfScope ps_(HARMONIA_PROF_PSA_HIST, st);
    k_psa2_rank<Digit, C><<<g, C::NT, 0, st>>>(q, n, dg, ws.counts, ws.tile_counts, ws.packed, ws.cta_counts);
  }
  HM_LAUNCHED();
  if (h_counts) {
    uint32_t tmp[C::BINS];
    HM_CUDA(cudaMemcpyAsync(tmp, ws.counts, nbins * 4, cudaMemcpyDeviceToHost, st));
    HM_CUDA(cudaStreamSynchronize(st));
    for (uint32_t b = 0; b < nbins; ++b) h_counts[b] = tmp[b];
  }
  {
    ProfScope ps_(HARMONIA_PROF_PSA_SCATTER, st);
    if (idx) {
      constexpr size_t smb = move_smem<C, true, kRecompute>();
      static bool cfg = false;
      if (!cfg) {
        HM_CUDA(cudaFuncSetAttribute(k_psa2_move<Digit, C, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smb));
        cfg = true;
      }
      k_psa2_move<Digit, C, true><<<gm, C::NT, smb, st>>>(q, n, dg, ws.counts, ws.counts + C::BINS, ws.tile_counts,
                                                         ws.packed, ws.cta_counts, ws.cta_base, sorted_q, idx);
    } else {
      constexpr size_t smb = move_smem<C, false, kRecompute>();
      static bool cfg = false;
      if (!cfg) {
        HM_CUDA(cudaFuncSetAttribute(k_psa2_move<Digit, C, false>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smb));
        cfg = true;
      }
      k_psa2_move<Digit, C, false><<<gm, C::NT, smb, st>>>(q, n, dg, ws.counts, ws.counts + C::BINS, ws.tile_counts,
                                                          ws.packed, ws.cta_counts, ws.cta_base, sorted_q, nullptr);
    }
  }
  HM_LAUNCHED();
  return HARMONIA_OK;
}

template <class C>
harmonia_status unpartition(const PsaWs& ws, const uint64_t* res1, uint64_t n, uint64_t* out, int sm,
                            cudaStream_t st) {
  constexpr size_t smb = unmove_smem<C>();
  static bool cfg = false;
  if (!cfg) {
    HM_CUDA(cudaFuncSetAttribute(k_psa2_unmove<C>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smb));
    cfg = true;
  }
  ProfScope ps_(HARMONIA_PROF_RETURN, st);
  k_psa2_unmove<C><<<l1_grid_mv<C>(n, sm), C::NT, smb, st>>>(ws.tile_counts, ws.cta_base, ws.packed, res1, n, out);
  HM_LAUNCHED();
  return HARMONIA_OK;
}

// copy nseg segments: dst_addr[s] <- src[src_off[s] .. + len[s]) (peer-mapped destinations);
// grid.y = segment, 16-byte vector stores when both ends are aligned
__global__ void __launch_bounds__(256) k_segments_push(const uint64_t* __restrict__ src,
                                                       const uint64_t* __restrict__ desc) {
  const uint64_t off = desc[blockIdx.y * 3], len = desc[blockIdx.y * 3 + 1];
  uint64_t* dst = reinterpret_cast<uint64_t*>(desc[blockIdx.y * 3 + 2]);
  const uint64_t* s = src + off;
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  const uint64_t t0 = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if ((((uintptr_t)s | (uintptr_t)dst) & 15) == 0) {
    const uint64_t pairs = len / 2;
    for (uint64_t i = t0; i < pairs; i += stride)
      reinterpret_cast<ulonglong2*>(dst)[i] = __ldg(reinterpret_cast<const ulonglong2*>(s) + i);
    if (t0 == 0 && (len & 1)) dst[len - 1] = s[len - 1];
  } else {
    for (uint64_t i = t0; i < len; i += stride) dst[i] = s[i];
  }
}

}  // namespace

// fused routing (partitioned mode, peer memory): pass 1 = destination ranks and counts
harmonia_status route_count2(const uint64_t* q, uint64_t n, const BucketSplit& f, uint32_t P, const PsaWs& ws, int sm,
                             cudaStream_t st, uint64_t* h_counts) {
  using C = Narrow;
  if (P > (uint32_t)C::BINS) return HARMONIA_ERR_INVALID_ARG;
  HM_CUDA(cudaMemsetAsync(ws.counts, 0, 2 * C::BINS * 4, st));
  {
    ProfScope ps_(HARMONIA_PROF_PSA_HIST, st);
    k_psa2_rank<BucketSplit, C><<<l1_grid<C>(n, sm), C::NT, 0, st>>>(q, n, f, ws.counts, ws.tile_counts, ws.packed,
                                                                    ws.cta_counts);
  }
  HM_LAUNCHED();
  uint32_t tmp[C::BINS];
  HM_CUDA(cudaMemcpyAsync(tmp, ws.counts, P * 4, cudaMemcpyDeviceToHost, st));
  HM_CUDA(cudaStreamSynchronize(st));
  for (uint32_t b = 0; b < P; ++b) h_counts[b] = tmp[b];
  return HARMONIA_OK;
}

// pass 2: every destination's run stored straight into its receive buffer (d_push[d])
harmonia_status route_push2(const uint64_t* q, uint64_t n, const BucketSplit& f, uint32_t P, const PsaWs& ws,
                            const uint64_t* d_push, int sm, cudaStream_t st) {
  using C = Narrow;
  if (P > (uint32_t)C::BINS) return HARMONIA_ERR_INVALID_ARG;
  constexpr size_t smb = move_smem<C, false, false>();
  static bool cfg = false;
  if (!cfg) {
    HM_CUDA(cudaFuncSetAttribute(k_psa2_move<BucketSplit, C, false, true>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                 (int)smb));
    cfg = true;
  }
  {
    ProfScope ps_(HARMONIA_PROF_PSA_SCATTER, st);
    k_psa2_move<BucketSplit, C, false, true><<<l1_grid_mv<C>(n, sm), C::NT, smb, st>>>(
        q, n, f, ws.counts, ws.counts + C::BINS, ws.tile_counts, ws.packed, ws.cta_counts, ws.cta_base, nullptr,
        nullptr, d_push);
  }
  HM_LAUNCHED();
  return HARMONIA_OK;
}

// results in routed (destination-major) order -> caller order: the inverse move
harmonia_status route_return2(const PsaWs& ws, const uint64_t* back, uint64_t n, uint64_t* out, int sm,
                              cudaStream_t st) {
  if (n == 0) return HARMONIA_OK;
  return unpartition<Narrow>(ws, back, n, out, sm, st);
}

harmonia_status segments_push(const uint64_t* src, uint32_t nseg, const uint64_t* d_desc, uint64_t max_len, int sm,
                              cudaStream_t st) {
  if (nseg == 0 || max_len == 0) return HARMONIA_OK;
  const uint64_t blocks = std::min<uint64_t>(ceil_div(max_len, 2 * 256), (uint64_t)sm * 8);
  {
    ProfScope ps_(HARMONIA_PROF_RETURN, st);
    k_segments_push<<<dim3((unsigned)std::max<uint64_t>(blocks, 1), nseg), 256, 0, st>>>(src, d_desc);
  }
  HM_LAUNCHED();
  return HARMONIA_OK;
}

// multi-GPU router: destination-major grouping by splitters (P <= 256 shards)
harmonia_status route_partition2(const uint64_t* q, uint64_t n, const BucketSplit& f, uint32_t P, const PsaWs& ws,
                                 int sm, cudaStream_t st, uint64_t* h_counts) {
  if (P > (uint32_t)Narrow::BINS) return HARMONIA_ERR_INVALID_ARG;
  return coarse_partition<Narrow>(q, n, f, ws, ws.sorted_q, ws.idx, sm, st, h_counts, P);
}

harmonia_status psa_partition2(const uint64_t* q, uint64_t n, const BucketBits& f, int nb, const PsaWs& ws, int sm,
                               cudaStream_t st, int level2, bool local, bool wide, uint32_t chunk) {
  harmonia_status s;
  if (wide) {  // staged-return mode only (no idx)
    const uint32_t b1 = (uint32_t)std::min(nb, Wide::BITS);
    s = coarse_partition<Wide>(q, n, CoarseDigit{f, (uint32_t)nb - b1}, ws, ws.sorted_q, nullptr, sm, st, nullptr,
                               0);
  } else {
    const uint32_t b1 = (uint32_t)std::min(nb, Narrow::BITS);
    s = coarse_partition<Narrow>(q, n, CoarseDigit{f, (uint32_t)nb - b1}, ws, ws.sorted_q, local ? nullptr : ws.idx,
                                 sm, st, nullptr, 0);
  }
  if (s != HARMONIA_OK) return s;
  if (level2 == 2) return HARMONIA_OK;  // coarse partition only (ablation / fused chunk sort)
  {
    ProfScope ps_(HARMONIA_PROF_PSA_SCAN, st);  // reported in the "scan" class: level-2 sort
    static bool configured = false;
    if (!configured) {
      HM_CUDA(cudaFuncSetAttribute(k_psa2_local_sort, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kSortSmem));
      HM_CUDA(cudaFuncSetAttribute(k_psa2_count_sort<false, kChunk>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                   (int)count_sort_smem<kChunk>()));
      HM_CUDA(cudaFuncSetAttribute(k_psa2_count_sort<true, kChunk>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                   (int)count_sort_smem<kChunk>()));
      HM_CUDA(cudaFuncSetAttribute(k_psa2_count_sort<true, (int)kPsaChunkMax>,
                                   cudaFuncAttributeMaxDynamicSharedMemorySize, (int)count_sort_smem<kPsaChunkMax>()));
      configured = true;
    }
#ifndef HM_SORT_CTAS_PER_SM
#define HM_SORT_CTAS_PER_SM 4
#endif
    const uint32_t ch = (local && level2 == 0 && chunk == kPsaChunkMax) ? kPsaChunkMax : (uint32_t)kChunk;
#ifndef HM_SORT_CTAS_PER_SM_8K
#define HM_SORT_CTAS_PER_SM_8K 1  // one resident CTA per SM: persistent, one TMA prefetch chain each
#endif
    const int cps = ch == kPsaChunkMax ? HM_SORT_CTAS_PER_SM_8K : HM_SORT_CTAS_PER_SM;
    const int g = (int)std::min<uint64_t>(ceil_div(n, ch), (uint64_t)sm * cps);
    if (level2 == 1)  // two stable LSD passes of ballot multisplit (ablation)
      k_psa2_local_sort<<<std::max(g, 1), kSortThreads, kSortSmem, st>>>(ws.sorted_q, ws.idx, n, f);
    else if (local && ch == kPsaChunkMax)  // 8192-query chunks (denser key ranges per warp)
      k_psa2_count_sort<true, (int)kPsaChunkMax>
          <<<std::max(g, 1), kSortThreads, count_sort_smem<kPsaChunkMax>(), st>>>(ws.sorted_q, ws.idx, n, f);
    else if (local)   // one counting pass with shared-memory atomics (default, measured faster)
      k_psa2_count_sort<true, kChunk><<<std::max(g, 1), kSortThreads, count_sort_smem<kChunk>(), st>>>(ws.sorted_q, ws.idx, n, f);
    else
      k_psa2_count_sort<false, kChunk><<<std::max(g, 1), kSortThreads, count_sort_smem<kChunk>(), st>>>(ws.sorted_q, ws.idx, n, f);
  }
  HM_LAUNCHED();
  return HARMONIA_OK;
}

harmonia_status psa_unpartition2(const PsaWs& ws, const uint64_t* res1, uint64_t n, uint64_t* out, int sm,
                                 cudaStream_t st, bool wide) {
  if (n == 0) return HARMONIA_OK;
  return wide ? unpartition<Wide>(ws, res1, n, out, sm, st) : unpartition<Narrow>(ws, res1, n, out, sm, st);
}

}  // namespace hm
