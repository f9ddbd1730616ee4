// Partially-sorted aggregation (PSA, §4.1) as MSD partition passes.
//
// "the queries will be sorted based on their most significant N bits", N from
// Eq 2.  On sm_100a a one-pass partition over 2^N buckets costs one global atomic per query
// (the one-pass form is kept in psa.cu as the literal ablation), so the N-bit order is built
// from shared-memory passes:
//   level 1  MSB partition of the PSA window on the top 8 bits of the N-bit bucket: a rank
//            pass (digit + rank in the 2048-query tile by one shared-memory atomic), then a
//            move pass that stages each tile in digit order so that every bin's run is
//            written by consecutive lanes; persistent CTAs reserve bin space once per bin;
//   level 2  (psa_levels = 2, large trees) the same rank + move on the next 8 bits inside
//            every level-1 segment, tile bases from per-segment column scans;
//   chunk    every 4096/8192-query chunk of that order (bucket-aligned chunks after level 2)
//            is counting-sorted by its full N-bit bucket in shared memory.
// One level orders each chunk by all N bits and the chunks by the top 8 bits; two levels
// order the whole window.  Order inside a bucket is free (C-A12).
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
// 4096-query tiles (the two-level path, both levels): 3 resident CTAs per SM, so the 16
// queries per thread fit in registers (at 4 the 64-register cap spilled; c4 move 1.16 -> 1.08
// ms, return 1.41 -> 1.27 ms; the 2048-query tiles of the one-level path keep 4)
#ifndef HM_MOVE_MINB4
#define HM_MOVE_MINB4 3
#endif
#ifndef HM_UNMOVE_MINB4
#define HM_UNMOVE_MINB4 3
#endif
#ifndef HM_L1_WAVES
#define HM_L1_WAVES 6
#endif
#ifndef HM_L1_WAVES_MV
#define HM_L1_WAVES_MV 16
#endif

namespace {

#ifndef HM_SORT_THREADS
#define HM_SORT_THREADS 512
#endif
constexpr int kSortThreads = HM_SORT_THREADS;
constexpr int kChunk = (int)kPsaChunk;                   // queries per chunk-sort chunk (4096)
constexpr int kLocalBits = 11;                           // chunk sort: 2048 local buckets

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
// per thread).  Narrow: 256 bins, 2048-query tiles (runs of ~8 queries per bin): the PSA levels
// and the multi-GPU router.  (An 11-bit level with 4096-query tiles was measured slower: its
// 2-query runs made the moves 3x slower.)
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
__global__ void __launch_bounds__(C::NT, (C::BINS == 256 ? (C::TILE == 4096 ? HM_MOVE_MINB4 : HM_MOVE_MINB) : C::MINB)) k_psa2_move(const uint64_t* __restrict__ q, uint64_t n, Digit dg,
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
__global__ void __launch_bounds__(C::NT, (C::BINS == 256 ? (C::TILE == 4096 ? HM_UNMOVE_MINB4 : HM_UNMOVE_MINB) : C::MINB)) k_psa2_unmove(const uint32_t* __restrict__ tile_counts,
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
    // rounds of <= 8 slots per thread: all loads of a round in flight before its stores (16
    // per thread at 4096-query tiles spilled past the 64-register cap)
#ifndef HM_UNMOVE_R
#define HM_UNMOVE_R 8
#endif
    constexpr int R = C::PER < HM_UNMOVE_R ? C::PER : HM_UNMOVE_R;
#pragma unroll
    for (int k0 = 0; k0 < C::PER; k0 += R) {
      uint64_t rv[R];
      uint32_t oo[R];
#pragma unroll
      for (int k = 0; k < R; ++k) {
        const uint32_t i = (k0 + k) * C::NT + threadIdx.x;
        if (i < tile_n) {
          const uint32_t od = st_od[i], dd = od >> C::TILE_SHIFT;
          oo[k] = od & (C::TILE - 1);
          rv[k] = __ldg(res1 + gbase[dd] + (i - bin_start[dd]));
        }
      }
#pragma unroll
      for (int k = 0; k < R; ++k)
        if ((k0 + k) * C::NT + threadIdx.x < tile_n) st_r[oo[k]] = rv[k];
    }
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

// ---- second MSD level (Plan::psa_levels == 2) ----------------------------------------------
// P:L418-L428 sorts the window by its top Nb bits.  Level 1 orders it by the top 8 bits; this
// level orders every level-1 segment (one 8-bit bucket) by the next 8 bits with the same rank
// + staged-move scheme on segment-aligned 2048-query tiles, so the level-2 order is sorted by
// the top 16 bits.  The chunk sort then runs on chunks made of whole 16-bit buckets (groups of
// Plan::l2_group consecutive buckets, each group padded to a multiple of 8 slots), which makes
// the whole window sorted by all Nb bits.  Tile bases are computed by per-segment column scans
// (deterministic; no global atomics).
#ifndef HM_L2_TILE
#define HM_L2_TILE 4096  // measured: 4096-query tiles (runs of ~16) beat 2048 in the two-level path
#endif
using L2C = L1Cfg<8, HM_L2_TILE, 256>;
// the two-level path's level 1 uses the same tile (its moves gain more than its unmoves lose)
using Narrow4 = L1Cfg<8, HM_L2_TILE, 256>;

struct L2Digit {
  BucketBits f;
  uint32_t shift;  // nb - 16
  __device__ __forceinline__ uint32_t operator()(uint64_t q) const { return (f(q) >> shift) & 255u; }
};

// segment starts from the level-1 bin counts, and the first level-2 tile of every segment
__global__ void __launch_bounds__(256) k_l2_segs(const uint32_t* __restrict__ counts, uint32_t* __restrict__ seg) {
  __shared__ uint32_t tmp[256 / 32 + 1];
  const uint32_t c = counts[threadIdx.x];
  uint32_t tot_n, tot_t;
  const uint32_t s0 = block_scan<256>(c, tmp, &tot_n);
  const uint32_t t0 = block_scan<256>((c + L2C::TILE - 1) / L2C::TILE, tmp, &tot_t);
  seg[threadIdx.x] = s0;
  seg[257 + threadIdx.x] = t0;
  if (threadIdx.x == 0) {
    seg[256] = tot_n;
    seg[257 + 256] = tot_t;
  }
}

// tile t of level 2 -> its segment, first level-1 position and length (s_seg: seg[] in smem)
__device__ __forceinline__ void l2_tile(const uint32_t* s_seg, uint32_t t, uint32_t* s, uint32_t* t0, uint32_t* len) {
  const uint32_t* tf = s_seg + 257;
  uint32_t lo = 0, hi = 256;  // largest s with tf[s] <= t
  while (hi - lo > 1) {
    const uint32_t mid = (lo + hi) >> 1;
    if (tf[mid] <= t) lo = mid;
    else hi = mid;
  }
  *s = lo;
  *t0 = s_seg[lo] + (t - tf[lo]) * L2C::TILE;
  const uint32_t end = s_seg[lo + 1];
  *len = end - *t0 < (uint32_t)L2C::TILE ? end - *t0 : (uint32_t)L2C::TILE;
}
__device__ __forceinline__ void l2_tile_range(const uint32_t* s_seg, uint32_t* tb, uint32_t* te) {
  const uint64_t T = s_seg[257 + 256];
  *tb = (uint32_t)((uint64_t)blockIdx.x * T / gridDim.x);
  *te = (uint32_t)((uint64_t)(blockIdx.x + 1) * T / gridDim.x);
}
__device__ __forceinline__ void l2_load_seg(uint32_t* s_seg, const uint32_t* __restrict__ seg) {
  for (int i = threadIdx.x; i < 2 * 257; i += blockDim.x) s_seg[i] = seg[i];
  __syncthreads();
}

// rank pass: each query's level-2 digit and its rank among the tile's queries with that digit
__global__ void __launch_bounds__(L2C::NT, L2C::MINB) k_psa2_rank_s(const uint64_t* __restrict__ q1, L2Digit dg,
                                                                   const uint32_t* __restrict__ seg,
                                                                   uint32_t* __restrict__ packed2,
                                                                   uint32_t* __restrict__ tile_counts2) {
  __shared__ uint32_t s_seg[2 * 257];
  __shared__ uint32_t cnt[L2C::BINS];
  l2_load_seg(s_seg, seg);
  uint32_t tb, te;
  l2_tile_range(s_seg, &tb, &te);
  for (uint32_t tile = tb; tile < te; ++tile) {
    uint32_t s, t0, len;
    l2_tile(s_seg, tile, &s, &t0, &len);
    uint64_t v[L2C::PER];
#pragma unroll
    for (int k = 0; k < L2C::PER; ++k) {
      const uint32_t i = k * L2C::NT + threadIdx.x;
      v[k] = i < len ? __ldg(q1 + t0 + i) : 0;
    }
    cnt[threadIdx.x] = 0;
    __syncthreads();
#pragma unroll
    for (int k = 0; k < L2C::PER; ++k) {
      const uint32_t i = k * L2C::NT + threadIdx.x;
      if (i < len) {
        const uint32_t d = dg(v[k]);
        packed2[t0 + i] = d | (atomicAdd(&cnt[d], 1u) << 8);
      }
    }
    __syncthreads();
    tile_counts2[(uint64_t)tile * 256 + threadIdx.x] = cnt[threadIdx.x];
    __syncthreads();
  }
}

// per segment (one CTA) and digit (one thread): queries per 16-bit bucket
__global__ void __launch_bounds__(256) k_l2_colsum(const uint32_t* __restrict__ seg,
                                                   const uint32_t* __restrict__ tile_counts2,
                                                   uint32_t* __restrict__ comp_cnt) {
  const uint32_t s = blockIdx.x, t0 = seg[257 + s], t1 = seg[257 + s + 1];
  uint32_t acc = 0;
  for (uint32_t t = t0; t < t1; ++t) acc += __ldg(tile_counts2 + (uint64_t)t * 256 + threadIdx.x);
  comp_cnt[s * 256 + threadIdx.x] = acc;
}

// level-2 layout: 16-bit buckets in groups of K, every group starts at a multiple of 8;
// comp_start[b] = level-2 position of bucket b; the chunk table lists each group (split into
// pieces of <= cap queries when larger); nch[0] = chunks, nch[1] = padded length.  Three short
// kernels (one thread per group): per-CTA scans, a scan of the CTA totals, then the writes.
constexpr int kLayNT = 1024;
__device__ __forceinline__ uint32_t l2_group_size(const uint32_t* __restrict__ comp_cnt, uint32_t g, uint32_t K) {
  uint32_t sz = 0;
  const uint32_t b1 = min(kL2Buckets, (g + 1) * K);
  for (uint32_t b = g * K; b < b1; ++b) sz += __ldg(comp_cnt + b);
  return sz;
}
// pass 1: per group (thread) its padded size, pieces and size; CTA-local exclusive prefixes
// of the three go to gpre[3 x ng], the CTA totals to ctot[3 x nctas]
__global__ void __launch_bounds__(kLayNT) k_l2_layout_a(const uint32_t* __restrict__ comp_cnt, uint32_t K, uint32_t cap,
                                                        uint32_t* __restrict__ gpre, uint32_t* __restrict__ ctot) {
  __shared__ uint32_t tmp[kLayNT / 32 + 1];
  const uint32_t ng = (kL2Buckets + K - 1) / K, g = blockIdx.x * kLayNT + threadIdx.x;
  const uint32_t sz = g < ng ? l2_group_size(comp_cnt, g, K) : 0;
  uint32_t t0, t1, t2;
  const uint32_t p0 = block_scan<kLayNT>((sz + 7) & ~7u, tmp, &t0);
  const uint32_t p1 = block_scan<kLayNT>((sz + cap - 1) / cap, tmp, &t1);
  const uint32_t p2 = block_scan<kLayNT>(sz, tmp, &t2);
  if (g < ng) {
    gpre[g] = p0;
    gpre[ng + g] = p1;
    gpre[2 * ng + g] = p2;
  }
  if (threadIdx.x == 0) {
    ctot[blockIdx.x] = t0;
    ctot[gridDim.x + blockIdx.x] = t1;
    ctot[2 * gridDim.x + blockIdx.x] = t2;
  }
}
// pass 2 (one CTA): exclusive scans of the CTA totals in place; the grand totals to nch
__global__ void __launch_bounds__(kLayNT) k_l2_layout_b(uint32_t* __restrict__ ctot, uint32_t nctas,
                                                        uint32_t* __restrict__ nch) {
  __shared__ uint32_t tmp[kLayNT / 32 + 1];
  for (int k = 0; k < 3; ++k) {
    const uint32_t v = threadIdx.x < nctas ? ctot[k * nctas + threadIdx.x] : 0;
    uint32_t tot;
    const uint32_t ex = block_scan<kLayNT>(v, tmp, &tot);
    if (threadIdx.x < nctas) ctot[k * nctas + threadIdx.x] = ex;
    if (threadIdx.x == 0 && k == 0) nch[1] = tot;
    if (threadIdx.x == 0 && k == 1) nch[0] = tot;
  }
}
// pass 3: bucket positions and the group's chunk entries
__global__ void __launch_bounds__(kLayNT) k_l2_layout_c(const uint32_t* __restrict__ comp_cnt, uint32_t K, uint32_t cap,
                                                        const uint32_t* __restrict__ gpre,
                                                        const uint32_t* __restrict__ ctot,
                                                        uint32_t* __restrict__ comp_start, uint2* __restrict__ chunks,
                                                        uint32_t* __restrict__ chunk_pos, const uint32_t* __restrict__ nch) {
  const uint32_t ng = (kL2Buckets + K - 1) / K, g = blockIdx.x * kLayNT + threadIdx.x;
  if (g == 0) comp_start[kL2Buckets] = nch[1];
  if (g >= ng) return;
  const uint32_t nct = gridDim.x;
  const uint32_t pos = gpre[g] + ctot[blockIdx.x];
  uint32_t ci = gpre[ng + g] + ctot[nct + blockIdx.x];
  const uint32_t rpos = gpre[2 * ng + g] + ctot[2 * nct + blockIdx.x];
  uint32_t run = pos;
  const uint32_t b1 = min(kL2Buckets, (g + 1) * K);
  for (uint32_t b = g * K; b < b1; ++b) {
    comp_start[b] = run;
    run += __ldg(comp_cnt + b);
  }
  const uint32_t sz = run - pos;
  for (uint32_t o = 0; o < sz; o += cap) {
    chunks[ci] = make_uint2(pos + o, min(cap, sz - o));
    chunk_pos[ci++] = rpos + o;
  }
}

// per segment and digit: level-2 position of every tile's digit run (column scan)
__global__ void __launch_bounds__(256) k_l2_tilebase(const uint32_t* __restrict__ seg,
                                                     const uint32_t* __restrict__ tile_counts2,
                                                     const uint32_t* __restrict__ comp_start,
                                                     uint32_t* __restrict__ tile_base2) {
  const uint32_t s = blockIdx.x, t0 = seg[257 + s], t1 = seg[257 + s + 1];
  uint32_t run = comp_start[s * 256 + threadIdx.x];
  for (uint32_t t = t0; t < t1; ++t) {
    const uint64_t i = (uint64_t)t * 256 + threadIdx.x;
    tile_base2[i] = run;
    run += __ldg(tile_counts2 + i);
  }
}

// staged move of every level-2 tile: level-1 order -> level-2 order (runs by consecutive lanes)
__global__ void __launch_bounds__(L2C::NT, (L2C::TILE == 4096 ? HM_MOVE_MINB4 : HM_MOVE_MINB)) k_psa2_move_s(const uint64_t* __restrict__ q1, L2Digit dg,
                                                                       const uint32_t* __restrict__ seg,
                                                                       const uint32_t* __restrict__ packed2,
                                                                       const uint32_t* __restrict__ tile_counts2,
                                                                       const uint32_t* __restrict__ tile_base2,
                                                                       uint64_t* __restrict__ q2) {
  __shared__ uint32_t s_seg[2 * 257];
  __shared__ __align__(16) uint64_t st_q[L2C::TILE];
  __shared__ uint32_t bin_start[L2C::BINS], gbase[L2C::BINS], tmp[L2C::NT / 32 + 1];
  l2_load_seg(s_seg, seg);
  uint32_t tb, te;
  l2_tile_range(s_seg, &tb, &te);
  for (uint32_t tile = tb; tile < te; ++tile) {
    uint32_t s, t0, len;
    l2_tile(s_seg, tile, &s, &t0, &len);
    uint64_t v[L2C::PER];
    uint32_t pk[L2C::PER];
#pragma unroll
    for (int k = 0; k < L2C::PER; ++k) {
      const uint32_t i = k * L2C::NT + threadIdx.x;
      v[k] = i < len ? __ldg(q1 + t0 + i) : 0;
      pk[k] = i < len ? __ldg(packed2 + t0 + i) : 0;
    }
    const uint64_t ti = (uint64_t)tile * 256 + threadIdx.x;
    const uint32_t c = __ldg(tile_counts2 + ti);
    gbase[threadIdx.x] = __ldg(tile_base2 + ti);
    bin_start[threadIdx.x] = block_scan<L2C::NT>(c, tmp, nullptr);
    __syncthreads();
#pragma unroll
    for (int k = 0; k < L2C::PER; ++k) {
      const uint32_t i = k * L2C::NT + threadIdx.x;
      if (i < len) st_q[bin_start[pk[k] & 255u] + (pk[k] >> 8)] = v[k];
    }
    __syncthreads();
    for (uint32_t i = threadIdx.x; i < len; i += L2C::NT) {
      const uint64_t x = st_q[i];
      const uint32_t d = dg(x);
      q2[gbase[d] + (i - bin_start[d])] = x;
    }
    __syncthreads();
  }
}

// inverse of k_psa2_move_s: res1[level-1 position] = res2[level-2 position]; reads res2 in
// runs, writes res1 contiguously
__global__ void __launch_bounds__(L2C::NT, (L2C::TILE == 4096 ? HM_UNMOVE_MINB4 : HM_UNMOVE_MINB)) k_psa2_unmove_s(const uint32_t* __restrict__ seg,
                                                                           const uint32_t* __restrict__ packed2,
                                                                           const uint32_t* __restrict__ tile_counts2,
                                                                           const uint32_t* __restrict__ tile_base2,
                                                                           const uint64_t* __restrict__ res2,
                                                                           uint64_t* __restrict__ res1) {
  __shared__ uint32_t s_seg[2 * 257];
  extern __shared__ __align__(16) unsigned char l2u_smem[];
  uint64_t* st_r = reinterpret_cast<uint64_t*>(l2u_smem);                      // TILE results
  uint32_t* st_od = reinterpret_cast<uint32_t*>(l2u_smem + L2C::TILE * 8);     // TILE offsets | digit
  __shared__ uint32_t bin_start[L2C::BINS], gbase[L2C::BINS], tmp[L2C::NT / 32 + 1];
  l2_load_seg(s_seg, seg);
  uint32_t tb, te;
  l2_tile_range(s_seg, &tb, &te);
  for (uint32_t tile = tb; tile < te; ++tile) {
    uint32_t s, t0, len;
    l2_tile(s_seg, tile, &s, &t0, &len);
    uint32_t pk[L2C::PER];
#pragma unroll
    for (int k = 0; k < L2C::PER; ++k) {
      const uint32_t i = k * L2C::NT + threadIdx.x;
      pk[k] = i < len ? __ldg(packed2 + t0 + i) : 0;
    }
    const uint64_t ti = (uint64_t)tile * 256 + threadIdx.x;
    const uint32_t c = __ldg(tile_counts2 + ti);
    gbase[threadIdx.x] = __ldg(tile_base2 + ti);
    bin_start[threadIdx.x] = block_scan<L2C::NT>(c, tmp, nullptr);
    __syncthreads();
#pragma unroll
    for (int k = 0; k < L2C::PER; ++k) {
      const uint32_t i = k * L2C::NT + threadIdx.x;
      if (i < len) st_od[bin_start[pk[k] & 255u] + (pk[k] >> 8)] = i | ((pk[k] & 255u) << L2C::TILE_SHIFT);
    }
    __syncthreads();
    constexpr int R = L2C::PER < 8 ? L2C::PER : 8;  // rounds: loads in flight before the stores
#pragma unroll
    for (int k0 = 0; k0 < L2C::PER; k0 += R) {
      uint64_t rv[R];
      uint32_t oo[R];
#pragma unroll
      for (int k = 0; k < R; ++k) {
        const uint32_t i = (k0 + k) * L2C::NT + threadIdx.x;
        if (i < len) {
          const uint32_t od = st_od[i], d = od >> L2C::TILE_SHIFT;
          oo[k] = od & (L2C::TILE - 1);
          rv[k] = __ldg(res2 + gbase[d] + (i - bin_start[d]));
        }
      }
#pragma unroll
      for (int k = 0; k < R; ++k)
        if ((k0 + k) * L2C::NT + threadIdx.x < len) st_r[oo[k]] = rv[k];
    }
    __syncthreads();
    for (uint32_t i = threadIdx.x; i < len; i += L2C::NT) res1[t0 + i] = st_r[i];
    __syncthreads();
  }
}
constexpr size_t kUnmoveSSmem = (size_t)L2C::TILE * 12;

// the queries of the level-2 chunks, pads skipped, in the order the search visits them
// (harmonia_psa_inspect)
__global__ void __launch_bounds__(256) k_l2_compact(const uint64_t* __restrict__ q2, const uint2* __restrict__ chunks,
                                                    const uint32_t* __restrict__ nch, const uint32_t* __restrict__ cpos,
                                                    uint64_t* __restrict__ out) {
  for (uint32_t c = blockIdx.x; c < nch[0]; c += gridDim.x) {
    const uint2 e = chunks[c];
    for (uint32_t i = threadIdx.x; i < e.y; i += blockDim.x) out[cpos[c] + i] = q2[e.x + i];
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
      HM_CUDA(smem_attr(k_psa2_move<Digit, C, true>, smb));
      k_psa2_move<Digit, C, true><<<gm, C::NT, smb, st>>>(q, n, dg, ws.counts, ws.counts + C::BINS, ws.tile_counts,
                                                         ws.packed, ws.cta_counts, ws.cta_base, sorted_q, idx);
    } else {
      constexpr size_t smb = move_smem<C, false, kRecompute>();
      HM_CUDA(smem_attr(k_psa2_move<Digit, C, false>, smb));
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
  HM_CUDA(smem_attr(k_psa2_unmove<C>, smb));
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
  HM_CUDA(smem_attr(k_psa2_move<BucketSplit, C, false, true>, smb));
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
                               cudaStream_t st, int level2, bool local, uint32_t chunk) {
  harmonia_status s;
  {
    const uint32_t b1 = (uint32_t)std::min(nb, Narrow::BITS);
    s = coarse_partition<Narrow>(q, n, CoarseDigit{f, (uint32_t)nb - b1}, ws, ws.sorted_q, local ? nullptr : ws.idx,
                                 sm, st, nullptr, 0);
  }
  if (s != HARMONIA_OK) return s;
  if (level2 == 2) return HARMONIA_OK;  // coarse partition only (ablation)
  {
    ProfScope ps_(HARMONIA_PROF_PSA_SCAN, st);  // reported in the "scan" class: level-2 sort
    HM_CUDA(smem_attr(k_psa2_count_sort<false, kChunk>, count_sort_smem<kChunk>()));
    HM_CUDA(smem_attr(k_psa2_count_sort<true, kChunk>, count_sort_smem<kChunk>()));
    HM_CUDA(smem_attr(k_psa2_count_sort<true, (int)kPsaChunkMax>, count_sort_smem<kPsaChunkMax>()));
#ifndef HM_SORT_CTAS_PER_SM
#define HM_SORT_CTAS_PER_SM 4
#endif
    const uint32_t ch = (local && level2 == 0 && chunk == kPsaChunkMax) ? kPsaChunkMax : (uint32_t)kChunk;
#ifndef HM_SORT_CTAS_PER_SM_8K
#define HM_SORT_CTAS_PER_SM_8K 1  // one resident CTA per SM: persistent, one TMA prefetch chain each
#endif
    const int cps = ch == kPsaChunkMax ? HM_SORT_CTAS_PER_SM_8K : HM_SORT_CTAS_PER_SM;
    const int g = (int)std::min<uint64_t>(ceil_div(n, ch), (uint64_t)sm * cps);
    if (local && ch == kPsaChunkMax)  // 8192-query chunks (denser key ranges per warp)
      k_psa2_count_sort<true, (int)kPsaChunkMax>
          <<<std::max(g, 1), kSortThreads, count_sort_smem<kPsaChunkMax>(), st>>>(ws.sorted_q, ws.idx, n, f, nullptr,
                                                                                 nullptr, ws.cbounds);
    else if (local)   // one counting pass with shared-memory atomics (default, measured faster)
      k_psa2_count_sort<true, kChunk><<<std::max(g, 1), kSortThreads, count_sort_smem<kChunk>(), st>>>(
          ws.sorted_q, ws.idx, n, f, nullptr, nullptr, ws.cbounds);
    else
      k_psa2_count_sort<false, kChunk><<<std::max(g, 1), kSortThreads, count_sort_smem<kChunk>(), st>>>(ws.sorted_q, ws.idx, n, f);
  }
  HM_LAUNCHED();
  return HARMONIA_OK;
}


// two-level PSA (Plan::psa_levels == 2) for the staged return: level 1 (rank + move on the top
// 8 bits) into ws.sorted_q, level 2 (segmented rank + move on the next 8 bits) into
// ws.sorted2, then the counting sort of the bucket-aligned chunks (K 16-bit buckets per
// group, <= cap queries per chunk) in place; ws.idx receives the chunk-local offsets.
harmonia_status psa_partition2_l2(const uint64_t* q, uint64_t n, const BucketBits& f, int nb, const PsaWs& ws, int sm,
                                  cudaStream_t st, uint32_t K, uint32_t cap) {
  if (nb < 16 || (cap != kPsaChunk && cap != kPsaChunkMax)) return HARMONIA_ERR_INVALID_ARG;
  harmonia_status s =
      coarse_partition<Narrow4>(q, n, CoarseDigit{f, (uint32_t)nb - 8}, ws, ws.sorted_q, nullptr, sm, st, nullptr, 0);
  if (s != HARMONIA_OK) return s;
  const L2Digit dg{f, (uint32_t)nb - 16};
  const int g = l1_grid<L2C>(n + 256ull * L2C::TILE, sm), gm = l1_grid_mv<L2C>(n + 256ull * L2C::TILE, sm);
  {
    ProfScope ps_(HARMONIA_PROF_PSA_HIST, st);
    k_l2_segs<<<1, 256, 0, st>>>(ws.counts, ws.seg);
    k_psa2_rank_s<<<g, L2C::NT, 0, st>>>(ws.sorted_q, dg, ws.seg, ws.packed2, ws.tile_counts2);
  }
  HM_LAUNCHED();
  {
    ProfScope ps_(HARMONIA_PROF_PSA_SCAN, st);
    k_l2_colsum<<<256, 256, 0, st>>>(ws.seg, ws.tile_counts2, ws.comp_cnt);
    const uint32_t ng = (kL2Buckets + K - 1) / K, nct = (ng + kLayNT - 1) / kLayNT;  // nct <= 64
    uint32_t* gpre = ws.l2_scratch;
    uint32_t* ctot = ws.seg + 2 * 257;
    k_l2_layout_a<<<nct, kLayNT, 0, st>>>(ws.comp_cnt, K, cap, gpre, ctot);
    k_l2_layout_b<<<1, kLayNT, 0, st>>>(ctot, nct, ws.nchunks);
    k_l2_layout_c<<<nct, kLayNT, 0, st>>>(ws.comp_cnt, K, cap, gpre, ctot, ws.comp_start, ws.chunks, ws.chunk_pos,
                                          ws.nchunks);
    k_l2_tilebase<<<256, 256, 0, st>>>(ws.seg, ws.tile_counts2, ws.comp_start, ws.tile_base2);
  }
  HM_LAUNCHED();
  {
    ProfScope ps_(HARMONIA_PROF_PSA_SCATTER, st);
    k_psa2_move_s<<<gm, L2C::NT, 0, st>>>(ws.sorted_q, dg, ws.seg, ws.packed2, ws.tile_counts2, ws.tile_base2,
                                          ws.sorted2);
  }
  HM_LAUNCHED();
  {
    ProfScope ps_(HARMONIA_PROF_PSA_SCAN, st);
    if (cap == kPsaChunkMax) {
      auto kern = k_psa2_count_sort<true, (int)kPsaChunkMax, true>;
      HM_CUDA(smem_attr(kern, count_sort_smem<kPsaChunkMax>()));
      kern<<<sm * HM_SORT_CTAS_PER_SM_8K, kSortThreads, count_sort_smem<kPsaChunkMax>(), st>>>(ws.sorted2, ws.idx, n, f,
                                                                                              ws.chunks, ws.nchunks,
                                                                                              ws.cbounds);
    } else {
      auto kern = k_psa2_count_sort<true, kChunk, true>;
      HM_CUDA(smem_attr(kern, count_sort_smem<kChunk>()));
      kern<<<sm * HM_SORT_CTAS_PER_SM, kSortThreads, count_sort_smem<kChunk>(), st>>>(ws.sorted2, ws.idx, n, f,
                                                                                      ws.chunks, ws.nchunks, ws.cbounds);
    }
  }
  HM_LAUNCHED();
  return HARMONIA_OK;
}

// inverse of the two-level partition: res2 (level-2 order) -> ws.sorted_q as level-1-order
// results (its queries are dead by now) -> out (caller order)
harmonia_status psa_unpartition2_l2(const PsaWs& ws, const uint64_t* res2, uint64_t n, uint64_t* out, int sm,
                                    cudaStream_t st) {
  if (n == 0) return HARMONIA_OK;
  {
    ProfScope ps_(HARMONIA_PROF_RETURN, st);
    HM_CUDA(smem_attr(k_psa2_unmove_s, kUnmoveSSmem));
    k_psa2_unmove_s<<<l1_grid_mv<L2C>(n + 256ull * L2C::TILE, sm), L2C::NT, kUnmoveSSmem, st>>>(
        ws.seg, ws.packed2, ws.tile_counts2, ws.tile_base2, res2, ws.sorted_q);
  }
  HM_LAUNCHED();
  return unpartition<Narrow4>(ws, ws.sorted_q, n, out, sm, st);
}

// harmonia_psa_inspect: the queries of the search's chunks in visiting order (two-level PSA)
harmonia_status psa_compact_l2(const PsaWs& ws, uint64_t* out, int sm, cudaStream_t st) {
  k_l2_compact<<<sm * 4, 256, 0, st>>>(ws.sorted2, ws.chunks, ws.nchunks, ws.chunk_pos, out);
  HM_LAUNCHED();
  return HARMONIA_OK;
}

harmonia_status psa_unpartition2(const PsaWs& ws, const uint64_t* res1, uint64_t n, uint64_t* out, int sm,
                                 cudaStream_t st) {
  if (n == 0) return HARMONIA_OK;
  return unpartition<Narrow>(ws, res1, n, out, sm, st);
}

}  // namespace hm
