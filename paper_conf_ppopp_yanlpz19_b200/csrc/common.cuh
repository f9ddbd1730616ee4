// Internal declarations shared by the translation units of libharmonia.so.
// (Product code only: nothing here is shared with oracle/.)
#pragma once

#include <cuda_runtime.h>

#include <cstddef>
#include <cstdint>

#include "../../include/harmonia.h"

namespace hm {

constexpr uint64_t kPad = 0xFFFFFFFFFFFFFFFFull;       // HARMONIA_KEY_PAD
constexpr uint64_t kNotFound = 0xFFFFFFFFFFFFFFFFull;  // HARMONIA_NOT_FOUND
constexpr unsigned kFull = 0xFFFFFFFFu;
constexpr int kBlock = 256;        // threads per CTA for the streaming kernels
#ifndef HM_QUERY_BLOCK
#define HM_QUERY_BLOCK 1024
#endif
#ifndef HM_QBPSM
#define HM_QBPSM 2
#endif
constexpr int kQueryBlocksPerSM = HM_QBPSM;
constexpr int kQueryBlock = HM_QUERY_BLOCK;  // search/range CTAs: 2 per SM, so the staged tree top is
                                   // duplicated twice per SM and L1 keeps most of its capacity

// ---- error plumbing --------------------------------------------------------------
harmonia_status cuda_fail(cudaError_t e);
void count_launch(uint64_t k = 1);

#define HM_CUDA(x)                                  \
  do {                                              \
    cudaError_t e_ = (x);                           \
    if (e_ != cudaSuccess) return hm::cuda_fail(e_); \
  } while (0)
#define HM_LAUNCHED()                                \
  do {                                               \
    hm::count_launch();                              \
    cudaError_t e_ = cudaGetLastError();             \
    if (e_ != cudaSuccess) return hm::cuda_fail(e_); \
  } while (0)

// raise a kernel's dynamic shared-memory limit to >= bytes on the current device (once per
// kernel and device; thread-safe)
cudaError_t smem_attr(const void* kern, size_t bytes);
template <class... A>
inline cudaError_t smem_attr(void (*kern)(A...), size_t bytes) {
  return smem_attr(reinterpret_cast<const void*>(kern), bytes);
}

__host__ __device__ inline uint64_t ceil_div(uint64_t a, uint64_t b) { return (a + b - 1) / b; }
// whole warps iterate a grid-stride loop uniformly when its bound is a multiple of 32
__host__ __device__ inline uint64_t round_up_dev(uint64_t n) { return (n + 31) & ~31ull; }
inline uint64_t round_up(uint64_t a, uint64_t b) { return ceil_div(a, b) * b; }

// ---- kernel timing (harmonia_profile_*): RAII event pair around one launch ---------------
void prof_record(int kind, cudaStream_t st, bool start);
extern bool g_prof_on;
struct ProfScope {
  int kind;
  cudaStream_t st;
  bool on;
  ProfScope(int k, cudaStream_t s) : kind(k), st(s), on(g_prof_on) {
    if (on) prof_record(kind, st, true);
  }
  ~ProfScope() {
    if (on) prof_record(kind, st, false);
  }
};

// ---- 1-D TMA bulk copies (cp.async.bulk, global -> shared) on an mbarrier ----------------
__device__ __forceinline__ uint32_t smem_addr(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_addr(bar)), "r"(count) : "memory");
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}
// one thread: the phase's single arrival, announcing `bytes` of transactions
__device__ __forceinline__ void bulk_expect(uint64_t* bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_addr(bar)), "r"(bytes) : "memory");
}
// copy `bytes` (% 16 == 0, both addresses 16-byte aligned) completing on bar; chunks of at
// most 64 KiB per instruction.  Every copy of a phase must be covered by its bulk_expect.
__device__ __forceinline__ void bulk_copy(void* dst, const void* src, uint32_t bytes, uint64_t* bar) {
  const uint32_t b = smem_addr(bar);
  for (uint32_t off = 0; off < bytes; off += 65536) {
    const uint32_t sz = bytes - off < 65536 ? bytes - off : 65536;
    asm volatile(
        "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
            smem_addr((char*)dst + off)),
        "l"((const char*)src + off), "r"(sz), "r"(b)
        : "memory");
  }
}
// one copy per phase: arrival + copy
__device__ __forceinline__ void bulk_load(void* dst, const void* src, uint32_t bytes, uint64_t* bar) {
  bulk_expect(bar, bytes);
  bulk_copy(dst, src, bytes, bar);
}
// shared -> global bulk copy (TMA store; bytes % 16 == 0, 16-byte aligned), one bulk group
__device__ __forceinline__ void bulk_store(void* gdst, const void* ssrc, uint32_t bytes) {
  for (uint32_t off = 0; off < bytes; off += 65536) {
    const uint32_t sz = bytes - off < 65536 ? bytes - off : 65536;
    asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"((char*)gdst + off),
                 "r"(smem_addr((const char*)ssrc + off)), "r"(sz)
                 : "memory");
  }
}
__device__ __forceinline__ void bulk_store_commit() { asm volatile("cp.async.bulk.commit_group;" ::: "memory"); }
// the issuing thread: every committed bulk store has finished READING shared memory
__device__ __forceinline__ void bulk_store_wait_read() { asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory"); }
// the issuing thread: every committed bulk store has completed (global writes performed)
__device__ __forceinline__ void bulk_store_wait_all() { asm volatile("cp.async.bulk.wait_group 0;" ::: "memory"); }
// generic-proxy shared-memory writes become visible to the async (TMA) proxy
__device__ __forceinline__ void fence_proxy_async_smem() { asm volatile("fence.proxy.async.shared::cta;" ::: "memory"); }
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
  const uint32_t b = smem_addr(bar);
  uint32_t done = 0;
  while (!done) {
    asm volatile(
        "{ .reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2; selp.u32 %0, 1, 0, p; }"
        : "=r"(done)
        : "r"(b), "r"(parity)
        : "memory");
  }
}

// ---- PSA bucket function (C-A11): bits [span-Nb, span) of clamp(q, kmin, kmax) -------
struct BucketBits {
  uint64_t kmin, kmax;
  uint32_t shift, mask;
  __device__ __forceinline__ uint32_t operator()(uint64_t q) const {
    uint64_t c = q < kmin ? kmin : (q > kmax ? kmax : q);
    return (uint32_t)(c >> shift) & mask;
  }
};

// ---- destination by splitters (partitioned multi-GPU mode) --------------------------
struct BucketSplit {
  const uint64_t* split;  // P-1 strictly increasing splitters
  uint32_t nsplit;
  __device__ __forceinline__ uint32_t operator()(uint64_t q) const {
    uint32_t lo = 0, hi = nsplit;  // count of splitters <= q
    while (lo < hi) {
      uint32_t mid = (lo + hi) >> 1;
      if (__ldg(split + mid) <= q) lo = mid + 1;
      else hi = mid;
    }
    return lo;
  }
};

}  // namespace hm

// The opaque tree of the C ABI.
struct harmonia_tree {
  int device = 0;
  uint32_t F = 0, h = 0;
  uint64_t n_keys = 0, N = 0, I = 0, L = 0;
  uint64_t level_start[HARMONIA_MAX_LEVELS + 1] = {};
  uint64_t* d_keys = nullptr;       // key region, N*F slots, BFS order
  uint32_t* d_ps = nullptr;         // prefix-sum child region, I+1 entries (+pad to 16 B)
  uint64_t* d_vals = nullptr;       // leaf-aligned values, L*F
  uint64_t* d_leaf_base = nullptr;  // records before leaf j, L+1 entries (range counts)
  uint64_t min_key = 0, max_key = 0;
  // capacities of the live arrays, spare arrays of the previous layout (an update builds into
  // them and hands the old ones back: no cudaMalloc/cudaFree per batch in steady state), and
  // build scratch (per-level subtree minima)
  size_t cap_keys = 0, cap_vals = 0, cap_ps = 0, cap_lb = 0;
  uint64_t *sp_keys = nullptr, *sp_vals = nullptr, *sp_lb = nullptr;
  uint32_t* sp_ps = nullptr;
  size_t sp_cap_keys = 0, sp_cap_vals = 0, sp_cap_ps = 0, sp_cap_lb = 0;
  uint64_t* scratch = nullptr;
  size_t scratch_cap = 0;
  float fill = 1.0f;
  int sm_count = 148;
  size_t smem_optin = 0;
  size_t smem_per_sm = 0;
  size_t l2_bytes = 0;
  size_t l2_persist_max = 0, l2_window_max = 0;  // device limits for the access-policy window
  size_t l2_persist_set = 0;                     // cudaLimitPersistingL2CacheSize this tree set
  int last_update_mode = 0;                      // 1 in place, 2 full rebuild (last update batch)
  // host-pipeline streams/events (harmonia_search_batch_host)
  cudaStream_t s_h2d = nullptr, s_d2h = nullptr;
  cudaEvent_t ev_start = nullptr, ev_in[2] = {}, ev_done[2] = {}, ev_out[2] = {};
};

namespace hm {

// ---- query plan (host) ----------------------------------------------------------------
struct Plan {
  int G = 4;
  bool g_auto = true;        // group size chosen by the library (search: G=1; range: by cap)
  bool psa = false;
  int nb = 0;                // PSA bits
  uint64_t window = 0;       // queries per PSA window
  BucketBits bucket{};
  uint32_t nbins = 0;
  int smem_levels = 0;       // staged top levels
  uint32_t smem_nodes = 0;   // nodes [0, smem_nodes) staged
  bool ps_smem = false;
  uint32_t ps_smem_bytes = 0;
  uint32_t smem_bytes = 0;   // dynamic smem of the search kernel
  bool gather = false;
  int kary = 1;              // in-node search: 1 = k-ary NTG, 0 = linear NTG (Fig 9)
  bool ilp2 = true;          // k-ary: two queries per lane group (k_ntg_search2)
  int lane_ilp = 2;          // G = 1: queries interleaved per lane (k_lane_search_u)
  int psa_level2 = 0;        // chunk sort: 0 counting, 2 none (coarse only, ablation)
  bool psa_global = false;   // one-pass Eq-2 partition with global atomics (ablation)
  bool ret = false;          // staged inverse return (chunk-local result staging + unmove)
  bool coop = false;         // G = 1 PSA path: warp-shared descent (k_lane_search_c<.., true>)
  bool range_warp = true;    // ranges: one warp per range, resolve then stream-copy (k_range_warp)
  bool range_lane = false;   // short ranges: one lane per range on the warp-shared descent
  uint32_t chunk = 4096;     // staged return: level-2 chunk (4096 or kPsaChunkMax queries)
  int psa_levels = 1;        // staged return: global MSD partition levels before the chunk sort:
                             // 1 = 8 bits; 2 = 8 + 8 bits with bucket-aligned chunks (the whole
                             // window in Eq-2 order)
  uint32_t l2_group = 0;     // psa_levels 2: 16-bit buckets per chunk group
  const void* l2_base = nullptr;  // L2 access-policy window over the unstaged internal levels
  size_t l2_bytes = 0;
  float l2_hit = 0.f;
};

// Launch kern(a) on st, carrying the plan's L2 access-policy window (if any) as a launch
// attribute: hits on the window persist in L2, everything else streams (north_star (c)).
template <typename Kern, typename Args>
cudaError_t launch_win(Kern kern, dim3 grid, dim3 block, size_t smem, cudaStream_t st, const Plan& p, const Args& a) {
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = grid;
  cfg.blockDim = block;
  cfg.dynamicSmemBytes = smem;
  cfg.stream = st;
  cudaLaunchAttribute at[1];
  if (p.l2_bytes) {
    at[0].id = cudaLaunchAttributeAccessPolicyWindow;
    at[0].val.accessPolicyWindow.base_ptr = const_cast<void*>(p.l2_base);
    at[0].val.accessPolicyWindow.num_bytes = p.l2_bytes;
    at[0].val.accessPolicyWindow.hitRatio = p.l2_hit;
    at[0].val.accessPolicyWindow.hitProp = cudaAccessPropertyPersisting;
    at[0].val.accessPolicyWindow.missProp = cudaAccessPropertyStreaming;
    cfg.attrs = at;
    cfg.numAttrs = 1;
  }
  return cudaLaunchKernelEx(&cfg, kern, a);
}

harmonia_status make_plan(const harmonia_tree* t, uint64_t n, const harmonia_query_opts* o,
                          Plan* p);
int auto_group_size(uint32_t F);
int psa_bits_for(uint64_t n_keys);

// workspace carve-up for one PSA window
struct PsaWs {
  uint32_t* counts;     // nbins
  uint32_t* tile_sums;  // ceil(nbins / kScanTile)
  uint64_t* sorted_q;   // window
  uint32_t* idx;        // window
  uint64_t* sorted_out; // window (gather mode only)
  uint32_t* packed;     // window: coarse digit | rank-in-tile << 8 (two-level PSA / router)
  uint32_t* tile_counts;// ceil(window / 2048) x 256 per-tile coarse bin counts
  uint32_t* cta_counts; // kL1CtaRows: per level-1 CTA bin totals
  uint32_t* cta_base;   // kL1CtaRows: per level-1 CTA first global slot of each bin
  // ---- second MSD level (Plan::psa_levels == 2), inside the level-1 segments
  uint32_t* seg;        // [0..256] level-1 segment starts, [257..513] first level-2 tile per segment,
                        // then 3 x 64 words of the layout's CTA totals
  uint32_t* l2_scratch; // 3 x 65536 words: the layout's per-group prefixes
  uint32_t* packed2;    // window: level-2 digit | rank-in-tile << 8, at level-1 positions
  uint32_t* tile_counts2;  // level-2 tiles x 256 digit counts
  uint32_t* tile_base2;    // level-2 tiles x 256: level-2 position of each tile's digit run
  uint32_t* comp_cnt;   // 65536 queries per 16-bit bucket
  uint32_t* comp_start; // 65537 level-2 position of each 16-bit bucket (chunk groups padded to 8)
  uint2* chunks;        // chunk table (start, queries): bucket-aligned chunks of <= Plan::chunk
  uint32_t* chunk_pos;  // queries before each chunk (unpadded; harmonia_psa_inspect)
  uint32_t* nchunks;    // [0] chunks, [1] padded level-2 length
  uint64_t* sorted2;    // level-2 order (window + padding)
  uint64_t* res2;       // results in level-2 order (window + padding)
  uint2* cbounds;       // staged return: per chunk, its smallest and largest Nb-bit bucket (the
                        // chunk sort writes them; the search starts every warp below the
                        // chunk's shared path)
};
constexpr uint32_t kL2Buckets = 65536;  // 16-bit composite buckets of the two MSD levels
inline uint64_t cbounds_entries(uint64_t window) { return window / 4096 + kL2Buckets + 4; }  // x 8 bytes
constexpr uint64_t kL1CtaRows = 2048 * 2048;  // >= (level-1 CTAs) x (bins) for every tiling
constexpr uint32_t kPsaTile = 2048;   // level-1 tile (queries), 256-bin configuration
// bytes of one per-(tile, bin) array: max over the level-1 tilings (256 bins / 2048-query
// tiles; 2048 bins / 4096- or 8192-query tiles), 4 bytes per (tile, bin)
inline uint64_t l1_rows_bytes(uint64_t window) {
  const uint64_t a = (window + 2047) / 2048 * 256 * 4, b = (window + 4095) / 4096 * 2048 * 4,
                 c = (window + 8191) / 8192 * 2048 * 4;
  return a > b ? (a > c ? a : c) : (b > c ? b : c);
}
#ifndef HM_IDX16
#define HM_IDX16 1  // staged return: chunk-local level-1 offsets stored as uint16 (< 2^16)
#endif
constexpr uint32_t kPsaChunk = 4096;     // level-2 chunk (queries): the LSD / non-staged sorts
constexpr uint32_t kPsaChunkMax = 8192;  // staged-return chunk sizes: 4096 or 8192 (Plan::chunk)
#ifndef HM_CHUNK8K_QPL
#define HM_CHUNK8K_QPL 192
#endif
constexpr uint64_t kChunk8kMinQueriesPerLeaf = HM_CHUNK8K_QPL;  // auto 8192 chunks from this density
constexpr uint32_t kScanTile = 4096;
// second MSD level: level-2 tiles (segment-aligned 2048-query tiles), chunk-table entries and
// the padded level-2 length (every chunk group is padded to a multiple of 8 queries, so chunk
// starts stay 16-byte aligned for the TMA copies)
struct L2Sizes {
  uint64_t tiles, chunks, padded;
};
inline L2Sizes l2_sizes(uint64_t window, uint32_t chunk) {
  return {(window + 2047) / 2048 + 256, window / chunk + kL2Buckets + 1, window + 8 * kL2Buckets};
}
inline uint64_t l2_ws_bytes(uint64_t window, uint32_t chunk) {
  const L2Sizes z = l2_sizes(window, chunk);
  auto r = [](uint64_t b) { return (b + 255) / 256 * 256; };
  return r((2 * 257 + 3 * 64) * 4) + r(3 * kL2Buckets * 4) + r(window * 4) + 2 * r(z.tiles * 256 * 4) + r(kL2Buckets * 4) + r((kL2Buckets + 1) * 4) +
         r(z.chunks * 8) + r(z.chunks * 4) + 256 + 2 * r(z.padded * 8) + r(z.padded * 2);
}
size_t psa_ws_bytes(const Plan& p);
PsaWs psa_ws_carve(const Plan& p, void* base);

// ---- kernels launchers (each returns after enqueue) ----------------------------------
template <class Bucket>
harmonia_status psa_partition(const uint64_t* q, uint64_t n, const Bucket& f, uint32_t nbins,
                              const PsaWs& ws, int sm_count, cudaStream_t st,
                              uint64_t* h_counts /* optional: sync copy of counts */);

// rank-mode results (update locate, short ranges): (leaf << 32) | #keys <= q | kRankHit when
// the leaf holds q (the in-place update needs no second read of the key)
constexpr uint32_t kRankHit = 0x80000000u;

struct SearchArgs {
  const uint64_t* keys;
  const uint32_t* ps;
  const uint64_t* vals;
  uint64_t leaf_start;
  uint32_t h;
  uint32_t smem_levels;
  uint32_t smem_nodes;
  uint32_t ps_smem_bytes;  // 0 = PS read from global
  const uint64_t* q;       // queries (PSA-sorted or caller order)
  const uint32_t* idx;     // original position within the window (nullptr = identity)
  uint64_t n;
  uint64_t* out;           // results: out[idx ? idx[j] : j]
  BucketBits bucket;       // PSA bucket (two-level PSA: the chunks' key intervals)
  uint32_t staged;         // staged return: idx holds chunk-local level-1 offsets and results
                           // go through shared memory (at dynamic-smem offset res_smem_off)
                           // to out[] in level-1 order, chunk by chunk (kPsaChunk)
  uint32_t res_smem_off;
  uint32_t chunk;          // staged return: level-2 chunk (queries), 4096 or 8192
  const uint2* ctab;       // chunk table (start, queries) instead of fixed chunks (psa_levels 2)
  const uint2* cbounds;    // per chunk: min/max PSA bucket (nullptr = descend from the root)
  const uint32_t* nctab;   // device: chunks in ctab
  // warp-shared descent (G = 1 PSA path): clamp(q) -> (clamp(q) - kmin) >> cshift is a
  // monotone 32-bit image of the key, so two 32-bit warp reductions bound the warp's queries
  uint32_t coop;
  uint32_t cshift;
  uint64_t kmin, kmax;
};
harmonia_status psa_partition2(const uint64_t* q, uint64_t n, const BucketBits& f, int nb, const PsaWs& ws,
                               int sm_count, cudaStream_t st, int level2 = 0, bool local = false,
                               uint32_t chunk = kPsaChunk);
// inverse of the level-1 move for the staged return: out[e] = res1[level-1 position of e]
harmonia_status psa_unpartition2(const PsaWs& ws, const uint64_t* res1, uint64_t n, uint64_t* out, int sm,
                                 cudaStream_t st);
// two-level PSA (Plan::psa_levels == 2): partition into ws.sorted2 (chunk table ws.chunks),
// and the inverse from level-2-order results; psa_compact_l2 = the chunks without padding
harmonia_status psa_partition2_l2(const uint64_t* q, uint64_t n, const BucketBits& f, int nb, const PsaWs& ws, int sm,
                                  cudaStream_t st, uint32_t K, uint32_t cap);
harmonia_status psa_unpartition2_l2(const PsaWs& ws, const uint64_t* res2, uint64_t n, uint64_t* out, int sm,
                                    cudaStream_t st);
harmonia_status psa_compact_l2(const PsaWs& ws, uint64_t* out, int sm, cudaStream_t st);

// Entry points run on the tree's device: the current device is switched for the call and
// restored; a stream of another device is HARMONIA_ERR_DEVICE_MISMATCH.
struct DevGuard {
  int prev = -1;
  int dev = -1;
  harmonia_status status = HARMONIA_OK;
  DevGuard(int d, cudaStream_t s) : dev(d) {
    if (cudaGetDevice(&prev) != cudaSuccess) {
      status = cuda_fail(cudaGetLastError());
      prev = -1;
      return;
    }
    if (prev != dev && cudaSetDevice(dev) != cudaSuccess) {
      status = cuda_fail(cudaGetLastError());
      return;
    }
    int sd = dev;
    if (s && cudaStreamGetDevice(s, &sd) == cudaSuccess && sd != dev) status = HARMONIA_ERR_DEVICE_MISMATCH;
    cudaGetLastError();
  }
  ~DevGuard() {
    if (prev >= 0 && prev != dev) cudaSetDevice(prev);
  }
};
harmonia_status route_partition2(const uint64_t* q, uint64_t n, const BucketSplit& f, uint32_t P, const PsaWs& ws,
                                 int sm, cudaStream_t st, uint64_t* h_counts);
// fused routing over peer memory (partitioned multi-GPU mode)
harmonia_status route_count2(const uint64_t* q, uint64_t n, const BucketSplit& f, uint32_t P, const PsaWs& ws, int sm,
                             cudaStream_t st, uint64_t* h_counts);
harmonia_status route_push2(const uint64_t* q, uint64_t n, const BucketSplit& f, uint32_t P, const PsaWs& ws,
                            const uint64_t* d_push, int sm, cudaStream_t st);
harmonia_status route_return2(const PsaWs& ws, const uint64_t* back, uint64_t n, uint64_t* out, int sm,
                              cudaStream_t st);
harmonia_status segments_push(const uint64_t* src, uint32_t nseg, const uint64_t* d_desc, uint64_t max_len, int sm,
                              cudaStream_t st);
harmonia_status launch_search(const harmonia_tree* t, const Plan& p, const SearchArgs& a,
                              cudaStream_t st);

struct RangeArgs {
  const uint64_t* keys;
  const uint32_t* ps;
  const uint64_t* vals;
  const uint64_t* leaf_base;
  uint64_t leaf_start, n_nodes;
  uint32_t h;
  uint32_t smem_levels, smem_nodes, ps_smem_bytes;
  const uint64_t* lo;      // (PSA-sorted) lower bounds
  const uint64_t* hi;      // upper bounds in caller order (indexed through idx)
  const uint32_t* idx;     // nullptr = identity
  uint64_t n;
  uint32_t cap;
  uint64_t* kout;
  uint64_t* vout;
  uint32_t* counts;
};
harmonia_status launch_range(const harmonia_tree* t, const Plan& p, const RangeArgs& a,
                             cudaStream_t st);
// in-place update: out[i] = (leaf index << 32) | #keys <= q[i] in that leaf (q sorted)
harmonia_status launch_locate(const harmonia_tree* t, const uint64_t* q, uint64_t n, uint64_t* out, cudaStream_t st);
// short ranges (cap < 512, PSA-ordered lo): one lane per range on the warp-shared descent
harmonia_status launch_range_lane(const harmonia_tree* t, const Plan& p, const RangeArgs& ra, const SearchArgs& sa,
                                  cudaStream_t st);

harmonia_status launch_gather(const uint64_t* sorted_out, const uint32_t* idx, uint64_t n,
                              uint64_t* out, int sm_count, cudaStream_t st);
harmonia_status launch_scatter_back(const uint64_t* vals, const uint32_t* pos, uint64_t n,
                                    uint64_t* out, int sm_count, cudaStream_t st);

// persisting-L2 bookkeeping of the access-policy window (capi.cu): drop the persisting lines
// after a layout swap; on destroy also restore the device limit when the last tree goes
void l2_persist_reset(const harmonia_tree* t);
void l2_persist_release(harmonia_tree* t);

// layout construction (tree.cu)
harmonia_status build_layout(harmonia_tree* t, const uint64_t* d_keys, const uint64_t* d_vals,
                             uint64_t n, cudaStream_t st);
// grow a device buffer to >= need bytes (contents not kept); 1/8 headroom on reallocation
harmonia_status reserve_bytes(void** p, size_t* cap, size_t need);
// the live arrays become the spares and the spares the live arrays (pointers and capacities)
void swap_layout_buffers(harmonia_tree* t);
uint32_t level_shape(uint64_t n, uint32_t F, double fill, uint64_t* bottom_up_nodes);

}  // namespace hm
