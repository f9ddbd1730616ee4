// Query-side C ABI: planning, search/range orchestration over PSA windows, the host-buffer
// pipeline, and the multi-GPU routing helpers.  Every arithmetic step of the query path runs
// in the kernels of psa.cu / search.cu; this file only sequences launches on the caller's
// stream.
#include <algorithm>
#include <cmath>
#include <cstring>
#include <mutex>

#include "common.cuh"

namespace hm {

namespace {
#ifndef HM_L2_WINDOW
#define HM_L2_WINDOW 1
#endif
#ifndef HM_L2_WINDOW_DIV
#define HM_L2_WINDOW_DIV 8
#endif
constexpr uint32_t kSmemBudget = 48 * 1024;  // auto plan: keeps >= 4 CTAs (32 warps) per SM
constexpr uint64_t kAutoWindow = 1ull << 27;  // auto PSA window (queries): measured best, DESIGN.md §8
#ifndef HM_L16_DENSITY
#define HM_L16_DENSITY 0.5
#endif
constexpr double kL16MaxChunkDensity = HM_L16_DENSITY;  // two PSA levels below this density
constexpr uint64_t kL16MinKeys = 1ull << 27;

bool pow2(int x) { return x > 0 && (x & (x - 1)) == 0; }
}  // namespace

harmonia_status make_plan(const harmonia_tree* t, uint64_t n, const harmonia_query_opts* o, Plan* p) {
  harmonia_query_opts z;
  std::memset(&z, 0, sizeof(z));
  if (!o) o = &z;
  Plan P;
  // ---- NTG group size
  int G = o->group_size;
  if (G == 0) {
    G = auto_group_size(t->F);
    while (2 * G > (int)t->F) G /= 2;
  }
  if (!pow2(G) || G < 1 || G > 32 || 2 * G > (int)t->F) return HARMONIA_ERR_INVALID_ARG;
  P.G = G;
  P.g_auto = o->group_size == 0;
  // ---- PSA bits (Eq 2) over the occupied key span (C-A11)
  int nb = o->psa_bits;
  if (nb == 0) nb = psa_bits_for(t->n_keys);
  if (nb > 28) return HARMONIA_ERR_INVALID_ARG;
  uint64_t window = o->window ? round_up(o->window, 1024) : std::min<uint64_t>(round_up(std::max<uint64_t>(n, 1), 1024), kAutoWindow);
  if (window > (1ull << 31)) return HARMONIA_ERR_INVALID_ARG;
  P.window = window;
  if (nb > 0 && t->n_keys >= 2 && t->min_key < t->max_key) {
    const uint32_t span = 64 - __builtin_clzll(t->min_key ^ t->max_key);
    uint32_t lw = 0;
    while ((1ull << lw) < window) ++lw;
    nb = std::min<int>({nb, (int)span, (int)lw});  // more buckets than window queries only costs
    if (nb > 0) {
      P.psa = true;
      P.nb = nb;
      P.bucket.kmin = t->min_key;
      P.bucket.kmax = t->max_key;
      P.bucket.shift = span - nb;
      P.bucket.mask = (uint32_t)((1ull << nb) - 1);
      P.nbins = 1u << nb;
    }
  }
  P.gather = (o->flags & HARMONIA_QF_GATHER) != 0;
  P.kary = (o->flags & HARMONIA_QF_LINEAR) ? 0 : 1;
  P.ilp2 = (o->flags & HARMONIA_QF_ILP1) == 0;
  if (o->lane_queries != 0 && o->lane_queries != 1 && o->lane_queries != 2 && o->lane_queries != 4)
    return HARMONIA_ERR_INVALID_ARG;
#ifndef HM_LANE_ILP
#define HM_LANE_ILP 2
#endif
  P.lane_ilp = o->lane_queries ? (int)o->lane_queries : HM_LANE_ILP;
  // flag bits of removed ablations (ABI 1: fused chunk sort, LSD chunk sort, 11-bit level 1;
  // all measured slower) are rejected
  if (o->flags & (HARMONIA_QF_REMOVED_FUSE_SORT | HARMONIA_QF_REMOVED_PSA_LSD | HARMONIA_QF_REMOVED_PSA_WIDE))
    return HARMONIA_ERR_INVALID_ARG;
  P.psa_level2 = (o->flags & HARMONIA_QF_PSA_COARSE) ? 2 : 0;
  P.psa_global = (o->flags & HARMONIA_QF_PSA_GLOBAL) != 0;
  // ---- shared-memory staging plan: PS first (P:L272 keeps the PS top on chip), then the
  // top levels in BFS order while they fit
  const uint32_t ps_bytes = (uint32_t)round_up((t->I + 1) * 4, 16);
  const uint32_t limit = (uint32_t)std::min<size_t>(t->smem_optin > 1024 ? t->smem_optin - 1024 : 0, 200 * 1024);
  const uint32_t budget = o->smem_levels > 0 ? limit : std::min(kSmemBudget, limit);
  // (a larger budget that stages the PS of bigger trees was measured 1.7-2.4x slower at c3:
  // the shared memory it takes comes out of the L1 that caches the leaves)
  const uint64_t qpl = t->L ? std::min<uint64_t>(n, P.window) / t->L : 0;
  P.chunk = o->sort_chunk == kPsaChunkMax || (o->sort_chunk == 0 && qpl >= kChunk8kMinQueriesPerLeaf)
                ? kPsaChunkMax : kPsaChunk;
  uint32_t used = 0;
  int lv = 0;
  if (o->smem_levels >= 0) {
    if (!(o->flags & HARMONIA_QF_NO_PS_SMEM) && t->I > 0 && ps_bytes <= budget) {
      P.ps_smem = true;
      P.ps_smem_bytes = ps_bytes;
      used = ps_bytes;
    }
    const int want = o->smem_levels > 0 ? std::min<int>(o->smem_levels, (int)t->h) : (int)t->h;
    while (lv < want && used + t->level_start[lv + 1] * t->F * 8 <= budget) ++lv;
  }
  P.smem_levels = lv;
  P.smem_nodes = (uint32_t)t->level_start[lv];
  P.smem_bytes = used + P.smem_nodes * t->F * 8;
  // staged return (default for the G = 1 PSA path): results leave the search in level-1
  // order through a chunk x 8-byte shared-memory stage, k_psa2_unmove restores the caller's
  // order; two 1024-thread CTAs per SM must still fit.  Chunk: 8192 queries when the window
  // holds >= 192 queries per leaf (a warp's 64 queries then span ~4 leaves instead of ~8;
  // measured +5 % at 504 and 252 queries per leaf), else 4096 (at 126, 63 and 32 the 8192
  // chunk loses 3-30 %: the denser warps gain little and the 8192 sort runs 1 CTA/SM).
  P.ret = P.psa && P.G == 1 && !P.psa_global && P.psa_level2 == 0 && !P.gather &&
          !(o->flags & HARMONIA_QF_SCATTER_RETURN) &&
          2 * (round_up(P.smem_bytes, 16) + P.chunk * 8 + 1024) <= t->smem_per_sm;
  if (!P.ret) P.chunk = kPsaChunk;
  // L2 access-policy window over the internal levels below the staged top (north_star (c):
  // the upper levels are pinned in L2 while leaves, values and query streams pass through)
  if (HM_L2_WINDOW && !(o->flags & HARMONIA_QF_NO_L2_WINDOW) && t->l2_window_max && t->l2_persist_max && t->h > 1 &&
      t->d_keys) {
    const uint64_t leaf0 = t->level_start[t->h - 1];
    const uint64_t first = std::min<uint64_t>(P.smem_nodes, leaf0);
    uint64_t bytes = (leaf0 - first) * t->F * 8;
    if (o->l2_window_bytes) bytes = std::min<uint64_t>(bytes, o->l2_window_bytes);
    bytes = std::min<uint64_t>(bytes, t->l2_window_max);
    // at most L2 / HM_L2_WINDOW_DIV: lines pinned across calls take L2 from the streaming PSA
    // passes (an 88 MB window at c3 F8 made the move pass 3x slower)
    bytes = std::min<uint64_t>(bytes, t->l2_bytes / HM_L2_WINDOW_DIV);
    if (bytes) {
      P.l2_base = t->d_keys + first * t->F;
      P.l2_bytes = bytes;
      P.l2_hit = (float)std::min(1.0, (double)t->l2_persist_max / (double)bytes);
    }
  }
  // two MSD levels (8 + 8 bits) before a bucket-aligned chunk sort puts the whole window in
  // Eq-2 order.  It costs a second rank/move/unmove round (~0.9 ms per 2^26
  // queries), which the search repays only when a level-1 chunk is very sparse in the tree:
  // 4096 x 256 / leaves queries per leaf (c2 63, 2^26 keys 0.98 -> one level; 2^28 keys 0.25
  // -> two levels: search 4.5 -> 2.1 ms, step 6.65 -> 6.19 ms).
  P.psa_levels = 1;
  if (P.ret && P.nb >= 16 && !(o->flags & HARMONIA_QF_PSA_L8)) {
    const double dens = t->L ? (double)kPsaChunk * 256.0 / (double)t->L : 1e9;
    // and only for trees far beyond L2 (>= 2^27 keys): with 2^26 keys a Zipf batch (c3) lost
    // 30 % with two levels, uniform ones broke even
    if ((o->flags & HARMONIA_QF_PSA_L16) || (dens < kL16MaxChunkDensity && t->n_keys >= kL16MinKeys))
      P.psa_levels = 2;
  }
  if (P.psa_levels == 2) {
    if (o->sort_chunk == 0) P.chunk = kPsaChunkMax;  // measured: 8192 beats 4096 at every size
    // buckets per chunk group: the group (mean + 4 sigma + padding) fits one chunk
    const double mean = (double)std::min<uint64_t>(n, P.window) / (double)kL2Buckets;
    const double fit = (double)P.chunk / (mean + 4.0 * std::sqrt(mean) + 8.0);
    P.l2_group = (uint32_t)std::max(1.0, std::min(fit, (double)kL2Buckets));
  }
  P.coop = P.ret && !(o->flags & HARMONIA_QF_PER_LANE);
  // ranges: the warp-per-range copy kernel unless a group size was requested explicitly or
  // the G-lane group walk is asked for (HARMONIA_QF_RANGE_GROUP)
  P.range_warp = o->group_size == 0 && !(o->flags & HARMONIA_QF_RANGE_GROUP);
  *p = P;
  return HARMONIA_OK;
}

static SearchArgs search_args(const harmonia_tree* t, const Plan& p) {
  SearchArgs a{};
  a.keys = t->d_keys;
  a.ps = t->d_ps;
  a.vals = t->d_vals;
  a.leaf_start = t->level_start[t->h - 1];
  a.h = t->h;
  a.smem_levels = (uint32_t)p.smem_levels;
  a.smem_nodes = p.smem_nodes;
  a.ps_smem_bytes = p.ps_smem ? p.ps_smem_bytes : 0;
  a.coop = p.coop ? 1u : 0u;
  a.kmin = t->min_key;
  a.kmax = t->max_key;
  const uint32_t span = t->min_key < t->max_key ? 64 - __builtin_clzll(t->min_key ^ t->max_key) : 0;
  a.cshift = span > 32 ? span - 32 : 0;
  return a;
}

// The device's persisting-L2 set-aside must cover the window (cudaLimitPersistingL2CacheSize
// is device-wide).  The first tree that raises it records the device's previous limit; the
// last such tree to be destroyed restores it (l2_persist_release), and a layout swap or a
// destroy drops the persisting lines (cudaCtxResetPersistingL2Cache) so stale key regions do
// not stay pinned.  false: no window this call.
namespace {
std::mutex g_l2_mu;
struct L2Dev {
  int users = 0;
  size_t saved = 0;
};
L2Dev g_l2[64];
}  // namespace

static bool ensure_l2_persist(const harmonia_tree* tc, size_t bytes) {
  harmonia_tree* t = const_cast<harmonia_tree*>(tc);
  const size_t want = std::min(bytes, t->l2_persist_max);
  if (t->l2_persist_set >= want) return true;
  std::lock_guard<std::mutex> lk(g_l2_mu);
  size_t cur = 0;
  if (cudaDeviceGetLimit(&cur, cudaLimitPersistingL2CacheSize) != cudaSuccess) {
    cudaGetLastError();
    return false;
  }
  L2Dev& d = g_l2[t->device & 63];
  const bool first_use = t->l2_persist_set == 0;
  if (cur < want) {
    if (d.users == 0) d.saved = cur;
    if (cudaDeviceSetLimit(cudaLimitPersistingL2CacheSize, want) != cudaSuccess) {
      cudaGetLastError();
      return false;
    }
    cur = want;
  } else if (d.users == 0 && first_use) {
    d.saved = cur;
  }
  if (first_use) ++d.users;
  t->l2_persist_set = cur;
  return true;
}

void l2_persist_reset(const harmonia_tree* t) {
  if (t->l2_persist_set) {
    cudaCtxResetPersistingL2Cache();
    cudaGetLastError();
  }
}

void l2_persist_release(harmonia_tree* t) {
  if (!t->l2_persist_set) return;
  std::lock_guard<std::mutex> lk(g_l2_mu);
  cudaCtxResetPersistingL2Cache();
  L2Dev& d = g_l2[t->device & 63];
  if (d.users > 0 && --d.users == 0) cudaDeviceSetLimit(cudaLimitPersistingL2CacheSize, d.saved);
  cudaGetLastError();
  t->l2_persist_set = 0;
}

static harmonia_status search_device(const harmonia_tree* t, const uint64_t* q, uint64_t n, uint64_t* out,
                                     void* ws, const Plan& p_in, cudaStream_t st) {
  if (n == 0) return HARMONIA_OK;
  Plan p = p_in;
  if (p.l2_bytes && !ensure_l2_persist(t, p.l2_bytes)) p.l2_bytes = 0;
  if (t->n_keys == 0) {  // C-A17: empty tree, every query is absent
    HM_CUDA(cudaMemsetAsync(out, 0xFF, n * 8, st));
    return HARMONIA_OK;
  }
  SearchArgs a = search_args(t, p);
  if (!p.psa) {
    a.q = q;
    a.idx = nullptr;
    a.n = n;
    a.out = out;
    return launch_search(t, p, a, st);
  }
  const PsaWs w = psa_ws_carve(p, ws);
  for (uint64_t w0 = 0; w0 < n; w0 += p.window) {
    const uint64_t nw = std::min<uint64_t>(p.window, n - w0);
    harmonia_status s = HARMONIA_OK;
    if (!p.ret) {
      s = p.psa_global ? psa_partition(q + w0, nw, p.bucket, p.nbins, w, t->sm_count, st, nullptr)
                       : psa_partition2(q + w0, nw, p.bucket, p.nb, w, t->sm_count, st, p.psa_level2);
      if (s != HARMONIA_OK) return s;
    }
    a.q = w.sorted_q;
    a.n = nw;
    if (p.ret && p.psa_levels == 2) {  // two MSD levels + bucket-aligned chunks
      if ((s = psa_partition2_l2(q + w0, nw, p.bucket, p.nb, w, t->sm_count, st, p.l2_group, p.chunk)) != HARMONIA_OK)
        return s;
      a.q = w.sorted2;
      a.idx = w.idx;
      a.out = w.res2;
      a.staged = 1;
      a.res_smem_off = (uint32_t)round_up(p.smem_bytes, 16);
      a.chunk = p.chunk;
      a.ctab = w.chunks;
      a.nctab = w.nchunks;
      a.cbounds = w.cbounds;
      a.bucket = p.bucket;
      if ((s = launch_search(t, p, a, st)) != HARMONIA_OK) return s;
      if ((s = psa_unpartition2_l2(w, w.res2, nw, out + w0, t->sm_count, st)) != HARMONIA_OK) return s;
      a.ctab = nullptr;
      a.nctab = nullptr;
      a.cbounds = nullptr;
      continue;
    }
    if (p.ret) {  // staged return: level-1-order results, then the inverse move
      s = psa_partition2(q + w0, nw, p.bucket, p.nb, w, t->sm_count, st, 0, true, p.chunk);
      if (s != HARMONIA_OK) return s;
      a.idx = w.idx;
      a.out = w.sorted_out;
      a.staged = 1;
      a.res_smem_off = (uint32_t)round_up(p.smem_bytes, 16);
      a.chunk = p.chunk;
      a.bucket = p.bucket;
      a.cbounds = w.cbounds;
      if ((s = launch_search(t, p, a, st)) != HARMONIA_OK) return s;
      a.cbounds = nullptr;
      if ((s = psa_unpartition2(w, w.sorted_out, nw, out + w0, t->sm_count, st)) != HARMONIA_OK) return s;
      continue;
    }
    if (p.gather) {
      a.idx = nullptr;
      a.out = w.sorted_out;
      if ((s = launch_search(t, p, a, st)) != HARMONIA_OK) return s;
      if ((s = launch_gather(w.sorted_out, w.idx, nw, out + w0, t->sm_count, st)) != HARMONIA_OK) return s;
    } else {
      a.idx = w.idx;
      a.out = out + w0;
      if ((s = launch_search(t, p, a, st)) != HARMONIA_OK) return s;
    }
  }
  return HARMONIA_OK;
}

static bool on_device(const void* ptr, int dev) {
  cudaPointerAttributes pa;
  if (cudaPointerGetAttributes(&pa, ptr) != cudaSuccess) {
    cudaGetLastError();
    return false;
  }
  return (pa.type == cudaMemoryTypeDevice || pa.type == cudaMemoryTypeManaged) && pa.device == dev;
}

}  // namespace hm

using namespace hm;

extern "C" size_t harmonia_search_workspace_bytes(const harmonia_tree* t, uint64_t n, const harmonia_query_opts* o) {
  if (!t) return 0;
  Plan p;
  if (make_plan(t, n, o, &p) != HARMONIA_OK) return 0;
  return psa_ws_bytes(p) + 256;
}

extern "C" harmonia_status harmonia_search_batch(const harmonia_tree* t, const uint64_t* d_q, uint64_t n,
                                                 uint64_t* d_out, void* ws, size_t ws_bytes,
                                                 const harmonia_query_opts* o, void* stream) {
  if (!t) return HARMONIA_ERR_INVALID_ARG;
  if (n == 0) return HARMONIA_OK;
  if (!d_q || !d_out) return HARMONIA_ERR_INVALID_ARG;
  DevGuard g(t->device, (cudaStream_t)stream);
  if (g.status != HARMONIA_OK) return g.status;
  if (!on_device(d_q, t->device) || !on_device(d_out, t->device)) return HARMONIA_ERR_DEVICE_MISMATCH;
  Plan p;
  harmonia_status s = make_plan(t, n, o, &p);
  if (s != HARMONIA_OK) return s;
  const size_t need = psa_ws_bytes(p);
  if (need) {
    if (!ws || ws_bytes < need) return HARMONIA_ERR_INVALID_ARG;
    if (((uintptr_t)ws & 255) != 0) {  // carve from the first 256-B boundary
      const size_t adj = 256 - ((uintptr_t)ws & 255);
      if (ws_bytes < need + adj) return HARMONIA_ERR_INVALID_ARG;
      ws = (char*)ws + adj;
    }
  }
  return search_device(t, d_q, n, d_out, ws, p, (cudaStream_t)stream);
}

extern "C" harmonia_status harmonia_query_plan(const harmonia_tree* t, uint64_t n, const harmonia_query_opts* o,
                                               harmonia_plan* out) {
  if (!t || !out) return HARMONIA_ERR_INVALID_ARG;
  Plan p;
  harmonia_status s = make_plan(t, n, o, &p);
  if (s != HARMONIA_OK) return s;
  std::memset(out, 0, sizeof(*out));
  out->group_size = p.G;
  out->psa_bits = p.psa ? p.nb : 0;
  out->smem_levels = p.smem_levels;
  out->ps_in_smem = p.ps_smem ? 1 : 0;
  out->window = p.psa ? p.window : 0;
  out->smem_bytes = p.smem_bytes;
  out->smem_nodes = p.smem_nodes;
  out->staged_return = p.ret ? 1u : 0u;
  out->lane_queries = p.G == 1 ? (uint32_t)p.lane_ilp : 0u;
  out->warp_shared = p.coop ? 1u : 0u;
  out->sort_chunk = p.ret ? p.chunk : 0u;
  out->l2_window_bytes = p.l2_bytes;
  out->psa_levels = p.psa ? (p.ret ? (uint32_t)p.psa_levels : 1u) : 0u;
  out->chunk_group = p.psa_levels == 2 ? p.l2_group : 0u;
  return HARMONIA_OK;
}

// ---- PSA order inspection (tests of the Eq-2 order) --------------------------------------
extern "C" harmonia_status harmonia_psa_inspect(const harmonia_tree* t, const uint64_t* d_q, uint64_t n,
                                                const harmonia_query_opts* o, void* ws, size_t ws_bytes,
                                                uint64_t* d_order_out, void* stream) {
  if (!t) return HARMONIA_ERR_INVALID_ARG;
  if (n == 0) return HARMONIA_OK;
  if (!d_q || !d_order_out) return HARMONIA_ERR_INVALID_ARG;
  DevGuard g(t->device, (cudaStream_t)stream);
  if (g.status != HARMONIA_OK) return g.status;
  if (!on_device(d_q, t->device) || !on_device(d_order_out, t->device)) return HARMONIA_ERR_DEVICE_MISMATCH;
  Plan p;
  harmonia_status s = make_plan(t, n, o, &p);
  if (s != HARMONIA_OK) return s;
  cudaStream_t st = (cudaStream_t)stream;
  if (!p.psa || t->n_keys == 0) {  // no partition: the search visits the caller's order
    HM_CUDA(cudaMemcpyAsync(d_order_out, d_q, n * 8, cudaMemcpyDeviceToDevice, st));
    return HARMONIA_OK;
  }
  const size_t need = psa_ws_bytes(p);
  if (!ws || ws_bytes < need) return HARMONIA_ERR_INVALID_ARG;
  if (((uintptr_t)ws & 255) != 0) {
    const size_t adj = 256 - ((uintptr_t)ws & 255);
    if (ws_bytes < need + adj) return HARMONIA_ERR_INVALID_ARG;
    ws = (char*)ws + adj;
  }
  const PsaWs w = psa_ws_carve(p, ws);
  for (uint64_t w0 = 0; w0 < n; w0 += p.window) {
    const uint64_t nw = std::min<uint64_t>(p.window, n - w0);
    if (p.ret && p.psa_levels == 2) {
      if ((s = psa_partition2_l2(d_q + w0, nw, p.bucket, p.nb, w, t->sm_count, st, p.l2_group, p.chunk)) != HARMONIA_OK)
        return s;
      if ((s = psa_compact_l2(w, d_order_out + w0, t->sm_count, st)) != HARMONIA_OK) return s;
      continue;
    }
    if (p.psa_global) s = psa_partition(d_q + w0, nw, p.bucket, p.nbins, w, t->sm_count, st, nullptr);
    else if (p.ret) s = psa_partition2(d_q + w0, nw, p.bucket, p.nb, w, t->sm_count, st, 0, true, p.chunk);
    else s = psa_partition2(d_q + w0, nw, p.bucket, p.nb, w, t->sm_count, st, p.psa_level2);
    if (s != HARMONIA_OK) return s;
    HM_CUDA(cudaMemcpyAsync(d_order_out + w0, w.sorted_q, nw * 8, cudaMemcpyDeviceToDevice, st));
  }
  return HARMONIA_OK;
}

// ---- host-buffer pipeline --------------------------------------------------------------
#ifndef HM_HOST_CHUNK_LOG
#define HM_HOST_CHUNK_LOG 22
#endif
static uint64_t host_chunk(const Plan& p, uint64_t n) {
  // 4M-query chunks: the copies (PCIe-bound) dominate, so a deeper pipeline beats larger
  // PSA windows here
  constexpr uint64_t kC = 1ull << HM_HOST_CHUNK_LOG;
  uint64_t c = std::min<uint64_t>(p.psa ? p.window : kC, kC);
  return std::max<uint64_t>(1024, std::min<uint64_t>(c, round_up(std::max<uint64_t>(n, 1), 1024)));
}

extern "C" size_t harmonia_search_host_workspace_bytes(const harmonia_tree* t, uint64_t n,
                                                       const harmonia_query_opts* o) {
  if (!t) return 0;
  Plan p;
  if (make_plan(t, std::min<uint64_t>(n, 1ull << 22), o, &p) != HARMONIA_OK) return 0;
  const uint64_t c = host_chunk(p, n);
  return psa_ws_bytes(p) + 4 * round_up(c * 8, 256) + 512;
}

extern "C" harmonia_status harmonia_search_batch_host(const harmonia_tree* tc, const uint64_t* h_q, uint64_t n,
                                                      uint64_t* h_out, void* ws, size_t ws_bytes,
                                                      const harmonia_query_opts* o, void* stream) {
  harmonia_tree* t = const_cast<harmonia_tree*>(tc);
  if (!t) return HARMONIA_ERR_INVALID_ARG;
  if (n == 0) return HARMONIA_OK;
  if (!h_q || !h_out || !ws) return HARMONIA_ERR_INVALID_ARG;
  DevGuard g(t->device, (cudaStream_t)stream);
  if (g.status != HARMONIA_OK) return g.status;
  Plan p;
  harmonia_status s = make_plan(t, std::min<uint64_t>(n, 1ull << 22), o, &p);
  if (s != HARMONIA_OK) return s;
  const uint64_t C = host_chunk(p, n);
  const size_t psa_b = psa_ws_bytes(p);
  if (ws_bytes < psa_b + 4 * round_up(C * 8, 256) + 256) return HARMONIA_ERR_INVALID_ARG;
  char* base = (char*)ws;
  if ((uintptr_t)base & 255) base += 256 - ((uintptr_t)base & 255);
  void* psa_ws = base;
  uint64_t* din[2] = {(uint64_t*)(base + psa_b), (uint64_t*)(base + psa_b + round_up(C * 8, 256))};
  uint64_t* dout[2] = {(uint64_t*)(base + psa_b + 2 * round_up(C * 8, 256)),
                       (uint64_t*)(base + psa_b + 3 * round_up(C * 8, 256))};
  cudaStream_t st = (cudaStream_t)stream;
  if (!t->s_h2d) {
    HM_CUDA(cudaStreamCreateWithFlags(&t->s_h2d, cudaStreamNonBlocking));
    HM_CUDA(cudaStreamCreateWithFlags(&t->s_d2h, cudaStreamNonBlocking));
    HM_CUDA(cudaEventCreateWithFlags(&t->ev_start, cudaEventDisableTiming));
    for (int i = 0; i < 2; ++i) {
      HM_CUDA(cudaEventCreateWithFlags(&t->ev_in[i], cudaEventDisableTiming));
      HM_CUDA(cudaEventCreateWithFlags(&t->ev_done[i], cudaEventDisableTiming));
      HM_CUDA(cudaEventCreateWithFlags(&t->ev_out[i], cudaEventDisableTiming));
    }
  }
  // order the pipeline after the caller's prior work (the query copies only when the caller
  // has not declared the host queries ready: HARMONIA_QF_HOST_UNORDERED)
  const bool unordered = o && (o->flags & HARMONIA_QF_HOST_UNORDERED);
  HM_CUDA(cudaEventRecord(t->ev_start, st));
  if (!unordered) HM_CUDA(cudaStreamWaitEvent(t->s_h2d, t->ev_start, 0));
  HM_CUDA(cudaStreamWaitEvent(t->s_d2h, t->ev_start, 0));
  const uint64_t chunks = ceil_div(n, C);
  for (uint64_t k = 0; k < chunks; ++k) {
    const int b = (int)(k & 1);
    const uint64_t off = k * C, m = std::min<uint64_t>(C, n - off);
    // din[b] consumed: by this call's chunk k-2, or (unordered) by the last chunk of an earlier
    // call that used it (an event never recorded is complete)
    if (k >= 2 || unordered) HM_CUDA(cudaStreamWaitEvent(t->s_h2d, t->ev_done[b], 0));
    HM_CUDA(cudaMemcpyAsync(din[b], h_q + off, m * 8, cudaMemcpyHostToDevice, t->s_h2d));
    HM_CUDA(cudaEventRecord(t->ev_in[b], t->s_h2d));
    HM_CUDA(cudaStreamWaitEvent(st, t->ev_in[b], 0));
    if (k >= 2) HM_CUDA(cudaStreamWaitEvent(st, t->ev_out[b], 0));  // dout[b] drained
    s = search_device(t, din[b], m, dout[b], psa_ws, p, st);
    if (s != HARMONIA_OK) return s;
    HM_CUDA(cudaEventRecord(t->ev_done[b], st));
    HM_CUDA(cudaStreamWaitEvent(t->s_d2h, t->ev_done[b], 0));
    HM_CUDA(cudaMemcpyAsync(h_out + off, dout[b], m * 8, cudaMemcpyDeviceToHost, t->s_d2h));
    HM_CUDA(cudaEventRecord(t->ev_out[b], t->s_d2h));
  }
  for (uint64_t k = (chunks >= 2 ? chunks - 2 : 0); k < chunks; ++k)
    HM_CUDA(cudaStreamWaitEvent(st, t->ev_out[k & 1], 0));
  return HARMONIA_OK;
}

// ---- range -------------------------------------------------------------------------------
extern "C" size_t harmonia_range_workspace_bytes(const harmonia_tree* t, uint64_t n, const harmonia_query_opts* o) {
  return harmonia_search_workspace_bytes(t, n, o);
}

extern "C" harmonia_status harmonia_range_batch(const harmonia_tree* t, const uint64_t* d_lo, const uint64_t* d_hi,
                                                uint64_t n, uint32_t cap, uint64_t* d_kout, uint64_t* d_vout,
                                                uint32_t* d_counts, void* ws, size_t ws_bytes,
                                                const harmonia_query_opts* o, void* stream) {
  if (!t) return HARMONIA_ERR_INVALID_ARG;
  if (n == 0) return HARMONIA_OK;
  if (!d_lo || !d_hi || !d_counts || (cap > 0 && (!d_kout || !d_vout))) return HARMONIA_ERR_INVALID_ARG;
  DevGuard g(t->device, (cudaStream_t)stream);
  if (g.status != HARMONIA_OK) return g.status;
  if (!on_device(d_lo, t->device) || !on_device(d_counts, t->device)) return HARMONIA_ERR_DEVICE_MISMATCH;
  cudaStream_t st = (cudaStream_t)stream;
  Plan p;
  harmonia_status s = make_plan(t, n, o, &p);
  if (s == HARMONIA_OK && p.l2_bytes && !ensure_l2_persist(t, p.l2_bytes)) p.l2_bytes = 0;
  if (s != HARMONIA_OK) return s;
  if (t->n_keys == 0) {
    HM_CUDA(cudaMemsetAsync(d_counts, 0, n * 4, st));
    return HARMONIA_OK;
  }
  const size_t need = psa_ws_bytes(p);
  if (need) {
    if (!ws || ws_bytes < need) return HARMONIA_ERR_INVALID_ARG;
    if (((uintptr_t)ws & 255) != 0) {
      const size_t adj = 256 - ((uintptr_t)ws & 255);
      if (ws_bytes < need + adj) return HARMONIA_ERR_INVALID_ARG;
      ws = (char*)ws + adj;
    }
  }
  RangeArgs a{};
  a.keys = t->d_keys;
  a.ps = t->d_ps;
  a.vals = t->d_vals;
  a.leaf_base = t->d_leaf_base;
  a.leaf_start = t->level_start[t->h - 1];
  a.n_nodes = t->N;
  a.h = t->h;
  a.smem_levels = (uint32_t)p.smem_levels;
  a.smem_nodes = p.smem_nodes;
  a.ps_smem_bytes = p.ps_smem ? p.ps_smem_bytes : 0;
  a.cap = cap;
  // long slabs (cap >= 512): one warp per range, resolve then stream-copy (164 G records/s at
  // len 1024); shorter ones: one lane per range on the warp-shared descent, copies by the
  // whole warp (98 / 179 / 204 G records/s at len 16 / 64 / 256 against 39 / 96 / 136 for the
  // G-lane group walk and the warp kernel), measured at c2
  const bool auto_kernel = p.range_warp;  // no group size, no QF_RANGE_GROUP
#ifndef HM_RANGE_LANE_MAX
#define HM_RANGE_LANE_MAX 512  // measured: lane kernel 1.5x at cap 256, warp kernel 1.5x at 1024
#endif
  p.range_warp = p.range_warp && cap >= HM_RANGE_LANE_MAX;
  // short slabs: one lane per range on the warp-shared descent of the PSA-ordered lo (needs
  // the PSA partition with positions, i.e. the non-staged path); DESIGN.md §8
  p.range_lane = auto_kernel && cap < HM_RANGE_LANE_MAX && p.psa && !p.psa_global && !(o && (o->flags & HARMONIA_QF_NO_RANGE_LANE));
  if (p.g_auto) {  // the leaf scan wants wide groups for long ranges (measured)
    int G = 8;
    while (G < 32 && (uint32_t)(4 * G) < cap) G *= 2;
    while (2 * G > (int)t->F) G /= 2;
    p.G = G;
  }
  if (!p.psa) {
    a.lo = d_lo;
    a.hi = d_hi;
    a.idx = nullptr;
    a.n = n;
    a.kout = d_kout;
    a.vout = d_vout;
    a.counts = d_counts;
    return launch_range(t, p, a, st);
  }
  const PsaWs w = psa_ws_carve(p, ws);
  for (uint64_t w0 = 0; w0 < n; w0 += p.window) {
    const uint64_t nw = std::min<uint64_t>(p.window, n - w0);
    s = p.psa_global ? psa_partition(d_lo + w0, nw, p.bucket, p.nbins, w, t->sm_count, st, nullptr)
                     : psa_partition2(d_lo + w0, nw, p.bucket, p.nb, w, t->sm_count, st, p.psa_level2);
    if (s != HARMONIA_OK) return s;
    a.lo = w.sorted_q;
    a.hi = d_hi + w0;
    a.idx = w.idx;
    a.n = nw;
    a.kout = d_kout ? d_kout + w0 * cap : nullptr;
    a.vout = d_vout ? d_vout + w0 * cap : nullptr;
    a.counts = d_counts + w0;
    if (p.range_lane) {
      SearchArgs sa = search_args(t, p);
      sa.n = nw;
      if ((s = launch_range_lane(t, p, a, sa, st)) != HARMONIA_OK) return s;
      continue;
    }
    if ((s = launch_range(t, p, a, st)) != HARMONIA_OK) return s;
  }
  return HARMONIA_OK;
}

// ---- multi-GPU routing helpers ---------------------------------------------------------
// the fused-routing calls keep their small host-built tables (push destinations, segment
// descriptors) in the first kRouteTables bytes of the workspace; the PSA arrays follow
constexpr size_t kRouteTables = 32 * 1024;
constexpr uint32_t kMaxSegments = 1024;

extern "C" size_t harmonia_route_workspace_bytes(uint32_t P, uint64_t n) {
  Plan p;
  p.psa = true;
  p.nbins = std::max<uint32_t>(P, 1);
  p.window = round_up(std::max<uint64_t>(n, 1), 1024);
  return psa_ws_bytes(p) + 256 + kRouteTables;
}

namespace {
// carve the routing workspace: tables first, then the PSA arrays of an n-query window
harmonia_status route_carve(uint32_t P, uint64_t n, void* ws, size_t ws_bytes, PsaWs* w, uint64_t** tables) {
  if (!ws) return HARMONIA_ERR_INVALID_ARG;
  Plan p;
  p.psa = true;
  p.nbins = std::max<uint32_t>(P, 1);
  p.window = round_up(std::max<uint64_t>(n, 1), 1024);
  if (ws_bytes < psa_ws_bytes(p) + 256 + kRouteTables) return HARMONIA_ERR_INVALID_ARG;
  if ((uintptr_t)ws & 255) ws = (char*)ws + (256 - ((uintptr_t)ws & 255));
  *tables = reinterpret_cast<uint64_t*>(ws);
  *w = psa_ws_carve(p, (char*)ws + kRouteTables);
  return HARMONIA_OK;
}
int device_sms() {
  int dev = 0, sm = 148;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sm, cudaDevAttrMultiProcessorCount, dev);
  return sm;
}
}  // namespace

extern "C" harmonia_status harmonia_route_count(const uint64_t* d_split, uint32_t P, const uint64_t* d_q, uint64_t n,
                                                uint64_t* h_counts, void* ws, size_t ws_bytes, void* stream) {
  if (P == 0 || P > 256 || !h_counts || (P > 1 && !d_split) || n >= (1ull << 32)) return HARMONIA_ERR_INVALID_ARG;
  if (n == 0) {
    for (uint32_t i = 0; i < P; ++i) h_counts[i] = 0;
    return HARMONIA_OK;
  }
  if (!d_q) return HARMONIA_ERR_INVALID_ARG;
  PsaWs w;
  uint64_t* tab;
  harmonia_status s = route_carve(P, n, ws, ws_bytes, &w, &tab);
  if (s != HARMONIA_OK) return s;
  return route_count2(d_q, n, BucketSplit{d_split, P - 1}, P, w, device_sms(), (cudaStream_t)stream, h_counts);
}

extern "C" harmonia_status harmonia_route_push(const uint64_t* d_split, uint32_t P, const uint64_t* d_q, uint64_t n,
                                               const uint64_t* h_dst, void* ws, size_t ws_bytes, void* stream) {
  if (P == 0 || P > 256 || !h_dst || (P > 1 && !d_split) || n >= (1ull << 32)) return HARMONIA_ERR_INVALID_ARG;
  if (n == 0) return HARMONIA_OK;
  if (!d_q) return HARMONIA_ERR_INVALID_ARG;
  PsaWs w;
  uint64_t* tab;
  harmonia_status s = route_carve(P, n, ws, ws_bytes, &w, &tab);
  if (s != HARMONIA_OK) return s;
  uint64_t table[256] = {};
  for (uint32_t d = 0; d < P; ++d) table[d] = h_dst[d];
  HM_CUDA(cudaMemcpyAsync(tab, table, sizeof(table), cudaMemcpyHostToDevice, (cudaStream_t)stream));
  return route_push2(d_q, n, BucketSplit{d_split, P - 1}, P, w, tab, device_sms(), (cudaStream_t)stream);
}

extern "C" harmonia_status harmonia_route_return(uint32_t P, const uint64_t* d_back, uint64_t n, uint64_t* d_out,
                                                 void* ws, size_t ws_bytes, void* stream) {
  if (P == 0 || P > 256 || n >= (1ull << 32)) return HARMONIA_ERR_INVALID_ARG;
  if (n == 0) return HARMONIA_OK;
  if (!d_back || !d_out) return HARMONIA_ERR_INVALID_ARG;
  PsaWs w;
  uint64_t* tab;
  harmonia_status s = route_carve(P, n, ws, ws_bytes, &w, &tab);
  if (s != HARMONIA_OK) return s;
  return route_return2(w, d_back, n, d_out, device_sms(), (cudaStream_t)stream);
}

extern "C" harmonia_status harmonia_segments_push(const uint64_t* d_src, uint32_t nseg, const uint64_t* h_src_off,
                                                  const uint64_t* h_len, const uint64_t* h_dst, void* ws,
                                                  size_t ws_bytes, void* stream) {
  if (nseg == 0) return HARMONIA_OK;
  if (nseg > kMaxSegments || !d_src || !h_src_off || !h_len || !h_dst || !ws || ws_bytes < kRouteTables + 256)
    return HARMONIA_ERR_INVALID_ARG;
  if ((uintptr_t)ws & 255) ws = (char*)ws + (256 - ((uintptr_t)ws & 255));
  uint64_t* tab = reinterpret_cast<uint64_t*>(ws) + 256;  // after the push-destination table
  uint64_t desc[3 * kMaxSegments];
  uint64_t max_len = 0;
  for (uint32_t s = 0; s < nseg; ++s) {
    desc[3 * s] = h_src_off[s];
    desc[3 * s + 1] = h_len[s];
    desc[3 * s + 2] = h_dst[s];
    if (h_len[s] && !h_dst[s]) return HARMONIA_ERR_INVALID_ARG;
    max_len = std::max(max_len, h_len[s]);
  }
  HM_CUDA(cudaMemcpyAsync(tab, desc, nseg * 24, cudaMemcpyHostToDevice, (cudaStream_t)stream));
  return segments_push(d_src, nseg, tab, max_len, device_sms(), (cudaStream_t)stream);
}

// ---- peer memory (CUDA IPC) for the fused routing ------------------------------------------
extern "C" harmonia_status harmonia_peer_alloc(size_t bytes, void** d_ptr, void* handle_out) {
  if (!d_ptr || !handle_out || bytes == 0) return HARMONIA_ERR_INVALID_ARG;
  void* p = nullptr;
  cudaError_t e = cudaMalloc(&p, bytes);
  if (e == cudaErrorMemoryAllocation) {
    cudaGetLastError();
    return HARMONIA_ERR_OUT_OF_MEMORY;
  }
  HM_CUDA(e);
  e = cudaMemset(p, 0, bytes);  // zero-filled (the peer barrier's flags start at epoch 0)
  if (e != cudaSuccess) {
    cudaFree(p);
    return cuda_fail(e);
  }
  cudaIpcMemHandle_t h;
  e = cudaIpcGetMemHandle(&h, p);
  if (e != cudaSuccess) {
    cudaFree(p);
    return cuda_fail(e);
  }
  std::memcpy(handle_out, &h, sizeof(h));
  *d_ptr = p;
  return HARMONIA_OK;
}

// ---- device-side barrier over peer memory (replaces the host barrier of the fused routing) ----
// Thread p (< P) publishes `epoch` into slot `me` of rank p's flag array (fence.sc.sys, then a
// system-scope release store: every store this rank's earlier kernels made on the stream --
// the pushed runs -- is visible to p before the flag), then spins with system-scope acquire
// loads until rank p's flag in this rank's array reaches `epoch`.  The kernels after it on the
// stream (the search of the receive buffer, the inverse partition) therefore see every peer's
// pushes, and no host thread waits.  A wait longer than timeout_ns sets *d_error = 1 and ends
// the kernel instead of hanging the device.
namespace hm_peer {
__device__ __forceinline__ uint64_t globaltimer_ns() {
  uint64_t t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}
__global__ void __launch_bounds__(256) k_peer_barrier(uint32_t P, uint32_t me, const uint64_t* __restrict__ flag_addrs,
                                                      const uint64_t* my_flags, uint64_t epoch, uint32_t* err,
                                                      uint64_t timeout_ns) {
  const uint32_t p = threadIdx.x;
  if (p >= P) return;
  uint64_t* f = reinterpret_cast<uint64_t*>(flag_addrs[p]) + me;
  asm volatile("fence.sc.sys;" ::: "memory");
  asm volatile("st.release.sys.global.u64 [%0], %1;" ::"l"(f), "l"(epoch) : "memory");
  const uint64_t t0 = globaltimer_ns();
  for (;;) {
    uint64_t v;
    asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(my_flags + p) : "memory");
    if (v >= epoch) break;
    if (globaltimer_ns() - t0 > timeout_ns) {
      atomicExch(err, 1u);
      break;
    }
    __nanosleep(256);
  }
}
}  // namespace hm_peer

extern "C" harmonia_status harmonia_peer_barrier(uint32_t P, uint32_t me, const uint64_t* d_flag_addrs,
                                                 uint64_t* d_my_flags, uint64_t epoch, uint32_t* d_error,
                                                 uint64_t timeout_ns, void* stream) {
  if (P == 0 || P > 256 || me >= P || !d_flag_addrs || !d_my_flags || !d_error || epoch == 0)
    return HARMONIA_ERR_INVALID_ARG;
  hm_peer::k_peer_barrier<<<1, 256, 0, (cudaStream_t)stream>>>(P, me, d_flag_addrs, d_my_flags, epoch, d_error,
                                                      timeout_ns ? timeout_ns : 30ull * 1000000000ull);
  count_launch();
  HM_CUDA(cudaGetLastError());
  return HARMONIA_OK;
}

extern "C" harmonia_status harmonia_peer_open(const void* handle, void** d_ptr) {
  if (!handle || !d_ptr) return HARMONIA_ERR_INVALID_ARG;
  cudaIpcMemHandle_t h;
  std::memcpy(&h, handle, sizeof(h));
  HM_CUDA(cudaIpcOpenMemHandle(d_ptr, h, cudaIpcMemLazyEnablePeerAccess));
  return HARMONIA_OK;
}

extern "C" harmonia_status harmonia_peer_close(void* d_ptr) {
  if (!d_ptr) return HARMONIA_ERR_INVALID_ARG;
  HM_CUDA(cudaIpcCloseMemHandle(d_ptr));
  return HARMONIA_OK;
}

extern "C" harmonia_status harmonia_peer_free(void* d_ptr) {
  if (!d_ptr) return HARMONIA_ERR_INVALID_ARG;
  HM_CUDA(cudaFree(d_ptr));
  return HARMONIA_OK;
}

extern "C" harmonia_status harmonia_route_partition(const uint64_t* d_split, uint32_t P, const uint64_t* d_q,
                                                    uint64_t n, uint64_t* d_routed, uint32_t* d_pos,
                                                    uint64_t* h_counts, void* ws, size_t ws_bytes, void* stream) {
  if (P == 0 || P > 1024 || !h_counts || (P > 1 && !d_split)) return HARMONIA_ERR_INVALID_ARG;
  if (n >= (1ull << 32)) return HARMONIA_ERR_INVALID_ARG;
  if (n == 0) {
    for (uint32_t i = 0; i < P; ++i) h_counts[i] = 0;
    return HARMONIA_OK;
  }
  if (!d_q || !d_routed || !d_pos || !ws) return HARMONIA_ERR_INVALID_ARG;
  Plan p;
  p.psa = true;
  p.nbins = P;
  p.window = round_up(n, 1024);
  if (ws_bytes < psa_ws_bytes(p) + 256) return HARMONIA_ERR_INVALID_ARG;
  if ((uintptr_t)ws & 255) ws = (char*)ws + (256 - ((uintptr_t)ws & 255));
  PsaWs w = psa_ws_carve(p, ws);
  w.sorted_q = d_routed;
  w.idx = d_pos;
  int dev = 0, sm = 148;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sm, cudaDevAttrMultiProcessorCount, dev);
  BucketSplit f{d_split, P - 1};
  if (P <= 256)  // SMEM-aggregated two-level router (one atomic per tile and shard)
    return route_partition2(d_q, n, f, P, w, sm, (cudaStream_t)stream, h_counts);
  return psa_partition(d_q, n, f, P, w, sm, (cudaStream_t)stream, h_counts);
}

extern "C" harmonia_status harmonia_scatter_results(const uint64_t* d_vals, const uint32_t* d_pos, uint64_t n,
                                                    uint64_t* d_out, void* stream) {
  if (n == 0) return HARMONIA_OK;
  if (!d_vals || !d_pos || !d_out) return HARMONIA_ERR_INVALID_ARG;
  int dev = 0, sm = 148;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sm, cudaDevAttrMultiProcessorCount, dev);
  return launch_scatter_back(d_vals, d_pos, n, d_out, sm, (cudaStream_t)stream);
}
