// Batched update (§3.2.2; C-A18) as bulk-synchronous device passes.
//
// The paper applies updates on the CPU with two-grained locks, auxiliary nodes for splits and
// a post-batch "movement" of the key region (Alg 1).  Here the phase model
// (the update phase has the tree to itself) lets the whole batch be applied at once:
//   1. validate (no PAD keys, no NOT_FOUND upsert values)            k_upd_validate
//   2. stable sort of the batch by key (CUB radix sort, positions as payload)
//   3. last op per key wins (sequential semantics, C-A18)             k_upd_winners + scan
//   4. extract the current record sequence from the leaves            k_upd_extract
//   5. classify winners against it: update value in place / delete / insert
//                                                                     k_upd_classify + scans
//   6. merge kept records with the inserts (merge path by ranks)       k_upd_merge_*
//   7. rebuild the layout from the merged sequence (build_layout): the "movement" of P:L314.
// Step 4' first tries the batch in place: when every leaf it changes keeps between
// ceil((F-1)/2) and F-1 records (trees built with fill < 1 have room: the paper's
// insertion-built trees are about 69 % full), the winners are located by the Eq-1
// descent, values are overwritten, the changed leaves are re-packed where the separators route
// their keys, and leaf_base is recomputed -- the key region and PS keep their positions (the
// paper's auxiliary-node-free case).  Otherwise the affected region is the leaf suffix from
// the batch's smallest key; on the GPU re-packing that suffix and the (small) internal levels
// costs the same passes as the closed form over all leaves, so the layout is rebuilt in full
// and stays bit-identical to a fresh harmonia_build of the record set (invariant I8).
#include <cub/cub.cuh>

#include <algorithm>

#include "common.cuh"

namespace hm {
namespace {
#ifndef HM_UPDATE_IN_PLACE
#define HM_UPDATE_IN_PLACE 1
#endif
constexpr double kInPlaceMaxFill = 0.95;  // attempt in place only when the leaves have room

__global__ void k_upd_validate(const uint8_t* __restrict__ ops, const uint64_t* __restrict__ keys,
                               const uint64_t* __restrict__ vals, uint64_t n, unsigned* flags) {
  unsigned f = 0;
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x) {
    if (keys[i] == kPad) f |= 2u;
    if (ops[i] == 0 && vals[i] == kNotFound) f |= 2u;
    if (ops[i] > 1) f |= 4u;
  }
  f = __reduce_or_sync(kFull, f);
  if (f && (threadIdx.x & 31) == 0) atomicOr(flags, f);
}

__global__ void k_iota(uint32_t* __restrict__ p, uint64_t n) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x)
    p[i] = (uint32_t)i;
}

__global__ void k_gather_keys(const uint64_t* __restrict__ src, const uint32_t* __restrict__ idx, uint64_t n,
                              uint64_t* __restrict__ dst) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x)
    dst[i] = src[idx[i]];
}

// routed update payload: op, value and sequence number of routed entry i come from batch
// position pos[i]; seq = rank << 32 | pos (global batch order = rank-major, C-A18)
__global__ void k_route_update_payload(const uint8_t* __restrict__ ops, const uint64_t* __restrict__ vals,
                                       const uint32_t* __restrict__ pos, uint64_t n, uint64_t rank,
                                       uint8_t* __restrict__ ops_out, uint64_t* __restrict__ vals_out,
                                       uint64_t* __restrict__ seq_out) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x) {
    const uint32_t p = pos[i];
    ops_out[i] = ops[p];
    vals_out[i] = vals[p];
    seq_out[i] = rank << 32 | p;
  }
}

// flag[i] = 1 if sorted entry i is the last op on its key
__global__ void k_upd_winners(const uint64_t* __restrict__ sk, uint64_t n, uint32_t* __restrict__ flag) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x)
    flag[i] = (i + 1 == n || sk[i + 1] != sk[i]) ? 1u : 0u;
}

__global__ void k_upd_compact_winners(const uint64_t* __restrict__ sk, const uint32_t* __restrict__ spos,
                                      const uint32_t* __restrict__ flag, const uint32_t* __restrict__ at, uint64_t n,
                                      const uint8_t* __restrict__ ops, const uint64_t* __restrict__ vals,
                                      uint64_t* __restrict__ wk, uint8_t* __restrict__ wop, uint64_t* __restrict__ wv) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x) {
    if (flag[i]) {
      const uint32_t d = at[i], p = spos[i];
      wk[d] = sk[i];
      wop[d] = ops[p];
      wv[d] = vals[p];
    }
  }
}

// current records in key order: record r lives in leaf j at slot r - leaf_base[j]
__global__ void k_upd_extract(const uint64_t* __restrict__ kr, const uint64_t* __restrict__ lv,
                              const uint64_t* __restrict__ leaf_base, uint64_t leaf_start, uint64_t L, uint32_t F,
                              uint64_t* __restrict__ K, uint64_t* __restrict__ V) {
  for (uint64_t s = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; s < L * F; s += (uint64_t)gridDim.x * blockDim.x) {
    const uint64_t j = s / F, slot = s % F;
    const uint64_t b = leaf_base[j], c = leaf_base[j + 1] - b;
    if (slot < c) {
      K[b + slot] = kr[(leaf_start + j) * F + slot];
      V[b + slot] = lv[s];
    }
  }
}

__device__ __forceinline__ uint64_t lower_bound_u64(const uint64_t* a, uint64_t n, uint64_t x) {
  uint64_t lo = 0, hi = n;
  while (lo < hi) {
    const uint64_t mid = (lo + hi) >> 1;
    if (a[mid] < x) lo = mid + 1;
    else hi = mid;
  }
  return lo;
}

// winners vs current records: in-place value update, delete mark, or insert flag
__global__ void k_upd_classify(const uint64_t* __restrict__ wk, const uint8_t* __restrict__ wop,
                               const uint64_t* __restrict__ wv, uint64_t nw, const uint64_t* __restrict__ K,
                               uint64_t* __restrict__ V, uint64_t nk, uint32_t* __restrict__ keep,
                               uint32_t* __restrict__ ins_flag) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < nw; i += (uint64_t)gridDim.x * blockDim.x) {
    const uint64_t p = lower_bound_u64(K, nk, wk[i]);
    const bool exists = p < nk && K[p] == wk[i];
    uint32_t ins = 0;
    if (wop[i] == 0) {
      if (exists) V[p] = wv[i];  // update an existing record's value
      else ins = 1;              // insert a new record
    } else if (exists) {
      keep[p] = 0;               // delete an existing record; a missing key is a no-op
    }
    ins_flag[i] = ins;
  }
}

__global__ void k_fill_u32(uint32_t* p, uint64_t n, uint32_t v) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x)
    p[i] = v;
}

// kept record i goes to kpos[i] + #inserts with a smaller key
__global__ void k_upd_merge_kept(const uint64_t* __restrict__ K, const uint64_t* __restrict__ V,
                                 const uint32_t* __restrict__ keep, const uint32_t* __restrict__ kpos, uint64_t nk,
                                 const uint64_t* __restrict__ ik, uint64_t ni, uint64_t* __restrict__ NK,
                                 uint64_t* __restrict__ NV) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < nk; i += (uint64_t)gridDim.x * blockDim.x) {
    if (keep[i]) {
      const uint64_t d = kpos[i] + lower_bound_u64(ik, ni, K[i]);
      NK[d] = K[i];
      NV[d] = V[i];
    }
  }
}

// insert j goes to j + #kept records with a smaller key
__global__ void k_upd_merge_ins(const uint64_t* __restrict__ ik, const uint64_t* __restrict__ iv, uint64_t ni,
                                const uint64_t* __restrict__ K, const uint32_t* __restrict__ kpos, uint64_t nk,
                                uint64_t* __restrict__ NK, uint64_t* __restrict__ NV) {
  for (uint64_t j = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; j < ni; j += (uint64_t)gridDim.x * blockDim.x) {
    const uint64_t p = lower_bound_u64(K, nk, ik[j]);
    const uint64_t d = j + kpos[p];
    NK[d] = ik[j];
    NV[d] = iv[j];
  }
}

__global__ void k_upd_compact_ins(const uint64_t* __restrict__ wk, const uint64_t* __restrict__ wv,
                                  const uint32_t* __restrict__ ins_flag, const uint32_t* __restrict__ ins_at, uint64_t nw,
                                  uint64_t* __restrict__ ik, uint64_t* __restrict__ iv) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < nw; i += (uint64_t)gridDim.x * blockDim.x)
    if (ins_flag[i]) {
      ik[ins_at[i]] = wk[i];
      iv[ins_at[i]] = wv[i];
    }
}

// ---- in-place path (leaves with room: trees built with fill < 1) -------------------------
// Winners (sorted, distinct keys) located by the Eq-1 descent (launch_locate): value updates
// of existing keys are written into the leaf value array at once; inserts and deletes become
// +1 / -1 deltas of the leaf the separators route them to, and those leaves are marked.
__global__ void k_upd_ip_classify(const uint64_t* __restrict__ wk, const uint8_t* __restrict__ wop,
                                  const uint64_t* __restrict__ wv, uint64_t nw, const uint64_t* __restrict__ loc,
                                  const uint64_t* __restrict__ kr, uint64_t* __restrict__ lv, uint64_t leaf_start,
                                  uint32_t F, int32_t* __restrict__ ldelta, uint8_t* __restrict__ lflag,
                                  uint32_t* __restrict__ wleaf) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < nw; i += (uint64_t)gridDim.x * blockDim.x) {
    const uint32_t leaf = (uint32_t)(loc[i] >> 32), r = (uint32_t)loc[i] & ~kRankHit;
    const bool exists = ((uint32_t)loc[i] & kRankHit) != 0;  // the locate saw key[r-1] == wk[i]
    wleaf[i] = leaf;
    if (wop[i] == 0) {
      if (exists) {
        lv[(uint64_t)leaf * F + r - 1] = wv[i];  // update an existing record's value
      } else {
        atomicAdd(ldelta + leaf, 1);  // insert into the routed leaf
        lflag[leaf] = 1;
      }
    } else if (exists) {
      atomicAdd(ldelta + leaf, -1);  // delete; a missing key is a no-op
      lflag[leaf] = 1;
    }
  }
}

// record counts after the batch (cnt[L] = 0 for the scan); a changed leaf outside
// [min occupancy, F-1] (I3) sends the batch to the full rebuild
__global__ void k_upd_ip_check(const uint64_t* __restrict__ leaf_base, const int32_t* __restrict__ ldelta,
                               const uint8_t* __restrict__ lflag, uint64_t L, uint32_t F, uint32_t minocc,
                               uint64_t* __restrict__ cnt, unsigned* __restrict__ bad) {
  for (uint64_t j = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; j <= L; j += (uint64_t)gridDim.x * blockDim.x) {
    if (j == L) {
      cnt[L] = 0;
      continue;
    }
    const int64_t c = (int64_t)(leaf_base[j + 1] - leaf_base[j]) + ldelta[j];
    cnt[j] = (uint64_t)(c < 0 ? 0 : c);
    if (lflag[j] && (c > (int64_t)F - 1 || c < (int64_t)minocc)) atomicOr(bad, 1u);
  }
}

__device__ __forceinline__ uint64_t lower_bound_u32(const uint32_t* a, uint64_t n, uint32_t x) {
  uint64_t lo = 0, hi = n;
  while (lo < hi) {
    const uint64_t mid = (lo + hi) >> 1;
    if (a[mid] < x) lo = mid + 1;
    else hi = mid;
  }
  return lo;
}

// re-pack every marked leaf: its records merged with its winners (both ascending), PAD tail
template <int F>
__global__ void __launch_bounds__(128) k_upd_ip_leaf(const uint8_t* __restrict__ lflag, uint64_t L,
                                                     const uint64_t* __restrict__ leaf_base,
                                                     const uint32_t* __restrict__ wleaf, const uint64_t* __restrict__ wk,
                                                     const uint8_t* __restrict__ wop, const uint64_t* __restrict__ wv,
                                                     uint64_t nw, uint64_t* __restrict__ kr, uint64_t* __restrict__ lv,
                                                     uint64_t leaf_start) {
  for (uint64_t j = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; j < L; j += (uint64_t)gridDim.x * blockDim.x) {
    if (!lflag[j]) continue;
    const uint64_t wb = lower_bound_u32(wleaf, nw, (uint32_t)j), we = lower_bound_u32(wleaf, nw, (uint32_t)j + 1);
    const uint32_t c = (uint32_t)(leaf_base[j + 1] - leaf_base[j]);
    uint64_t* K = kr + (leaf_start + j) * F;
    uint64_t* V = lv + j * F;
    uint64_t ok[F - 1], ov[F - 1];
    for (uint32_t i = 0; i < c; ++i) {
      ok[i] = K[i];
      ov[i] = V[i];
    }
    uint32_t o = 0, i = 0;
    uint64_t p = wb;
    while (i < c || p < we) {
      if (p < we && (i >= c || wk[p] < ok[i])) {  // a key not in the leaf: insert (or delete no-op)
        if (wop[p] == 0) {
          K[o] = wk[p];
          V[o] = wv[p];
          ++o;
        }
        ++p;
      } else if (p < we && wk[p] == ok[i]) {      // an existing key: updated value, or deleted
        if (wop[p] == 0) {
          K[o] = ok[i];
          V[o] = wv[p];
          ++o;
        }
        ++i;
        ++p;
      } else {
        K[o] = ok[i];
        V[o] = ov[i];
        ++o;
        ++i;
      }
    }
    for (; o < F; ++o) {
      K[o] = kPad;
      V[o] = kNotFound;
    }
  }
}

// n_keys, min and max key of the tree after an in-place batch
__global__ void k_upd_ip_info(const uint64_t* __restrict__ kr, const uint64_t* __restrict__ leaf_base, uint64_t L,
                              uint64_t leaf_start, uint32_t F, uint64_t* __restrict__ info) {
  const uint64_t n = leaf_base[L];
  const uint64_t clast = leaf_base[L] - leaf_base[L - 1];
  info[0] = n;
  info[1] = kr[leaf_start * F];
  info[2] = clast ? kr[(leaf_start + L - 1) * F + clast - 1] : 0;
}

int grid_of(uint64_t n, int sm) {
  return (int)std::max<uint64_t>(1, std::min<uint64_t>(ceil_div(std::max<uint64_t>(n, 1), kBlock), (uint64_t)sm * 8));
}

// workspace layout (byte offsets), for batch n and current record count nk
struct UpdWs {
  size_t cub, sk, sk2, pos, pos2, flag, at, wk, wop, wv, K, V, keep, kpos, insf, insat, ik, iv, NK, NV, total;
};

UpdWs upd_layout(uint64_t n, uint64_t nk, size_t cub_bytes) {
  UpdWs w{};
  size_t o = 0;
  auto take = [&](size_t b) {
    size_t r = o;
    o += round_up(std::max<size_t>(b, 1), 256);
    return r;
  };
  w.cub = take(cub_bytes);
  w.sk = take(n * 8);
  w.sk2 = take(n * 8);
  w.pos = take(n * 4);
  w.pos2 = take(n * 4);
  w.flag = take((n + 1) * 4);
  w.at = take((n + 1) * 4);
  w.wk = take(n * 8);
  w.wop = take(n);
  w.wv = take(n * 8);
  w.K = take(nk * 8);
  w.V = take(nk * 8);
  w.keep = take((nk + 1) * 4);
  w.kpos = take((nk + 1) * 4);
  w.insf = take((n + 1) * 4);
  w.insat = take((n + 1) * 4);
  w.ik = take(n * 8);
  w.iv = take(n * 8);
  w.NK = take((nk + n) * 8);
  w.NV = take((nk + n) * 8);
  w.total = o;
  return w;
}

size_t cub_temp_bytes(uint64_t n, uint64_t nk) {
  size_t a = 0, b = 0, c = 0;
  cub::DeviceRadixSort::SortPairs(nullptr, a, (const uint64_t*)nullptr, (uint64_t*)nullptr, (const uint32_t*)nullptr,
                                  (uint32_t*)nullptr, (int)std::max<uint64_t>(n, 1));
  cub::DeviceScan::ExclusiveSum(nullptr, b, (const uint32_t*)nullptr, (uint32_t*)nullptr,
                                (int)std::max<uint64_t>(n + 1, 1));
  cub::DeviceScan::ExclusiveSum(nullptr, c, (const uint32_t*)nullptr, (uint32_t*)nullptr,
                                (int)std::max<uint64_t>(nk + 1, 1));
  size_t d = 0;  // in-place path: leaf_base from the leaf counts (<= nk + 1 entries)
  cub::DeviceScan::ExclusiveSum(nullptr, d, (const uint64_t*)nullptr, (uint64_t*)nullptr,
                                (int)std::max<uint64_t>(nk + 1, 1));
  return std::max({a, b, c, d});
}

}  // namespace
}  // namespace hm

using namespace hm;

extern "C" size_t harmonia_update_workspace_bytes(const harmonia_tree* t, uint64_t n) {
  if (!t) return 0;
  return upd_layout(n, t->n_keys, cub_temp_bytes(n, t->n_keys)).total + 256;
}

extern "C" harmonia_status harmonia_update_batch(harmonia_tree* t, const uint8_t* d_ops, const uint64_t* d_keys,
                                                 const uint64_t* d_values, uint64_t n, void* ws, size_t ws_bytes,
                                                 void* stream) {
  return harmonia_update_batch_seq(t, d_ops, d_keys, d_values, nullptr, n, ws, ws_bytes, stream);
}

extern "C" harmonia_status harmonia_update_batch_seq(harmonia_tree* t, const uint8_t* d_ops, const uint64_t* d_keys,
                                                     const uint64_t* d_values, const uint64_t* d_seq, uint64_t n,
                                                     void* ws, size_t ws_bytes, void* stream) {
  if (!t) return HARMONIA_ERR_INVALID_ARG;
  if (n == 0) return HARMONIA_OK;
  if (!d_ops || !d_keys || !d_values || !ws) return HARMONIA_ERR_INVALID_ARG;
  if (n >= (1ull << 31)) return HARMONIA_ERR_INVALID_ARG;
  // the CUB scans and the keep/position arrays count records in 32 bits: the
  // merged sequence of at most n_keys + n records must stay below 2^31
  if (t->n_keys + n >= (1ull << 31) - 1) return HARMONIA_ERR_TOO_LARGE;
  DevGuard dg_(t->device, (cudaStream_t)stream);
  if (dg_.status != HARMONIA_OK) return dg_.status;
  cudaStream_t st = (cudaStream_t)stream;
  const uint64_t nk = t->n_keys;
  const size_t cubb = cub_temp_bytes(n, nk);
  const UpdWs L_ = upd_layout(n, nk, cubb);
  char* base = (char*)ws;
  if ((uintptr_t)base & 255) {
    const size_t adj = 256 - ((uintptr_t)base & 255);
    if (ws_bytes < adj) return HARMONIA_ERR_INVALID_ARG;
    base += adj;
    ws_bytes -= adj;
  }
  if (ws_bytes < L_.total) return HARMONIA_ERR_INVALID_ARG;
  auto P = [&](size_t off) { return (void*)(base + off); };
  const int sm = t->sm_count;
  ProfScope prof(HARMONIA_PROF_UPDATE, st);

  // 1. validate
  unsigned* d_flags = (unsigned*)P(L_.flag);
  HM_CUDA(cudaMemsetAsync(d_flags, 0, 4, st));
  k_upd_validate<<<grid_of(n, sm), kBlock, 0, st>>>(d_ops, d_keys, d_values, n, d_flags);
  HM_LAUNCHED();
  unsigned flags = 0;
  HM_CUDA(cudaMemcpyAsync(&flags, d_flags, 4, cudaMemcpyDeviceToHost, st));
  HM_CUDA(cudaStreamSynchronize(st));
  if (flags & 2u) return HARMONIA_ERR_RESERVED;
  if (flags & 4u) return HARMONIA_ERR_INVALID_ARG;

  // 2. stable sort by key, batch position as payload
  uint64_t *sk = (uint64_t*)P(L_.sk), *sk2 = (uint64_t*)P(L_.sk2);
  uint32_t *pos = (uint32_t*)P(L_.pos), *pos2 = (uint32_t*)P(L_.pos2);
  k_iota<<<grid_of(n, sm), kBlock, 0, st>>>(pos, n);
  HM_LAUNCHED();
  size_t cb = cubb;
  if (d_seq) {  // batch order = ascending seq: present the keys in that order to the stable key sort
    HM_CUDA(cub::DeviceRadixSort::SortPairs(P(L_.cub), cb, d_seq, sk, pos, pos2, (int)n, 0, 64, st));
    count_launch(4);
    k_gather_keys<<<grid_of(n, sm), kBlock, 0, st>>>(d_keys, pos2, n, sk);
    HM_LAUNCHED();
    cb = cubb;
    HM_CUDA(cub::DeviceRadixSort::SortPairs(P(L_.cub), cb, sk, sk2, pos2, pos, (int)n, 0, 64, st));
    count_launch(4);
    std::swap(pos, pos2);  // pos2 = original batch index of each key-sorted entry
  } else {
    HM_CUDA(cub::DeviceRadixSort::SortPairs(P(L_.cub), cb, d_keys, sk2, pos, pos2, (int)n, 0, 64, st));
    count_launch(4);
  }
  // 3. winners (last op per key) and their compaction
  uint32_t *flag = (uint32_t*)P(L_.flag), *at = (uint32_t*)P(L_.at);
  k_upd_winners<<<grid_of(n, sm), kBlock, 0, st>>>(sk2, n, flag);
  HM_LAUNCHED();
  HM_CUDA(cudaMemsetAsync(flag + n, 0, 4, st));
  cb = cubb;
  HM_CUDA(cub::DeviceScan::ExclusiveSum(P(L_.cub), cb, flag, at, (int)(n + 1), st));
  count_launch(2);
  uint32_t nw32 = 0;
  HM_CUDA(cudaMemcpyAsync(&nw32, at + n, 4, cudaMemcpyDeviceToHost, st));
  uint64_t *wk = (uint64_t*)P(L_.wk), *wv = (uint64_t*)P(L_.wv);
  uint8_t* wop = (uint8_t*)P(L_.wop);
  k_upd_compact_winners<<<grid_of(n, sm), kBlock, 0, st>>>(sk2, pos2, flag, at, n, d_ops, d_values, wk, wop, wv);
  HM_LAUNCHED();
  HM_CUDA(cudaStreamSynchronize(st));
  const uint64_t nw = nw32;

  // 4'. in place when the tree has room (fill < 1): the leaves the batch changes are re-packed
  // where the separators route their keys, internal levels and PS stay (every separator still
  // bounds its subtree, I5; it need not equal the subtree minimum after deletes), leaf_base is
  // recomputed.  If a changed leaf would leave [ceil((F-1)/2), F-1] records (I3), the batch
  // takes the full rebuild below (the value writes done here are repeated there).
  t->last_update_mode = 2;
  const uint64_t L = t->L, ls0 = t->level_start[t->h - 1];
  if (HM_UPDATE_IN_PLACE && t->h >= 2 && nk >= 64 && nw > 0 &&
      (double)nk <= kInPlaceMaxFill * (double)L * (double)(t->F - 1)) {
    uint64_t* loc = (uint64_t*)P(L_.NK);
    uint64_t* cnt = (uint64_t*)P(L_.NV);
    uint64_t* info = cnt + L + 1;
    int32_t* ldelta = (int32_t*)P(L_.K);
    uint8_t* lflag = (uint8_t*)(ldelta + L);
    uint32_t* wleaf = (uint32_t*)P(L_.insf);
    unsigned* bad = (unsigned*)P(L_.flag);
    HM_CUDA(cudaMemsetAsync(ldelta, 0, L * 4 + L, st));
    HM_CUDA(cudaMemsetAsync(bad, 0, 4, st));
    harmonia_status ls_ = launch_locate(t, wk, nw, loc, st);
    if (ls_ != HARMONIA_OK) return ls_;
    k_upd_ip_classify<<<grid_of(nw, sm), kBlock, 0, st>>>(wk, wop, wv, nw, loc, t->d_keys, t->d_vals, ls0, t->F, ldelta,
                                                          lflag, wleaf);
    HM_LAUNCHED();
    k_upd_ip_check<<<grid_of(L + 1, sm), kBlock, 0, st>>>(t->d_leaf_base, ldelta, lflag, L, t->F, t->F / 2, cnt, bad);
    HM_LAUNCHED();
    unsigned hbad = 0;
    HM_CUDA(cudaMemcpyAsync(&hbad, bad, 4, cudaMemcpyDeviceToHost, st));
    HM_CUDA(cudaStreamSynchronize(st));
    if (!hbad) {
      const int g = (int)std::max<uint64_t>(1, std::min<uint64_t>(ceil_div(L, 128), (uint64_t)sm * 16));
      switch (t->F) {
#define HM_IPL(F_)                                                                                                   \
  case F_:                                                                                                           \
    k_upd_ip_leaf<F_><<<g, 128, 0, st>>>(lflag, L, t->d_leaf_base, wleaf, wk, wop, wv, nw, t->d_keys, t->d_vals, ls0); \
    break;
        HM_IPL(4) HM_IPL(8) HM_IPL(16) HM_IPL(32) HM_IPL(64) HM_IPL(128) HM_IPL(256)
#undef HM_IPL
        default:
          return HARMONIA_ERR_INVALID_ARG;
      }
      HM_LAUNCHED();
      size_t cb2 = cubb;
      HM_CUDA(cub::DeviceScan::ExclusiveSum(P(L_.cub), cb2, cnt, t->d_leaf_base, (int)(L + 1), st));
      count_launch(2);
      k_upd_ip_info<<<1, 1, 0, st>>>(t->d_keys, t->d_leaf_base, L, ls0, t->F, info);
      HM_LAUNCHED();
      uint64_t hinfo[3];
      HM_CUDA(cudaMemcpyAsync(hinfo, info, 24, cudaMemcpyDeviceToHost, st));
      HM_CUDA(cudaStreamSynchronize(st));
      t->n_keys = hinfo[0];
      t->min_key = hinfo[1];
      t->max_key = hinfo[2];
      t->last_update_mode = 1;
      return HARMONIA_OK;
    }
  }

  // 4. current records
  uint64_t *K = (uint64_t*)P(L_.K), *V = (uint64_t*)P(L_.V);
  if (nk > 0) {
    k_upd_extract<<<grid_of(t->L * t->F, sm), kBlock, 0, st>>>(t->d_keys, t->d_vals, t->d_leaf_base,
                                                               t->level_start[t->h - 1], t->L, t->F, K, V);
    HM_LAUNCHED();
  }
  // 5. classify
  uint32_t *keep = (uint32_t*)P(L_.keep), *kpos = (uint32_t*)P(L_.kpos);
  uint32_t *insf = (uint32_t*)P(L_.insf), *insat = (uint32_t*)P(L_.insat);
  k_fill_u32<<<grid_of(nk + 1, sm), kBlock, 0, st>>>(keep, nk + 1, 1u);
  HM_LAUNCHED();
  HM_CUDA(cudaMemsetAsync(keep + nk, 0, 4, st));
  HM_CUDA(cudaMemsetAsync(insf + nw, 0, 4, st));
  k_upd_classify<<<grid_of(nw, sm), kBlock, 0, st>>>(wk, wop, wv, nw, K, V, nk, keep, insf);
  HM_LAUNCHED();
  cb = cubb;
  HM_CUDA(cub::DeviceScan::ExclusiveSum(P(L_.cub), cb, keep, kpos, (int)(nk + 1), st));
  count_launch(2);
  cb = cubb;
  HM_CUDA(cub::DeviceScan::ExclusiveSum(P(L_.cub), cb, insf, insat, (int)(nw + 1), st));
  count_launch(2);
  uint32_t nkeep = 0, nins = 0;
  HM_CUDA(cudaMemcpyAsync(&nkeep, kpos + nk, 4, cudaMemcpyDeviceToHost, st));
  HM_CUDA(cudaMemcpyAsync(&nins, insat + nw, 4, cudaMemcpyDeviceToHost, st));
  uint64_t *ik = (uint64_t*)P(L_.ik), *iv = (uint64_t*)P(L_.iv);
  k_upd_compact_ins<<<grid_of(nw, sm), kBlock, 0, st>>>(wk, wv, insf, insat, nw, ik, iv);
  HM_LAUNCHED();
  HM_CUDA(cudaStreamSynchronize(st));

  // 6. merge
  const uint64_t nn = (uint64_t)nkeep + nins;
  uint64_t *NK = (uint64_t*)P(L_.NK), *NV = (uint64_t*)P(L_.NV);
  if (nk > 0) {
    k_upd_merge_kept<<<grid_of(nk, sm), kBlock, 0, st>>>(K, V, keep, kpos, nk, ik, nins, NK, NV);
    HM_LAUNCHED();
  }
  if (nins > 0) {
    k_upd_merge_ins<<<grid_of(nins, sm), kBlock, 0, st>>>(ik, iv, nins, K, kpos, nk, NK, NV);
    HM_LAUNCHED();
  }
  // 7. rebuild the layout into the spare arrays (the previous layout's buffers, kept by the
  // tree); on success the old arrays become the spares, on failure the tree is unchanged
  harmonia_tree old = *t;
  swap_layout_buffers(t);
  harmonia_status s = build_layout(t, NK, NV, nn, st);
  if (s != HARMONIA_OK) {
    swap_layout_buffers(t);  // live arrays back; whatever build_layout grew stays spare
    t->h = old.h;
    t->N = old.N;
    t->I = old.I;
    t->L = old.L;
    t->n_keys = old.n_keys;
    for (int l = 0; l <= HARMONIA_MAX_LEVELS; ++l) t->level_start[l] = old.level_start[l];
    return s;
  }
  l2_persist_reset(t);  // the old key region (now the spare) must not stay pinned in L2
  if (nn > 0) {
    HM_CUDA(cudaMemcpyAsync(&t->min_key, NK, 8, cudaMemcpyDeviceToHost, st));
    HM_CUDA(cudaMemcpyAsync(&t->max_key, NK + nn - 1, 8, cudaMemcpyDeviceToHost, st));
    HM_CUDA(cudaStreamSynchronize(st));
  } else {
    t->min_key = kPad;
    t->max_key = 0;
  }
  return HARMONIA_OK;
}

extern "C" int harmonia_update_last_mode(const harmonia_tree* t) { return t ? t->last_update_mode : 0; }

extern "C" harmonia_status harmonia_update_validate(const uint8_t* d_ops, const uint64_t* d_keys,
                                                    const uint64_t* d_values, uint64_t n, uint32_t* d_flags,
                                                    void* stream) {
  if (!d_flags) return HARMONIA_ERR_INVALID_ARG;
  cudaStream_t st = (cudaStream_t)stream;
  HM_CUDA(cudaMemsetAsync(d_flags, 0, 4, st));
  if (n == 0) return HARMONIA_OK;
  if (!d_ops || !d_keys || !d_values) return HARMONIA_ERR_INVALID_ARG;
  int dev = 0, sm = 148;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sm, cudaDevAttrMultiProcessorCount, dev);
  k_upd_validate<<<grid_of(n, sm), kBlock, 0, st>>>(d_ops, d_keys, d_values, n, (unsigned*)d_flags);
  HM_LAUNCHED();
  return HARMONIA_OK;
}

extern "C" harmonia_status harmonia_route_update_payload(const uint8_t* d_ops, const uint64_t* d_values,
                                                         const uint32_t* d_pos, uint64_t n, uint32_t rank,
                                                         uint8_t* d_ops_out, uint64_t* d_values_out,
                                                         uint64_t* d_seq_out, void* stream) {
  if (n == 0) return HARMONIA_OK;
  if (!d_ops || !d_values || !d_pos || !d_ops_out || !d_values_out || !d_seq_out || n >= (1ull << 32))
    return HARMONIA_ERR_INVALID_ARG;
  int dev = 0, sm = 148;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sm, cudaDevAttrMultiProcessorCount, dev);
  k_route_update_payload<<<grid_of(n, sm), kBlock, 0, (cudaStream_t)stream>>>(d_ops, d_values, d_pos, n, rank,
                                                                              d_ops_out, d_values_out, d_seq_out);
  HM_LAUNCHED();
  return HARMONIA_OK;
}
