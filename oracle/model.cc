// O5: analytic models of §4 (PSA bit count, NTG steps and size choice, Fig 2 transactions)
// and O6: the update oracle (std::map).  TEST INFRASTRUCTURE ONLY — see oracle.h.
#include "oracle.h"

#include <algorithm>
#include <cmath>
#include <map>
#include <set>
#include <vector>

namespace {

uint64_t node_cnt(const uint64_t* kr, uint64_t node, uint32_t F) {
  uint64_t c = 0;
  while (c < F && kr[node * F + c] != ORC_PAD) ++c;
  return c;
}

// Eq-1 descent recording the node visited at each level
void path_of(const uint64_t* kr, const uint32_t* ps, uint32_t F, uint32_t h, uint64_t q,
             std::vector<uint64_t>& nodes) {
  nodes.assign(h, 0);
  uint64_t node = 0;
  for (uint32_t l = 0; l < h; ++l) {
    nodes[l] = node;
    if (l + 1 == h) break;
    uint64_t i = 1;
    for (uint32_t s = 0; s < F; ++s)
      if (kr[node * F + s] != ORC_PAD && kr[node * F + s] <= q) ++i;
    node = (uint64_t)ps[node] + i - 1;
  }
}

}  // namespace

// Eq 2: N = B - log2(2^B / T * K).  P:L428: B=64, T=2^23, K=16 -> 19.
extern "C" uint32_t orc_psa_bits(uint32_t B, double T, uint32_t K) {
  if (T <= 0) return 0;
  long double cover = std::log2(std::pow(2.0L, (long double)B) / (long double)T * (long double)K);
  long double N = (long double)B - cover;
  if (N <= 0) return 0;
  uint32_t r = (uint32_t)std::ceil(N - 1e-12L);
  return std::min(r, B);
}

// C-A11: the N most significant bits of the occupied key span [min_key, max_key].
extern "C" uint64_t orc_psa_bucket(uint64_t q, uint32_t nbits, uint64_t min_key,
                                   uint64_t max_key) {
  if (nbits == 0 || min_key >= max_key) return 0;
  uint64_t c = std::min(std::max(q, min_key), max_key);
  uint32_t span = 64 - (uint32_t)__builtin_clzll(min_key ^ max_key);  // bit length
  uint32_t nb = std::min(nbits, span);
  uint32_t shift = span - nb;
  uint64_t mask = nb >= 64 ? ~0ull : ((1ull << nb) - 1);
  return (c >> shift) & mask;
}

// orc_psa_bucket over an array (test convenience: one call instead of one per query)
extern "C" void orc_psa_buckets(const uint64_t* q, uint64_t nq, uint32_t nbits, uint64_t min_key,
                                uint64_t max_key, uint64_t* out) {
  for (uint64_t i = 0; i < nq; ++i) out[i] = orc_psa_bucket(q[i], nbits, min_key, max_key);
}

// "the queries will be sorted based on their most significant N bits" (stable).
extern "C" void orc_psa_order(const uint64_t* q, uint64_t nq, uint32_t nbits,
                              uint64_t min_key, uint64_t max_key, uint64_t* perm) {
  std::vector<uint64_t> idx(nq);
  for (uint64_t i = 0; i < nq; ++i) idx[i] = i;
  std::stable_sort(idx.begin(), idx.end(), [&](uint64_t a, uint64_t b) {
    return orc_psa_bucket(q[a], nbits, min_key, max_key) <
           orc_psa_bucket(q[b], nbits, min_key, max_key);
  });
  for (uint64_t i = 0; i < nq; ++i) perm[i] = idx[i];
}

// C-A13 (Fig 9): a group of gs threads compares gs*kpl keys per step and
// stops in the step that holds the target; a node of cnt keys needs at most
// ceil(cnt / (gs*kpl)) steps.
extern "C" uint32_t orc_ntg_steps(uint32_t r, uint32_t cnt, uint32_t gs, uint32_t kpl) {
  uint32_t w = gs * kpl;
  uint32_t full = (cnt + w - 1) / w;
  return std::min(r / w + 1, full);
}

// Eq 3/4 inputs: S = the max comparison steps a warp executes, summed over
// the profiled levels; averaged over the warps of the sample.
extern "C" double orc_ntg_warp_steps(const uint64_t* kr, const uint32_t* ps, uint32_t F,
                                     uint32_t h, const uint64_t* ls, const uint64_t* q,
                                     uint64_t nq, uint32_t gs, uint32_t kpl, uint32_t lev0,
                                     uint32_t warp) {
  (void)ls;
  // "the number of queries processed by one warp equals to warpsize/GS"; Fig 9 uses
  // a warp of 8 threads, the B200 a warp of 32.
  const uint32_t qpw = std::max<uint32_t>(1, warp / gs);
  std::vector<uint64_t> path;
  double total = 0;
  uint64_t warps = 0;
  for (uint64_t w0 = 0; w0 < nq; w0 += qpw, ++warps) {
    std::vector<uint32_t> smax(h, 0);
    for (uint64_t j = w0; j < std::min<uint64_t>(nq, w0 + qpw); ++j) {
      path_of(kr, ps, F, h, q[j], path);
      for (uint32_t l = lev0; l < h; ++l) {
        uint64_t node = path[l];
        uint32_t cnt = (uint32_t)node_cnt(kr, node, F);
        uint32_t r = 0;  // keys before the target: <= q internally, < q at the leaf
        for (uint32_t s = 0; s < cnt; ++s)
          if (l + 1 < h ? kr[node * F + s] <= q[j] : kr[node * F + s] < q[j]) ++r;
        smax[l] = std::max(smax[l], orc_ntg_steps(r, cnt, gs, kpl));
      }
    }
    for (uint32_t l = lev0; l < h; ++l) total += smax[l];
  }
  return warps ? total / (double)warps : 0.0;
}

// "the best NTG size is decided based on Equation 4.  If its value is greater
// than 1 ... narrowing the thread group can further improve performance.  This step is
// repeated until its value is smaller than 1."  Eq 4 with GS_b = 2*GS_a:
// TP_a/TP_b = (S_b * GS_b) / (S_a * GS_a) = 2 * S_b / S_a.   C-A14: GS >= 2.
extern "C" uint32_t orc_ntg_choose_gs(const uint64_t* kr, const uint32_t* ps, uint32_t F,
                                      uint32_t h, const uint64_t* ls, const uint64_t* q,
                                      uint64_t nq, uint32_t gs0, uint32_t kpl,
                                      uint32_t lev0, uint32_t warp) {
  uint32_t gs = gs0;
  double sb = orc_ntg_warp_steps(kr, ps, F, h, ls, q, nq, gs, kpl, lev0, warp);
  while (gs / 2 >= 2) {
    double sa = orc_ntg_warp_steps(kr, ps, F, h, ls, q, nq, gs / 2, kpl, lev0, warp);
    double ratio = sa > 0 ? 2.0 * sb / sa : 0.0;
    if (!(ratio > 1.0)) break;
    gs /= 2;
    sb = sa;
  }
  return gs;
}

// Fig 2: transactions per warp = distinct nodes the warp's queries touch at
// a level (one node per transaction), averaged over levels and warps.
extern "C" double orc_warp_transactions(const uint64_t* kr, const uint32_t* ps, uint32_t F,
                                        uint32_t h, const uint64_t* ls, const uint64_t* q,
                                        uint64_t nq, uint32_t qpw) {
  (void)ls;
  std::vector<uint64_t> path;
  double total = 0;
  uint64_t samples = 0;
  for (uint64_t w0 = 0; w0 < nq; w0 += qpw) {
    std::vector<std::set<uint64_t>> distinct(h);
    for (uint64_t j = w0; j < std::min<uint64_t>(nq, w0 + qpw); ++j) {
      path_of(kr, ps, F, h, q[j], path);
      for (uint32_t l = 0; l < h; ++l) distinct[l].insert(path[l]);
    }
    for (uint32_t l = 0; l < h; ++l, ++samples) total += (double)distinct[l].size();
  }
  return samples ? total / (double)samples : 0.0;
}

// ---------------- O6: update oracle, C-A18 (sequential semantics in batch order) --------
extern "C" void* orc_map_create(const uint64_t* keys, const uint64_t* vals, uint64_t n) {
  auto* m = new std::map<uint64_t, uint64_t>;
  for (uint64_t i = 0; i < n; ++i) (*m)[keys[i]] = vals[i];
  return m;
}
extern "C" void orc_map_destroy(void* m) { delete (std::map<uint64_t, uint64_t>*)m; }
extern "C" uint64_t orc_map_apply(void* mp, const uint8_t* ops, const uint64_t* keys,
                                  const uint64_t* vals, uint64_t n) {
  auto& m = *(std::map<uint64_t, uint64_t>*)mp;
  for (uint64_t i = 0; i < n; ++i) {
    if (ops[i] == 0) m[keys[i]] = vals[i];  // insert, or update an existing record
    else m.erase(keys[i]);                  // delete; a missing key is a no-op
  }
  return m.size();
}
extern "C" uint64_t orc_map_dump(void* mp, uint64_t* keys, uint64_t* vals, uint64_t cap) {
  auto& m = *(std::map<uint64_t, uint64_t>*)mp;
  uint64_t i = 0;
  for (auto& kv : m) {
    if (i >= cap) break;
    keys[i] = kv.first;
    vals[i] = kv.second;
    ++i;
  }
  return m.size();
}
