// O1 (std::lower_bound over the sorted key array) and O3 (brute force).
// TEST INFRASTRUCTURE ONLY — see oracle.h.
//
// The definition followed (§3.2.1): a point query traverses to the leaf
// and "the target key is found" -> return its record; a range query returns the records
// "from the first target key to the last target key in the query range".  C-A10: the
// range is inclusive [lo, hi], results ascending, count = true total, at most cap stored.
#include "oracle.h"

#include <algorithm>
#include <thread>
#include <vector>

namespace {

template <class F>
void parallel_for(uint64_t n, int nthreads, F&& body) {
  if (nthreads <= 0) nthreads = (int)std::max(1u, std::thread::hardware_concurrency());
  if (n < 4096 || nthreads == 1) {
    body(0, n);
    return;
  }
  std::vector<std::thread> th;
  uint64_t chunk = (n + nthreads - 1) / nthreads;
  for (int t = 0; t < nthreads; ++t) {
    uint64_t b = std::min<uint64_t>(n, t * chunk), e = std::min<uint64_t>(n, b + chunk);
    if (b < e) th.emplace_back([&, b, e] { body(b, e); });
  }
  for (auto& x : th) x.join();
}

}  // namespace

extern "C" void orc_sorted_search(const uint64_t* keys, const uint64_t* vals, uint64_t n,
                                  const uint64_t* q, uint64_t nq, uint64_t* out,
                                  int nthreads) {
  parallel_for(nq, nthreads, [&](uint64_t b, uint64_t e) {
    for (uint64_t j = b; j < e; ++j) {
      const uint64_t* p = std::lower_bound(keys, keys + n, q[j]);
      out[j] = (p != keys + n && *p == q[j]) ? vals[p - keys] : ORC_NOT_FOUND;
    }
  });
}

extern "C" void orc_sorted_range(const uint64_t* keys, const uint64_t* vals, uint64_t n,
                                 const uint64_t* lo, const uint64_t* hi, uint64_t nq,
                                 uint32_t cap, uint64_t* kout, uint64_t* vout,
                                 uint32_t* counts, int nthreads) {
  parallel_for(nq, nthreads, [&](uint64_t b, uint64_t e) {
    for (uint64_t j = b; j < e; ++j) {
      if (lo[j] > hi[j]) {
        counts[j] = 0;
        continue;
      }
      const uint64_t* first = std::lower_bound(keys, keys + n, lo[j]);
      const uint64_t* last = std::upper_bound(keys, keys + n, hi[j]);
      uint64_t cnt = (uint64_t)(last - first);
      counts[j] = (uint32_t)cnt;
      uint64_t m = std::min<uint64_t>(cnt, cap);
      for (uint64_t t = 0; t < m; ++t) {
        kout[j * (uint64_t)cap + t] = first[t];
        vout[j * (uint64_t)cap + t] = vals[(first - keys) + t];
      }
    }
  });
}

extern "C" void orc_brute_search(const uint64_t* keys, const uint64_t* vals, uint64_t n,
                                 const uint64_t* q, uint64_t nq, uint64_t* out) {
  for (uint64_t j = 0; j < nq; ++j) {
    out[j] = ORC_NOT_FOUND;
    for (uint64_t i = 0; i < n; ++i)
      if (keys[i] == q[j]) out[j] = vals[i];
  }
}

extern "C" void orc_brute_range(const uint64_t* keys, const uint64_t* vals, uint64_t n,
                                const uint64_t* lo, const uint64_t* hi, uint64_t nq,
                                uint32_t cap, uint64_t* kout, uint64_t* vout,
                                uint32_t* counts) {
  for (uint64_t j = 0; j < nq; ++j) {
    uint32_t c = 0;
    for (uint64_t i = 0; i < n; ++i) {
      if (keys[i] >= lo[j] && keys[i] <= hi[j]) {
        if (c < cap) {
          kout[j * (uint64_t)cap + c] = keys[i];
          vout[j * (uint64_t)cap + c] = vals[i];
        }
        ++c;
      }
    }
    counts[j] = c;
  }
}
