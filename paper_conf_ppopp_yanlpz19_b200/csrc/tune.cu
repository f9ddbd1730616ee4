// NTG group-size model (§4.2, "static profiling"): choose the thread-group size
// GS from a small sample of PSA-ordered queries instead of a full sweep.
//
//   * Fig 9 / C-A13: a group of GS lanes compares GS*kpl keys per step (kpl = 2 with one
//     128-bit load per lane) and stops in the step that holds the target, so a query whose
//     target has r keys before it in a node of cnt keys needs min(r/(GS*kpl)+1,
//     ceil(cnt/(GS*kpl))) steps.
//   * Eq 3: a warp runs 32/GS queries together and waits for the slowest, so
//     its cost at a level is the max of its queries' steps; S(GS) = that max summed over the
//     profiled levels, averaged over the sample's warps.
//   * Eq 4: halving GS doubles the queries per warp; throughput improves while
//     TP_a/TP_b = (S_b * GS_b) / (S_a * GS_a) = 2 * S_b / S_a > 1 (C-A22), starting from
//     GS = min(32, F/2) and stopping at GS = 2 (C-A14).
//
// The per-query (r, cnt) of every level comes from a small GPU kernel (one thread per
// sample, a plain Eq-1 descent); the model itself is O(samples * levels) host arithmetic
// ("CPU, O(1000 h)"), exported separately so it can be checked on a
// machine without a GPU.  Offline per tree and workload: not on the query path.
#include <algorithm>
#include <cstring>
#include <numeric>
#include <vector>

#include "common.cuh"

namespace hm {
namespace {

// one thread per sample: PSA bucket (C-A11) and, per level, r = keys before the target
// (<= q in internal nodes: Eq 1's rank; < q at the leaf: the slot of q) and the node's key
// count cnt
__global__ void k_ntg_profile(const uint64_t* __restrict__ keys, const uint32_t* __restrict__ ps, uint32_t F,
                              uint32_t h, const uint64_t* __restrict__ q, uint32_t n, BucketBits f, int psa,
                              uint32_t* __restrict__ prof, uint32_t* __restrict__ bucket) {
  const uint32_t j = blockIdx.x * blockDim.x + threadIdx.x;
  if (j >= n) return;
  const uint64_t x = q[j];
  bucket[j] = psa ? f(x) : 0u;
  uint32_t node = 0;
  for (uint32_t l = 0; l < h; ++l) {
    const uint64_t* nk = keys + (uint64_t)node * F;
    uint32_t cnt = 0, le = 0, lt = 0;
    for (uint32_t s = 0; s < F; ++s) {
      const uint64_t k = nk[s];
      if (k == kPad) break;  // valid keys occupy slots 0..cnt-1 (I6)
      ++cnt;
      le += k <= x;
      lt += k < x;
    }
    const bool leaf = l + 1 == h;
    prof[((uint64_t)j * h + l) * 2] = leaf ? lt : le;
    prof[((uint64_t)j * h + l) * 2 + 1] = cnt;
    if (!leaf) node = ps[node] + le;  // Eq 1 (i = le + 1)
  }
}

uint32_t fig9_steps(uint32_t r, uint32_t cnt, uint32_t gs, uint32_t kpl) {
  const uint32_t w = gs * kpl, full = (cnt + w - 1) / w;
  return std::min(r / w + 1, full);
}

}  // namespace
}  // namespace hm

using namespace hm;

extern "C" harmonia_status harmonia_ntg_choose(const uint32_t* prof, const uint32_t* bucket, uint32_t n, uint32_t h,
                                               uint32_t lev0, uint32_t gs0, uint32_t kpl, int32_t* gs_out,
                                               double* steps_out) {
  if (!prof || !gs_out || n == 0 || h == 0 || h > HARMONIA_MAX_LEVELS || kpl == 0 || gs0 < 1 || gs0 > 32 ||
      (gs0 & (gs0 - 1)))
    return HARMONIA_ERR_INVALID_ARG;
  // PSA order of the sample: stable by bucket
  std::vector<uint32_t> ord(n);
  std::iota(ord.begin(), ord.end(), 0u);
  if (bucket) std::stable_sort(ord.begin(), ord.end(), [&](uint32_t a, uint32_t b) { return bucket[a] < bucket[b]; });
  auto S = [&](uint32_t gs) {  // Eq 3 input: mean over warps of the summed per-level max steps
    const uint32_t qpw = std::max(1u, 32u / gs);
    double total = 0;
    uint64_t warps = 0;
    std::vector<uint32_t> smax(h);
    for (uint32_t w0 = 0; w0 < n; w0 += qpw, ++warps) {
      std::fill(smax.begin(), smax.end(), 0u);
      for (uint32_t j = w0; j < std::min(n, w0 + qpw); ++j)
        for (uint32_t l = lev0; l < h; ++l) {
          const uint32_t* rc = prof + ((uint64_t)ord[j] * h + l) * 2;
          smax[l] = std::max(smax[l], fig9_steps(rc[0], rc[1], gs, kpl));
        }
      for (uint32_t l = lev0; l < h; ++l) total += smax[l];
    }
    return warps ? total / (double)warps : 0.0;
  };
  if (steps_out)
    for (int i = 0; i < 6; ++i) steps_out[i] = (1u << i) <= gs0 ? S(1u << i) : 0.0;
  // Eq 4 narrowing loop, GS >= 2 (C-A14)
  uint32_t gs = gs0;
  double sb = S(gs);
  while (gs / 2 >= 2) {
    const double sa = S(gs / 2);
    if (!(sa > 0 && 2.0 * sb / sa > 1.0)) break;
    gs /= 2;
    sb = sa;
  }
  *gs_out = (int32_t)gs;
  return HARMONIA_OK;
}

extern "C" harmonia_status harmonia_tune_group_size(const harmonia_tree* t, const uint64_t* d_samples, uint32_t n,
                                                    const harmonia_query_opts* o, int32_t* gs_out,
                                                    double* steps_out) {
  if (!t || !d_samples || !gs_out || n == 0 || n > (1u << 20)) return HARMONIA_ERR_INVALID_ARG;
  if (t->n_keys == 0) {
    *gs_out = 2;
    if (steps_out) std::memset(steps_out, 0, 6 * sizeof(double));
    return HARMONIA_OK;
  }
  cudaPointerAttributes pa;
  if (cudaPointerGetAttributes(&pa, d_samples) != cudaSuccess) {
    cudaGetLastError();
    return HARMONIA_ERR_DEVICE_MISMATCH;
  }
  if (pa.type != cudaMemoryTypeDevice && pa.type != cudaMemoryTypeManaged) return HARMONIA_ERR_DEVICE_MISMATCH;
  if (pa.device != t->device) return HARMONIA_ERR_DEVICE_MISMATCH;
  Plan p;  // the plan of a full batch (the sample is ordered with the production PSA buckets)
  harmonia_status s = make_plan(t, 1ull << 27, o, &p);
  if (s != HARMONIA_OK) return s;
  const uint32_t h = t->h;
  uint32_t* d = nullptr;
  HM_CUDA(cudaMalloc(&d, ((size_t)n * h * 2 + n) * 4));
  k_ntg_profile<<<(n + 255) / 256, 256>>>(t->d_keys, t->d_ps, t->F, h, d_samples, n, p.bucket, p.psa ? 1 : 0, d,
                                          d + (size_t)n * h * 2);
  count_launch();
  cudaError_t e = cudaGetLastError();
  std::vector<uint32_t> prof((size_t)n * h * 2), bucket(n);
  if (e == cudaSuccess) e = cudaMemcpy(prof.data(), d, prof.size() * 4, cudaMemcpyDeviceToHost);
  if (e == cudaSuccess) e = cudaMemcpy(bucket.data(), d + (size_t)n * h * 2, (size_t)n * 4, cudaMemcpyDeviceToHost);
  cudaFree(d);
  if (e != cudaSuccess) return cuda_fail(e);
  // C-A14: start at min(32, F/2); profile the levels below the shared-memory-staged top
  const uint32_t gs0 = std::min(32u, t->F / 2), lev0 = std::min<uint32_t>((uint32_t)p.smem_levels, h - 1);
  return harmonia_ntg_choose(prof.data(), bucket.data(), n, h, lev0, gs0, 2, gs_out, steps_out);
}
