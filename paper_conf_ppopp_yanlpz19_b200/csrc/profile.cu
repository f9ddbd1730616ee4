// harmonia_profile_*: CUDA-event timing of the library's kernels, per kernel class, on the
// stream each kernel is launched on (used by bench.py for the roofline's kernel duration).
#include <map>
#include <mutex>
#include <utility>
#include <vector>

#include "common.cuh"

namespace hm {

bool g_prof_on = false;

// cudaFuncAttributeMaxDynamicSharedMemorySize is a per-device property of a kernel: remember
// what was set per (kernel, device) so that a process driving trees on several devices sets
// it on each (the per-process function-local caches skipped the second device).
cudaError_t smem_attr(const void* kern, size_t bytes) {
  static std::mutex mu;
  static std::map<std::pair<const void*, int>, size_t> done;
  int dev = 0;
  cudaError_t e = cudaGetDevice(&dev);
  if (e != cudaSuccess) return e;
  std::lock_guard<std::mutex> lk(mu);
  size_t& cur = done[{kern, dev}];
  if (cur >= bytes) return cudaSuccess;
  e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)bytes);
  if (e == cudaSuccess) cur = bytes;
  return e;
}

namespace {
struct Rec {
  int kind;
  cudaEvent_t a, b;
};
std::mutex g_mu;
std::vector<Rec> g_recs;
std::vector<cudaEvent_t> g_pool;
cudaEvent_t take() {
  cudaEvent_t e = nullptr;
  if (!g_pool.empty()) {
    e = g_pool.back();
    g_pool.pop_back();
  } else {
    cudaEventCreate(&e);
  }
  return e;
}
}  // namespace

void prof_record(int kind, cudaStream_t st, bool start) {
  std::lock_guard<std::mutex> lk(g_mu);
  if (start) {
    Rec r{kind, take(), nullptr};
    cudaEventRecord(r.a, st);
    g_recs.push_back(r);
  } else {
    for (auto it = g_recs.rbegin(); it != g_recs.rend(); ++it)
      if (it->kind == kind && it->b == nullptr) {
        it->b = take();
        cudaEventRecord(it->b, st);
        break;
      }
  }
}

}  // namespace hm

extern "C" void harmonia_profile_enable(int on) { hm::g_prof_on = on != 0; }

extern "C" harmonia_status harmonia_profile_read(double* total_ms, uint64_t* launches) {
  using namespace hm;
  std::lock_guard<std::mutex> lk(g_mu);
  for (int k = 0; k < HARMONIA_PROF_KINDS; ++k) {
    if (total_ms) total_ms[k] = 0;
    if (launches) launches[k] = 0;
  }
  harmonia_status s = HARMONIA_OK;
  for (auto& r : g_recs) {
    if (r.b) {
      float ms = 0;
      cudaError_t e = cudaEventSynchronize(r.b);
      if (e == cudaSuccess) e = cudaEventElapsedTime(&ms, r.a, r.b);
      if (e != cudaSuccess) s = cuda_fail(e);
      if (total_ms) total_ms[r.kind] += ms;
      if (launches) launches[r.kind] += 1;
      g_pool.push_back(r.b);
    }
    g_pool.push_back(r.a);
  }
  g_recs.clear();
  return s;
}
