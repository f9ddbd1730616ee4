// Harmonia layout construction on the device (Fig 4(b)) and the tree-level
// C ABI (build / destroy / info / export / status helpers).
//
// Layout:
//   key region  uint64[N*F]  node n at [n*F, n*F+F), BFS order; internal nodes hold
//                            c-1 separators, leaves <= F-1 keys, unused slots = PAD (C-A2)
//   PS          uint32[I+1]  PS[n] = index of node n's first child, PS[I] = N (C-A7)
//   values      uint64[L*F]  value of leaf j slot s at [j*F+s] (C-A3), pads = NOT_FOUND
//   leaf_base   uint64[L+1]  records stored before leaf j (for range counts)
// Level sizes follow the even-distribution closed form (C-A6); every node's position and
// every PS entry is then a closed-form function of its index, so each device pass below is
// one thread per record (leaves) or one thread per child (internal levels).
#include <algorithm>
#include <cmath>
#include <cstring>
#include <new>

#include "common.cuh"

namespace hm {

namespace {
thread_local int g_last_cuda_error = 0;
unsigned long long g_launches = 0;  // updated with __atomic builtins
}  // namespace

harmonia_status cuda_fail(cudaError_t e) {
  g_last_cuda_error = (int)e;
  if (e == cudaErrorMemoryAllocation) return HARMONIA_ERR_OUT_OF_MEMORY;
  return HARMONIA_ERR_CUDA;
}

void count_launch(uint64_t k) { __atomic_fetch_add(&g_launches, (unsigned long long)k, __ATOMIC_RELAXED); }

// C-A6 (product implementation): nodes for n items at capacity cap and fill target.
static uint64_t nodes_needed(uint64_t n, uint64_t cap, double fill) {
  uint64_t target = std::max<uint64_t>((cap + 1) / 2, (uint64_t)std::floor(fill * (double)cap));
  uint64_t m = std::max<uint64_t>(ceil_div(n, cap), n / target);
  return std::max<uint64_t>(m, 1);
}

uint32_t level_shape(uint64_t n, uint32_t F, double fill, uint64_t* bottom_up) {
  uint32_t h = 0;
  uint64_t m = nodes_needed(n, F - 1, fill);
  bottom_up[h++] = m;
  while (m > 1 && h < HARMONIA_MAX_LEVELS) {
    m = nodes_needed(m, F, fill);
    bottom_up[h++] = m;
  }
  return m > 1 ? 0 : h;  // 0 = too tall
}

// position of item i among m nodes sharing n items (first n%m nodes get one extra)
struct Locate {
  uint64_t q, r, big;
  __host__ __device__ Locate(uint64_t n, uint64_t m) : q(n / m), r(n % m), big((n % m) * (n / m + 1)) {}
  __device__ __forceinline__ void operator()(uint64_t i, uint64_t* node, uint64_t* pos) const {
    if (i < big) {
      *node = i / (q + 1);
      *pos = i % (q + 1);
    } else {
      uint64_t k = i - big;
      *node = r + k / q;
      *pos = k % q;
    }
  }
};

__global__ void k_validate(const uint64_t* __restrict__ keys, const uint64_t* __restrict__ vals,
                           uint64_t n, unsigned* flags) {
  unsigned f = 0;
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n;
       i += (uint64_t)gridDim.x * blockDim.x) {
    uint64_t k = keys[i];
    if (k == kPad || vals[i] == kNotFound) f |= 2u;
    if (i > 0 && !(keys[i - 1] < k)) f |= 1u;
  }
  f = __reduce_or_sync(kFull, f);
  if (f && (threadIdx.x & 31) == 0) atomicOr(flags, f);
}

__global__ void k_fill_leaves(const uint64_t* __restrict__ keys, const uint64_t* __restrict__ vals,
                              uint64_t n, Locate loc, uint32_t F, uint64_t leaf_start,
                              uint64_t* __restrict__ kr, uint64_t* __restrict__ lv,
                              uint64_t* __restrict__ mins, uint64_t* __restrict__ leaf_base) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n;
       i += (uint64_t)gridDim.x * blockDim.x) {
    uint64_t j, s;
    loc(i, &j, &s);
    uint64_t k = keys[i];
    kr[(leaf_start + j) * F + s] = k;
    lv[j * F + s] = vals[i];
    if (s == 0) {
      mins[j] = k;
      leaf_base[j] = i;
    }
  }
}

// one thread per child c of level l+1: separator (C-A5) or first-child PS entry
__global__ void k_fill_internal(uint64_t nc, Locate loc, uint32_t F, uint64_t ls_l,
                                uint64_t ls_next, const uint64_t* __restrict__ child_min,
                                uint64_t* __restrict__ parent_min, uint64_t* __restrict__ kr,
                                uint32_t* __restrict__ ps) {
  for (uint64_t c = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; c < nc;
       c += (uint64_t)gridDim.x * blockDim.x) {
    uint64_t p, k;
    loc(c, &p, &k);
    uint64_t mk = child_min[c];
    if (k > 0) {
      kr[(ls_l + p) * F + (k - 1)] = mk;
    } else {
      parent_min[p] = mk;
      ps[ls_l + p] = (uint32_t)(ls_next + c);
    }
  }
}

static int grid_for(uint64_t n, int sm) {
  uint64_t g = ceil_div(std::max<uint64_t>(n, 1), kBlock);
  return (int)std::min<uint64_t>(g, (uint64_t)sm * 16);
}

harmonia_status build_layout(harmonia_tree* t, const uint64_t* d_keys, const uint64_t* d_vals,
                             uint64_t n, cudaStream_t st) {
  const uint32_t F = t->F;
  uint64_t bu[HARMONIA_MAX_LEVELS];
  uint32_t h = level_shape(n, F, t->fill, bu);
  if (h == 0) return HARMONIA_ERR_TOO_LARGE;
  t->h = h;
  t->level_start[0] = 0;
  for (uint32_t l = 0; l < h; ++l) t->level_start[l + 1] = t->level_start[l] + bu[h - 1 - l];
  t->N = t->level_start[h];
  t->I = t->level_start[h - 1];
  t->L = bu[0];
  t->n_keys = n;
  if (t->N >= 0xFFFFFFFFull) return HARMONIA_ERR_TOO_LARGE;

  const size_t kr_bytes = (size_t)t->N * F * 8, lv_bytes = (size_t)t->L * F * 8;
  const size_t ps_bytes = round_up((t->I + 1) * 4, 16);
  // the layout is built into the tree's current arrays, grown only when too small
  harmonia_status rs;
  if ((rs = reserve_bytes((void**)&t->d_keys, &t->cap_keys, kr_bytes)) != HARMONIA_OK) return rs;
  if ((rs = reserve_bytes((void**)&t->d_vals, &t->cap_vals, lv_bytes)) != HARMONIA_OK) return rs;
  if ((rs = reserve_bytes((void**)&t->d_ps, &t->cap_ps, ps_bytes)) != HARMONIA_OK) return rs;
  if ((rs = reserve_bytes((void**)&t->d_leaf_base, &t->cap_lb, (t->L + 1) * 8)) != HARMONIA_OK) return rs;
  HM_CUDA(cudaMemsetAsync(t->d_keys, 0xFF, kr_bytes, st));
  HM_CUDA(cudaMemsetAsync(t->d_vals, 0xFF, lv_bytes, st));
  HM_CUDA(cudaMemsetAsync(t->d_ps, 0, ps_bytes, st));
  HM_CUDA(cudaMemsetAsync(t->d_leaf_base, 0, (t->L + 1) * 8, st));
  uint32_t sentinel = (uint32_t)t->N;
  HM_CUDA(cudaMemcpyAsync(t->d_ps + t->I, &sentinel, 4, cudaMemcpyHostToDevice, st));
  uint64_t nrec = n;
  HM_CUDA(cudaMemcpyAsync(t->d_leaf_base + t->L, &nrec, 8, cudaMemcpyHostToDevice, st));

  if ((rs = reserve_bytes((void**)&t->scratch, &t->scratch_cap, 2 * round_up(t->L * 8, 256))) != HARMONIA_OK)
    return rs;
  uint64_t *mins_a = t->scratch, *mins_b = t->scratch + round_up(t->L * 8, 256) / 8;
  harmonia_status s = HARMONIA_OK;
  if (n > 0) {
    k_fill_leaves<<<grid_for(n, t->sm_count), kBlock, 0, st>>>(
        d_keys, d_vals, n, Locate(n, t->L), F, t->level_start[h - 1], t->d_keys, t->d_vals,
        mins_a, t->d_leaf_base);
    count_launch();
    for (int l = (int)h - 2; l >= 0; --l) {
      uint64_t nl = t->level_start[l + 1] - t->level_start[l];
      uint64_t nc = t->level_start[l + 2] - t->level_start[l + 1];
      k_fill_internal<<<grid_for(nc, t->sm_count), kBlock, 0, st>>>(
          nc, Locate(nc, nl), F, t->level_start[l], t->level_start[l + 1], mins_a, mins_b,
          t->d_keys, t->d_ps);
      count_launch();
      std::swap(mins_a, mins_b);
    }
  }
  cudaError_t e = cudaGetLastError();
  if (e == cudaSuccess) e = cudaStreamSynchronize(st);
  if (e != cudaSuccess) s = cuda_fail(e);
  return s;
}

harmonia_status reserve_bytes(void** p, size_t* cap, size_t need) {
  need = std::max<size_t>(need, 16);
  if (*p && *cap >= need) return HARMONIA_OK;
  if (*p) cudaFree(*p);
  *p = nullptr;
  *cap = 0;
  const size_t want = need + need / 8;
  cudaError_t e = cudaMalloc(p, want);
  if (e != cudaSuccess) {
    cudaGetLastError();
    *p = nullptr;
    if (e == cudaErrorMemoryAllocation) {  // retry without headroom
      if (cudaMalloc(p, need) == cudaSuccess) {
        *cap = need;
        return HARMONIA_OK;
      }
      cudaGetLastError();
      *p = nullptr;
      return HARMONIA_ERR_OUT_OF_MEMORY;
    }
    return cuda_fail(e);
  }
  *cap = want;
  return HARMONIA_OK;
}

void swap_layout_buffers(harmonia_tree* t) {
  std::swap(t->d_keys, t->sp_keys);
  std::swap(t->cap_keys, t->sp_cap_keys);
  std::swap(t->d_vals, t->sp_vals);
  std::swap(t->cap_vals, t->sp_cap_vals);
  std::swap(t->d_ps, t->sp_ps);
  std::swap(t->cap_ps, t->sp_cap_ps);
  std::swap(t->d_leaf_base, t->sp_lb);
  std::swap(t->cap_lb, t->sp_cap_lb);
}

int psa_bits_for(uint64_t n_keys) {
  // Eq 2: N = B - log2(2^B / T * K) = log2(T / K), K = 16 keys per 128-B line
  if (n_keys <= 16) return 0;
  double b = std::ceil(std::log2((double)n_keys / 16.0) - 1e-9);
  return (int)std::min(28.0, std::max(0.0, b));
}

}  // namespace hm

using namespace hm;

static void free_tree(harmonia_tree* t) {
  if (!t) return;
  int cur = 0;
  cudaGetDevice(&cur);
  cudaSetDevice(t->device);
  cudaDeviceSynchronize();
  l2_persist_release(t);
  cudaFree(t->d_keys);
  cudaFree(t->d_vals);
  cudaFree(t->d_ps);
  cudaFree(t->d_leaf_base);
  cudaFree(t->sp_keys);
  cudaFree(t->sp_vals);
  cudaFree(t->sp_ps);
  cudaFree(t->sp_lb);
  cudaFree(t->scratch);
  if (t->s_h2d) cudaStreamDestroy(t->s_h2d);
  if (t->s_d2h) cudaStreamDestroy(t->s_d2h);
  if (t->ev_start) cudaEventDestroy(t->ev_start);
  for (int i = 0; i < 2; ++i) {
    if (t->ev_in[i]) cudaEventDestroy(t->ev_in[i]);
    if (t->ev_done[i]) cudaEventDestroy(t->ev_done[i]);
    if (t->ev_out[i]) cudaEventDestroy(t->ev_out[i]);
  }
  delete t;
  cudaSetDevice(cur);
}

extern "C" harmonia_status harmonia_build(const uint64_t* keys, const uint64_t* values, uint64_t n,
                                          const harmonia_build_opts* opts, void* stream,
                                          harmonia_tree** out) {
  if (!out || (n > 0 && (!keys || !values))) return HARMONIA_ERR_INVALID_ARG;
  *out = nullptr;
  uint32_t F = opts && opts->fanout ? opts->fanout : 64;
  float fill = opts && opts->fill > 0 ? opts->fill : 1.0f;
  if (F < 4 || F > 256 || (F & (F - 1))) return HARMONIA_ERR_INVALID_ARG;
  if (fill < 0.5f || fill > 1.0f) return HARMONIA_ERR_INVALID_ARG;
  bool on_dev = opts && opts->keys_on_device;
  cudaStream_t st = (cudaStream_t)stream;

  harmonia_tree* t = new (std::nothrow) harmonia_tree;
  if (!t) return HARMONIA_ERR_OUT_OF_MEMORY;
  t->F = F;
  t->fill = fill;
  cudaError_t e = cudaGetDevice(&t->device);
  if (e != cudaSuccess) {
    delete t;
    return cuda_fail(e);
  }
  cudaDeviceProp prop;
  if ((e = cudaGetDeviceProperties(&prop, t->device)) != cudaSuccess) {
    delete t;
    return cuda_fail(e);
  }
  t->sm_count = prop.multiProcessorCount;
  t->smem_optin = prop.sharedMemPerBlockOptin;
  t->smem_per_sm = prop.sharedMemPerMultiprocessor;
  t->l2_bytes = prop.l2CacheSize;
  t->l2_persist_max = prop.persistingL2CacheMaxSize;
  t->l2_window_max = prop.accessPolicyMaxWindowSize;

  if (on_dev && n > 0) {
    cudaPointerAttributes pa;
    if (cudaPointerGetAttributes(&pa, keys) != cudaSuccess || pa.type != cudaMemoryTypeDevice ||
        pa.device != t->device) {
      cudaGetLastError();
      delete t;
      return HARMONIA_ERR_DEVICE_MISMATCH;
    }
  }

  const uint64_t *dk = keys, *dv = values;
  uint64_t *tmpk = nullptr, *tmpv = nullptr;
  unsigned* d_flags = nullptr;
  harmonia_status s = HARMONIA_OK;
  auto fail = [&](harmonia_status x) {
    cudaFree(tmpk);
    cudaFree(tmpv);
    cudaFree(d_flags);
    free_tree(t);
    return x;
  };
  if (n > 0 && !on_dev) {
    if ((e = cudaMalloc(&tmpk, n * 8)) != cudaSuccess) return fail(cuda_fail(e));
    if ((e = cudaMalloc(&tmpv, n * 8)) != cudaSuccess) return fail(cuda_fail(e));
    if ((e = cudaMemcpyAsync(tmpk, keys, n * 8, cudaMemcpyHostToDevice, st)) != cudaSuccess)
      return fail(cuda_fail(e));
    if ((e = cudaMemcpyAsync(tmpv, values, n * 8, cudaMemcpyHostToDevice, st)) != cudaSuccess)
      return fail(cuda_fail(e));
    dk = tmpk;
    dv = tmpv;
  }
  if (n > 0) {
    if ((e = cudaMalloc(&d_flags, 4)) != cudaSuccess) return fail(cuda_fail(e));
    cudaMemsetAsync(d_flags, 0, 4, st);
    k_validate<<<grid_for(n, t->sm_count), kBlock, 0, st>>>(dk, dv, n, d_flags);
    count_launch();
    unsigned flags = 0;
    if ((e = cudaMemcpyAsync(&flags, d_flags, 4, cudaMemcpyDeviceToHost, st)) != cudaSuccess)
      return fail(cuda_fail(e));
    if ((e = cudaStreamSynchronize(st)) != cudaSuccess) return fail(cuda_fail(e));
    if (flags & 2u) return fail(HARMONIA_ERR_RESERVED);
    if (flags & 1u) return fail(HARMONIA_ERR_UNSORTED);
    if ((e = cudaMemcpyAsync(&t->min_key, dk, 8, cudaMemcpyDeviceToHost, st)) != cudaSuccess)
      return fail(cuda_fail(e));
    if ((e = cudaMemcpyAsync(&t->max_key, dk + n - 1, 8, cudaMemcpyDeviceToHost, st)) != cudaSuccess)
      return fail(cuda_fail(e));
  } else {
    t->min_key = kPad;
    t->max_key = 0;
  }
  s = build_layout(t, dk, dv, n, st);
  if (s != HARMONIA_OK) return fail(s);
  cudaFree(tmpk);
  cudaFree(tmpv);
  cudaFree(d_flags);
  *out = t;
  return HARMONIA_OK;
}

extern "C" void harmonia_destroy(harmonia_tree* t) { free_tree(t); }

extern "C" harmonia_status harmonia_get_info(const harmonia_tree* t, harmonia_info* info) {
  if (!t || !info) return HARMONIA_ERR_INVALID_ARG;
  std::memset(info, 0, sizeof(*info));
  info->n_keys = t->n_keys;
  info->fanout = t->F;
  info->height = t->h;
  info->psa_bits_auto = (uint32_t)psa_bits_for(t->n_keys);
  info->group_size_auto = (uint32_t)auto_group_size(t->F);
  info->n_nodes = t->N;
  info->n_internal = t->I;
  info->n_leaves = t->L;
  for (uint32_t l = 0; l <= t->h; ++l) info->level_start[l] = t->level_start[l];
  info->key_region_bytes = t->N * t->F * 8;
  info->ps_bytes = (t->I + 1) * 4;
  info->value_bytes = t->L * t->F * 8;
  info->min_key = t->min_key;
  info->max_key = t->max_key;
  info->device = t->device;
  return HARMONIA_OK;
}

extern "C" harmonia_status harmonia_export_layout(const harmonia_tree* t, uint64_t* h_kr,
                                                  uint32_t* h_ps, uint64_t* h_lv) {
  if (!t || !h_kr || !h_ps || !h_lv) return HARMONIA_ERR_INVALID_ARG;
  HM_CUDA(cudaMemcpy(h_kr, t->d_keys, t->N * t->F * 8, cudaMemcpyDeviceToHost));
  HM_CUDA(cudaMemcpy(h_ps, t->d_ps, (t->I + 1) * 4, cudaMemcpyDeviceToHost));
  HM_CUDA(cudaMemcpy(h_lv, t->d_vals, t->L * t->F * 8, cudaMemcpyDeviceToHost));
  return HARMONIA_OK;
}

extern "C" int32_t harmonia_psa_bits_auto(uint64_t n_keys) { return psa_bits_for(n_keys); }

extern "C" const char* harmonia_status_string(harmonia_status s) {
  switch (s) {
    case HARMONIA_OK: return "ok";
    case HARMONIA_ERR_INVALID_ARG: return "invalid argument";
    case HARMONIA_ERR_UNSORTED: return "build keys not strictly increasing";
    case HARMONIA_ERR_RESERVED: return "reserved key (UINT64_MAX) or value (UINT64_MAX)";
    case HARMONIA_ERR_OUT_OF_MEMORY: return "out of device memory";
    case HARMONIA_ERR_CUDA: return "CUDA error";
    case HARMONIA_ERR_DEVICE_MISMATCH: return "pointer or stream not on the tree's device";
    case HARMONIA_ERR_TOO_LARGE: return "tree too large (nodes >= 2^32 or height > 64)";
  }
  return "unknown status";
}

extern "C" int harmonia_last_cuda_error(void) { return hm::g_last_cuda_error; }
extern "C" uint64_t harmonia_kernel_launches(void) {
  return __atomic_load_n(&hm::g_launches, __ATOMIC_RELAXED);
}
extern "C" int harmonia_abi_version(void) { return HARMONIA_ABI_VERSION; }
