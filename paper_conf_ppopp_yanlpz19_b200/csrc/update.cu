// Batched update: implemented in a later milestone; the ABI slot is fixed.
#include "common.cuh"

extern "C" size_t harmonia_update_workspace_bytes(const harmonia_tree* t, uint64_t n) {
  (void)t;
  (void)n;
  return 0;
}

extern "C" harmonia_status harmonia_update_batch(harmonia_tree* t, const uint8_t* d_ops, const uint64_t* d_keys,
                                                 const uint64_t* d_values, uint64_t n, void* ws, size_t ws_bytes,
                                                 void* stream) {
  (void)t; (void)d_ops; (void)d_keys; (void)d_values; (void)n; (void)ws; (void)ws_bytes; (void)stream;
  return HARMONIA_ERR_INVALID_ARG;
}
