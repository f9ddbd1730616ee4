/*
 * harmonia.h — C ABI of libharmonia.so: batched B+tree point and range queries over the
 * Harmonia layout on NVIDIA B200 (sm_100a).
 *
 * Method: Yan, Lin, Peng, Zhang, "Harmonia: A High Throughput B+tree for GPUs", PPoPP'19.
 * Citations "P:Lnnn" are lines of the paper text (reference PAPER.md); "C-Axx" are the
 * readings of ambiguous passages listed in DESIGN.md §3.
 *
 * Conventions (all functions):
 *   - Plain C11, no exceptions cross the ABI; every fallible call returns harmonia_status.
 *   - `stream` is a cudaStream_t passed as void* (NULL = the legacy default stream).
 *   - "d_" pointers are device memory on the tree's device, "h_" pointers host memory.
 *   - Keys and values are uint64.  Keys are compared unsigned (C-A1).
 *   - *_batch calls only enqueue work on `stream` and return after launch; launch errors
 *     return HARMONIA_ERR_CUDA; execution errors surface at the caller's synchronisation.
 *   - Query, result and workspace buffers are caller-owned; the library performs no device
 *     allocation on any query path (search, range, host search).
 *   - Query inputs are never errors: a query equal to HARMONIA_KEY_PAD returns NOT_FOUND,
 *     a range with lo > hi returns count 0.
 *   - Results are bit-identical whatever group size, PSA bits, window, staging plan or GPU
 *     count is used.
 *   - A tree is immutable during search/range calls; calls on different streams need
 *     separate workspaces; harmonia_update_batch needs exclusive access (the paper's phase
 *     model: query phase, then update phase).
 */
#ifndef HARMONIA_H
#define HARMONIA_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define HARMONIA_ABI_VERSION 2
#define HARMONIA_NOT_FOUND UINT64_C(0xFFFFFFFFFFFFFFFF) /* result of an absent key (C-A4)     */
#define HARMONIA_KEY_PAD   UINT64_C(0xFFFFFFFFFFFFFFFF) /* unused node slot; never a key (C-A2) */
#define HARMONIA_MAX_LEVELS 64

typedef enum {
  HARMONIA_OK = 0,
  HARMONIA_ERR_INVALID_ARG = 1,  /* null pointer, bad fanout/group size/opts, short workspace  */
  HARMONIA_ERR_UNSORTED = 2,     /* build keys not strictly increasing (duplicates included)  */
  HARMONIA_ERR_RESERVED = 3,     /* a key == HARMONIA_KEY_PAD or a value == HARMONIA_NOT_FOUND */
  HARMONIA_ERR_OUT_OF_MEMORY = 4,
  HARMONIA_ERR_CUDA = 5,         /* CUDA API/launch failure; see harmonia_last_cuda_error()   */
  HARMONIA_ERR_DEVICE_MISMATCH = 6,
  HARMONIA_ERR_TOO_LARGE = 7     /* more than 2^32-1 nodes, or height > HARMONIA_MAX_LEVELS    */
} harmonia_status;

/* Opaque: one Harmonia layout (key region + prefix-sum child region + values) resident on
 * one device.  Owned by the library; release with harmonia_destroy. */
typedef struct harmonia_tree harmonia_tree;

typedef struct {
  uint32_t fanout;        /* F: max children per internal node, power of two in [4, 256].
                             Internal nodes hold <= F-1 separator keys, leaves <= F-1 records
                             (P:L120, L268).  0 => 64.                                       */
  float fill;             /* bulk-load target occupancy in [0.5, 1]; 0 => 1.0 (C-A6)         */
  int32_t keys_on_device; /* 1: keys/values are device pointers on the current device; 0: host */
  int32_t reserved;
} harmonia_build_opts;

/* Query options.  An all-zero struct (or a NULL pointer) selects every default. */
typedef struct {
  int32_t group_size;   /* NTG lanes per query G: 0 = auto = 1 (the measured
                           B200 choice for every fanout: the narrowing of
                           Eq 4 continued to one lane per query); else a power of two in
                           [1, 32] with 2G <= F.  G = 1 is a deviation from §8(b)'s 2..32:
                           the paper's group narrowed to a single lane (lane-local binary
                           rank instead of a ballot).                                        */
  int32_t psa_bits;     /* PSA sort bits Nb (Eq 2): 0 = auto = ceil(log2(T/K)), K=16;
                           < 0 = PSA off (queries searched in arrival order); else 1..28.   */
  int32_t smem_levels;  /* top tree levels staged in shared memory: 0 = auto plan (fits the
                           smem budget), < 0 = none, else that many levels (clamped).        */
  int32_t flags;        /* HARMONIA_QF_* bits                                                 */
  uint64_t window;      /* PSA window = queries partitioned together (the paper's "time
                           window"): 0 = auto; otherwise rounded to a multiple of 1024 */
  uint32_t lane_queries; /* group_size = 1 only: independent queries interleaved per lane
                           (1, 2 or 4; 0 = auto)                                            */
  uint32_t sort_chunk;   /* staged-return PSA: level-2 chunk in queries, 4096 or 8192; 0 = auto
                           (8192 when the window holds >= 192 queries per leaf)            */
  uint64_t l2_window_bytes; /* search kernels: bytes of the unstaged internal key region pinned
                           in L2 by an access-policy window (persisting hits, streaming
                           misses): 0 = auto = all of it (capped by the device's window and
                           persisting-L2 limits); disable with HARMONIA_QF_NO_L2_WINDOW.  The
                           first windowed call sets the device's cudaLimitPersistingL2CacheSize. */
} harmonia_query_opts;

#define HARMONIA_QF_NO_PS_SMEM 1u  /* do not stage the prefix-sum array in shared memory     */
#define HARMONIA_QF_GATHER     2u  /* PSA return via a separate gather pass instead of the
                                      search kernel scattering results in place             */
#define HARMONIA_QF_ILP1       16u /* k-ary search with one query per lane group instead of two */
/* 64, 128, 512: ablations of ABI 1 removed in ABI 2 (LSD chunk sort, fused chunk sort + search,
 * 11-bit level-1 partition; all measured slower).  Set, they are INVALID_ARG. */
#define HARMONIA_QF_REMOVED_PSA_LSD   64u
#define HARMONIA_QF_REMOVED_FUSE_SORT 128u
#define HARMONIA_QF_REMOVED_PSA_WIDE  512u
#define HARMONIA_QF_SCATTER_RETURN 256u /* G = 1 PSA path: the search scatters results to
                                      out[original position] instead of the default staged
                                      return (chunk-local smem permutation + k_psa2_unmove) */
#define HARMONIA_QF_PER_LANE 1024u /* G = 1 PSA path: every lane descends on its own instead of
                                      the default warp-shared descent (the warp's PSA-ordered
                                      queries share the path down to the level where their
                                      key interval splits)                           */
#define HARMONIA_QF_RANGE_GROUP 2048u /* ranges: the G-lane group walk of the leaves (one
                                      load-ballot-store step per 2G slots) instead of the
                                      default lane-per-range (max_results < 512) or
                                      warp-per-range kernel; also implied by an explicit
                                      group_size                                             */
#define HARMONIA_QF_NO_L2_WINDOW 4096u /* no L2 access-policy window on the search kernels   */
#define HARMONIA_QF_NO_RANGE_LANE 32768u /* ranges with max_results < 512: the G-lane group walk
                                      instead of the default lane-per-range kernel (one lane
                                      per range on the warp-shared descent of PSA-ordered lo) */
#define HARMONIA_QF_PSA_COARSE 32u /* PSA level 1 only (8-bit coarse partition, no chunk sort) */
#define HARMONIA_QF_PSA_GLOBAL 8u  /* PSA as one global pass over all 2^Nb buckets (one atomic
                                      per query) instead of the default two-level partition  */
#define HARMONIA_QF_PSA_L16 8192u /* staged-return PSA: force two MSD levels (8 + 8 bits) and
                                      bucket-aligned chunks, i.e. the whole window in Eq-2
                                      order (default: chosen by the plan, see harmonia_plan) */
#define HARMONIA_QF_HOST_UNORDERED 65536u /* harmonia_search_batch_host: the caller guarantees that
                                      h_queries is ready when the call is made (written by the host,
                                      not by earlier work on `stream`), so the first chunks' H2D
                                      copies wait only for their device buffers, not for earlier
                                      work on `stream`: back-to-back calls then overlap one call's
                                      last D2H copy with the next call's first H2D copy.  Results
                                      are unchanged; h_values_out stays ordered after the call's
                                      own work as before. */
#define HARMONIA_QF_PSA_L8 16384u /* staged-return PSA: force one MSD level (8 bits) + chunk
                                      sort (the window is Eq-2 ordered inside each chunk)    */
#define HARMONIA_QF_LINEAR     4u  /* in-node search = the paper's linear NTG walk (Fig 9:
                                      2G keys per step, early exit) instead of the default
                                      k-ary NTG (same G lanes, fixed log-depth steps)         */

typedef struct {
  uint64_t n_keys;
  uint32_t fanout, height, psa_bits_auto, group_size_auto;
  uint64_t n_nodes, n_internal, n_leaves;
  uint64_t level_start[HARMONIA_MAX_LEVELS + 1]; /* BFS level boundaries, [0, N]            */
  uint64_t key_region_bytes, ps_bytes, value_bytes;
  uint64_t min_key, max_key;                     /* PAD/0 when the tree is empty             */
  int32_t device;
  int32_t reserved;
} harmonia_info;

/* ---------------------------------------------------------------------------------------
 * harmonia_build — bulk-load a Harmonia layout from n records (Fig 4(b)).
 *   keys[n]: strictly increasing, none equal to HARMONIA_KEY_PAD (C-A9);
 *   values[n]: none equal to HARMONIA_NOT_FOUND.  Host or device per opts->keys_on_device;
 *   caller-owned, copied (not retained).  n may be 0 (every query then returns NOT_FOUND).
 *   Layout: key region = N nodes x F uint64 slots in breadth-first order, unused slots =
 *   HARMONIA_KEY_PAD (C-A2); PS = uint32[I+1], PS[n] = key-region index of node n's first
 *   child, PS[I] = N (C-A7); values = uint64[L x F] aligned with leaf slots (C-A3).
 *   Node counts per level follow the even-distribution closed form (C-A6).
 *   Synchronises `stream` (validation result is read back).  *out receives the tree.
 *   Errors: INVALID_ARG, UNSORTED, RESERVED, OUT_OF_MEMORY, TOO_LARGE, CUDA.
 * ------------------------------------------------------------------------------------- */
harmonia_status harmonia_build(const uint64_t* keys, const uint64_t* values, uint64_t n,
                               const harmonia_build_opts* opts, void* stream,
                               harmonia_tree** out);

/* Frees the tree's device memory (synchronises the device). NULL is a no-op. */
void harmonia_destroy(harmonia_tree* tree);

harmonia_status harmonia_get_info(const harmonia_tree* tree, harmonia_info* info);

/* Copies the layout to caller-owned host arrays (for the oracle's layout checker):
 * h_key_region[n_nodes*F], h_ps[n_internal+1], h_leaf_values[n_leaves*F].  Synchronous. */
harmonia_status harmonia_export_layout(const harmonia_tree* tree, uint64_t* h_key_region,
                                       uint32_t* h_ps, uint64_t* h_leaf_values);

/* ---------------------------------------------------------------------------------------
 * harmonia_search_batch — n point queries (§3.2.1; PSA §4.1; NTG §4.2).
 *   d_queries[n] -> d_values_out[n]: the value of each query's key, or HARMONIA_NOT_FOUND.
 *   Pipeline per PSA window (default: the whole batch up to 2^27 queries): PSA (Eq 2) on the
 *   top Nb key bits -- one or two 8-bit MSD rank + move rounds (harmonia_plan.psa_levels),
 *   then a counting sort of 4096/8192-query chunks on all Nb bits -- the descent with Eq 1
 *   (child = PS[node] + i - 1) and leaf probe, then the results go back to the caller's
 *   order through a chunk-local shared-memory permutation and the inverse moves.  d_queries
 *   and d_values_out may not overlap.  d_workspace must hold
 *   harmonia_search_workspace_bytes(tree, n, opts) bytes (about 36 bytes per window query),
 *   16-byte aligned.   Errors: INVALID_ARG, DEVICE_MISMATCH, CUDA.
 * ------------------------------------------------------------------------------------- */
size_t harmonia_search_workspace_bytes(const harmonia_tree* tree, uint64_t n,
                                       const harmonia_query_opts* opts);
harmonia_status harmonia_search_batch(const harmonia_tree* tree, const uint64_t* d_queries,
                                      uint64_t n, uint64_t* d_values_out, void* d_workspace,
                                      size_t workspace_bytes, const harmonia_query_opts* opts,
                                      void* stream);

/* Host-buffer variant (end-to-end): h_queries[n] / h_values_out[n] in host memory (pinned
 * for overlap; pageable works but serialises).  Chunks are copied H2D, searched and copied
 * D2H on a three-stage pipeline; everything is ordered after prior work on `stream` and the
 * caller synchronises `stream` to consume h_values_out.  d_workspace must hold
 * harmonia_search_host_workspace_bytes(tree, n, opts).  Not reentrant per tree. */
size_t harmonia_search_host_workspace_bytes(const harmonia_tree* tree, uint64_t n,
                                            const harmonia_query_opts* opts);
harmonia_status harmonia_search_batch_host(const harmonia_tree* tree, const uint64_t* h_queries,
                                           uint64_t n, uint64_t* h_values_out,
                                           void* d_workspace, size_t workspace_bytes,
                                           const harmonia_query_opts* opts, void* stream);

/* ---------------------------------------------------------------------------------------
 * harmonia_range_batch — n inclusive range queries [lo, hi] ("use the basic query
 *   operation to get the first target key in the range, and scan the key region from the
 *   first target key to the last target key"; C-A10).
 *   Query j writes its first min(count, max_results) records, ascending, to
 *   d_keys_out[j*max_results + t] / d_values_out[j*max_results + t]; d_counts_out[j] = the
 *   true total (> max_results signals truncation).  Slab entries past the count are not
 *   written.  max_results may be 0 (counts only).  Workspace as for search.
 * ------------------------------------------------------------------------------------- */
size_t harmonia_range_workspace_bytes(const harmonia_tree* tree, uint64_t n,
                                      const harmonia_query_opts* opts);
harmonia_status harmonia_range_batch(const harmonia_tree* tree, const uint64_t* d_lo,
                                     const uint64_t* d_hi, uint64_t n, uint32_t max_results,
                                     uint64_t* d_keys_out, uint64_t* d_values_out,
                                     uint32_t* d_counts_out, void* d_workspace,
                                     size_t workspace_bytes, const harmonia_query_opts* opts,
                                     void* stream);

/* ---------------------------------------------------------------------------------------
 * harmonia_update_batch — batched upsert/delete (§3.2.2; C-A18).
 *   d_ops[n] (0 = upsert: insert a new record or update an existing record's value;
 *   1 = delete: remove if present), d_keys[n], d_values[n] (ignored for deletes).
 *   Sequential semantics in batch order: the last op on a key wins.  Keys equal to
 *   HARMONIA_KEY_PAD or upsert values equal to HARMONIA_NOT_FOUND are rejected
 *   (HARMONIA_ERR_RESERVED, tree unchanged).  In place when the leaves have room: if every
 *   leaf the batch changes keeps between ceil((F-1)/2) and F-1 records (trees built with fill
 *   < 1), values are overwritten, the changed leaves re-packed where the separators route their
 *   keys and the leaf record counts recomputed; the key region, PS and internal levels keep
 *   their positions (separators still bound their subtrees, I5, but need not equal subtree
 *   minima after deletes).  Otherwise the whole layout is rebuilt from the merged record
 *   sequence (the paper's post-batch "movement", as bulk-synchronous device passes;
 *   bit-identical to a fresh harmonia_build, invariant I8).  harmonia_update_last_mode tells
 *   which (1 in place, 2 rebuilt).  The batch sort and scans use CUB (a library primitive,
 *   like cuBLAS for a GEMM; not on the query path).  A tree of 2^31 - 1 or more records after
 *   the batch is HARMONIA_ERR_TOO_LARGE (32-bit scan counts).  May reallocate the tree's
 *   arrays; synchronises `stream`.
 *   d_workspace must hold harmonia_update_workspace_bytes(tree, n).
 * ------------------------------------------------------------------------------------- */
size_t harmonia_update_workspace_bytes(const harmonia_tree* tree, uint64_t n);
int harmonia_update_last_mode(const harmonia_tree* tree); /* 0 none yet, 1 in place, 2 rebuilt */
harmonia_status harmonia_update_batch(harmonia_tree* tree, const uint8_t* d_ops,
                                      const uint64_t* d_keys, const uint64_t* d_values,
                                      uint64_t n, void* d_workspace, size_t workspace_bytes,
                                      void* stream);
/* harmonia_update_batch_seq: the same with the batch order given explicitly: op i counts as
 * issued at d_seq[i] (uint64, distinct), so the last op per key is the one with the largest
 * seq (C-A18).  d_seq = NULL is harmonia_update_batch.  Used by the partitioned mode, where a
 * shard receives the ops of several ranks in routed order.  Same workspace size.
 * harmonia_route_update_payload: after harmonia_route_partition of the update keys (d_pos =
 * its positions), d_ops_out[i] = d_ops[d_pos[i]], d_values_out[i] = d_values[d_pos[i]] and
 * d_seq_out[i] = rank << 32 | d_pos[i] (global batch order = rank-major, then batch order). */
harmonia_status harmonia_update_batch_seq(harmonia_tree* tree, const uint8_t* d_ops, const uint64_t* d_keys,
                                          const uint64_t* d_values, const uint64_t* d_seq, uint64_t n,
                                          void* d_workspace, size_t workspace_bytes, void* stream);
/* harmonia_update_validate: *d_flags (uint32, device) = OR over the batch of 2 (a key equal to
 * HARMONIA_KEY_PAD or an upsert value equal to HARMONIA_NOT_FOUND: the batch would be
 * HARMONIA_ERR_RESERVED) and 4 (an op code other than 0/1).  Asynchronous.  The partitioned
 * mode validates every rank's batch before routing so that all shards accept or all reject. */
harmonia_status harmonia_update_validate(const uint8_t* d_ops, const uint64_t* d_keys, const uint64_t* d_values,
                                         uint64_t n, uint32_t* d_flags, void* stream);
harmonia_status harmonia_route_update_payload(const uint8_t* d_ops, const uint64_t* d_values,
                                              const uint32_t* d_pos, uint64_t n, uint32_t rank,
                                              uint8_t* d_ops_out, uint64_t* d_values_out,
                                              uint64_t* d_seq_out, void* stream);

/* ---------------------------------------------------------------------------------------
 * Key-range partitioning across P devices (multi-GPU mode).
 * harmonia_route_partition: dest(q) = #{ s in d_splitters[0..P-2] : s <= q }  (splitters
 *   strictly increasing; shard p owns [splitter[p-1], splitter[p]) ).  Writes the queries
 *   grouped by destination (d_routed[n], destination-major), the original position of each
 *   routed query (d_pos[n], uint32 — n < 2^32), and h_counts[P] (host, synchronous).
 * harmonia_scatter_results: d_out[d_pos[i]] = d_routed_values[i] for i < n.
 * ------------------------------------------------------------------------------------- */
size_t harmonia_route_workspace_bytes(uint32_t P, uint64_t n);
harmonia_status harmonia_route_partition(const uint64_t* d_splitters, uint32_t P,
                                         const uint64_t* d_queries, uint64_t n,
                                         uint64_t* d_routed, uint32_t* d_pos, uint64_t* h_counts,
                                         void* d_workspace, size_t workspace_bytes, void* stream);
harmonia_status harmonia_scatter_results(const uint64_t* d_routed_values, const uint32_t* d_pos,
                                         uint64_t n, uint64_t* d_out, void* stream);

/* ---------------------------------------------------------------------------------------
 * Fused routing over peer memory (partitioned mode without NCCL data collectives; the
 * north_star's "queries routed ... and results returned" step).  Per batch,
 * all calls on one rank use the same workspace (harmonia_route_workspace_bytes(P, n)):
 *   1. harmonia_route_count: dest(q) as in harmonia_route_partition; the per-query rank
 *      inside its destination run is kept in the workspace; h_counts[P] (host, synchronous).
 *   2. (caller) exchange the P x P count matrix; rank p's run for destination d starts at
 *      sum_{p' < p} counts[p'][d] in d's receive buffer.
 *   3. harmonia_route_push: the destination-major partition writes the run of destination d
 *      straight to h_dst[d] (a device address: this rank's own buffer or a peer buffer mapped
 *      with harmonia_peer_open; NVLink stores); the order inside a run is unspecified.
 *      No local copy of the routed batch exists.  Asynchronous on `stream`.
 *   4. (caller) barrier; each rank searches its receive buffer (harmonia_search_batch) and
 *      returns the results of source p's segment with harmonia_segments_push to p's "back"
 *      buffer at the offset of this rank's run in p's routed order; barrier.
 *   5. harmonia_route_return: d_out[i] = d_back[routed position of query i] (the inverse of
 *      step 3's partition; reads back in runs, writes d_out contiguously).
 * harmonia_segments_push: for s < nseg, copy d_src[h_src_off[s] .. + h_len[s]) to the device
 *   address h_dst[s] (16-byte stores when aligned).  nseg <= 1024.  Workspace: any buffer of
 *   harmonia_route_workspace_bytes(1, 1) bytes not in use by a pending route call.
 * P <= 256, n < 2^32; INVALID_ARG on violations or a short workspace.
 * harmonia_peer_alloc: cudaMalloc(bytes) + its CUDA IPC handle (64 bytes written to
 *   handle_out) for the other ranks; harmonia_peer_open maps a peer's handle into this
 *   process (cudaIpcOpenMemHandle, lazy peer access); harmonia_peer_close unmaps it;
 *   harmonia_peer_free releases an own buffer.  Setup-time calls, never on a query path.
 *   Buffers from harmonia_peer_alloc are zero-filled.
 * harmonia_peer_barrier: device-side barrier of the P ranks of the fused routing (steps 4's
 *   "barrier"; no host thread waits).  d_flag_addrs[P] (device array): the address of rank p's
 *   flag array (P uint64, a harmonia_peer_alloc buffer, mapped into this process with
 *   harmonia_peer_open; this rank's own for p = me); d_my_flags: this rank's own flag array.
 *   Every rank calls it with the same strictly increasing epoch (1, 2, ...).  The kernel
 *   stores `epoch` to slot `me` of every rank's flags (system-scope fence + release store, so
 *   the stores of this rank's earlier work on `stream` -- its pushed runs -- are visible
 *   first) and returns when every rank's slot in d_my_flags holds >= epoch (system-scope
 *   acquire), so the work queued after it on `stream` sees every peer's pushes.  After
 *   timeout_ns (0: 30 s) without all flags, it sets *d_error = 1 and returns (the caller
 *   checks d_error; the batch's results are then invalid).  Asynchronous; P <= 256.
 * ------------------------------------------------------------------------------------- */
harmonia_status harmonia_route_count(const uint64_t* d_splitters, uint32_t P, const uint64_t* d_queries,
                                     uint64_t n, uint64_t* h_counts, void* d_workspace,
                                     size_t workspace_bytes, void* stream);
harmonia_status harmonia_route_push(const uint64_t* d_splitters, uint32_t P, const uint64_t* d_queries,
                                    uint64_t n, const uint64_t* h_dst, void* d_workspace,
                                    size_t workspace_bytes, void* stream);
harmonia_status harmonia_route_return(uint32_t P, const uint64_t* d_back, uint64_t n, uint64_t* d_out,
                                      void* d_workspace, size_t workspace_bytes, void* stream);
harmonia_status harmonia_segments_push(const uint64_t* d_src, uint32_t nseg, const uint64_t* h_src_off,
                                       const uint64_t* h_len, const uint64_t* h_dst, void* d_workspace,
                                       size_t workspace_bytes, void* stream);
/* ---------------------------------------------------------------------------------------
 * Range queries over key-range shards (partitioned mode; C-A10).  A range
 * [lo, hi] is cut at every splitter it crosses: its piece on shard d is
 * [max(lo, s_{d-1}), min(hi, s_d - 1)] (s = d_splitters, P-1 strictly increasing; shard d owns
 * [s_{d-1}, s_d)); lo > hi gives one piece on dest(lo) that answers count 0.  Pieces of range
 * i get ids pbase[i] .. pbase[i+1]-1 in shard (= key) order.
 * harmonia_range_split_count: d_npieces[n+1] (per range, [n] = 0), d_pbase[n+1] (exclusive
 *   prefix: piece ids), h_counts[P] pieces per destination, *h_total = pieces (host, sync).
 * harmonia_range_split_emit (same workspace, after _count): the pieces destination-major:
 *   d_plo/d_phi[total] and their ids d_pid[total]; order inside a destination's run is
 *   unspecified.
 *   (caller) route the pieces to their shards, run harmonia_range_batch there with the same
 *   cap, bring the answers back in the routed order.
 * harmonia_range_assemble: for the m = total routed answers (d_counts[m] true totals,
 *   d_keys/d_values[m][cap] slabs, d_pid[m] their piece ids), range i receives its pieces'
 *   records in shard order, cut at cap (d_keys_out/d_values_out[n][cap]; entries past the
 *   count are not written) and d_total_out[i] = the summed true count.  d_row_scratch: m
 *   uint32.  Asynchronous.
 * ------------------------------------------------------------------------------------- */
size_t harmonia_range_split_workspace_bytes(uint64_t n);
harmonia_status harmonia_range_split_count(const uint64_t* d_splitters, uint32_t P, const uint64_t* d_lo,
                                           const uint64_t* d_hi, uint64_t n, uint32_t* d_npieces,
                                           uint32_t* d_pbase, uint64_t* h_counts, uint64_t* h_total,
                                           void* d_workspace, size_t workspace_bytes, void* stream);
harmonia_status harmonia_range_split_emit(const uint64_t* d_splitters, uint32_t P, const uint64_t* d_lo,
                                          const uint64_t* d_hi, uint64_t n, const uint32_t* d_pbase,
                                          uint64_t* d_plo, uint64_t* d_phi, uint32_t* d_pid,
                                          void* d_workspace, size_t workspace_bytes, void* stream);
harmonia_status harmonia_range_assemble(uint64_t n, uint32_t cap, const uint32_t* d_pbase,
                                        const uint32_t* d_pid, uint64_t m, const uint32_t* d_counts,
                                        const uint64_t* d_keys, const uint64_t* d_values,
                                        uint32_t* d_row_scratch, uint64_t* d_keys_out,
                                        uint64_t* d_values_out, uint64_t* d_total_out, void* stream);
harmonia_status harmonia_peer_alloc(size_t bytes, void** d_ptr, void* handle_out);
harmonia_status harmonia_peer_open(const void* handle, void** d_ptr);
harmonia_status harmonia_peer_close(void* d_ptr);
harmonia_status harmonia_peer_free(void* d_ptr);
harmonia_status harmonia_peer_barrier(uint32_t P, uint32_t me, const uint64_t* d_flag_addrs, uint64_t* d_my_flags,
                                      uint64_t epoch, uint32_t* d_error, uint64_t timeout_ns, void* stream);

/* The plan a search/range call with these options would use (for reporting). */
typedef struct {
  int32_t group_size, psa_bits, smem_levels, ps_in_smem;
  uint64_t window;
  uint32_t smem_bytes, smem_nodes;
  uint32_t staged_return;  /* 1: results return through the chunk-local stage + inverse move */
  uint32_t lane_queries;   /* G = 1: queries interleaved per lane */
  uint32_t warp_shared;    /* 1: G = 1 warp-shared descent (see HARMONIA_QF_PER_LANE) */
  uint32_t sort_chunk;     /* staged return: level-2 chunk (queries); 0 when not staged */
  uint64_t l2_window_bytes; /* bytes of the internal key region pinned in L2 (0 = none) */
  uint32_t psa_levels;     /* global MSD partition levels before the chunk sort: 1 = 8 bits
                              (Eq-2 order inside each sort_chunk piece), 2 = 8 + 8 bits with
                              chunks of whole 16-bit buckets (the whole window in Eq-2 order);
                              0 = PSA off.  Auto: 2 when a level-1 chunk would hold fewer
                              than 4 queries per leaf (large trees), else 1.                */
  uint32_t chunk_group;    /* psa_levels 2: 16-bit buckets per chunk group (0 otherwise)     */
} harmonia_plan;
harmonia_status harmonia_query_plan(const harmonia_tree* tree, uint64_t n,
                                    const harmonia_query_opts* opts, harmonia_plan* out);

/* ---------------------------------------------------------------------------------------
 * harmonia_psa_inspect — run only the PSA stages (Eq 2) that
 *   harmonia_search_batch would run for (n, opts) and write the queries to d_order_out[n] in
 *   the order the search kernel visits them (window by window, chunk by chunk, no padding).
 *   With the plan's psa_levels = 2 every window is non-decreasing in its Nb-bit bucket
 *   (C-A11) except inside a chunk group larger than sort_chunk queries (skewed batches); with
 *   psa_levels = 1 the top min(8, Nb) bucket bits are non-decreasing over each window and all
 *   Nb bits inside each sort_chunk piece.  d_order_out is a permutation of d_queries.
 *   Workspace as for harmonia_search_batch.  Asynchronous.  For tests and reports; it is not
 *   part of the query path.  Errors: INVALID_ARG, DEVICE_MISMATCH, CUDA.
 * ------------------------------------------------------------------------------------- */
harmonia_status harmonia_psa_inspect(const harmonia_tree* tree, const uint64_t* d_queries, uint64_t n,
                                     const harmonia_query_opts* opts, void* d_workspace,
                                     size_t workspace_bytes, uint64_t* d_order_out, void* stream);

/* ---------------------------------------------------------------------------------------
 * NTG static profiling (§4.2): the paper's model for the thread-group size.
 *
 * harmonia_ntg_choose — host-only arithmetic (no GPU needed).
 *   prof[n][h][2]: per sample query j and level l, prof[j][l][0] = r = keys of the node on
 *     j's path before the target (<= q in internal nodes, < q at the leaf) and
 *     prof[j][l][1] = cnt = valid keys in that node.  bucket[n] (may be NULL = identity):
 *     PSA bucket per sample; the samples are taken in stable bucket order.
 *   Fig 9 steps (C-A13): min(r/(GS*kpl)+1, ceil(cnt/(GS*kpl))).  Eq 3: S(GS) = mean over
 *   warps of 32/GS consecutive samples of the per-level max steps summed over levels
 *   [lev0, h).  Eq 4 (C-A22): starting at gs0, halve GS while 2*S(GS)/S(GS/2) > 1, GS >= 2
 *   (C-A14).  *gs_out = the chosen GS; steps_out[6] (may be NULL) = S(1), S(2), ..., S(32)
 *   (0 for GS > gs0).  INVALID_ARG on null prof/gs_out, n == 0, h == 0, kpl == 0 or gs0 not a
 *   power of two in [1, 32].
 *
 * harmonia_tune_group_size — the same model on a device sample: one profiling kernel (a plain
 *   Eq-1 descent per sample on the legacy default stream), a synchronous copy of the n*h*2
 *   counters, then harmonia_ntg_choose with gs0 = min(32, F/2), kpl = 2 (128-bit loads),
 *   lev0 = the shared-memory-staged levels of the plan `opts` selects and the plan's PSA
 *   bucket.  d_samples: n <= 2^20 device queries.  Offline (allocates a temporary device
 *   buffer); the result is advice for harmonia_query_opts.group_size, which stays 0 = the
 *   measured auto choice unless the caller passes it.
 * --------------------------------------------------------------------------------------- */
harmonia_status harmonia_ntg_choose(const uint32_t* prof, const uint32_t* bucket, uint32_t n, uint32_t h,
                                    uint32_t lev0, uint32_t gs0, uint32_t kpl, int32_t* gs_out,
                                    double* steps_out);
harmonia_status harmonia_tune_group_size(const harmonia_tree* tree, const uint64_t* d_samples, uint32_t n,
                                         const harmonia_query_opts* opts, int32_t* gs_out, double* steps_out);

/* Eq 2 as used by psa_bits = 0: ceil(log2(T/K)) clamped to [0, 28], K = 16. */
int32_t harmonia_psa_bits_auto(uint64_t n_keys);

/* Kernel timing for benchmarks.  While enabled, every kernel the library launches is
 * bracketed by a CUDA event pair recorded on its launch stream, per kernel class.
 * harmonia_profile_read synchronises those events, writes the summed milliseconds and
 * launch counts per class (arrays of HARMONIA_PROF_KINDS) and clears the record. */
#define HARMONIA_PROF_KINDS 8
enum { HARMONIA_PROF_SEARCH = 0, HARMONIA_PROF_RANGE = 1, HARMONIA_PROF_PSA_HIST = 2,
       HARMONIA_PROF_PSA_SCAN = 3, HARMONIA_PROF_PSA_SCATTER = 4, HARMONIA_PROF_RETURN = 5,
       HARMONIA_PROF_BUILD = 6, HARMONIA_PROF_UPDATE = 7 };
void harmonia_profile_enable(int on);
harmonia_status harmonia_profile_read(double* total_ms, uint64_t* launches);

const char* harmonia_status_string(harmonia_status s);
int harmonia_last_cuda_error(void);          /* cudaError_t of the last ERR_CUDA (thread-local) */
uint64_t harmonia_kernel_launches(void);     /* kernels this library launched (process total)  */
int harmonia_abi_version(void);

#ifdef __cplusplus
}
#endif
#endif /* HARMONIA_H */
