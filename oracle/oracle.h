/*
 * oracle.h — CPU ORACLE for Harmonia (Yan, Lin, Peng, Zhang, PPoPP'19).
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and bench.py's
 * cpu_baseline / --impl reference legs may load liboracle.so.  The product path
 * (paper_conf_ppopp_yanlpz19_b200/, libharmonia.so) never includes, links or calls
 * anything here, and nothing here includes the product's headers: the two share no
 * code, no constants and no helpers.
 *
 * Citations "P:Lnnn" are /root/reference/PAPER.md line numbers (the paper text);
 * "C-Axx" are the readings listed in DESIGN.md §3 (ambiguities the paper leaves open).
 *
 * Parity status of each function is stated beside it; every function is pinned by a
 * `-m "not gpu"` test except where "parity unpinned" is written.
 */
#ifndef HARMONIA_ORACLE_H
#define HARMONIA_ORACLE_H
#include <stdint.h>
#include <stddef.h>

#ifdef __cplusplus
extern "C" {
#endif

/* Oracle-private sentinels (C-A2, C-A4).  Deliberately re-declared here, not shared. */
#define ORC_NOT_FOUND 0xFFFFFFFFFFFFFFFFull
#define ORC_PAD       0xFFFFFFFFFFFFFFFFull

/* ---------------- O1: sorted array + std::lower_bound (the authority) -------------
 * P:L282-L288 (§3.2.1): a point query returns the record of the target key; a range
 * query returns every record from the first to the last target key of the range.
 * Plain definition (DESIGN.md §3 "oracle"): point(q) = v(q) if q in K else NOT_FOUND;
 * range(lo,hi) = ascending (k, v(k)) with lo <= k <= hi, count = true total.
 * keys must be strictly increasing.  nthreads <= 0 => hardware_concurrency().
 * Pinned by: brute force O3 (tests/test_oracle_search.py), closed forms. */
void orc_sorted_search(const uint64_t* keys, const uint64_t* vals, uint64_t n,
                       const uint64_t* q, uint64_t nq, uint64_t* out, int nthreads);
/* Slab layout per query j: kout[j*cap + t], vout[j*cap + t] for t < min(count,cap);
 * counts[j] = true total (may exceed cap).  Unwritten slab entries are untouched. */
void orc_sorted_range(const uint64_t* keys, const uint64_t* vals, uint64_t n,
                      const uint64_t* lo, const uint64_t* hi, uint64_t nq, uint32_t cap,
                      uint64_t* kout, uint64_t* vout, uint32_t* counts, int nthreads);

/* ---------------- O3: brute-force linear scan (tiny inputs) ----------------------- */
void orc_brute_search(const uint64_t* keys, const uint64_t* vals, uint64_t n,
                      const uint64_t* q, uint64_t nq, uint64_t* out);
void orc_brute_range(const uint64_t* keys, const uint64_t* vals, uint64_t n,
                     const uint64_t* lo, const uint64_t* hi, uint64_t nq, uint32_t cap,
                     uint64_t* kout, uint64_t* vout, uint32_t* counts);

/* ---------------- O2: regular (pointer) B+tree, Fig 4(a) ------------
 * Internal node: <= F-1 keys, <= F children.  Leaf: <= F-1 (key,value) with
 * a sibling link.  Separator rule C-A5 (key equal to a separator descends right).
 * Insert splits, delete borrows/merges at the textbook minimum occupancy (C-A6/I2/I3).
 * Pinned by: O1 on random insert/delete sequences, O6 std::map, structural check. */
void*    orc_bpt_create(uint32_t fanout);
void     orc_bpt_destroy(void* t);
int      orc_bpt_insert(void* t, uint64_t key, uint64_t value); /* 1 new, 0 replaced */
int      orc_bpt_erase(void* t, uint64_t key);                  /* 1 erased, 0 absent */
void     orc_bpt_search(void* t, const uint64_t* q, uint64_t nq, uint64_t* out);
void     orc_bpt_search_mt(void* t, const uint64_t* q, uint64_t nq, uint64_t* out, int nthreads);
uint64_t orc_bpt_insert_array(void* t, const uint64_t* keys, const uint64_t* vals, uint64_t n);
void     orc_bpt_range(void* t, const uint64_t* lo, const uint64_t* hi, uint64_t nq,
                       uint32_t cap, uint64_t* kout, uint64_t* vout, uint32_t* counts);
uint64_t orc_bpt_size(void* t);
uint32_t orc_bpt_height(void* t);
/* 0 = ok; otherwise a positive code naming the violated rule (see bptree.cc). */
int      orc_bpt_check(void* t);
/* Test hook pinning the checker: apply one targeted corruption (kinds 1-6, bptree.cc). */
int      orc_bpt_debug_mutate(void* t, int kind);
/* In-order dump via the leaf chain. */
void     orc_bpt_dump(void* t, uint64_t* keys, uint64_t* vals);
/* Level statistics: nodes[l], entries[l] (keys in leaves, children in internals). */
void     orc_bpt_level_stats(void* t, uint64_t* nodes, uint64_t* entries, uint32_t maxlev);
/* Fig 10: for each query and every level, the sequential in-node search
 * stops at slot p (first key > q, or the last valid key); counts[quarter(p)]++ where the
 * F-1 key slots are cut into 4 equal parts.  Weak statistical pin only (T9). */
void     orc_bpt_quarter_stats(void* t, const uint64_t* q, uint64_t nq, uint64_t counts[4]);
/* Fig 3: comparisons per level for each query, sequential in-node search.
 * out[j*h + l] = comparisons of query j at level l (h = orc_bpt_height). */
void     orc_bpt_comparisons(void* t, const uint64_t* q, uint64_t nq, uint32_t* out);

/* ---------------- O4: Harmonia layout (Fig 4(b)) ---------------------
 * Key region: nodes in breadth-first order, fixed item of F slots (C-A2: (F-1) keys of
 * P:L268 plus one PAD slot), unused slots = ORC_PAD.  Child region: prefix-sum array,
 * PS[n] = index of node n's first child = number of nodes before it, over the
 * I internal nodes plus the sentinel PS[I] = N (C-A7).  Values: leaf-aligned,
 * vals[(leaf - level_start[h-1])*F + slot] (C-A3), pads = ORC_NOT_FOUND.
 * Bulk load = even-distribution closed form (C-A6).
 * level_nodes / level_start have room for 64 levels; returns height h (>= 1). */
uint32_t orc_layout_shape(uint64_t n, uint32_t fanout, double fill, uint64_t level_nodes[64]);
/* Fills caller-allocated arrays sized from orc_layout_shape:
 * key_region[N*F], ps[I+1], leaf_vals[L*F].  Returns 0 on success. */
int      orc_layout_build(const uint64_t* keys, const uint64_t* vals, uint64_t n,
                          uint32_t fanout, double fill,
                          uint64_t* key_region, uint32_t* ps, uint64_t* leaf_vals);
/* Invariants I1..I7 and I9 of DESIGN.md §3 over an arbitrary layout (GPU-exported or
 * oracle-built).  keys/vals: the expected record set (strictly increasing keys).
 * Returns 0 if all hold, else the invariant number; msg gets a description. */
int      orc_layout_check(const uint64_t* key_region, const uint32_t* ps,
                          const uint64_t* leaf_vals, uint32_t fanout, uint32_t height,
                          const uint64_t* level_start /* h+1 entries */,
                          const uint64_t* keys, const uint64_t* vals, uint64_t n,
                          char* msg, int msglen);
/* The same with strict_sep = 0: the equality half of I5 (separator == subtree minimum, a
 * property of a fresh build) is not required -- for layouts updated in place. */
int      orc_layout_check2(const uint64_t* key_region, const uint32_t* ps,
                           const uint64_t* leaf_vals, uint32_t fanout, uint32_t height,
                           const uint64_t* level_start, const uint64_t* keys, const uint64_t* vals,
                           uint64_t n, char* msg, int msglen, int strict_sep);
/* Scalar Eq-1 interpreter: child_idx = PrefixSum[node_idx] + i - 1. */
void     orc_layout_search(const uint64_t* key_region, const uint32_t* ps,
                           const uint64_t* leaf_vals, uint32_t fanout, uint32_t height,
                           const uint64_t* level_start, const uint64_t* q, uint64_t nq,
                           uint64_t* out);
/* Range over the layout: Eq-1 descent to lo, then scan the key region. */
void     orc_layout_range(const uint64_t* key_region, const uint32_t* ps,
                          const uint64_t* leaf_vals, uint32_t fanout, uint32_t height,
                          const uint64_t* level_start, const uint64_t* lo, const uint64_t* hi,
                          uint64_t nq, uint32_t cap, uint64_t* kout, uint64_t* vout,
                          uint32_t* counts);
/* One Eq-1 step, for the worked example P:L286. */
uint64_t orc_eq1_child(const uint32_t* ps, uint64_t node_idx, uint64_t i);

/* ---------------- O5: analytic models (§4) ----------------------------------------- */
/* Eq 2: N = B - log2(2^B / T * K), literally; rounded up, clamped to [0,B]. */
uint32_t orc_psa_bits(uint32_t B, double T, uint32_t K);
/* PSA as the paper states it: stable order of the queries by their most
 * significant N bits (C-A11: bits of the occupied key span [min_key, max_key]).
 * perm[j] = original index of the j-th query in partially-sorted order.           */
void     orc_psa_order(const uint64_t* q, uint64_t nq, uint32_t nbits,
                       uint64_t min_key, uint64_t max_key, uint64_t* perm);
uint64_t orc_psa_bucket(uint64_t q, uint32_t nbits, uint64_t min_key, uint64_t max_key);
void     orc_psa_buckets(const uint64_t* q, uint64_t nq, uint32_t nbits, uint64_t min_key,
                         uint64_t max_key, uint64_t* out);
/* Fig 9, C-A13: comparison steps of one query whose target sits after r
 * keys (r = #keys <= q) in a node of cnt keys, with GS threads and kpl keys per thread
 * per step. */
uint32_t orc_ntg_steps(uint32_t r, uint32_t cnt, uint32_t gs, uint32_t kpl);
/* Eq 3/4: average over warps of the per-warp maximum step count summed
 * over the profiled levels [lev0, h), for thread-group size gs; a warp of `warp` threads
 * serves warp/gs consecutive queries (Fig 9 uses warp = 8, the B200 32). */
double   orc_ntg_warp_steps(const uint64_t* key_region, const uint32_t* ps, uint32_t fanout,
                            uint32_t height, const uint64_t* level_start, const uint64_t* q,
                            uint64_t nq, uint32_t gs, uint32_t kpl, uint32_t lev0, uint32_t warp);
/* Static-profile choice: start at gs0, halve while Eq 4 ratio 2*S_b/S_a > 1. */
uint32_t orc_ntg_choose_gs(const uint64_t* key_region, const uint32_t* ps, uint32_t fanout,
                           uint32_t height, const uint64_t* level_start, const uint64_t* q,
                           uint64_t nq, uint32_t gs0, uint32_t kpl, uint32_t lev0, uint32_t warp);
/* Fig 2: memory transactions per warp per level = distinct nodes touched
 * by the warp's queries at that level, averaged over levels and warps. */
double   orc_warp_transactions(const uint64_t* key_region, const uint32_t* ps,
                               uint32_t fanout, uint32_t height, const uint64_t* level_start,
                               const uint64_t* q, uint64_t nq, uint32_t queries_per_warp);

/* ---------------- O6: update oracle (std::map), C-A18 ------------------------------ */
/* ops[i] = 0 upsert, 1 delete; applied in batch order; returns new size.  The result
 * record set is written to out_keys/out_vals (capacity cap). */
void*    orc_map_create(const uint64_t* keys, const uint64_t* vals, uint64_t n);
void     orc_map_destroy(void* m);
uint64_t orc_map_apply(void* m, const uint8_t* ops, const uint64_t* keys,
                       const uint64_t* vals, uint64_t n);
uint64_t orc_map_dump(void* m, uint64_t* keys, uint64_t* vals, uint64_t cap);

#ifdef __cplusplus
}
#endif
#endif
