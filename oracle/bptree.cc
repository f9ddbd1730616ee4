// O2: the paper's "regular B+tree" (Fig 4(a)) — a textbook pointer tree.
// TEST INFRASTRUCTURE ONLY — see oracle.h.
//
// "Each internal node can store no more than fanout-1 keys and fanout child
// references."  Leaves hold <= F-1 (key, value) records and a sibling link (the leaf
// level is what a range scan walks).  Search: "compares with the keys
// held by current node to find a child whose corresponding range contains the target
// key", then follows the child reference.  Separator rule C-A5: child i holds keys in
// [sep[i-1], sep[i]); a key equal to a separator descends right.
// Minimum occupancy (paper silent, C-A6 / I2 / I3): non-root internal >= ceil(F/2)
// children, non-root leaf >= ceil((F-1)/2) records.
#include "oracle.h"

#include <algorithm>
#include <cstdint>
#include <thread>
#include <vector>

namespace {

struct Node {
  bool leaf;
  std::vector<uint64_t> keys;   // separators (internal) or record keys (leaf)
  std::vector<Node*> child;     // internal only
  std::vector<uint64_t> vals;   // leaf only
  Node* next = nullptr;         // leaf sibling link
  explicit Node(bool l) : leaf(l) {}
};

struct Tree {
  uint32_t F;
  Node* root;
  uint64_t size = 0;
  size_t min_children() const { return (F + 1) / 2; }  // ceil(F/2)
  size_t min_records() const { return F / 2; }         // ceil((F-1)/2)
  size_t max_keys() const { return F - 1; }
};

void free_node(Node* n) {
  if (!n->leaf)
    for (Node* c : n->child) free_node(c);
  delete n;
}

// index of the child whose range contains k = number of separators <= k
size_t child_index(const Node* n, uint64_t k) {
  return std::upper_bound(n->keys.begin(), n->keys.end(), k) - n->keys.begin();
}

struct Split {
  bool happened = false;
  uint64_t sep = 0;
  Node* right = nullptr;
};

Split insert_rec(Tree* t, Node* n, uint64_t k, uint64_t v, int* is_new) {
  Split s;
  if (n->leaf) {
    auto it = std::lower_bound(n->keys.begin(), n->keys.end(), k);
    size_t pos = it - n->keys.begin();
    if (it != n->keys.end() && *it == k) {
      n->vals[pos] = v;
      *is_new = 0;
      return s;
    }
    *is_new = 1;
    n->keys.insert(n->keys.begin() + pos, k);
    n->vals.insert(n->vals.begin() + pos, v);
    if (n->keys.size() <= t->max_keys()) return s;
    // split a leaf of F records into F/2 + F/2 ("the target node needs to be split")
    size_t mid = n->keys.size() / 2;
    Node* r = new Node(true);
    r->keys.assign(n->keys.begin() + mid, n->keys.end());
    r->vals.assign(n->vals.begin() + mid, n->vals.end());
    n->keys.resize(mid);
    n->vals.resize(mid);
    r->next = n->next;
    n->next = r;
    s.happened = true;
    s.sep = r->keys[0];
    s.right = r;
    return s;
  }
  size_t i = child_index(n, k);
  Split cs = insert_rec(t, n->child[i], k, v, is_new);
  if (!cs.happened) return s;
  n->keys.insert(n->keys.begin() + i, cs.sep);
  n->child.insert(n->child.begin() + i + 1, cs.right);
  if (n->child.size() <= t->F) return s;
  // split an internal node of F+1 children: left ceil((F+1)/2), right the rest;
  // the separator between them moves up.
  size_t lc = (n->child.size() + 1) / 2;
  Node* r = new Node(false);
  s.happened = true;
  s.sep = n->keys[lc - 1];
  r->keys.assign(n->keys.begin() + lc, n->keys.end());
  r->child.assign(n->child.begin() + lc, n->child.end());
  n->keys.resize(lc - 1);
  n->child.resize(lc);
  s.right = r;
  return s;
}

bool underflow(const Tree* t, const Node* n) {
  return n->leaf ? n->keys.size() < t->min_records() : n->child.size() < t->min_children();
}
bool can_lend(const Tree* t, const Node* n) {
  return n->leaf ? n->keys.size() > t->min_records() : n->child.size() > t->min_children();
}

// repair child i of internal node p after it underflowed (borrow, else merge)
void fix_child(Tree* t, Node* p, size_t i) {
  Node* c = p->child[i];
  Node* L = i > 0 ? p->child[i - 1] : nullptr;
  Node* R = i + 1 < p->child.size() ? p->child[i + 1] : nullptr;
  if (L && can_lend(t, L)) {
    if (c->leaf) {
      c->keys.insert(c->keys.begin(), L->keys.back());
      c->vals.insert(c->vals.begin(), L->vals.back());
      L->keys.pop_back();
      L->vals.pop_back();
      p->keys[i - 1] = c->keys[0];
    } else {
      c->keys.insert(c->keys.begin(), p->keys[i - 1]);
      c->child.insert(c->child.begin(), L->child.back());
      p->keys[i - 1] = L->keys.back();
      L->keys.pop_back();
      L->child.pop_back();
    }
    return;
  }
  if (R && can_lend(t, R)) {
    if (c->leaf) {
      c->keys.push_back(R->keys.front());
      c->vals.push_back(R->vals.front());
      R->keys.erase(R->keys.begin());
      R->vals.erase(R->vals.begin());
      p->keys[i] = R->keys[0];
    } else {
      c->keys.push_back(p->keys[i]);
      c->child.push_back(R->child.front());
      p->keys[i] = R->keys.front();
      R->keys.erase(R->keys.begin());
      R->child.erase(R->child.begin());
    }
    return;
  }
  // merge (the inverse of a split, "delete is the inverse")
  size_t li = L ? i - 1 : i;  // merge child[li+1] into child[li]
  Node* a = p->child[li];
  Node* b = p->child[li + 1];
  if (a->leaf) {
    a->keys.insert(a->keys.end(), b->keys.begin(), b->keys.end());
    a->vals.insert(a->vals.end(), b->vals.begin(), b->vals.end());
    a->next = b->next;
  } else {
    a->keys.push_back(p->keys[li]);
    a->keys.insert(a->keys.end(), b->keys.begin(), b->keys.end());
    a->child.insert(a->child.end(), b->child.begin(), b->child.end());
    b->child.clear();
  }
  p->keys.erase(p->keys.begin() + li);
  p->child.erase(p->child.begin() + li + 1);
  b->leaf = true;  // children already moved; free only the shell
  delete b;
}

int erase_rec(Tree* t, Node* n, uint64_t k) {
  if (n->leaf) {
    auto it = std::lower_bound(n->keys.begin(), n->keys.end(), k);
    if (it == n->keys.end() || *it != k) return 0;
    size_t pos = it - n->keys.begin();
    n->keys.erase(it);
    n->vals.erase(n->vals.begin() + pos);
    return 1;
  }
  size_t i = child_index(n, k);
  int r = erase_rec(t, n->child[i], k);
  if (r && underflow(t, n->child[i])) fix_child(t, n, i);
  return r;
}

const Node* find_leaf(const Tree* t, uint64_t k) {
  const Node* n = t->root;
  while (!n->leaf) n = n->child[child_index(n, k)];
  return n;
}

// structural check: returns 0 or a rule code
//  1 key order, 2 leaf depth, 3 occupancy, 4 separator bounds, 5 leaf chain, 6 size
int check_rec(const Tree* t, const Node* n, int depth, int* leaf_depth, bool is_root,
              bool has_lo, uint64_t lo, bool has_hi, uint64_t hi) {
  for (size_t j = 1; j < n->keys.size(); ++j)
    if (!(n->keys[j - 1] < n->keys[j])) return 1;
  for (uint64_t k : n->keys) {
    if (has_lo && k < lo) return 4;
    if (has_hi && k >= hi) return 4;
  }
  if (n->leaf) {
    if (*leaf_depth < 0) *leaf_depth = depth;
    if (*leaf_depth != depth) return 2;
    if (n->keys.size() > t->max_keys()) return 3;
    if (!is_root && n->keys.size() < t->min_records()) return 3;
    if (n->vals.size() != n->keys.size()) return 3;
    return 0;
  }
  if (n->child.size() != n->keys.size() + 1) return 3;
  if (n->child.size() > t->F) return 3;
  if (is_root ? n->child.size() < 2 : n->child.size() < t->min_children()) return 3;
  for (size_t j = 0; j < n->child.size(); ++j) {
    bool hl = j > 0 ? true : has_lo;
    uint64_t l = j > 0 ? n->keys[j - 1] : lo;
    bool hh = j < n->keys.size() ? true : has_hi;
    uint64_t h = j < n->keys.size() ? n->keys[j] : hi;
    int r = check_rec(t, n->child[j], depth + 1, leaf_depth, false, hl, l, hh, h);
    if (r) return r;
  }
  return 0;
}

}  // namespace

extern "C" void* orc_bpt_create(uint32_t fanout) {
  Tree* t = new Tree;
  t->F = fanout;
  t->root = new Node(true);
  return t;
}

extern "C" void orc_bpt_destroy(void* tp) {
  Tree* t = (Tree*)tp;
  free_node(t->root);
  delete t;
}

extern "C" int orc_bpt_insert(void* tp, uint64_t key, uint64_t value) {
  Tree* t = (Tree*)tp;
  int is_new = 0;
  Split s = insert_rec(t, t->root, key, value, &is_new);
  if (s.happened) {  // grow a new root
    Node* r = new Node(false);
    r->keys.push_back(s.sep);
    r->child.push_back(t->root);
    r->child.push_back(s.right);
    t->root = r;
  }
  t->size += is_new;
  return is_new;
}

extern "C" int orc_bpt_erase(void* tp, uint64_t key) {
  Tree* t = (Tree*)tp;
  int r = erase_rec(t, t->root, key);
  if (!t->root->leaf && t->root->child.size() == 1) {  // shrink the root
    Node* old = t->root;
    t->root = old->child[0];
    old->child.clear();
    old->leaf = true;
    delete old;
  }
  t->size -= r;
  return r;
}

extern "C" void orc_bpt_search(void* tp, const uint64_t* q, uint64_t nq, uint64_t* out) {
  const Tree* t = (const Tree*)tp;
  for (uint64_t j = 0; j < nq; ++j) {
    const Node* n = find_leaf(t, q[j]);
    auto it = std::lower_bound(n->keys.begin(), n->keys.end(), q[j]);
    out[j] = (it != n->keys.end() && *it == q[j]) ? n->vals[it - n->keys.begin()]
                                                    : ORC_NOT_FOUND;
  }
}

// The same search split over nthreads host threads (static chunks; the tree is read-only
// here), for the CPU baseline timing of the paper's pointer B+tree.
extern "C" void orc_bpt_search_mt(void* tp, const uint64_t* q, uint64_t nq, uint64_t* out, int nthreads) {
  if (nthreads <= 0) nthreads = (int)std::max(1u, std::thread::hardware_concurrency());
  if (nthreads == 1 || nq < 4096) {
    orc_bpt_search(tp, q, nq, out);
    return;
  }
  std::vector<std::thread> th;
  const uint64_t chunk = (nq + nthreads - 1) / nthreads;
  for (int i = 0; i < nthreads; ++i) {
    const uint64_t b = std::min<uint64_t>(nq, i * chunk), e = std::min<uint64_t>(nq, b + chunk);
    if (b < e) th.emplace_back([=] { orc_bpt_search(tp, q + b, e - b, out + b); });
  }
  for (auto& x : th) x.join();
}

// n inserts in array order (one orc_bpt_insert each); returns the number of new keys
extern "C" uint64_t orc_bpt_insert_array(void* tp, const uint64_t* keys, const uint64_t* vals, uint64_t n) {
  uint64_t fresh = 0;
  for (uint64_t i = 0; i < n; ++i) fresh += (uint64_t)orc_bpt_insert(tp, keys[i], vals[i]);
  return fresh;
}

extern "C" void orc_bpt_range(void* tp, const uint64_t* lo, const uint64_t* hi, uint64_t nq,
                              uint32_t cap, uint64_t* kout, uint64_t* vout,
                              uint32_t* counts) {
  const Tree* t = (const Tree*)tp;
  for (uint64_t j = 0; j < nq; ++j) {
    uint32_t c = 0;
    if (lo[j] <= hi[j]) {
      // find the first target key with a search, then walk the leaf level
      const Node* n = find_leaf(t, lo[j]);
      size_t pos = std::lower_bound(n->keys.begin(), n->keys.end(), lo[j]) - n->keys.begin();
      while (n) {
        for (; pos < n->keys.size(); ++pos) {
          if (n->keys[pos] > hi[j]) goto done;
          if (c < cap) {
            kout[j * (uint64_t)cap + c] = n->keys[pos];
            vout[j * (uint64_t)cap + c] = n->vals[pos];
          }
          ++c;
        }
        n = n->next;
        pos = 0;
      }
    }
  done:
    counts[j] = c;
  }
}

extern "C" uint64_t orc_bpt_size(void* tp) { return ((Tree*)tp)->size; }

extern "C" uint32_t orc_bpt_height(void* tp) {
  const Node* n = ((Tree*)tp)->root;
  uint32_t h = 1;
  while (!n->leaf) {
    n = n->child[0];
    ++h;
  }
  return h;
}

extern "C" int orc_bpt_check(void* tp) {
  const Tree* t = (const Tree*)tp;
  int leaf_depth = -1;
  int r = check_rec(t, t->root, 0, &leaf_depth, true, false, 0, false, 0);
  if (r) return r;
  // leaf chain: in-order, strictly increasing, total = size
  const Node* n = t->root;
  while (!n->leaf) n = n->child[0];
  uint64_t cnt = 0;
  bool have = false;
  uint64_t prev = 0;
  for (; n; n = n->next) {
    for (uint64_t k : n->keys) {
      if (have && !(prev < k)) return 5;
      prev = k;
      have = true;
      ++cnt;
    }
  }
  return cnt == t->size ? 0 : 6;
}

// Test hook for the checker's own pin: corrupt the tree in one targeted way so that a test
// can assert orc_bpt_check reports the rule it breaks.  Returns 1 if the mutation applied
// (the tree must have height >= 2 and a leaf with >= 2 records for kinds 1-5).
//  1 swap two keys of a leaf (order)        2 underfill a leaf (occupancy)
//  3 move a leaf key outside its separator bounds (bounds)
//  4 break the leaf sibling chain (chain)   5 size counter off by one (size)
//  6 drop a child of an internal node (occupancy: children != keys + 1)
extern "C" int orc_bpt_debug_mutate(void* tp, int kind) {
  Tree* t = (Tree*)tp;
  Node* n = t->root;
  if (n->leaf) return 0;
  Node* parent = n;
  while (!n->leaf) {
    parent = n;
    n = n->child[n->child.size() / 2];
  }
  Node* leaf = n;  // a middle leaf: it has a predecessor and separator bounds on both sides
  if (leaf->keys.size() < 2) return 0;
  switch (kind) {
    case 1:
      std::swap(leaf->keys[0], leaf->keys[1]);
      return 1;
    case 2:  // underfill below ceil((F-1)/2) records (keeps order and bounds)
      if (t->min_records() < 2) return 0;
      leaf->keys.resize(1);
      leaf->vals.resize(1);
      return 1;
    case 3:
      leaf->keys[0] = 0;  // below the separator that routes to this middle leaf
      return leaf->keys[1] > 0 ? 1 : 0;
    case 4: {  // relink leaves 0 -> 2 -> 1 -> 3: every record still reachable, order broken
      Node* l0 = t->root;
      while (!l0->leaf) l0 = l0->child[0];
      Node* l1 = l0->next;
      Node* l2 = l1 ? l1->next : nullptr;
      if (!l2) return 0;
      Node* l3 = l2->next;
      l0->next = l2;
      l2->next = l1;
      l1->next = l3;
      return 1;
    }
    case 5:
      t->size += 1;
      return 1;
    case 6:
      if (parent->child.size() < 2) return 0;
      parent->child.pop_back();
      return 1;
  }
  return 0;
}

extern "C" void orc_bpt_dump(void* tp, uint64_t* keys, uint64_t* vals) {
  const Node* n = ((Tree*)tp)->root;
  while (!n->leaf) n = n->child[0];
  uint64_t i = 0;
  for (; n; n = n->next)
    for (size_t j = 0; j < n->keys.size(); ++j, ++i) {
      keys[i] = n->keys[j];
      vals[i] = n->vals[j];
    }
}

extern "C" void orc_bpt_level_stats(void* tp, uint64_t* nodes, uint64_t* entries,
                                    uint32_t maxlev) {
  const Tree* t = (const Tree*)tp;
  for (uint32_t l = 0; l < maxlev; ++l) nodes[l] = entries[l] = 0;
  std::vector<const Node*> cur{t->root}, nxt;
  for (uint32_t l = 0; l < maxlev && !cur.empty(); ++l) {
    nxt.clear();
    for (const Node* n : cur) {
      nodes[l] += 1;
      entries[l] += n->leaf ? n->keys.size() : n->child.size();
      if (!n->leaf) nxt.insert(nxt.end(), n->child.begin(), n->child.end());
    }
    std::swap(cur, nxt);
  }
}

extern "C" void orc_bpt_quarter_stats(void* tp, const uint64_t* q, uint64_t nq,
                                      uint64_t counts[4]) {
  const Tree* t = (const Tree*)tp;
  for (int i = 0; i < 4; ++i) counts[i] = 0;
  const uint64_t slots = t->F - 1;
  for (uint64_t j = 0; j < nq; ++j) {
    const Node* n = t->root;
    for (;;) {
      // sequential search stops at the first key > q (internal) / >= q (leaf)
      size_t r = n->leaf ? std::lower_bound(n->keys.begin(), n->keys.end(), q[j]) - n->keys.begin()
                         : child_index(n, q[j]);
      size_t p = n->keys.empty() ? 0 : std::min(r, n->keys.size() - 1);
      counts[std::min<uint64_t>(3, (p * 4) / slots)] += 1;
      if (n->leaf) break;
      n = n->child[child_index(n, q[j])];
    }
  }
}

extern "C" void orc_bpt_comparisons(void* tp, const uint64_t* q, uint64_t nq, uint32_t* out) {
  const Tree* t = (const Tree*)tp;
  uint32_t h = orc_bpt_height(tp);
  for (uint64_t j = 0; j < nq; ++j) {
    const Node* n = t->root;
    for (uint32_t l = 0; l < h; ++l) {
      // sequential comparisons: compare keys until one exceeds q (or all are compared)
      uint32_t c = 0;
      for (size_t s = 0; s < n->keys.size(); ++s) {
        ++c;
        if (n->leaf ? n->keys[s] >= q[j] : n->keys[s] > q[j]) break;
      }
      out[j * h + l] = c;
      if (n->leaf) break;
      n = n->child[child_index(n, q[j])];
    }
  }
}
