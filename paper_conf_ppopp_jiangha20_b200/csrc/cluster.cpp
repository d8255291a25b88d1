// Host half of the reorder pipeline: Alg 3 clustering and the
// nnz-balanced panel partition.  The paper runs the clustering on the CPU because it is
// "inherently sequential, but fast"; so do we.
//
// Library design (differs from the oracle's plain heap, same result):
//  * the initial candidates arrive already sorted in heap order (J desc, then (i, j)
//    asc; R10) from the GPU, so the initial heap is a read cursor over that array, walked
//    with software prefetches of the union-find nodes a few pairs ahead;
//  * pairs re-inserted by Alg 3 line 28 with J > 0 go to an 8-ary heap; each pop takes the
//    larger of the cursor head and the heap top under the same total order;
//  * re-inserted pairs with J = 0 (95 % of them on R-MAT) sort after every J > 0 pair, in (i, j)
//    order: they are appended to an array and sorted once when the J > 0 pairs run out, then
//    read as a second cursor beside a small min-heap for J = 0 pairs re-inserted after that;
//  * the exact J of a re-inserted pair (R8) first tests 192-bit column-hash digests of the two
//    representing rows: disjoint digests prove inter = 0 without reading the column lists;
//  * union-find parent, cluster size and the deleted flag share one 8-byte node;
//  * candidate-pair membership (line 27, R9): one open-addressing hash set of the initial and
//    re-inserted pairs; above 2^26 candidates the initial ones are looked up by binary search
//    in the key-sorted pair array (the GPU's dedupe output) instead.
//  SR_DEBUG_CLUSTER=1 prints the phase times.
// Readings R3-R12 decide everything the paper leaves open.
#include <algorithm>
#include <atomic>
#include <thread>
#include <chrono>
#include <cstdio>
#include <cstdlib>
#include <parallel/algorithm>
#include <queue>
#include <cstring>
#include <memory>
#include <numeric>
#include <vector>

#ifdef _OPENMP
#include <omp.h>
#endif

#include "internal.h"

namespace sr {
namespace {

struct Cand {
  uint32_t inter, uni;
  uint32_t i, j;  // i < j
};

// true if a comes before b in heap order (a has higher priority)
inline bool before(const Cand& a, const Cand& b) {
  const uint64_t l = (uint64_t)a.inter * b.uni, r = (uint64_t)b.inter * a.uni;
  if (l != r) return l > r;
  if (a.i != b.i) return a.i < b.i;
  return a.j < b.j;
}

// 8-ary max-heap under `before` (re-inserted pairs, Alg 3 line 28): log8 levels of one or two
// cache lines each instead of log2 levels of one line — the heap can hold millions of pairs.
// Its elements are distinct pairs under a strict total order, so the pop sequence is the same
// as any other priority queue's.
class DHeap {
 public:
  bool empty() const { return v_.empty(); }
  const Cand& top() const { return v_[0]; }
  void push(const Cand& c) {
    size_t i = v_.size();
    v_.push_back(c);
    while (i > 0) {
      const size_t p = (i - 1) / kD;
      if (!before(c, v_[p])) break;
      v_[i] = v_[p];
      i = p;
    }
    v_[i] = c;
  }
  void pop() {
    const Cand last = v_.back();
    v_.pop_back();
    const size_t n = v_.size();
    if (n == 0) return;
    size_t i = 0;
    while (true) {
      const size_t c0 = i * kD + 1;
      if (c0 >= n) break;
      size_t best = c0;
      const size_t ce = std::min(n, c0 + kD);
      for (size_t c = c0 + 1; c < ce; ++c)
        if (before(v_[c], v_[best])) best = c;
      if (!before(v_[best], last)) break;
      v_[i] = v_[best];
      i = best;
    }
    v_[i] = last;
  }

 private:
  static constexpr size_t kD = 8;
  std::vector<Cand> v_;
};

class PairSet {
 public:
  explicit PairSet(size_t expected) {
    size_t cap = 16;
    while (cap < 2 * expected + 16) cap <<= 1;
    reset(cap);
  }
  void prefetch(uint64_t k) const { __builtin_prefetch(&slots_[hash(k) & mask_]); }
  bool contains(uint64_t k) const {  // relaxed atomic loads: may run beside concurrent CAS inserts
    size_t h = hash(k) & mask_;
    while (true) {
      const uint64_t v = __atomic_load_n(&slots_[h], __ATOMIC_RELAXED);
      if (v == k) return true;
      if (v == kEmpty) return false;
      h = (h + 1) & mask_;
    }
  }
  // concurrent insert of keys known to be distinct (initial build, OpenMP): CAS on the slot
  void insert_distinct_concurrent(uint64_t k) {
    size_t h = hash(k) & mask_;
    while (true) {
      uint64_t expected = kEmpty;
      if (__atomic_compare_exchange_n(&slots_[h], &expected, k, false, __ATOMIC_RELAXED, __ATOMIC_RELAXED)) return;
      h = (h + 1) & mask_;
    }
  }
  void set_size(size_t n) { size_ = n; }
  size_t size() const { return size_; }
  // make room for `more` insertions without growing inside a parallel region
  void reserve_more(size_t more) {
    while (2 * (size_ + more + 1) > cap_) grow();
  }
  void insert(uint64_t k) {
    if (2 * (size_ + 1) > cap_) grow();
    size_t h = hash(k) & mask_;
    while (slots_[h] != kEmpty) {
      if (slots_[h] == k) return;
      h = (h + 1) & mask_;
    }
    slots_[h] = k;
    ++size_;
  }

 private:
  static constexpr uint64_t kEmpty = ~0ull;
  static size_t hash(uint64_t k) {
    k ^= k >> 33;
    k *= 0xff51afd7ed558ccdull;
    k ^= k >> 33;
    k *= 0xc4ceb9fe1a85ec53ull;
    k ^= k >> 33;
    return (size_t)k;
  }
  void reset(size_t cap) {  // uninitialised allocation + parallel first-touch fill
    slots_.reset(new uint64_t[cap]);
    cap_ = cap;
    mask_ = cap - 1;
    uint64_t* sl = slots_.get();
#pragma omp parallel for schedule(static)
    for (int64_t k = 0; k < (int64_t)cap; ++k) sl[k] = kEmpty;
  }
  void grow() {
    std::unique_ptr<uint64_t[]> old = std::move(slots_);
    const size_t ocap = cap_;
    reset(2 * ocap);
    size_ = 0;
    for (size_t k = 0; k < ocap; ++k)
      if (old[k] != kEmpty) insert(old[k]);
  }
  std::unique_ptr<uint64_t[]> slots_;
  size_t cap_ = 0, mask_ = 0, size_ = 0;
};

// Keys inserted since the last flush into the big membership set (L2-resident, cleared through
// its list of used slots).
class SmallSet {
 public:
  SmallSet() : slots_(kCap, kEmpty) {}
  bool contains(uint64_t k) const {
    size_t h = mix(k);
    while (true) {
      const uint64_t v = slots_[h];
      if (v == k) return true;
      if (v == kEmpty) return false;
      h = (h + 1) & (kCap - 1);
    }
  }
  void insert(uint64_t k) {
    size_t h = mix(k);
    while (slots_[h] != kEmpty) {
      if (slots_[h] == k) return;
      h = (h + 1) & (kCap - 1);
    }
    slots_[h] = k;
    used_.push_back((uint32_t)h);
    keys_.push_back(k);
  }
  bool nearly_full() const { return used_.size() * 2 > kCap; }
  const std::vector<uint64_t>& keys() const { return keys_; }
  void clear() {
    for (uint32_t h : used_) slots_[h] = kEmpty;
    used_.clear();
    keys_.clear();
  }

 private:
  static constexpr size_t kCap = 1 << 16;
  static constexpr uint64_t kEmpty = ~0ull;
  static size_t mix(uint64_t k) { return (size_t)((k * 0x9E3779B97F4A7C15ull) >> 48) & (kCap - 1); }
  std::vector<uint64_t> slots_;
  std::vector<uint32_t> used_;
  std::vector<uint64_t> keys_;
};

inline void intersect(const int64_t* rowptr, const int32_t* col, int64_t a, int64_t b,
                      uint32_t* inter, uint32_t* uni) {
  const int32_t *p = col + rowptr[a], *pe = col + rowptr[a + 1];
  const int32_t *q = col + rowptr[b], *qe = col + rowptr[b + 1];
  int64_t na = pe - p, nb = qe - q;
  int64_t n = 0;
  if (na > nb) {
    std::swap(p, q);
    std::swap(pe, qe);
  }
  if ((qe - q) >= 16 * (pe - p)) {  // skewed sizes (hub rows): binary-search the short list's
    for (; p < pe && q < qe; ++p) {  // columns in the long one, O(short · log long)
      q = std::lower_bound(q, qe, *p);
      if (q < qe && *q == *p) ++n, ++q;
    }
    *inter = (uint32_t)n;
    *uni = (uint32_t)(na + nb - n);
    return;
  }
  while (p < pe && q < qe) {
    const int32_t x = *p, y = *q;
    n += (x == y);
    p += (x <= y);
    q += (y <= x);
  }
  *inter = (uint32_t)n;
  *uni = (uint32_t)(na + nb - n);
}

// Per-row digest for exact J = 0 detection without touching the column lists: a 192-bit mask
// of hashed columns and the row length.  Disjoint masks prove that two rows share no column
// (inter = 0, uni = |S_i| + |S_j|, exactly); overlapping masks fall back to the merge.  On R-MAT
// (C2) 95 % of Alg 3's re-inserted pairs have J = 0.
struct __align__(32) RowDigest {
  uint64_t m[3];
  uint32_t len, pad;
};
inline void digest_bit(uint32_t c, uint32_t* w, uint32_t* bit) {
  const uint32_t h = c * 0x9E3779B1u;
  *w = (h >> 8) % 3;
  *bit = h >> 26;
}

// Union-find node: parent and cluster size; bit 31 of the size marks a deleted (frozen) cluster.
struct Node {
  int32_t parent;
  uint32_t sz;
};
constexpr uint32_t kDeleted = 1u << 31;

}  // namespace

void cluster_rows(int64_t M, const int64_t* rowptr, const int32_t* col, int64_t npairs,
                  const uint64_t* pairs, const uint32_t* inter, const uint32_t* uni,
                  int32_t threshold_size, int32_t* perm, const uint64_t* pairs_by_key) {
  const bool dbg = getenv("SR_DEBUG_CLUSTER") != nullptr;
  auto now = [] { return std::chrono::duration<double>(std::chrono::steady_clock::now().time_since_epoch()).count(); };
  double t0 = now();
  // initial candidates in heap order; the heap order is a strict total order (R10), so any
  // sort gives the same array
  std::unique_ptr<Cand[]> init_buf(new Cand[(size_t)npairs]);  // filled below (no zeroing pass)
  Cand* const init = init_buf.get();
  // membership (line 27, R9): one open-addressing hash set of the initial candidates and the
  // re-inserted pairs (one cache miss per lookup); above 2^26 candidates the initial ones are
  // found by binary search in the key-sorted pair array instead (memory), if the caller has it
  const bool by_key = pairs_by_key != nullptr && npairs > (int64_t(1) << 26);
  PairSet members(by_key ? (size_t)npairs / 4 + 16 : (size_t)npairs + (size_t)npairs / 4);
  std::vector<int64_t> seg(by_key ? (size_t)M + 1 : 0);
  if (by_key) {
#pragma omp parallel for schedule(static)
    for (int64_t r = 0; r <= M; ++r)
      seg[r] = std::lower_bound(pairs_by_key, pairs_by_key + npairs, (uint64_t)r << 32) - pairs_by_key;
  }
  SmallSet recent;  // re-inserted pairs not yet flushed into `members` (see flush_recent)
  auto is_candidate_big = [&](uint64_t key) {
    if (by_key) {
      const int64_t lo = (int64_t)(key >> 32);
      if (std::binary_search(pairs_by_key + seg[lo], pairs_by_key + seg[lo + 1], key)) return true;
    }
    return members.contains(key);
  };
  auto is_candidate = [&](uint64_t key) { return recent.contains(key) || is_candidate_big(key); };
  // move the recent re-inserts into the big set (distinct keys, absent from it: parallel CAS)
  auto flush_recent = [&]() {
    const std::vector<uint64_t>& ks = recent.keys();
    if (ks.empty()) return;
    members.reserve_more(ks.size());
#pragma omp parallel for schedule(static) if (ks.size() > 4096)
    for (int64_t k = 0; k < (int64_t)ks.size(); ++k) members.insert_distinct_concurrent(ks[k]);
    members.set_size(members.size() + ks.size());
    recent.clear();
  };
  const double ta = now();
  std::vector<RowDigest> dig((size_t)M);
#pragma omp parallel for schedule(dynamic, 4096)
  for (int64_t r = 0; r < M; ++r) {
    RowDigest d{};
    d.len = (uint32_t)(rowptr[r + 1] - rowptr[r]);
    for (int64_t e = rowptr[r]; e < rowptr[r + 1]; ++e) {
      uint32_t w, bit;
      digest_bit((uint32_t)col[e], &w, &bit);
      d.m[w] |= 1ull << bit;
    }
    dig[r] = d;
  }
  const double tb = now();
#pragma omp parallel for schedule(static)
  for (int64_t e = 0; e < npairs; ++e) {
    Cand c;
    c.i = (uint32_t)(pairs[e] >> 32);
    c.j = (uint32_t)(pairs[e] & 0xFFFFFFFFu);
    if (inter) {
      c.inter = inter[e];
      c.uni = uni[e];
    } else {
      intersect(rowptr, col, c.i, c.j, &c.inter, &c.uni);
    }
    if (c.uni == 0) c.uni = 1;  // J(empty, empty) := 0/1 (R16)
    init[e] = c;
    if (!by_key) members.insert_distinct_concurrent(pairs[e]);
  }
  if (!by_key) members.set_size((size_t)npairs);
  bool sorted = true;
  for (int64_t e = 1; e < npairs && sorted; ++e) sorted = !before(init[e], init[e - 1]);
  const double t1 = now();
  if (!sorted) __gnu_parallel::sort(init, init + npairs, before);
  const double t2 = now();
  int64_t n_reinsert = 0, n_zero = 0;

  std::vector<Node> nd((size_t)M);
  for (int64_t x = 0; x < M; ++x) nd[x] = Node{(int32_t)x, 1u};
  // The union-find nodes are written only by the thread running Alg 3; the pipelined speculative
  // pass reads them concurrently, so the writes are relaxed atomic stores (plain moves on x86).
  auto set_parent = [&](int32_t x, int32_t v) { __atomic_store_n(&nd[x].parent, v, __ATOMIC_RELAXED); };
  auto set_size = [&](int32_t x, uint32_t v) { __atomic_store_n(&nd[x].sz, v, __ATOMIC_RELAXED); };
  auto root = [&](int32_t x) {  // path halving
    while (x != nd[x].parent) {
      set_parent(x, nd[nd[x].parent].parent);
      x = nd[x].parent;
    }
    return x;
  };
  // Exact J of the representing rows of a re-inserted pair (R8), with the digest early-out.
  auto similarity = [&](uint32_t lo, uint32_t hi, Cand* c) {
    const RowDigest &a = dig[lo], &b = dig[hi];
    c->i = lo;
    c->j = hi;
    if (((a.m[0] & b.m[0]) | (a.m[1] & b.m[1]) | (a.m[2] & b.m[2])) == 0) {
      c->inter = 0;
      c->uni = a.len + b.len;
    } else {
      intersect(rowptr, col, lo, hi, &c->inter, &c->uni);
    }
    if (c->uni == 0) c->uni = 1;
  };
  // Priority structure (R10 total order: J desc, then (i, j) asc), in three parts that pop in
  // exactly that order:
  //  * J > 0: the initial candidates as a sorted cursor (all have J > 0: an LSH candidate shares
  //    a band key, hence a column) and an 8-ary heap of re-inserted pairs with J > 0;
  //  * J = 0 (re-inserted pairs only), which pop after every J > 0 pair in (i, j) order: appended
  //    to a plain array while J > 0 pairs remain, sorted once, then read as a cursor together with
  //    a min-heap of the J = 0 pairs re-inserted after that point.
  DHeap extra;
  std::vector<uint64_t> zero_keys;
  std::priority_queue<uint64_t, std::vector<uint64_t>, std::greater<uint64_t>> zero_new;
  bool zero_phase = false;
  // initial candidates with J = 0 (never produced by the LSH, whose pairs share a column, but
  // a caller of sr_host_cluster may pass them) sort to the end of `init` and join the J = 0 part
  size_t init_pos = (size_t)npairs;
  while (init_pos > 0 && init[init_pos - 1].inter == 0) --init_pos;
  size_t cur = 0, zc = 0;
  int64_t nclusters = M;
  // roots changed by a merge since the current block's speculative evaluation: a 2^16-bit
  // filter (false positives only send a pop down the sequential path)
  uint64_t modbits[1024];
  auto mod_bit = [](int32_t x) { return (uint32_t)((uint32_t)x * 0x9E3779B1u) >> 16; };
  auto mark_mod = [&](int32_t x) { const uint32_t b = mod_bit(x); modbits[b >> 6] |= 1ull << (b & 63); };
  auto is_mod = [&](int32_t x) { const uint32_t b = mod_bit(x); return (modbits[b >> 6] >> (b & 63)) & 1ull; };
  std::memset(modbits, 0, sizeof(modbits));
  bool midflush = false;  // `recent` was flushed since the current block's evaluation
  auto reinsert = [&](const Cand& c, uint64_t key) {
    if (recent.nearly_full()) {
      flush_recent();
      midflush = true;
    }
    recent.insert(key);
    ++n_reinsert;
    if (c.inter > 0) {
      extra.push(c);
    } else {
      ++n_zero;
      if (zero_phase)
        zero_new.push(key);
      else
        zero_keys.push_back(key);
    }
  };
  // One popped pair, exactly as Alg 3 (lines 17-30 under R3-R12): the sequential path.
  auto process = [&](int32_t i, int32_t j) {
    if (nd[i].parent == i && nd[j].parent == j) {
      if ((nd[i].sz | nd[j].sz) & kDeleted) return;
      // the larger cluster absorbs the smaller; equal sizes: smaller index (R6)
      const bool i_wins = nd[i].sz > nd[j].sz || (nd[i].sz == nd[j].sz && i < j);
      const int32_t w = i_wins ? i : j, l = i_wins ? j : i;
      set_parent(l, w);
      set_size(w, nd[w].sz + nd[l].sz);  // R4
      --nclusters;
      if (nd[w].sz >= (uint32_t)threshold_size) {  // R7, R5
        set_size(w, nd[w].sz | kDeleted);
        --nclusters;
      }
      mark_mod(w);
      mark_mod(l);
    } else {
      i = root(i);
      j = root(j);
      if (((nd[i].sz | nd[j].sz) & kDeleted) || i == j) return;
      const uint32_t lo = (uint32_t)std::min(i, j), hi = (uint32_t)std::max(i, j);
      const uint64_t key = ((uint64_t)lo << 32) | hi;
      if (is_candidate(key)) return;
      Cand c;
      similarity(lo, hi, &c);  // representing rows (R8)
      reinsert(c, key);
    }
  };
  // Speculative evaluation of the initial-candidate cursor in blocks (parallel, read-only):
  // against the union-find state at the block's start, each pop is classified as
  //   0 both rows are roots -> merge path, done sequentially at its turn;
  //   1 the roots are equal or one is deleted -> skip (both facts are permanent: a deleted root
  //     never merges again and equal roots stay equal), valid whatever happens in between;
  //   2 the roots' pair is a candidate -> skip, valid if neither root changed since;
  //   3 not a candidate -> re-insert with the exact J computed here (the expensive part), valid
  //     if neither root changed since and no earlier pop of the block re-inserted the same pair.
  // The pops then run in the exact sequential order (interleaved with the re-insert heap); a
  // pop whose class 2/3 result may be stale (a root merged since, modbits) takes the
  // sequential path.  The result is identical to the plain loop.
  const bool spec = getenv("SR_CLUSTER_SEQ") == nullptr;
  struct Pre {
    int32_t ri, rj;
    uint32_t inter, uni;
    int32_t cls;
  };
  static const size_t BS = [] {  // block size of the speculative pass (SR_CLUSTER_BS, measurement knob)
    const char* e = getenv("SR_CLUSTER_BS");
    const long v = e ? atol(e) : 8192;
    return (size_t)(v < 64 ? 64 : v);
  }();
  std::vector<Pre> pre(BS);
  size_t blk0 = 0, blk1 = 0;
  int64_t n_spec_used = 0;
  auto find_ro = [&](int32_t x) {  // read-only root walk
    while (nd[x].parent != x) x = nd[x].parent;
    return x;
  };
  double t_eval = 0.0;
  auto evaluate_block = [&](size_t from) {
    const double te = dbg ? now() : 0.0;
    flush_recent();  // the speculative pass reads `members` only
    midflush = false;
    blk0 = from;
    blk1 = std::min(init_pos, from + BS);
    std::memset(modbits, 0, sizeof(modbits));
#pragma omp parallel for schedule(static, 64)
    for (int64_t k = (int64_t)blk0; k < (int64_t)blk1; ++k) {
      Pre& p = pre[(size_t)k - blk0];
      const int32_t i = (int32_t)init[k].i, j = (int32_t)init[k].j;
      if (nd[i].parent == i && nd[j].parent == j) {
        p.cls = 0;
        continue;
      }
      const int32_t ri = find_ro(i), rj = find_ro(j);
      p.ri = ri;
      p.rj = rj;
      if (((nd[ri].sz | nd[rj].sz) & kDeleted) || ri == rj) {
        p.cls = 1;
        continue;
      }
      const uint32_t lo = (uint32_t)std::min(ri, rj), hi = (uint32_t)std::max(ri, rj);
      if (is_candidate_big(((uint64_t)lo << 32) | hi)) {
        p.cls = 2;
        continue;
      }
      Cand c;
      similarity(lo, hi, &c);
      p.inter = c.inter;
      p.uni = c.uni;
      p.cls = 3;
    }
    if (dbg) t_eval += now() - te;
  };
  // ---- Pipelined variant of the speculative pass (the default with >= 3 OpenMP threads): the
  // evaluation of block b+1 runs on the other threads while this thread replays block b, so the
  // replay (the sequential part) is the phase's critical path.  The evaluators read the union-find
  // nodes while the replay writes them (relaxed atomics), so a block's results are checked against
  // every merge since its evaluation began (the merged-root filters of the current and the previous
  // block); skips because of equal or deleted roots stay valid under any interleaving (both facts
  // are permanent, and an observed parent chain only ever leads to an ancestor).  Re-inserted pairs
  // go to small per-block sets; the keys of block b-1 are added to the big set by the evaluators of
  // block b+1 before they evaluate it, so a block's "not a candidate" results are re-checked against
  // the sets of the previous and the current block only.
  int nthr = 1;
#ifdef _OPENMP
  nthr = std::min(omp_get_max_threads(), 16);
#endif
  if (spec && nthr >= 3 && init_pos > 0 && getenv("SR_CLUSTER_NOPIPE") == nullptr) {
    const int64_t nblocks = (int64_t)((init_pos + BS - 1) / BS);
    std::vector<Pre> ring[2] = {std::vector<Pre>(BS), std::vector<Pre>(BS)};
    constexpr size_t kNodeAhead = 24;
    // per 64 pops of a block: bit t set unless pop t was classified 1 (equal or deleted roots: a
    // permanent skip), so the replay jumps over those pops without reading their records
    std::vector<uint64_t> live[2] = {std::vector<uint64_t>(BS / 64 + 1), std::vector<uint64_t>(BS / 64 + 1)};
    SmallSet kset[2];  // keys re-inserted while replaying the previous / the current block
    int kprev = 0, kcur = 1;
    uint64_t fbits[2][1024];
    std::memset(fbits, 0, sizeof(fbits));
    int fprev = 0, fcur = 1;
    auto fmark = [&](int32_t x) { const uint32_t b = mod_bit(x); fbits[fcur][b >> 6] |= 1ull << (b & 63); };
    auto fmod = [&](int32_t x) {
      const uint32_t b = mod_bit(x);
      return ((fbits[fprev][b >> 6] | fbits[fcur][b >> 6]) >> (b & 63)) & 1ull;
    };
    bool overflow = false;  // a block's key set was flushed early: re-check class 3 against `members`
    // work cursors tagged with their request (request << 40 | position): a thread still looking
    // at an earlier request can never claim work of a newer one, so no request waits for
    // stragglers; a request is issued only after the previous one completed (all its claimed
    // chunks counted)
    constexpr int kTag = 40;
    constexpr uint64_t kPos = (1ull << kTag) - 1;
    std::atomic<int64_t> req{-1}, ready{-1};
    std::atomic<uint64_t> flush_cur{0}, eval_cur{0};
    std::atomic<int64_t> flush_done{0}, eval_done{0};
    std::atomic<bool> stop{false};
    auto claim = [&](std::atomic<uint64_t>& c, int64_t r, int64_t len, int64_t step, int64_t* k) {
      uint64_t v = c.load(std::memory_order_acquire);
      while (true) {
        if ((int64_t)(v >> kTag) != r || (int64_t)(v & kPos) >= len) return false;
        if (c.compare_exchange_weak(v, v + (uint64_t)step, std::memory_order_acq_rel, std::memory_order_acquire)) {
          *k = (int64_t)(v & kPos);
          return true;
        }
      }
    };
    const uint64_t* flush_keys = nullptr;
    int64_t flush_n = 0, eval_b0 = 0, eval_len = 0;
    Pre* eval_out = nullptr;
    uint64_t* live_out = nullptr;
    // spin (the phase lasts about a second; yielding measured slower, r02l)
    auto pause = [] { __builtin_ia32_pause(); };
    std::atomic<int> team{0};
    auto cand_pipe = [&](uint64_t key) {
      return kset[kcur].contains(key) || kset[kprev].contains(key) || is_candidate_big(key);
    };
    // replay-side versions of process()/reinsert() that use the per-block key sets and filters
    auto reinsert_pipe = [&](const Cand& c, uint64_t key) {
      if (kset[kcur].nearly_full()) {  // rare: flush it here (CAS inserts; the big set was reserved)
        for (uint64_t k : kset[kcur].keys()) members.insert_distinct_concurrent(k);
        members.set_size(members.size() + kset[kcur].keys().size());
        kset[kcur].clear();
        overflow = true;
      }
      kset[kcur].insert(key);
      ++n_reinsert;
      if (c.inter > 0) {
        extra.push(c);
      } else {
        ++n_zero;
        zero_keys.push_back(key);
      }
    };
    auto process_pipe = [&](int32_t i, int32_t j) {
      if (nd[i].parent == i && nd[j].parent == j) {
        if ((nd[i].sz | nd[j].sz) & kDeleted) return;
        const bool i_wins = nd[i].sz > nd[j].sz || (nd[i].sz == nd[j].sz && i < j);
        const int32_t w = i_wins ? i : j, l = i_wins ? j : i;
        set_parent(l, w);
        set_size(w, nd[w].sz + nd[l].sz);  // R4
        --nclusters;
        if (nd[w].sz >= (uint32_t)threshold_size) {  // R7, R5
          set_size(w, nd[w].sz | kDeleted);
          --nclusters;
        }
        fmark(w);
        fmark(l);
      } else {
        i = root(i);
        j = root(j);
        if (((nd[i].sz | nd[j].sz) & kDeleted) || i == j) return;
        const uint32_t lo = (uint32_t)std::min(i, j), hi = (uint32_t)std::max(i, j);
        const uint64_t key = ((uint64_t)lo << 32) | hi;
        if (cand_pipe(key)) return;
        Cand c;
        similarity(lo, hi, &c);  // representing rows (R8)
        reinsert_pipe(c, key);
      }
    };
    auto evaluate_one = [&](int64_t k, Pre& p) {  // (declared before its use in evaluate_chunk)
      const int32_t i = (int32_t)init[k].i, j = (int32_t)init[k].j;
      const int32_t pi = __atomic_load_n(&nd[i].parent, __ATOMIC_RELAXED);
      const int32_t pj = __atomic_load_n(&nd[j].parent, __ATOMIC_RELAXED);
      if (pi == i && pj == j) {
        p.cls = 0;
        return;
      }
      int32_t ri = i, rj = j;
      for (int32_t q; (q = __atomic_load_n(&nd[ri].parent, __ATOMIC_RELAXED)) != ri;) ri = q;
      for (int32_t q; (q = __atomic_load_n(&nd[rj].parent, __ATOMIC_RELAXED)) != rj;) rj = q;
      p.ri = ri;
      p.rj = rj;
      const uint32_t si = __atomic_load_n(&nd[ri].sz, __ATOMIC_RELAXED);
      const uint32_t sj = __atomic_load_n(&nd[rj].sz, __ATOMIC_RELAXED);
      if (((si | sj) & kDeleted) || ri == rj) {
        p.cls = 1;
        return;
      }
      const uint32_t lo = (uint32_t)std::min(ri, rj), hi = (uint32_t)std::max(ri, rj);
      if (is_candidate_big(((uint64_t)lo << 32) | hi)) {
        p.cls = 2;
        return;
      }
      Cand c;
      similarity(lo, hi, &c);
      p.inter = c.inter;
      p.uni = c.uni;
      p.cls = 3;
    };
    // pops [k, e) of the current evaluation request, k a multiple of 64 (one live word)
    auto evaluate_chunk = [&](int64_t k, int64_t e) {
      uint64_t m = 0;
      for (int64_t t = k; t < e; ++t) {
        evaluate_one(eval_b0 + t, eval_out[t]);
        if (eval_out[t].cls != 1) m |= 1ull << (t - k);
      }
      live_out[k >> 6] = m;
    };
    // publish the next evaluation (the evaluators are idle: the previous one has completed)
    auto request = [&](int64_t b, const std::vector<uint64_t>* keys) {
      flush_n = keys ? (int64_t)keys->size() : 0;
      members.reserve_more((size_t)flush_n + (size_t)BS * 4 + 65536);
      members.set_size(members.size() + (size_t)flush_n);
      flush_keys = keys ? keys->data() : nullptr;
      eval_b0 = b * (int64_t)BS;
      eval_len = std::min<int64_t>((int64_t)init_pos, eval_b0 + (int64_t)BS) - eval_b0;
      eval_out = ring[b & 1].data();
      live_out = live[b & 1].data();
      flush_done.store(0, std::memory_order_relaxed);
      eval_done.store(0, std::memory_order_relaxed);
      flush_cur.store((uint64_t)b << kTag, std::memory_order_release);
      eval_cur.store((uint64_t)b << kTag, std::memory_order_release);
      req.store(b, std::memory_order_release);
    };
    auto wait_ready = [&](int64_t b) {
      const double te = dbg ? now() : 0.0;
      if (team.load(std::memory_order_relaxed) < 2) {  // the runtime gave no evaluator thread
        for (int64_t t = 0; t < flush_n; ++t) members.insert_distinct_concurrent(flush_keys[t]);
        for (int64_t t = 0; t < eval_len; t += 64) evaluate_chunk(t, std::min<int64_t>(eval_len, t + 64));
        ready.store(b, std::memory_order_release);
      }
      while (ready.load(std::memory_order_acquire) != b) pause();
      if (dbg) t_eval += now() - te;  // time the replay waited for the evaluators
    };
#pragma omp parallel num_threads(nthr)
    {
      if (omp_get_thread_num() == 0) team.store(omp_get_num_threads(), std::memory_order_release);
      if (omp_get_thread_num() != 0) {  // evaluators
        int64_t seen = -1;
        while (true) {
          int64_t r;
          while ((r = req.load(std::memory_order_acquire)) == seen && !stop.load(std::memory_order_acquire)) pause();
          if (r == seen) break;
          seen = r;
          int64_t k;
          while (claim(flush_cur, r, flush_n, 512, &k)) {
            const int64_t e = std::min(flush_n, k + 512);
            for (int64_t t = k; t < e; ++t) members.insert_distinct_concurrent(flush_keys[t]);
            flush_done.fetch_add(e - k, std::memory_order_release);
          }
          // every flush chunk of this request is in before any of its evaluation reads `members`
          while (req.load(std::memory_order_acquire) == r && flush_done.load(std::memory_order_acquire) < flush_n)
            pause();
          while (claim(eval_cur, r, eval_len, 64, &k)) {
            const int64_t e = std::min(eval_len, k + 64);
            evaluate_chunk(k, e);
            if (eval_done.fetch_add(e - k, std::memory_order_acq_rel) + (e - k) == eval_len)
              ready.store(r, std::memory_order_release);
          }
        }
      } else {  // the replay, in the exact order of Alg 3
        request(0, nullptr);
        for (int64_t b = 0; b < nblocks && nclusters > 0; ++b) {
          wait_ready(b);
          if (b > 0) {  // rotate: the previous block's keys / merges become "previous"
            kset[kprev].clear();
            std::swap(kprev, kcur);
            std::memset(fbits[fprev], 0, sizeof(fbits[fprev]));
            std::swap(fprev, fcur);
          }
          const bool overflow_prev = overflow;
          overflow = false;
          if (b + 1 < nblocks) request(b + 1, b > 0 ? &kset[kprev].keys() : nullptr);
          const Pre* pr = ring[b & 1].data();
          const uint64_t* lv = live[b & 1].data();
          const size_t b0 = (size_t)b * BS, b1 = std::min(init_pos, b0 + BS);
          for (size_t c = b0; c < b1 && nclusters > 0;) {
            {  // jump over permanently skipped pops (class 1): no effect, whatever pops between
              const size_t t = c - b0;
              const uint64_t m = lv[t >> 6] >> (t & 63);
              if (m == 0) {
                const size_t nxt = b0 + ((t >> 6) + 1) * 64;
                n_spec_used += (int64_t)(std::min(nxt, b1) - c);
                c = nxt;
                continue;
              }
              const size_t z = (size_t)__builtin_ctzll(m);
              n_spec_used += (int64_t)z;
              c += z;
              if (c + kNodeAhead < b1) {  // the union-find nodes a pop a little ahead reads first
                __builtin_prefetch(&nd[init[c + kNodeAhead].i]);
                __builtin_prefetch(&nd[init[c + kNodeAhead].j]);
              }
            }
            if (!extra.empty() && !before(init[c], extra.top())) {  // a re-inserted pair pops first
              const int32_t i = (int32_t)extra.top().i, j = (int32_t)extra.top().j;
              extra.pop();
              process_pipe(i, j);
              continue;
            }
            const Pre& p = pr[c - b0];
            const int32_t i = (int32_t)init[c].i, j = (int32_t)init[c].j;
            ++c;
            if (p.cls == 1) {
              ++n_spec_used;
              continue;
            }
            if ((p.cls == 2 || p.cls == 3) && !fmod(p.ri) && !fmod(p.rj)) {
              ++n_spec_used;
              if (p.cls == 2) continue;
              const uint32_t lo = (uint32_t)std::min(p.ri, p.rj), hi = (uint32_t)std::max(p.ri, p.rj);
              const uint64_t key = ((uint64_t)lo << 32) | hi;
              if (kset[kcur].contains(key) || kset[kprev].contains(key) ||
                  ((overflow || overflow_prev) && members.contains(key)))
                continue;  // re-inserted since this block's evaluation began
              Cand cc;
              cc.i = lo;
              cc.j = hi;
              cc.inter = p.inter;
              cc.uni = p.uni;
              reinsert_pipe(cc, key);
              continue;
            }
            process_pipe(i, j);
          }
        }
        // the cursor is done: the remaining re-inserted pairs with J > 0
        while (!extra.empty() && nclusters > 0) {
          const int32_t i = (int32_t)extra.top().i, j = (int32_t)extra.top().j;
          extra.pop();
          process_pipe(i, j);
        }
        stop.store(true, std::memory_order_release);
      }
    }
    // hand the remaining key sets to the sequential structures of the J = 0 phase
    for (int k = 0; k < 2; ++k) {
      members.reserve_more(kset[k].keys().size());
      for (uint64_t key : kset[k].keys()) members.insert(key);
      kset[k].clear();
    }
    cur = init_pos;
    blk0 = blk1 = init_pos;
  }
  constexpr size_t PF = 32, PF2 = 16, PF3 = 8;  // prefetch distances (sequential mode)
  while (nclusters > 0) {
    int32_t i, j;
    if (!zero_phase) {
      if (cur < init_pos && (extra.empty() || before(init[cur], extra.top()))) {
        i = (int32_t)init[cur].i;
        j = (int32_t)init[cur].j;
        if (spec) {
          if (cur >= blk1) evaluate_block(cur);
          if (cur + PF < blk1 && pre[cur + PF - blk0].cls == 0) {  // merge-path pops read both nodes
            __builtin_prefetch(&nd[init[cur + PF].i]);
            __builtin_prefetch(&nd[init[cur + PF].j]);
          }
          const Pre& p = pre[cur - blk0];
          ++cur;
          if (p.cls == 1) {
            ++n_spec_used;
            continue;
          }
          if ((p.cls == 2 || p.cls == 3) && !is_mod(p.ri) && !is_mod(p.rj)) {
            ++n_spec_used;
            if (p.cls == 2) continue;
            const uint32_t lo = (uint32_t)std::min(p.ri, p.rj), hi = (uint32_t)std::max(p.ri, p.rj);
            const uint64_t key = ((uint64_t)lo << 32) | hi;
            // re-inserted by an earlier pop of this block?
            if (recent.contains(key) || (midflush && members.contains(key))) continue;
            Cand c;
            c.i = lo;
            c.j = hi;
            c.inter = p.inter;
            c.uni = p.uni;
            reinsert(c, key);
            continue;
          }
          process(i, j);
          continue;
        }
        if (cur + PF < init_pos) {
          __builtin_prefetch(&nd[init[cur + PF].i]);
          __builtin_prefetch(&nd[init[cur + PF].j]);
        }
        if (cur + PF2 < init_pos) {  // second level: the (likely) roots of a nearer pair
          __builtin_prefetch(&nd[nd[init[cur + PF2].i].parent]);
          __builtin_prefetch(&nd[nd[init[cur + PF2].j].parent]);
        }
        if (cur + PF3 < init_pos) {
          // third level: a nearer pair's likely roots (read-only walk, merges are rare between
          // here and its pop), whose membership slot and digests the else branch will read
          int32_t a = (int32_t)init[cur + PF3].i, b = (int32_t)init[cur + PF3].j;
          if (nd[a].parent != a || nd[b].parent != b) {
            for (int k = 0; k < 4 && nd[a].parent != a; ++k) a = nd[a].parent;
            for (int k = 0; k < 4 && nd[b].parent != b; ++k) b = nd[b].parent;
            if (a != b) {
              const uint64_t key = ((uint64_t)std::min(a, b) << 32) | (uint64_t)std::max(a, b);
              if (!by_key) members.prefetch(key);
              __builtin_prefetch(&dig[a]);
              __builtin_prefetch(&dig[b]);
            }
          }
        }
        ++cur;
      } else if (!extra.empty()) {
        i = (int32_t)extra.top().i;
        j = (int32_t)extra.top().j;
        extra.pop();
      } else {
        zero_phase = true;
        if (dbg)
          fprintf(stderr, "  J>0 phase %.3f s (speculative blocks %.3f s), %lld clusters left, %zu J=0 pairs, %lld speculative results used\n",
                  now() - t2, t_eval, (long long)nclusters, zero_keys.size(), (long long)n_spec_used);
        for (size_t e = init_pos; e < (size_t)npairs; ++e) zero_keys.push_back(((uint64_t)init[e].i << 32) | init[e].j);
        __gnu_parallel::sort(zero_keys.begin(), zero_keys.end());
        continue;
      }
    } else {
      uint64_t key;
      if (!extra.empty()) {  // a J > 0 pair re-inserted during the J = 0 phase pops first
        i = (int32_t)extra.top().i;
        j = (int32_t)extra.top().j;
        extra.pop();
      } else {
        if (zc < zero_keys.size() && (zero_new.empty() || zero_keys[zc] < zero_new.top())) {
          if (zc + PF < zero_keys.size()) {  // the nodes (and their likely roots) of pops ahead
            __builtin_prefetch(&nd[(int32_t)(zero_keys[zc + PF] >> 32)]);
            __builtin_prefetch(&nd[(int32_t)(zero_keys[zc + PF] & 0xFFFFFFFFu)]);
          }
          if (zc + PF2 < zero_keys.size()) {
            __builtin_prefetch(&nd[nd[(int32_t)(zero_keys[zc + PF2] >> 32)].parent]);
            __builtin_prefetch(&nd[nd[(int32_t)(zero_keys[zc + PF2] & 0xFFFFFFFFu)].parent]);
          }
          key = zero_keys[zc++];
        } else if (!zero_new.empty()) {
          key = zero_new.top();
          zero_new.pop();
        } else {
          break;  // every structure is empty
        }
        i = (int32_t)(key >> 32);
        j = (int32_t)(key & 0xFFFFFFFFu);
      }
    }
    process(i, j);
  }
  if (dbg)
    fprintf(stderr, "cluster_rows: set %.3f s, digests %.3f s, build %.3f s, sort %.3f s (sorted=%d), loop %.3f s, %lld re-inserted (%lld with J = 0)\n",
            ta - t0, tb - ta, t1 - tb, t2 - t1, (int)sorted, now() - t2, (long long)n_reinsert, (long long)n_zero);
  // rule B (R11): clusters of >= 2 rows by ascending root, then singletons ascending
  std::vector<int32_t> r_of((size_t)M);
  std::vector<int64_t> count((size_t)M + 1, 0);
  for (int64_t x = 0; x < M; ++x) {
    r_of[x] = root((int32_t)x);
    ++count[r_of[x]];
  }
  // offsets: cluster roots ascending, members ascending (counting sort by root)
  std::vector<int64_t> off((size_t)M, 0);
  int64_t pos = 0;
  for (int64_t r = 0; r < M; ++r)
    if (count[r] >= 2) {
      off[r] = pos;
      pos += count[r];
    }
  int64_t spos = pos;
  for (int64_t x = 0; x < M; ++x) {
    const int32_t r = r_of[x];
    if (count[r] >= 2)
      perm[off[r]++] = (int32_t)x;
    else
      perm[spos++] = (int32_t)x;
  }
}

void partition_panels(int64_t npanels, const int64_t* w, int32_t G, int64_t* cuts) {
  std::vector<int64_t> prefix((size_t)npanels + 1, 0);
  for (int64_t p = 0; p < npanels; ++p) prefix[p + 1] = prefix[p] + w[p];
  const int64_t total = prefix[npanels];
  cuts[0] = 0;
  cuts[G] = npanels;
  for (int32_t g = 1; g < G; ++g) {
    // smallest p with prefix[p]·G >= g·total  (prefix is non-decreasing)
    auto it = std::partition_point(prefix.begin(), prefix.end(), [&](int64_t v) {
      return (unsigned __int128)v * (unsigned)G < (unsigned __int128)g * (uint64_t)total;
    });
    cuts[g] = std::min<int64_t>(it - prefix.begin(), npanels);
  }
}

}  // namespace sr
