// SONG oracle — TEST INFRASTRUCTURE ONLY.
//
// A plain, slow, single-threaded (per query) CPU implementation of the search
// that SONG (Zhao, Tan, Li; ICDE 2020) accelerates, written from PAPER.md.
// Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
// --impl reference legs may load this library.  The product path
// (paper_conf_icde_zhaotl20_b200/) never links, imports or calls it, and it
// shares no header, helper or constant table with the CUDA path.
//
// Citations: "P:<line>" = /root/reference/PAPER.md line.
//   Algorithm 1 (best-first search)
//   bounded priority queue, Observation 1    P:413-421  (§IV-C)
//   selected insertion                       P:425-431  (§IV-D)
//   visited deletion                         P:433-437  (§IV-E)
//   Bloom-filter visited set                 P:283      (§IV-B)
//   distance measures                        P:461      (§VI)
//
// Readings of the paper adopted here (all listed in DESIGN.md §3):
//   R1 topk is bounded at L = queue_len (Fig. 1 iteration 4 evicts vertex 1).
//   R2 every comparison uses the total order key(v) = (dist(p,v), v).
//   R3 selection applies only when |topk| = L (Fig. 4(b) iteration 1 admits 5).
//   R4 q capacity is exactly L (reproduces Fig. 1 and Fig. 4(c)).
//   R5 the entry vertex is a parameter (default id 0).
//   R6 -1 entries of an adjacency row are padding; a repeated id in one row is
//      located once (first occurrence).
//   R7 distances: squared L2; -<p,x>; 1 - cos (zero norm -> 1); accumulated in
//      fp64 in dimension order, rounded once to fp32; -0.0 canonicalised to +0.0.
//   R8 Bloom filter: k = 7 bits per id by double hashing
//      bit_i = (h1 + i*h2) mod m, h1 = fmix32(id), h2 = fmix32(id ^ 0x5bd1e995) | 1,
//      fmix32 = MurmurHash3's 32-bit finaliser.  No deletion.
//   R9 maintenance is a batch: selected candidates are inserted in candidate
//      order, then q's maximum is evicted while |q| > L (identical sets to the
//      per-candidate interleaving for exact visited sets; fixes the operation
//      order for the probabilistic filters).
//   R10 Cuckoo filter: see struct Cuckoo.
//   R11 1-bit random projection (§VII): bit j of a point's code is
//      1 iff <x, r_j> > 0 (sgn(0) -> bit 0), the projection accumulated in fp64
//      in dimension order; bit j lives in 32-bit word j / 32 at bit position
//      j % 32 ("h can be set as a multiple of 32 so that the bit vector can be
//      stored as several 32-bit unsigned integers").  R is [h][dim].
//   R13 multi-step probing (§V): an iteration pops up to `steps` vertices
//      (each checked against the termination rule with topk as updated by the
//      previous pops), locates the unvisited neighbours of all of them into ONE
//      candidate list (pop order, then row order, first occurrence), then runs
//      the distance and maintenance stages once.  n_exp counts pops.
//   R14 lazy visited deletion (a B200 schedule of P:435, flag ORACLE_LAZY with
//      DEL): the erasures of §IV-E are deferred; when inserting an iteration's
//      selected candidates would grow the exact visited set past a capacity C,
//      visited := ids(q) ∪ ids(topk) first (every deferred erasure at once).
//      Any schedule of the erasures leaves the result unchanged (a vertex
//      evicted from q ∪ topk has L better vertices there for good), so only
//      the counters move: fewer recomputed distances than eager deletion,
//      memory still bounded by C >= 2L + 32.
//   R15 graph construction (the step before the search: SONG loads NSW graphs,
//      P:477; HNSW layer-0 style): with every distance the search's
//      own (R7) and every order the (dist, id) key (R2), degree D:
//      1. forward F(i) = the D smallest keys (d(i, j), j) over j < i
//         (exact-insertion NSW: each vertex links to its D nearest earlier ones);
//      2. backward B(j) = the D smallest keys (d(i, j), i) over {i : j in F(i)};
//      3. C(v) = F(v) u B(v) ascending by key, as a set of vertices: v itself
//         is dropped and an id in both lists is kept once at its smaller key
//         (a no-op for 1.'s earlier-only lists, where F(v) < v < B(v); caller-
//         given kNN lists, song_build_graph_from_forward, can overlap);
//      4. HNSW heuristic: walk C(v) in order, keep c while fewer than D are kept
//         and d(c, k) > d(c, v) for every kept k ("closer to the base than to
//         every kept neighbour"); then refill with the skipped candidates in
//         C(v) order up to D; pad with -1.  Row = kept then refilled, in order.
//   R16 batched-insertion construction (the scale-out builder; the batch loop
//      is in oracle/__init__.py build_graph_batched): rows [0, P) take R15's
//      forward lists; each later batch [m, m + max(1, m >> s)) searches the
//      graph G_m = R15 steps 2-4 on the forward lists of rows [0, m)
//      (Algorithm 1, entry 0, K = D) and takes the top D as forward lists;
//      the graph is R15 steps 2-4 on all rows (oracle_forward_lists,
//      oracle_build_graph_from_forward below).
//   R12 Hamming search: the distance of two codes is the number of differing
//      bits ("the hamming distance between the bit-vectors"), used as the
//      key's distance (an integer, exact in fp32) with the same (dist, id)
//      order; the graph is the one built on the original vectors (the
//      index is kept, only the dataset is reduced).
//
// Parity status: every function below is pinned by tests/test_oracle_*.py
// (Fig. 1 / Fig. 4(c) traces, plain == optimized equivalence, brute-force
// exactness, greedy special case, invariants, Bloom FPR).  Nothing is
// "parity unpinned".

#include <algorithm>
#include <cmath>
#include <cstdint>
#include <cstring>
#include <set>
#include <thread>
#include <unordered_set>
#include <vector>

namespace {

enum Metric { ORACLE_L2 = 0, ORACLE_IP = 1, ORACLE_COSINE = 2, ORACLE_HAMMING = 3 };

// Mode flags.  ORACLE_PLAIN (= 0) is Algorithm 1 literally: unbounded q,
// exact visited set never deleted from, topk bounded at L (R1).
enum Flags {
  ORACLE_BOUNDED_Q = 1,  // §IV-C: q keeps at most L entries
  ORACLE_SEL = 2,        // §IV-D: selected insertion
  ORACLE_DEL = 4,        // §IV-E: visited deletion
  ORACLE_BLOOM = 8,      // §IV-B: visited is a Bloom filter (no deletion)
  ORACLE_CUCKOO = 16,    // visited is a Cuckoo filter (supports deletion)
  ORACLE_LAZY = 32,      // with DEL: deletions deferred until visited reaches a capacity (R14)
  ORACLE_UNION = 64,     // R17: q and topk kept as ONE bounded list (see search_one_union)
};

struct Key {
  float dist;
  int32_t id;
};

// R2: lexicographic (dist, id).
bool operator<(const Key& a, const Key& b) {
  if (a.dist < b.dist) return true;
  if (b.dist < a.dist) return false;
  return a.id < b.id;
}

// R12: Hamming distance of two h-bit codes stored as dim = h / 32 words (the
// float pointers carry the code words bit for bit); bits counted one by one.
float hamming(const float* p, const float* x, int words) {
  int64_t diff = 0;
  for (int i = 0; i < words; ++i) {
    uint32_t a, b;
    std::memcpy(&a, p + i, 4);
    std::memcpy(&b, x + i, 4);
    const uint32_t d = a ^ b;
    for (int bit = 0; bit < 32; ++bit) diff += (d >> bit) & 1u;
  }
  return (float)diff;
}

// R7: the distance of §VI, accumulated in fp64 in index order.
float distance(const float* p, const float* x, int dim, int metric) {
  if (metric == ORACLE_HAMMING) return hamming(p, x, dim);
  double out;
  if (metric == ORACLE_L2) {
    double acc = 0.0;
    for (int i = 0; i < dim; ++i) {
      double t = (double)p[i] - (double)x[i];
      acc += t * t;
    }
    out = acc;
  } else if (metric == ORACLE_IP) {
    double acc = 0.0;
    for (int i = 0; i < dim; ++i) acc += (double)p[i] * (double)x[i];
    out = -acc;
  } else {
    double dot = 0.0, np = 0.0, nx = 0.0;
    for (int i = 0; i < dim; ++i) {
      dot += (double)p[i] * (double)x[i];
      np += (double)p[i] * (double)p[i];
      nx += (double)x[i] * (double)x[i];
    }
    if (np == 0.0 || nx == 0.0)
      out = 1.0;
    else
      out = 1.0 - dot / (std::sqrt(np) * std::sqrt(nx));
  }
  float f = (float)out;
  if (f == 0.0f) f = 0.0f;  // -0.0 -> +0.0
  return f;
}

uint32_t fmix32(uint32_t h) {
  h ^= h >> 16;
  h *= 0x85ebca6bu;
  h ^= h >> 13;
  h *= 0xc2b2ae35u;
  h ^= h >> 16;
  return h;
}

// R8: the Bloom filter of §IV-B.
struct Bloom {
  std::vector<uint32_t> words;
  uint64_t m;  // number of bits
  explicit Bloom(uint64_t bits) : words((bits + 31) / 32, 0u), m(bits) {}
  uint64_t bit(int32_t id, int i) const {
    uint32_t h1 = fmix32((uint32_t)id);
    uint32_t h2 = fmix32((uint32_t)id ^ 0x5bd1e995u) | 1u;
    uint32_t h = h1 + (uint32_t)i * h2;  // 32-bit wrap-around
    return (uint64_t)h % m;
  }
  bool contains(int32_t id) const {
    for (int i = 0; i < 7; ++i) {
      uint64_t b = bit(id, i);
      if (!((words[b >> 5] >> (b & 31)) & 1u)) return false;
    }
    return true;
  }
  void insert(int32_t id) {
    for (int i = 0; i < 7; ++i) {
      uint64_t b = bit(id, i);
      words[b >> 5] |= 1u << (b & 31);
    }
  }
};

// R10: the Cuckoo filter of P:437 [14] ("supports deletion, so it works with
// visited deletion").  B = 2^b buckets of 4 slots holding 16-bit fingerprints
// (0 = empty); fp(v) = fmix32(v ^ 0x2545f491) & 0xffff, 0 -> 1;
// i1 = fmix32(v) mod B, i2 = (i1 ^ fmix32(fp)) mod B (partial-key cuckoo).
// insert: first empty slot of i1, else of i2, else kick: cur = i2, for
// n = 0..499 swap with slot n % 4 of cur, cur = alt(cur, fp'), stop at an empty
// slot; after 500 kicks the homeless fingerprint is dropped (counted).
// erase: clear the first slot holding fp in i1, else in i2.
struct Cuckoo {
  std::vector<uint16_t> slot;  // 4 * B
  uint32_t mask;
  int64_t drops = 0;
  explicit Cuckoo(uint64_t buckets) : slot(4 * buckets, 0), mask((uint32_t)buckets - 1) {}
  static uint16_t fp(int32_t v) {
    uint16_t f = (uint16_t)(fmix32((uint32_t)v ^ 0x2545f491u) & 0xffffu);
    return f ? f : 1;
  }
  uint32_t alt(uint32_t i, uint16_t f) const { return (i ^ fmix32((uint32_t)f)) & mask; }
  bool in_bucket(uint32_t b, uint16_t f) const {
    for (int j = 0; j < 4; ++j)
      if (slot[4 * b + j] == f) return true;
    return false;
  }
  bool put(uint32_t b, uint16_t f) {
    for (int j = 0; j < 4; ++j)
      if (slot[4 * b + j] == 0) {
        slot[4 * b + j] = f;
        return true;
      }
    return false;
  }
  bool contains(int32_t v) const {
    const uint16_t f = fp(v);
    const uint32_t i1 = fmix32((uint32_t)v) & mask;
    return in_bucket(i1, f) || in_bucket(alt(i1, f), f);
  }
  void insert(int32_t v) {
    uint16_t f = fp(v);
    const uint32_t i1 = fmix32((uint32_t)v) & mask;
    const uint32_t i2 = alt(i1, f);
    if (put(i1, f) || put(i2, f)) return;
    uint32_t cur = i2;
    for (int n = 0; n < 500; ++n) {
      std::swap(f, slot[4 * cur + (n & 3)]);
      cur = alt(cur, f);
      if (put(cur, f)) return;
    }
    ++drops;
  }
  void erase(int32_t v) {
    const uint16_t f = fp(v);
    const uint32_t i1 = fmix32((uint32_t)v) & mask;
    for (uint32_t b : {i1, alt(i1, f)})
      for (int j = 0; j < 4; ++j)
        if (slot[4 * b + j] == f) {
          slot[4 * b + j] = 0;
          return;
        }
  }
};

// The visited set: an exact hash set, a Bloom filter or a Cuckoo filter.
struct Visited {
  int kind;  // 0 exact, 1 Bloom, 2 Cuckoo
  std::unordered_set<int32_t> exact;
  Bloom filter;
  Cuckoo cuckoo;
  Visited(int k, uint64_t bloom_bits, uint64_t cuckoo_buckets)
      : kind(k), filter(k == 1 ? bloom_bits : 1), cuckoo(k == 2 ? cuckoo_buckets : 1) {}
  bool contains(int32_t v) const {
    return kind == 1 ? filter.contains(v) : kind == 2 ? cuckoo.contains(v) : exact.count(v) != 0;
  }
  void insert(int32_t v) {
    if (kind == 1)
      filter.insert(v);
    else if (kind == 2)
      cuckoo.insert(v);
    else
      exact.insert(v);
  }
  void erase(int32_t v) {
    if (kind == 0) exact.erase(v);
    if (kind == 2) cuckoo.erase(v);  // a Bloom filter cannot delete
  }
};

typedef void (*trace_fn)(void* ctx, int64_t iteration, const int32_t* q_ids, int64_t nq,
                         const int32_t* topk_ids, int64_t ntopk, const int32_t* visited_ids,
                         int64_t nvisited);

void emit_trace(trace_fn cb, void* ctx, int64_t it, const std::set<Key>& q,
                const std::set<Key>& topk, const Visited& vis) {
  if (!cb) return;
  std::vector<int32_t> qi, ti, vi;
  for (const Key& k : q) qi.push_back(k.id);
  for (const Key& k : topk) ti.push_back(k.id);
  int64_t nv = -1;  // a Bloom / Cuckoo filter cannot be enumerated
  if (vis.kind == 0) {
    vi.assign(vis.exact.begin(), vis.exact.end());
    std::sort(vi.begin(), vi.end());
    nv = (int64_t)vi.size();
  }
  cb(ctx, it, qi.data(), (int64_t)qi.size(), ti.data(), (int64_t)ti.size(), vi.data(), nv);
}

struct Problem {
  const float* data;
  int64_t n;
  int dim;
  const int32_t* adj;
  int degree;
  int metric;
  int K, L, flags, entry;
  uint64_t bloom_bits;  // Bloom: bits; Cuckoo: buckets
  int64_t max_iters;
  int steps;            // multi-step probing: pops per iteration (R13), >= 1
  int64_t lazy_cap;     // ORACLE_LAZY: visited capacity (R14)
};

// Algorithm 1 with the optimizations of §IV switched by flags.
// Step numbers refer to SURVEY.md §8(c) "Optimized mode, step by step".
// Returns 0, or 1 if the iteration cap was reached.
int search_one(const Problem& P, const float* p, int32_t* ids_out, float* dists_out,
               int64_t* counters, trace_fn cb, void* ctx) {
  const int L = P.L;
  const bool bounded = P.flags & ORACLE_BOUNDED_Q;
  const bool sel = P.flags & ORACLE_SEL;
  const bool lazy = (P.flags & ORACLE_LAZY) && (P.flags & ORACLE_DEL);
  const bool del = (P.flags & ORACLE_DEL) && !lazy;  // eager deletion
  Visited visited((P.flags & ORACLE_BLOOM) ? 1 : (P.flags & ORACLE_CUCKOO) ? 2 : 0, P.bloom_bits,
                  P.bloom_bits);
  std::set<Key> q;     // min-priority queue (begin() = min, prev(end()) = max)
  std::set<Key> topk;  // bounded max-priority queue (R1)
  int64_t n_dist = 0, n_exp = 0;
  int status = 0;

  // Step 1 — Alg. 1 line 1: q and visited start with the starting point.
  const int32_t e = P.entry;
  q.insert(Key{distance(p, P.data + (int64_t)e * P.dim, P.dim, P.metric), e});
  visited.insert(e);
  n_dist = 1;
  emit_trace(cb, ctx, 0, q, topk, visited);

  std::vector<int32_t> cand;
  std::vector<Key> popped;
  int64_t it = 0;
  // Step 2 — Alg. 1 line 2.
  while (!q.empty()) {
    if (it >= P.max_iters) {
      status = 1;
      break;
    }
    ++it;
    // 2.1 — line 3: pop the minimum of q.
    // 2.1 / 2.2 / 2.3 for each of up to P.steps pops (multi-step probing, §V
    // P:451, reading R13; steps = 1 is Alg. 1 exactly): pop the minimum of q
    // (line 3); stop when topk is full and its max is better (lines 4-5) —
    // before the first pop that ends the search, before a later pop that ends
    // only this iteration's popping; push into topk, evict its max beyond L and
    // [del] erase it from visited (line 7, R1).
    popped.clear();
    while ((int)popped.size() < P.steps && !q.empty()) {
      Key now = *q.begin();
      if ((int)topk.size() == L && *std::prev(topk.end()) < now) break;
      q.erase(q.begin());
      popped.push_back(now);
      topk.insert(now);
      if ((int)topk.size() > L) {
        Key y = *std::prev(topk.end());
        topk.erase(std::prev(topk.end()));
        if (del) visited.erase(y.id);
      }
    }
    if (popped.empty()) break;
    // 2.4 — candidate locating (§V): unvisited neighbours of the popped
    // vertices, in pop order then row order, skipping padding and repeats (R6)
    // — one candidate list for all pops ("fills more vertices into the
    // candidate list").
    cand.clear();
    for (const Key& now : popped) {
      const int32_t* row = P.adj + (int64_t)now.id * P.degree;
      for (int j = 0; j < P.degree; ++j) {
        int32_t v = row[j];
        if (v < 0) continue;
        if (visited.contains(v)) continue;
        if (std::find(cand.begin(), cand.end(), v) != cand.end()) continue;
        cand.push_back(v);
      }
    }
    // 2.5 — bulk distance computation (§VI).
    std::vector<Key> ck;
    ck.reserve(cand.size());
    for (int32_t v : cand) ck.push_back(Key{distance(p, P.data + (int64_t)v * P.dim, P.dim, P.metric), v});
    n_dist += (int64_t)cand.size();
    n_exp += (int64_t)popped.size();
    // 2.6 — maintenance, lines 12-13 with §IV-C/D/E, as a batch (R9: "the data
    // structure maintenance stage uses the distances to update the priority
    // queues and the hash table"): insert the selected candidates in
    // candidate order, then evict q's maximum while |q| > L.
    auto selected = [&](const Key& k) {
      // [sel] P:429: filtered when topk is full and k is worse than all of it (R3).
      return !(sel && (int)topk.size() == L && *std::prev(topk.end()) < k);
    };
    if (lazy) {
      // R14: the deferred deletions of P:435 are applied all at once — visited
      // becomes ids(q) ∪ ids(topk), the set eager deletion would hold — when
      // inserting this iteration's selected candidates would pass the capacity
      int64_t n_sel = 0;
      for (const Key& k : ck) n_sel += selected(k);
      if (n_sel > 0 && (int64_t)visited.exact.size() + n_sel > P.lazy_cap) {
        visited.exact.clear();
        for (const Key& k : q) visited.exact.insert(k.id);
        for (const Key& k : topk) visited.exact.insert(k.id);
      }
    }
    for (const Key& k : ck) {
      if (!selected(k)) continue;
      visited.insert(k.id);
      q.insert(k);
    }
    // [bounded] P:421: pop the worst once q grows past L (R4); [del] P:435.
    while (bounded && (int)q.size() > L) {
      Key w = *std::prev(q.end());
      q.erase(std::prev(q.end()));
      if (del) visited.erase(w.id);
    }
    emit_trace(cb, ctx, it, q, topk, visited);
  }

  // Step 3 — line 17: the first K of topk in ascending key order, padded.
  int i = 0;
  for (const Key& k : topk) {
    if (i >= P.K) break;
    ids_out[i] = k.id;
    dists_out[i] = k.dist;
    ++i;
  }
  for (; i < P.K; ++i) {
    ids_out[i] = -1;
    dists_out[i] = INFINITY;
  }
  if (counters) {
    counters[0] = n_dist;
    counters[1] = n_exp;
  }
  return status;
}

// Reading R17 — the bounded union.  q and topk of Algorithm 1 held as one
// list W of the L smallest keys discovered (the vertices of q ∪ topk that can
// still matter), each marked popped (in topk) or not (in q):
//   1. W = {(d_e, e)} unpopped; visited = {e}; n_dist = 1.
//   2. u = the smallest unpopped key of W; none -> stop (then every key of W
//      is popped: topk is full and its max beats q's min, Alg. 1 lines 4-5,
//      or q is empty).  Mark u popped (Alg. 1 lines 3, 7); n_exp += 1.
//   3. Locate the unvisited neighbours of u (row order, first occurrence).
//   4. Distances; n_dist += |cand|.
//   5. Maintain: [sel] skip c when |W| = L and key(c) > max(W) (a key beaten
//      by L discovered ones can never be popped nor returned: once full, W
//      stays full and its max only decreases); [lazy] if |visited| + |cand| > C
//      first set visited := ids(W), then mark EVERY candidate visited (a
//      skipped one can never enter W, so marking it saves recomputing it;
//      eager deletion keeps visited = ids(W) and marks only the selected);
//      insert the selected into W (unpopped); while |W| > L drop max(W) and
//      [del] erase it from visited.
//   6. Return the first K popped keys of W (all of W is popped at the end).
// Same popped sequence and result as Algorithm 1 (the popped key is q's min
// whenever it lies in the best L of q ∪ topk; otherwise topk is full and
// beats it — the stop rule), so the counters differ from the separate
// structures only in n_dist: a vertex dropped from W is no longer visited
// and is recomputed (then skipped by [sel]) if met again.
int search_one_union(const Problem& P, const float* p, int32_t* ids_out, float* dists_out,
                     int64_t* counters) {
  const int L = P.L;
  const bool sel = P.flags & ORACLE_SEL;
  const bool lazy = (P.flags & ORACLE_LAZY) && (P.flags & ORACLE_DEL);
  const bool del = (P.flags & ORACLE_DEL) && !lazy;
  std::set<Key> W;
  std::unordered_set<int32_t> popped;  // ids of W's popped keys
  std::unordered_set<int32_t> visited;
  int64_t n_dist = 0, n_exp = 0;
  int status = 0;
  const int32_t e = P.entry;
  W.insert(Key{distance(p, P.data + (int64_t)e * P.dim, P.dim, P.metric), e});
  visited.insert(e);
  n_dist = 1;
  std::vector<int32_t> cand;
  int64_t it = 0;
  while (true) {
    Key u{0.f, -1};
    for (const Key& k : W)
      if (!popped.count(k.id)) {
        u = k;
        break;
      }
    if (u.id < 0) break;
    if (it >= P.max_iters) {
      status = 1;
      break;
    }
    ++it;
    popped.insert(u.id);
    ++n_exp;
    cand.clear();
    const int32_t* row = P.adj + (int64_t)u.id * P.degree;
    for (int j = 0; j < P.degree; ++j) {
      const int32_t v = row[j];
      if (v < 0 || visited.count(v)) continue;
      if (std::find(cand.begin(), cand.end(), v) != cand.end()) continue;
      cand.push_back(v);
    }
    std::vector<Key> ck;
    for (int32_t v : cand) ck.push_back(Key{distance(p, P.data + (int64_t)v * P.dim, P.dim, P.metric), v});
    n_dist += (int64_t)cand.size();
    const bool full = (int)W.size() == L;
    const Key wmax = W.empty() ? Key{0.f, -1} : *std::prev(W.end());
    auto selected = [&](const Key& k) { return !(sel && full && wmax < k); };
    if (lazy && !ck.empty() && (int64_t)visited.size() + (int64_t)ck.size() > P.lazy_cap) {
      visited.clear();
      for (const Key& k : W) visited.insert(k.id);
    }
    for (const Key& k : ck) {
      if (!selected(k)) {
        if (lazy) visited.insert(k.id);
        continue;
      }
      visited.insert(k.id);
      W.insert(k);
    }
    while ((int)W.size() > L) {
      const Key w = *std::prev(W.end());
      W.erase(std::prev(W.end()));
      popped.erase(w.id);
      if (del) visited.erase(w.id);
    }
  }
  int i = 0;
  for (const Key& k : W) {
    if (i >= P.K) break;
    if (!popped.count(k.id)) continue;
    ids_out[i] = k.id;
    dists_out[i] = k.dist;
    ++i;
  }
  for (; i < P.K; ++i) {
    ids_out[i] = -1;
    dists_out[i] = INFINITY;
  }
  if (counters) {
    counters[0] = n_dist;
    counters[1] = n_exp;
  }
  return status;
}

int search_dispatch(const Problem& P, const float* p, int32_t* ids_out, float* dists_out,
                    int64_t* counters, trace_fn cb, void* ctx) {
  if (P.flags & ORACLE_UNION) return search_one_union(P, p, ids_out, dists_out, counters);
  return search_one(P, p, ids_out, dists_out, counters, cb, ctx);
}

}  // namespace

extern "C" {

// As oracle_search, with `steps` pops per iteration (multi-step probing, R13).
int64_t oracle_search_steps(const float* data, int64_t n, int32_t dim, const int32_t* adj,
                            int32_t degree, int32_t metric, const float* queries, int64_t nq,
                            int32_t K, int32_t L, int32_t flags, int64_t bloom_bits,
                            int32_t entry, int64_t max_iters, int32_t steps, int64_t lazy_cap,
                            int32_t* ids,
                            float* dists, int64_t* counters, int32_t nthreads, trace_fn cb,
                            void* ctx) {
  Problem P{data, n, dim, adj, degree, metric, K, L, flags, entry, (uint64_t)bloom_bits, max_iters,
            steps < 1 ? 1 : steps, lazy_cap};
  if (nthreads <= 1 || cb) {
    int64_t fails = 0;
    for (int64_t i = 0; i < nq; ++i)
      fails += search_dispatch(P, queries + i * dim, ids + i * K, dists + i * K,
                               counters ? counters + 2 * i : nullptr, cb, ctx);
    return fails;
  }
  std::vector<std::thread> pool;
  std::vector<int64_t> fails(nthreads, 0);
  for (int t = 0; t < nthreads; ++t) {
    pool.emplace_back([&, t]() {
      for (int64_t i = t; i < nq; i += nthreads)
        fails[t] += search_dispatch(P, queries + i * dim, ids + i * K, dists + i * K,
                                    counters ? counters + 2 * i : nullptr, nullptr, nullptr);
    });
  }
  for (auto& th : pool) th.join();
  int64_t total = 0;
  for (int64_t f : fails) total += f;
  return total;
}

// Search nq queries.  All pointers are host pointers; layouts are row-major:
// data [n][dim] fp32, adj [n][degree] int32 (-1 = padding), queries [nq][dim],
// ids/dists [nq][K], counters [nq][2] = (distance computations, expansions)
// or NULL.  nthreads > 1 partitions the queries over std::threads (no trace).
// Returns the number of queries that hit max_iters (0 = all finished).
int64_t oracle_search(const float* data, int64_t n, int32_t dim, const int32_t* adj,
                      int32_t degree, int32_t metric, const float* queries, int64_t nq,
                      int32_t K, int32_t L, int32_t flags, int64_t bloom_bits, int32_t entry,
                      int64_t max_iters, int32_t* ids, float* dists, int64_t* counters,
                      int32_t nthreads, trace_fn cb, void* ctx) {
  return oracle_search_steps(data, n, dim, adj, degree, metric, queries, nq, K, L, flags,
                             bloom_bits, entry, max_iters, 1, 0, ids, dists, counters, nthreads,
                             cb, ctx);
}

// The distance of §VI for one pair (exposed so tests can pin R7 directly).
float oracle_distance(const float* p, const float* x, int32_t dim, int32_t metric) {
  return distance(p, x, dim, metric);
}

// Exact top-K by scanning every point under the same key order (R2).  This is
// the ground truth B of the recall definition on small inputs.
void oracle_bruteforce(const float* data, int64_t n, int32_t dim, int32_t metric,
                       const float* queries, int64_t nq, int32_t K, int32_t* ids,
                       float* dists, int32_t nthreads) {
  auto one = [&](int64_t qi) {
    std::vector<Key> all((size_t)n);
    for (int64_t v = 0; v < n; ++v)
      all[v] = Key{distance(queries + qi * dim, data + v * dim, dim, metric), (int32_t)v};
    int64_t k = std::min<int64_t>(K, n);
    std::partial_sort(all.begin(), all.begin() + k, all.end());
    for (int64_t i = 0; i < K; ++i) {
      ids[qi * K + i] = i < k ? all[i].id : -1;
      dists[qi * K + i] = i < k ? all[i].dist : INFINITY;
    }
  };
  if (nthreads <= 1) {
    for (int64_t i = 0; i < nq; ++i) one(i);
    return;
  }
  std::vector<std::thread> pool;
  for (int t = 0; t < nthreads; ++t)
    pool.emplace_back([&, t]() {
      for (int64_t i = t; i < nq; i += nthreads) one(i);
    });
  for (auto& th : pool) th.join();
}

// 1-bit random projection of §VII (R11): codes[i] = the h-bit code
// of data[i], packed in h / 32 uint32 words.  R is [h][dim] row-major (row j =
// the random vector r_j).  h must be a multiple of 32.
void oracle_rp_encode(const float* data, int64_t n, int32_t dim, const float* R, int32_t h,
                      uint32_t* codes, int32_t nthreads) {
  const int words = h / 32;
  auto one = [&](int64_t i) {
    const float* x = data + i * dim;
    for (int w = 0; w < words; ++w) codes[i * words + w] = 0u;
    for (int j = 0; j < h; ++j) {
      double acc = 0.0;
      for (int t = 0; t < dim; ++t) acc += (double)x[t] * (double)R[(int64_t)j * dim + t];
      if (acc > 0.0) codes[i * words + j / 32] |= 1u << (j % 32);
    }
  };
  if (nthreads <= 1) {
    for (int64_t i = 0; i < n; ++i) one(i);
    return;
  }
  std::vector<std::thread> pool;
  for (int t = 0; t < nthreads; ++t)
    pool.emplace_back([&, t]() {
      for (int64_t i = t; i < n; i += nthreads) one(i);
    });
  for (auto& th : pool) th.join();
}

// R15 steps 2-4 (backward lists, candidates, heuristic) on given forward
// lists F (fwd_ids / fwd_dists [n][degree], -1 padded, ascending keys).
static void build_from_forward(const float* data, int64_t n, int32_t dim, int32_t metric,
                               int32_t degree, std::vector<std::vector<Key>>& F,
                               int32_t* adj_out, int32_t nthreads) {
  const int D = degree;
  auto dist = [&](int64_t a, int64_t b) {
    return distance(data + a * dim, data + b * dim, dim, metric);
  };
  auto parallel = [&](auto&& fn) {
    if (nthreads <= 1) {
      for (int64_t v = 0; v < n; ++v) fn(v);
      return;
    }
    std::vector<std::thread> pool;
    for (int t = 0; t < nthreads; ++t)
      pool.emplace_back([&, t]() {
        for (int64_t v = t; v < n; v += nthreads) fn(v);
      });
    for (auto& th : pool) th.join();
  };
  // 2. backward lists
  std::vector<std::vector<Key>> B(n);
  for (int64_t i = 0; i < n; ++i)
    for (const Key& e : F[i]) B[e.id].push_back(Key{e.dist, (int32_t)i});
  parallel([&](int64_t j) {
    auto& b = B[j];
    const size_t k = std::min<size_t>(D, b.size());
    std::partial_sort(b.begin(), b.begin() + k, b.end());
    b.resize(k);
  });
  // 3. + 4. candidates and the heuristic
  parallel([&](int64_t v) {
    std::vector<Key> all = F[v];
    all.insert(all.end(), B[v].begin(), B[v].end());
    std::sort(all.begin(), all.end());
    // C(v) = F(v) ∪ B(v) as a set of vertices (R15): v itself is not its own
    // neighbour, and an id in both lists is kept once, at its smaller key
    std::vector<Key> C;
    for (const Key& k : all) {
      if (k.id == (int32_t)v) continue;
      bool seen = false;
      for (const Key& c : C) seen = seen || c.id == k.id;
      if (!seen) C.push_back(k);
    }
    std::vector<int32_t> kept;
    std::vector<char> taken(C.size(), 0);
    for (size_t t = 0; t < C.size() && (int)kept.size() < D; ++t) {
      bool ok = true;
      for (int32_t k : kept)
        if (!(dist(C[t].id, k) > C[t].dist)) {
          ok = false;
          break;
        }
      if (ok) {
        kept.push_back(C[t].id);
        taken[t] = 1;
      }
    }
    for (size_t t = 0; t < C.size() && (int)kept.size() < D; ++t)
      if (!taken[t]) kept.push_back(C[t].id);
    for (int j = 0; j < D; ++j) adj_out[v * D + j] = j < (int)kept.size() ? kept[j] : -1;
  });
}

// R15 step 1: F(i) = the D smallest keys (d(i, j), j) over j < i.
static std::vector<std::vector<Key>> forward_lists(const float* data, int64_t n, int32_t dim,
                                                   int32_t metric, int32_t D, int32_t nthreads) {
  std::vector<std::vector<Key>> F(n);
  auto one = [&](int64_t i) {
    std::vector<Key> all;
    all.reserve(i);
    for (int64_t j = 0; j < i; ++j)
      all.push_back(Key{distance(data + i * dim, data + j * dim, dim, metric), (int32_t)j});
    const size_t k = std::min<size_t>(D, all.size());
    std::partial_sort(all.begin(), all.begin() + k, all.end());
    all.resize(k);
    F[i] = all;
  };
  if (nthreads <= 1) {
    for (int64_t i = 0; i < n; ++i) one(i);
  } else {
    std::vector<std::thread> pool;
    for (int t = 0; t < nthreads; ++t)
      pool.emplace_back([&, t]() {
        for (int64_t i = t; i < n; i += nthreads) one(i);
      });
    for (auto& th : pool) th.join();
  }
  return F;
}

// R15: graph construction (see the header).  data [n][dim] fp32, adj_out
// [n][degree] int32.  nthreads > 1 splits the per-vertex loops over threads.
void oracle_build_graph(const float* data, int64_t n, int32_t dim, int32_t metric, int32_t degree,
                        int32_t* adj_out, int32_t nthreads) {
  auto F = forward_lists(data, n, dim, metric, degree, nthreads);
  build_from_forward(data, n, dim, metric, degree, F, adj_out, nthreads);
}

// R15 step 1 alone: F as ids / dists [n][degree] (-1 / +inf past a row's |F|).
void oracle_forward_lists(const float* data, int64_t n, int32_t dim, int32_t metric,
                          int32_t degree, int32_t* ids_out, float* dists_out, int32_t nthreads) {
  auto F = forward_lists(data, n, dim, metric, degree, nthreads);
  for (int64_t i = 0; i < n; ++i)
    for (int j = 0; j < degree; ++j) {
      const bool ok = j < (int)F[i].size();
      ids_out[i * degree + j] = ok ? F[i][j].id : -1;
      dists_out[i * degree + j] = ok ? F[i][j].dist : INFINITY;
    }
}

// R16 steps on given forward lists: fwd_ids / fwd_dists [n][degree] (-1 /
// any padding past a row's entries); the rows' keys are taken as given.
void oracle_build_graph_from_forward(const float* data, int64_t n, int32_t dim, int32_t metric,
                                     int32_t degree, const int32_t* fwd_ids,
                                     const float* fwd_dists, int32_t* adj_out, int32_t nthreads) {
  std::vector<std::vector<Key>> F(n);
  for (int64_t i = 0; i < n; ++i)
    for (int j = 0; j < degree; ++j) {
      const int32_t id = fwd_ids[i * degree + j];
      if (id >= 0) F[i].push_back(Key{fwd_dists[i * degree + j], id});
    }
  build_from_forward(data, n, dim, metric, degree, F, adj_out, nthreads);
}

// Cuckoo filter probe for tests of R10: applies ops[i] (+id = insert,
// -(id+1) = erase) in order, then writes 1/0 membership of probe[] to out;
// returns the number of dropped fingerprints.
int64_t oracle_cuckoo_probe(int64_t buckets, const int64_t* ops, int64_t nops,
                            const int32_t* probe, int64_t nprobe, uint8_t* out) {
  Cuckoo c((uint64_t)buckets);
  for (int64_t i = 0; i < nops; ++i) {
    if (ops[i] >= 0)
      c.insert((int32_t)ops[i]);
    else
      c.erase((int32_t)(-ops[i] - 1));
  }
  for (int64_t i = 0; i < nprobe; ++i) out[i] = c.contains(probe[i]) ? 1 : 0;
  return c.drops;
}

// Bloom filter probe for tests of §IV-B: inserts ins[0..nins), then
// writes 1/0 membership of probe[0..nprobe) to out.
void oracle_bloom_probe(int64_t bits, const int32_t* ins, int64_t nins, const int32_t* probe,
                        int64_t nprobe, uint8_t* out) {
  Bloom b((uint64_t)bits);
  for (int64_t i = 0; i < nins; ++i) b.insert(ins[i]);
  for (int64_t i = 0; i < nprobe; ++i) out[i] = b.contains(probe[i]) ? 1 : 0;
}

}  // extern "C"
