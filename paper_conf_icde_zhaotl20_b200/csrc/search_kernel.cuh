// search_kernel.cuh — the SONG search hot path for sm_100a.
//
// One warp owns one query at a time (persistent: warps pull query tickets from
// an atomic counter, so long and short queries load-balance).  Each iteration
// of Algorithm 1 runs the paper's three stages (§III, Fig. 3)
// warp-cooperatively instead of on "one single thread":
//
//   locate (§V)    the adjacency row of the head (prefetched into registers
//                  during the previous iteration's maintenance) is filtered:
//                  padding, repeats (match.any, only if the index has them)
//                  and visited ids (32 parallel probes of a bucketed hash),
//                  compacted by a ballot
//   distance (§VI) rounds of 8 candidate rows: lane j resolves candidate j's
//                  row address, every row of the round is put in flight at
//                  once with cp.async (LDGSTS, 16 B per lane per row) into a
//                  per-warp shared-memory stage — no register cost — then each
//                  lane reduces its own 16 B slices with packed FFMA2/FADD2 and
//                  a transposed butterfly sums 8 rows in 9 shuffles (P:455's
//                  shfl_down reduction, batched)
//   maintain (§IV) selected insertion (§IV-D) against topk's max, compaction +
//                  bitonic sort of only the selected keys, visited insert,
//                  bitonic merge into the bounded q (§IV-C) with visited
//                  deletion of the evicted keys (§IV-E).  For queue_len <= 128
//                  q and topk live in registers (sorted, striped over the
//                  lanes); larger queues use shared-memory arrays and
//                  merge-path ranks.
//
// Priority-queue keys are u64 (orderable(dist) << 32 | id): the (dist, id)
// total order of DESIGN.md reading A3 as a single integer compare.
#pragma once

#include <cuda_runtime.h>

#include <cstdint>

namespace song {

constexpr unsigned FULL = 0xffffffffu;
constexpr int EMPTY = -1;  // hash slot never used
constexpr int TOMB = -2;   // hash slot whose key was deleted (§IV-E)
constexpr uint64_t KEY_MAX = ~0ull;
constexpr int STAGE_BYTES = 16384;  // per-warp row stage (32 rows of d = 128)

enum : int { STATUS_BAD_INPUT = 1, STATUS_ITER_CAP = 2, STATUS_TABLE_FULL = 4 };
// visited-set kinds (template parameter VK of the kernel)
enum : int { VK_HASH = 0, VK_BLOOM = 1, VK_GHASH = 2, VK_CUCKOO = 3 };
// MET_HAM: rows are h-bit codes of the 1-bit random projection (§VII),
// dpad 32-bit words each; the distance is the Hamming distance (reading R12)
enum : int { MET_L2 = 0, MET_DOT = 1, MET_HAM = 2 };

struct SearchArgs {
  const float* data;      // [n][dpad], 16 B aligned rows (MET_HAM: uint32 code words)
  const int32_t* adj;     // [n][degree]
  const float* queries;   // [nq][dim] (caller layout, unpadded; MET_HAM: [nq][dim] words)
  int32_t* ids_out;       // [nq][K]
  float* dists_out;       // [nq][K]
  int32_t* counters_out;  // [nq][2] or nullptr
  unsigned* ticket;       // work counter, zeroed before launch
  const int32_t* order;   // [nq] ticket -> query index, or nullptr (batch order)
  int* status;            // sticky STATUS_* bits
  int64_t n;
  int64_t nq;
  int dim, dpad, degree;
  int K, L;
  int table_log2;  // hash: log2 slots; bloom: log2 bits
  int entry, max_iters, id_offset;
  int steps;       // multi-step probing (§V, reading R13): pops per iteration
  int lazy;        // VK_HASH: deletions deferred to the rebuild at rebuild_at (reading R14)
  int cosine;      // MET_DOT: 1 -> 1 - dot, 0 -> -dot
  int dedup;       // 1 if some adjacency row repeats an id
  int rebuild_at;  // hash: rebuild when live + tombstones would exceed this
  int sel;         // selected insertion on (VK_GHASH: hashtable-sel vs hashtable)
  uint64_t* gtab;  // VK_GHASH: [grid warps][2^table_log2] u64
  uint32_t gen0;   // VK_GHASH: generation base of this launch
  int warp_smem_bytes;
  unsigned long long* stage_cycles;  // SONG_STAGE_TIMING builds: [4] SM cycles per stage
  int* gvis;       // QR == -2: [grid warps][2^table_log2] int32 visited tables (global)
};

// SONG_STAGE_TIMING (a separate build, never the product library): lane 0 of
// every warp reads clock64 at the stage boundaries of each iteration and adds
// the cycles of pop/topk (a3), locate (a4), distance (a5) and maintenance
// (a6) to stage_cycles[0..3] — the in-kernel split of Fig. 10
#ifdef SONG_STAGE_TIMING
#define SONG_ST_MARK(k)                      \
  do {                                       \
    if (lane == 0) {                         \
      const long long t_ = clock64();        \
      st_acc[k] += (unsigned long long)(t_ - st_t); \
      st_t = t_;                             \
    }                                        \
  } while (0)
#else
#define SONG_ST_MARK(k) \
  do {                  \
  } while (0)
#endif

// ------------------------------------------------------------------- keys --
__device__ __forceinline__ uint32_t f2ord(float f) {
  f = f + 0.0f;  // canonicalise -0.0 to +0.0 (reading A9)
  uint32_t u = __float_as_uint(f);
  return (u & 0x80000000u) ? ~u : (u | 0x80000000u);
}

__device__ __forceinline__ float ord2f(uint32_t o) {
  uint32_t u = (o & 0x80000000u) ? (o & 0x7fffffffu) : ~o;
  return __uint_as_float(u);
}

__device__ __forceinline__ uint64_t make_key(float d, int id) {
  return ((uint64_t)f2ord(d) << 32) | (uint32_t)id;
}

__device__ __forceinline__ int key_id(uint64_t k) { return (int)(uint32_t)(k & 0xffffffffu); }

// Reading R17 keys (the bounded union W): orderable(dist) << 32 | id << 1 |
// popped — ids < 2^31, so the (dist, id) order is unchanged and the popped
// mark rides in bit 0 without ever deciding a comparison between two keys
__device__ __forceinline__ uint64_t make_wkey(float d, int id) {
  return ((uint64_t)f2ord(d) << 32) | ((uint64_t)(uint32_t)id << 1);
}
__device__ __forceinline__ int wkey_id(uint64_t k) { return (int)((uint32_t)(k & 0xffffffffu) >> 1); }

__device__ __forceinline__ unsigned lanemask_lt() {
  unsigned m;
  asm("mov.u32 %0, %%lanemask_lt;" : "=r"(m));
  return m;
}

__device__ __forceinline__ uint64_t umin64(uint64_t a, uint64_t b) { return a < b ? a : b; }
__device__ __forceinline__ uint64_t umax64(uint64_t a, uint64_t b) { return a < b ? b : a; }

// warp-wide minimum of a u64 key (two REDUX ops)
__device__ __forceinline__ uint64_t warp_min_key(uint64_t k) {
  uint32_t hi = (uint32_t)(k >> 32);
  uint32_t mh = __reduce_min_sync(FULL, hi);
  uint32_t lo = (hi == mh) ? (uint32_t)k : 0xffffffffu;
  uint32_t ml = __reduce_min_sync(FULL, lo);
  return ((uint64_t)mh << 32) | ml;
}

// ------------------------------------------------------- shared addresses --
__device__ __forceinline__ uint32_t smem_u32(const void* p) {
  return (uint32_t)__cvta_generic_to_shared(p);
}

// ---------------------------------------------------------------- visited --
// Open-addressing hash in shared memory organised as buckets of four
// 4-byte slots: one LDS.128 reads a whole bucket, so at the table's low load
// (<= 1/4) almost every operation resolves with a single probe; buckets are
// probed linearly (open addressing).  Every lane runs its own probe sequence,
// so up to 32 operations proceed in parallel, and all loops are
// warp-collective (trip count decided by __any_sync) so the warp stays
// converged for the shuffles that follow.
// GLOBAL: the table lives in a per-warp region of global memory (L2-resident;
// the bounded union at large queue_len, where a shared-memory table would
// cost most of the SM's resident warps): buckets are read at L2 (ld.cg), so
// the reads see the atomicCAS / store results of the same warp.
template <bool GLOBAL = false>
struct HashSetT {
  int* slot;
  int log2;  // slots = 2^log2, buckets = 2^(log2 - 2)
  __device__ __forceinline__ unsigned home(int v) const {
    return ((uint32_t)v * 0x9E3779B1u) >> (34 - log2);
  }
  __device__ __forceinline__ int4 bucket(unsigned b) const {
    if constexpr (GLOBAL) return __ldcg(reinterpret_cast<const int4*>(slot) + b);
    return reinterpret_cast<const int4*>(slot)[b];
  }
  // every slot EMPTY (warp-collective; 16 B stores)
  __device__ __forceinline__ void clear(int lane) {
    int4* s4 = reinterpret_cast<int4*>(slot);
    for (int i = lane; i < (1 << (log2 - 2)); i += 32) s4[i] = make_int4(EMPTY, EMPTY, EMPTY, EMPTY);
    __syncwarp();
  }
  // membership of v for lanes with act; result false elsewhere
  __device__ __forceinline__ bool contains(int v, bool act) const {
    const unsigned mask = (1u << (log2 - 2)) - 1;
    unsigned b = home(v);
    bool found = false;
    while (__any_sync(FULL, act)) {
      if (act) {
        const int4 s = bucket(b);
        found = (s.x == v) | (s.y == v) | (s.z == v) | (s.w == v);
        const bool open = (s.x == EMPTY) | (s.y == EMPTY) | (s.z == EMPTY) | (s.w == EMPTY);
        act = !found && !open;
        b = (b + 1) & mask;
      }
    }
    return found;
  }
  // contains(), also returning (eslot) the first EMPTY slot of the bucket the
  // probe ended in — where an insert of v would go — or -1 when v was found
  __device__ __forceinline__ bool contains_slot(int v, bool act, int& eslot) const {
    const unsigned mask = (1u << (log2 - 2)) - 1;
    unsigned b = home(v);
    bool found = false;
    eslot = -1;
    while (__any_sync(FULL, act)) {
      if (act) {
        const int4 s = bucket(b);
        found = (s.x == v) | (s.y == v) | (s.z == v) | (s.w == v);
        const bool e0 = s.x == EMPTY, e1 = s.y == EMPTY, e2 = s.z == EMPTY, e3 = s.w == EMPTY;
        const bool open = e0 | e1 | e2 | e3;
        if (!found && open) eslot = 4 * (int)b + (e0 ? 0 : e1 ? 1 : e2 ? 2 : 3);
        act = !found && !open;
        b = (b + 1) & mask;
      }
    }
    return found;
  }
  // insert v (not present) for lanes with act; true when an EMPTY slot was used
  __device__ __forceinline__ bool insert(int v, bool act) {
    const unsigned mask = (1u << (log2 - 2)) - 1;
    unsigned b = home(v);
    bool took_empty = false;
    while (__any_sync(FULL, act)) {
      if (act) {
        const int4 s = bucket(b);
        const bool f0 = s.x < 0, f1 = s.y < 0, f2 = s.z < 0, f3 = s.w < 0;  // EMPTY or TOMB
        if (f0 | f1 | f2 | f3) {
          const int j = f0 ? 0 : f1 ? 1 : f2 ? 2 : 3;
          const int old_v = f0 ? s.x : f1 ? s.y : f2 ? s.z : s.w;
          const int old = atomicCAS(&slot[4 * b + j], old_v, v);
          if (old == old_v) {
            act = false;
            took_empty = (old_v == EMPTY);
          }  // else: lost the race for this slot, re-read the bucket
        } else {
          b = (b + 1) & mask;
        }
      }
    }
    return took_empty;
  }
  // delete v (present) for lanes with act (§IV-E): the slot becomes a tombstone
  __device__ __forceinline__ void erase(int v, bool act) {
    const unsigned mask = (1u << (log2 - 2)) - 1;
    unsigned b = home(v);
    while (__any_sync(FULL, act)) {
      if (act) {
        const int4 s = bucket(b);
        const bool h0 = s.x == v, h1 = s.y == v, h2 = s.z == v, h3 = s.w == v;
        if (h0 | h1 | h2 | h3) {
          slot[4 * b + (h0 ? 0 : h1 ? 1 : h2 ? 2 : 3)] = TOMB;
          act = false;
        } else {
          act = !((s.x == EMPTY) | (s.y == EMPTY) | (s.z == EMPTY) | (s.w == EMPTY));
          b = (b + 1) & mask;
        }
      }
    }
  }
};

using HashSet = HashSetT<false>;

// Bloom filter with the k = 7 double-hashing spec of reading A8:
// bit_i = (h1 + i*h2) mod m, h1 = fmix32(id), h2 = fmix32(id ^ 0x5bd1e995) | 1.
__device__ __forceinline__ uint32_t fmix32(uint32_t h) {
  h ^= h >> 16;
  h *= 0x85ebca6bu;
  h ^= h >> 13;
  h *= 0xc2b2ae35u;
  h ^= h >> 16;
  return h;
}

struct BloomSet {
  uint32_t* word;
  int log2;  // m = 2^log2 bits
  __device__ __forceinline__ bool contains(int v, bool act) const {
    const uint32_t h1 = fmix32((uint32_t)v), h2 = fmix32((uint32_t)v ^ 0x5bd1e995u) | 1u;
    const uint32_t mask = (1u << log2) - 1;
    bool all = true;
#pragma unroll
    for (int i = 0; i < 7; ++i) {
      const uint32_t b = (h1 + (uint32_t)i * h2) & mask;
      all = all && (act ? ((word[b >> 5] >> (b & 31)) & 1u) : 0u);
    }
    return act && all;
  }
  __device__ __forceinline__ void insert(int v, bool act) {
    const uint32_t h1 = fmix32((uint32_t)v), h2 = fmix32((uint32_t)v ^ 0x5bd1e995u) | 1u;
    const uint32_t mask = (1u << log2) - 1;
    if (act) {
#pragma unroll
      for (int i = 0; i < 7; ++i) {
        const uint32_t b = (h1 + (uint32_t)i * h2) & mask;
        atomicOr(&word[b >> 5], 1u << (b & 31));
      }
    }
    __syncwarp();
  }
};

// Exact visited set in GLOBAL memory for the variants without visited
// deletion ("hashtable" / "hashtable-sel" of Fig. 7; the paper keeps
// the unbounded table in global memory).  One table of 2^log2 u64 slots
// per resident warp; a slot holds (generation << 32 | id) and counts as empty
// unless its generation is the current query's, so tables are never cleared.
struct GHash {
  uint64_t* slot;
  int log2;
  uint32_t gen;
  __device__ __forceinline__ unsigned home(int v) const {
    return ((uint32_t)v * 0x9E3779B1u) >> (32 - log2);
  }
  __device__ __forceinline__ bool contains(int v, bool act) const {
    const unsigned mask = (1u << log2) - 1;
    const uint64_t want = ((uint64_t)gen << 32) | (uint32_t)v;
    unsigned h = home(v);
    bool found = false;
    while (__any_sync(FULL, act)) {
      if (act) {
        const uint64_t s = slot[h];
        found = (s == want);
        act = !found && (uint32_t)(s >> 32) == gen;
        h = (h + 1) & mask;
      }
    }
    return found;
  }
  __device__ __forceinline__ void insert(int v, bool act) {
    const unsigned mask = (1u << log2) - 1;
    const uint64_t want = ((uint64_t)gen << 32) | (uint32_t)v;
    unsigned h = home(v);
    while (__any_sync(FULL, act)) {
      if (act) {
        const uint64_t s = slot[h];
        if ((uint32_t)(s >> 32) != gen) {
          const unsigned long long old =
              atomicCAS(reinterpret_cast<unsigned long long*>(slot + h), (unsigned long long)s,
                        (unsigned long long)want);
          if (old == s) act = false;  // else: lost the race, re-read the slot
        } else {
          h = (h + 1) & mask;
        }
      }
    }
  }
};

// Cuckoo filter (reading R10; the oracle's struct Cuckoo): 2^log2
// buckets of 4 x 16-bit fingerprints in shared memory.  Lookups run on all
// lanes in parallel; inserts and erases are single-lane and issued in the
// oracle's order (kicks make the state order-dependent).
struct CuckooSet {
  uint16_t* slot;
  int log2;
  __device__ __forceinline__ uint32_t mask() const { return (1u << log2) - 1; }
  __device__ __forceinline__ static uint16_t fp(int v) {
    const uint16_t f = (uint16_t)(fmix32((uint32_t)v ^ 0x2545f491u) & 0xffffu);
    return f ? f : (uint16_t)1;
  }
  __device__ __forceinline__ uint32_t alt(uint32_t i, uint16_t f) const {
    return (i ^ fmix32((uint32_t)f)) & mask();
  }
  __device__ __forceinline__ bool in_bucket(uint32_t b, uint16_t f) const {
    const uint2 w = reinterpret_cast<const uint2*>(slot)[b];  // 4 fingerprints
    const uint32_t ff = (uint32_t)f;
    return ((w.x & 0xffffu) == ff) | ((w.x >> 16) == ff) | ((w.y & 0xffffu) == ff) |
           ((w.y >> 16) == ff);
  }
  __device__ __forceinline__ bool contains(int v, bool act) const {
    if (!act) return false;
    const uint16_t f = fp(v);
    const uint32_t i1 = fmix32((uint32_t)v) & mask();
    return in_bucket(i1, f) || in_bucket(alt(i1, f), f);
  }
  __device__ __forceinline__ bool put(uint32_t b, uint16_t f) {
#pragma unroll
    for (int j = 0; j < 4; ++j)
      if (slot[4 * b + j] == 0) {
        slot[4 * b + j] = f;
        return true;
      }
    return false;
  }
  // single lane; returns false when a fingerprint was dropped after 500 kicks
  __device__ __forceinline__ bool insert1(int v) {
    uint16_t f = fp(v);
    const uint32_t i1 = fmix32((uint32_t)v) & mask();
    const uint32_t i2 = alt(i1, f);
    if (put(i1, f) || put(i2, f)) return true;
    uint32_t cur = i2;
    for (int n = 0; n < 500; ++n) {
      const uint16_t victim = slot[4 * cur + (n & 3)];
      slot[4 * cur + (n & 3)] = f;
      f = victim;
      cur = alt(cur, f);
      if (put(cur, f)) return true;
    }
    return false;
  }
  __device__ __forceinline__ void erase1(int v) {
    const uint16_t f = fp(v);
    const uint32_t i1 = fmix32((uint32_t)v) & mask();
    const uint32_t b2 = alt(i1, f);
#pragma unroll
    for (int j = 0; j < 4; ++j)
      if (slot[4 * i1 + j] == f) {
        slot[4 * i1 + j] = 0;
        return;
      }
#pragma unroll
    for (int j = 0; j < 4; ++j)
      if (slot[4 * b2 + j] == f) {
        slot[4 * b2 + j] = 0;
        return;
      }
  }
};

// ------------------------------------------------------------- utilities --
template <bool DESC>
__device__ __forceinline__ uint64_t bitonic_sort32(uint64_t key, int lane) {
#pragma unroll
  for (int k = 2; k <= 32; k <<= 1) {
#pragma unroll
    for (int j = k >> 1; j > 0; j >>= 1) {
      const uint64_t other = __shfl_xor_sync(FULL, key, j);
      const bool take_min = (((lane & j) == 0) == (((lane & k) == 0) != DESC));
      key = ((other < key) == take_min) ? other : key;  // one 64-bit compare
    }
  }
  return key;
}

// ascending bitonic sort of each W-lane block (W <= 32, a power of two)
template <int W>
__device__ __forceinline__ uint64_t bitonic_sort_w(uint64_t key, int lane) {
#pragma unroll
  for (int k = 2; k <= W; k <<= 1) {
#pragma unroll
    for (int j = k >> 1; j > 0; j >>= 1) {
      const uint64_t other = __shfl_xor_sync(FULL, key, j);
      const bool take_min = (((lane & j) == 0) == ((lane & k) == 0));
      key = ((other < key) == take_min) ? other : key;
    }
  }
  return key;
}

// ascending sort of the n (warp-uniform) keys held by lanes [0, n); lanes >= n
// hold KEY_MAX.  Only the network for the next power of two >= n is run.
__device__ __forceinline__ uint64_t sort_prefix(uint64_t key, int n, int lane) {
  if (n <= 1) return key;
  if (n <= 2) return bitonic_sort_w<2>(key, lane);
  if (n <= 4) return bitonic_sort_w<4>(key, lane);
  if (n <= 8) return bitonic_sort_w<8>(key, lane);
  if (n <= 16) return bitonic_sort_w<16>(key, lane);
  return bitonic_sort_w<32>(key, lane);
}

// number of elements of sorted a[0..n) strictly below x
// (branch-free: the trip count depends only on the warp-uniform n)
__device__ __forceinline__ int count_below(const uint64_t* a, int n, uint64_t x) {
  int lo = 0;
  for (int step = 1 << (31 - __clz(n | 1)); step > 0; step >>= 1) {
    const int j = lo + step - 1;
    lo = (j < n && a[j] < x) ? lo + step : lo;
  }
  return lo;
}

template <int R>
struct Log2 {
  static constexpr int value = (R <= 1) ? 0 : 1 + Log2<R / 2>::value;
};
template <>
struct Log2<1> {
  static constexpr int value = 0;
};

// Transposed butterfly: on entry every lane holds R partial sums v[0..R); on
// exit every lane holds the warp-wide total of row (lane >> (5 - log2 R)).
template <int R>
__device__ __forceinline__ float transpose_reduce(float (&v)[R], int lane) {
  constexpr int LR = Log2<R>::value;
#pragma unroll
  for (int t = 0; t < LR; ++t) {
    const int n = R >> t;
    const int s = 16 >> t;
    const bool upper = (lane & s) != 0;
#pragma unroll
    for (int j = 0; j < n / 2; ++j) {
      float send = upper ? v[j] : v[j + n / 2];
      float keep = upper ? v[j + n / 2] : v[j];
      v[j] = keep + __shfl_xor_sync(FULL, send, s);
    }
  }
  float r = v[0];
#pragma unroll
  for (int s = 16 >> LR; s >= 1; s >>= 1) r += __shfl_xor_sync(FULL, r, s);
  return r;
}

// --------------------------------------------------- register queues (<=128)
// QR u64 registers per lane hold a sorted array of 32*QR keys: element
// e = r*32 + lane; unused slots are KEY_MAX.
template <int QR>
struct RegArr {
  uint64_t v[QR];

  __device__ __forceinline__ void clear() {
#pragma unroll
    for (int r = 0; r < QR; ++r) v[r] = KEY_MAX;
  }
  // element e (warp-uniform)
  // (mask-and-or over every register, not a select chain: nvcc turns a chain
  // keyed on a runtime index into an indexed local-memory access, which puts
  // the whole array on the stack)
  // (8 registers: the select chain, i.e. W indexed in local memory, measured
  // faster than 8 masked ORs per access — GloVe-IP L 160 1.63 vs 1.52 M QPS;
  // 2 / 4 registers: the masks — K = 100 6.11 -> 6.27 M, NYTimes 6.74 -> 6.91 M)
  __device__ __forceinline__ uint64_t get(int e) const {
    uint64_t x = 0;
    if constexpr (QR >= 8) {
      x = v[0];
#pragma unroll
      for (int r = 1; r < QR; ++r)
        if ((e >> 5) == r) x = v[r];
    } else {
#pragma unroll
      for (int r = 0; r < QR; ++r) x |= v[r] & (0ull - (uint64_t)((e >> 5) == r));
    }
    return __shfl_sync(FULL, x, e & 31);
  }
  // remove element 0 (the head), shifting the rest down
  __device__ __forceinline__ void pop_front(int lane) {
#pragma unroll
    for (int r = 0; r < QR; ++r) {
      uint64_t nxt = (r + 1 < QR) ? __shfl_sync(FULL, v[r + 1 < QR ? r + 1 : r], 0) : KEY_MAX;
      uint64_t d = __shfl_down_sync(FULL, v[r], 1);
      v[r] = (lane == 31) ? nxt : d;
    }
  }
  // insert x at its sorted position, capacity L; returns the evicted key
  // (old element L-1 when the array was full) or KEY_MAX
  __device__ __forceinline__ uint64_t insert_one(uint64_t x, int L, int lane) {
    int pos = 0;
#pragma unroll
    for (int r = 0; r < QR; ++r) pos += __popc(__ballot_sync(FULL, v[r] < x));
    const uint64_t evicted = get(L - 1);
    uint64_t prev[QR];
#pragma unroll
    for (int r = 0; r < QR; ++r) {
      uint64_t up = __shfl_up_sync(FULL, v[r], 1);
      uint64_t last = (r > 0) ? __shfl_sync(FULL, v[r > 0 ? r - 1 : 0], 31) : KEY_MAX;
      prev[r] = (lane == 0) ? last : up;
    }
#pragma unroll
    for (int r = 0; r < QR; ++r) {
      const int e = r * 32 + lane;
      uint64_t y = (e < pos) ? v[r] : ((e == pos) ? x : prev[r]);
      v[r] = (e < L) ? y : KEY_MAX;
    }
    return (pos < L) ? evicted : KEY_MAX;
  }
};

// Bitonic merge of the sorted queue q (QR regs) with 32 keys sorted
// DESCENDING (one reg): the 32*QR smallest stay in q (ascending) and the rest
// are returned in `out` (one reg, unordered, KEY_MAX where empty).  Entries of
// q at positions >= L are also moved out (to out2, one per lane per reg).
template <int QR>
__device__ __forceinline__ void merge_into(RegArr<QR>& q, uint64_t sdesc, int lane, uint64_t& out) {
  // first half-cleaner of the 64*QR-long bitonic sequence [q asc | MAX.. | s desc]
  // only touches the last q register (the MAX block pairs with the rest)
  {
    const bool lt = q.v[QR - 1] < sdesc;
    out = lt ? sdesc : q.v[QR - 1];
    q.v[QR - 1] = lt ? q.v[QR - 1] : sdesc;
  }
  // the lower half is bitonic: finish the merge (ascending)
#pragma unroll
  for (int m = QR / 2; m >= 1; m >>= 1) {
#pragma unroll
    for (int r = 0; r < QR; ++r) {
      if ((r & m) == 0) {
        const uint64_t a = q.v[r], b = q.v[r + m];
        const bool lt = a < b;
        q.v[r] = lt ? a : b;
        q.v[r + m] = lt ? b : a;
      }
    }
  }
#pragma unroll
  for (int j = 16; j >= 1; j >>= 1) {
    const bool lower = (lane & j) == 0;
#pragma unroll
    for (int r = 0; r < QR; ++r) {
      const uint64_t o = __shfl_xor_sync(FULL, q.v[r], j);
      q.v[r] = ((o < q.v[r]) == lower) ? o : q.v[r];
    }
  }
}

// ------------------------------------------- shared-memory queues (> 128)
// q and topk for queue_len > 128: sorted arrays in shared memory laid out as
// a TIERED VECTOR — blocks of 64 keys, each block a small ring with its own
// head, every block full except the last; lane c of the warp owns block c
// (queue_len <= 2048 = 32 blocks) and keeps its head in a register.  An
// insertion shifts keys inside ONE block and passes one key from each later
// block to the next (all lanes at once: each later block rotates by one
// slot); popping the minimum passes each block's first key down the same
// way.  So both are a constant number of warp operations whatever the queue
// length, where a flat sorted array moves O(L) keys per iteration (measured:
// ring moves were 45 % of the instructions at L = 1280).
struct Tier {
  uint64_t* a;  // nblk * 64 slots
  int size;     // logical elements (warp-uniform)
  int hd;       // lane c: physical offset of block c's first element
  __device__ __forceinline__ int nb() const { return (size + 63) >> 6; }
  // element i (per lane, 0 <= i < 32 * 64); every lane of the warp must call
  __device__ __forceinline__ uint64_t at(int i) const {
    const int b = (i >> 6) & 31;
    const int h = __shfl_sync(FULL, hd, b);
    return a[(b << 6) | ((h + i) & 63)];
  }
  // number of elements < x, x per lane (uniform trip count)
  __device__ __forceinline__ int rank_lane(uint64_t x) const {
    const int n = size;
    int lo = 0;
    for (int step = 1 << (31 - __clz(n | 1)); step > 0; step >>= 1) {
      const int j = lo + step - 1;
      const uint64_t v = at(j < n ? j : 0);
      lo = (j < n && v < x) ? lo + step : lo;
    }
    return lo;
  }
  // number of elements < x, x warp-uniform: the block (first keys, one per
  // lane), then the position inside it (two keys per lane)
  __device__ __forceinline__ int rank_warp(uint64_t x, int lane) const {
    const int n = size, nbk = nb();
    const uint64_t first = lane < nbk ? a[(lane << 6) | hd] : KEY_MAX;
    const int k = __popc(__ballot_sync(FULL, first < x));  // blocks starting below x
    if (k == 0) return 0;
    const int b = k - 1;
    const int cnt = min(64, n - (b << 6));
    const int h = __shfl_sync(FULL, hd, b);
    const uint64_t e0 = a[(b << 6) | ((h + lane) & 63)];
    const uint64_t e1 = a[(b << 6) | ((h + lane + 32) & 63)];
    return (b << 6) + __popc(__ballot_sync(FULL, lane < cnt && e0 < x)) +
           __popc(__ballot_sync(FULL, lane + 32 < cnt && e1 < x));
  }
  // insert x (warp-uniform, not present) at its sorted position; the caller
  // keeps size < 32 * 64 and within its block budget
  __device__ __forceinline__ int insert(uint64_t x, int lane) {
    const int n = size, nbk = nb();
    if (nbk == 0) {  // empty: x opens block 0
      if (lane == 0) {
        hd = 0;
        a[0] = x;
      }
      __syncwarp();
      size = 1;
      return 0;
    }
    // every block's first and (if full) last key at once: the first keys find
    // x's block b (the last one starting below x), the last keys are what the
    // cascade passes on
    const uint64_t first = lane < nbk ? a[(lane << 6) | hd] : KEY_MAX;
    const uint64_t last = (lane < nbk && ((lane + 1) << 6) <= n) ? a[(lane << 6) | ((hd + 63) & 63)] : 0;
    const int k = __popc(__ballot_sync(FULL, first < x));
    const int b = k > 0 ? k - 1 : 0;
    const int hb = __shfl_sync(FULL, hd, b);
    const int cnt = min(64, n - (b << 6));
    const int s0 = (b << 6) | ((hb + lane) & 63), s1 = (b << 6) | ((hb + lane + 32) & 63);
    const uint64_t e0 = a[s0], e1 = a[s1];
    // o = keys of block b below x (0..cnt); o == 64: x follows a full block b
    // and is itself what b passes on
    const int o = __popc(__ballot_sync(FULL, lane < cnt && e0 < x)) +
                  __popc(__ballot_sync(FULL, lane + 32 < cnt && e1 < x));
    const uint64_t v = (lane == b && o == 64) ? x : last;  // block c passes v on
    const uint64_t vin = __shfl_up_sync(FULL, v, 1);       // lane c: block c - 1's
    const uint64_t up0 = __shfl_up_sync(FULL, e0, 1), up1 = __shfl_up_sync(FULL, e1, 1);
    const uint64_t e0_31 = __shfl_sync(FULL, e0, 31);
    __syncwarp();
    // block b: offsets k <= cnt (k < 64) take old[k] (k < o), x (k = o) or
    // old[k - 1] (k > o); old[63] of a full block left as `last`
    if (o < 64) {
      const int k0 = lane, k1 = lane + 32;
      const uint64_t p1 = lane == 0 ? e0_31 : up1;
      if (k0 <= cnt) a[s0] = k0 < o ? e0 : (k0 == o ? x : up0);
      if (k1 <= cnt && k1 < 64) a[s1] = k1 < o ? e1 : (k1 == o ? x : p1);
    }
    // later blocks rotate by one slot and take the previous block's last key
    if (lane > b && lane < nbk) {
      hd = (hd + 63) & 63;
      a[(lane << 6) | hd] = vin;
    } else if (lane == nbk && (n & 63) == 0) {  // the last block was full: a new block
      hd = 0;
      a[lane << 6] = vin;
    }
    __syncwarp();
    size = n + 1;
    return (b << 6) + o;
  }
  // reading R17: set the popped mark (bit 0 of a W key) of element i
  __device__ __forceinline__ void set_flag(int i, int lane) {
    const int b = (i >> 6) & 31;
    const int h = __shfl_sync(FULL, hd, b);
    if (lane == 0) a[(b << 6) | ((h + i) & 63)] |= 1ull;
    __syncwarp();
  }
  // R17: index of the first element >= i without the popped mark, or size
  __device__ __forceinline__ int next_unpopped(int i, int lane) const {
    for (; i < size; i += 32) {
      const int j = i + lane;
      const uint64_t v = at(j < size ? j : 0);
      const unsigned m = __ballot_sync(FULL, j < size && !(v & 1ull));
      if (m) return i + __ffs(m) - 1;
    }
    return size;
  }
  // remove the minimum (element 0)
  __device__ __forceinline__ void pop_front(int lane) {
    const int nbk = nb();
    const uint64_t fo = lane < nbk ? a[(lane << 6) | hd] : 0;
    const uint64_t fin = __shfl_down_sync(FULL, fo, 1);  // lane c: block c + 1's first key
    __syncwarp();
    if (lane < nbk) {
      const int old = hd;
      hd = (hd + 1) & 63;
      if (lane < nbk - 1) a[(lane << 6) | old] = fin;  // the freed slot is block c's last
    }
    __syncwarp();
    --size;
  }
  // topk insertion (§IV-C, Alg. 1 line 7): insert x (x < the maximum when
  // full); returns the evicted maximum (old element L-1 when full) or KEY_MAX
  __device__ __forceinline__ uint64_t push1(uint64_t x, int L, int lane) {
    uint64_t ev = KEY_MAX;
    if (size == L) {
      ev = at(L - 1);
      --size;
    }
    insert(x, lane);
    return ev;
  }
};

// ------------------------------------------------------- bulk distance --
// §VI: distances of the nc candidates whose ids are in cid[0..nc) (shared).
// Rows are staged R at a time in `stage` by cp.async (LDGSTS, 16 B per lane
// per row, L1-bypassing): every row of the round is in flight at once with no
// register cost, then each lane reads back only its own 16 B slices (no
// cross-lane hazard) and a transposed butterfly reduces the R partial sums.
// Lane j (< nc) receives candidate j's distance.  NCH = 16 B chunks per lane.
#ifndef SONG_STAGE_ROWS
#define SONG_STAGE_ROWS 8
#endif
#ifndef SONG_L2_PREFETCH
#define SONG_L2_PREFETCH 2
#endif
#ifndef SONG_BULK_PF_NCH
#define SONG_BULK_PF_NCH 2
#endif
// rows prefetched ahead for rows of >= SONG_PF_WINDOW_NCH chunks per lane
// (32 = every later row at once).  GIST L 24 (1K queries x 10): window 32 /
// 16 / 8 / 6 / 4 / 2 = 4.12 / 4.21 / 4.27 / 4.28 / 4.31 / 4.39 M QPS;
// MNIST8m-shaped original vectors (25 GB, no reuse) at L 48: 1.11 M (32),
// 1.32 M (8), 1.48 M (4), 1.49 M (2) — 1.47 M with 8-row rounds; the 1 KB /
// 800 B rows of NYTimes / GloVe lose 0.5-2 % with a window (r03aq / r03ar A/B)
#ifndef SONG_PF_WINDOW
#define SONG_PF_WINDOW 2
#endif
#ifndef SONG_PF_WINDOW_NCH
#define SONG_PF_WINDOW_NCH 8
#endif
#ifndef SONG_STAGE_BUFS
#define SONG_STAGE_BUFS 1
#endif
#ifdef SONG_DIST_TEAM
constexpr bool kDistTeam = true;   // row-team distance path (query in shared memory)
#else
constexpr bool kDistTeam = false;  // lane-slice distance path (query in registers)
#endif
#ifndef SONG_UNION_WIDE_ROWS
#define SONG_UNION_WIDE_ROWS 4
#endif
// rows per round for rows wider than 256 floats (GIST-shaped, 3.75 KB rows):
// with one bulk L2 prefetch per later-round row, 2 rows per round at 16
// resident warps beat 4 (11 warps) and 8 (6 warps): GIST L = 24 4.12 / 3.93 /
// 3.27 M QPS (r03ak); with per-line prefetches 8 rows had won (2.67 vs 2.38 /
// 2.13 M, r03n / r03o)
#ifndef SONG_XWIDE_ROWS
#define SONG_XWIDE_ROWS 2
#endif
#ifndef SONG_XWIDE_LB_BLOCKS  // CTAs of 128 threads per SM the wide-row kernels are compiled for
#define SONG_XWIDE_LB_BLOCKS 4
#endif
#ifndef SONG_WIDE_ROWS  // rows per round for 129-256 floats (NYTimes / GloVe-shaped)
#define SONG_WIDE_ROWS 4
#endif
template <int NCH, bool UNION = false>
struct StageRows {  // rows per round: SONG_STAGE_ROWS for 128-float rows, 4 for wider ones
  // (NYTimes-shaped, 256 floats: 8 -> 4 rows frees 4 KB per warp, 14 -> 19 resident warps,
  // +12 % QPS; SIFT-shaped rows keep 8: at equal residency 4 rows cost 9 %)
  static constexpr int R = (NCH >= 2) ? (UNION ? SONG_UNION_WIDE_ROWS : NCH >= 4 ? SONG_XWIDE_ROWS : SONG_WIDE_ROWS)
                                      : SONG_STAGE_ROWS;
  static constexpr int NBUF = SONG_STAGE_BUFS;  // rounds in flight
};

__device__ __forceinline__ void cp_async16(void* dst, const void* src) {
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(smem_u32(dst)), "l"(src)
               : "memory");
}

// predicated form: no branch around the copy
__device__ __forceinline__ void cp_async16_if(bool p, uint32_t dst, const void* src) {
  asm volatile(
      "{\n\t.reg .pred q;\n\tsetp.ne.b32 q, %2, 0;\n\t"
      "@q cp.async.cg.shared.global [%0], [%1], 16;\n\t}" ::"r"(dst),
      "l"(src), "r"((int)p)
      : "memory");
}

__device__ __forceinline__ void cp_async_wait_all() {
  asm volatile("cp.async.wait_all;" ::: "memory");
}

// packed fp32x2 arithmetic (sm_100: FADD2 / FFMA2)
__device__ __forceinline__ uint64_t f2pack(float lo, float hi) {
  uint64_t r;
  asm("mov.b64 %0, {%1, %2};" : "=l"(r) : "f"(lo), "f"(hi));
  return r;
}

__device__ __forceinline__ float f2sum(uint64_t v) {
  float lo, hi;
  asm("mov.b64 {%0, %1}, %2;" : "=f"(lo), "=f"(hi) : "l"(v));
  return lo + hi;
}

template <int METRIC>
__device__ __forceinline__ uint64_t acc4(uint64_t acc, uint64_t q01, uint64_t q23, float4 x) {
#ifdef SONG_SCALAR_FMA
  float a0, a1, q0, q1, q2, q3;
  asm("mov.b64 {%0, %1}, %2;" : "=f"(a0), "=f"(a1) : "l"(acc));
  asm("mov.b64 {%0, %1}, %2;" : "=f"(q0), "=f"(q1) : "l"(q01));
  asm("mov.b64 {%0, %1}, %2;" : "=f"(q2), "=f"(q3) : "l"(q23));
  if (METRIC == MET_L2) {
    float t0 = q0 - x.x, t1 = q1 - x.y, t2 = q2 - x.z, t3 = q3 - x.w;
    a0 = fmaf(t0, t0, a0); a1 = fmaf(t1, t1, a1); a0 = fmaf(t2, t2, a0); a1 = fmaf(t3, t3, a1);
  } else {
    a0 = fmaf(q0, x.x, a0); a1 = fmaf(q1, x.y, a1); a0 = fmaf(q2, x.z, a0); a1 = fmaf(q3, x.w, a1);
  }
  return f2pack(a0, a1);
#endif
  const uint64_t x01 = f2pack(x.x, x.y), x23 = f2pack(x.z, x.w);
  if (METRIC == MET_L2) {
    uint64_t d01, d23;
    asm("sub.rn.f32x2 %0, %1, %2;" : "=l"(d01) : "l"(q01), "l"(x01));
    asm("sub.rn.f32x2 %0, %1, %2;" : "=l"(d23) : "l"(q23), "l"(x23));
    asm("fma.rn.f32x2 %0, %1, %1, %0;" : "+l"(acc) : "l"(d01));
    asm("fma.rn.f32x2 %0, %1, %1, %0;" : "+l"(acc) : "l"(d23));
  } else {
    asm("fma.rn.f32x2 %0, %1, %2, %0;" : "+l"(acc) : "l"(q01), "l"(x01));
    asm("fma.rn.f32x2 %0, %1, %2, %0;" : "+l"(acc) : "l"(q23), "l"(x23));
  }
  return acc;
}

__device__ __forceinline__ void cp_async_commit() {
  asm volatile("cp.async.commit_group;" ::: "memory");
}

// wait until at most n committed groups of this thread are still in flight
__device__ __forceinline__ void cp_async_wait_pending(int n) {
  if (n <= 0)
    asm volatile("cp.async.wait_group 0;" ::: "memory");
  else if (n == 1)
    asm volatile("cp.async.wait_group 1;" ::: "memory");
  else if (n == 2)
    asm volatile("cp.async.wait_group 2;" ::: "memory");
  else
    asm volatile("cp.async.wait_group 3;" ::: "memory");
}

// Rounds of R rows are software-pipelined over NBUF stage buffers: round k+1
// (and k+2 ...) are in flight while round k is reduced.  Staged rows have a
// compile-time stride of 128*NCH floats (512*NCH bytes) so every shared-memory
// address is an immediate offset; lane j holds candidate j's row pointer and
// rows are broadcast with SHFL (an LDS-sourced address makes ptxas pad every
// LDGSTS with three dummy LDS).
template <int NCH>
struct Stage {
  static constexpr int STRIDE = 128 * NCH;  // floats per staged row
};

// first chunk: no accumulator input (FMUL2 instead of a zeroed FFMA2)
template <int METRIC>
__device__ __forceinline__ uint64_t acc4_first(uint64_t q01, uint64_t q23, float4 x) {
  const uint64_t x01 = f2pack(x.x, x.y), x23 = f2pack(x.z, x.w);
  uint64_t acc;
  if (METRIC == MET_L2) {
    uint64_t d01, d23;
    asm("sub.rn.f32x2 %0, %1, %2;" : "=l"(d01) : "l"(q01), "l"(x01));
    asm("sub.rn.f32x2 %0, %1, %2;" : "=l"(d23) : "l"(q23), "l"(x23));
    asm("mul.rn.f32x2 %0, %1, %1;" : "=l"(acc) : "l"(d01));
    asm("fma.rn.f32x2 %0, %1, %1, %0;" : "+l"(acc) : "l"(d23));
  } else {
    asm("mul.rn.f32x2 %0, %1, %2;" : "=l"(acc) : "l"(q01), "l"(x01));
    asm("fma.rn.f32x2 %0, %1, %2, %0;" : "+l"(acc) : "l"(q23), "l"(x23));
  }
  return acc;
}

// zero this lane's slices of every staged row once per launch: slices past
// dpad are never written by the copies, so they keep contributing 0
template <int NCH>
__device__ __forceinline__ void zero_stage(float* stage, int rows, int lane) {
  float4* s4 = reinterpret_cast<float4*>(stage);
  for (int i = lane; i < rows * 32 * NCH; i += 32) s4[i] = make_float4(0.f, 0.f, 0.f, 0.f);
  __syncwarp();
}

// Hamming distance (§VII; reading R12): a code is dpad <= 4*NCH words
// (dpad = 1, 2 or a multiple of 4),
// so lane j gathers candidate j's whole code with NCH 16 B loads — all the
// warp's rows in flight at once, no staging and no cross-lane reduction — and
// XOR-popcounts it against the query code every lane holds in qv.
template <int NCH>
__device__ __forceinline__ float hamming_distance(const float* __restrict__ data, int dpad,
                                                  const int* cid, int nc,
                                                  const float4 (&qv)[NCH], int lane) {
  int d = 0;
  if (dpad < 4) {  // 32- and 64-bit codes are stored unpadded (1 or 2 words)
    if (lane < nc) {
      const uint32_t* w = reinterpret_cast<const uint32_t*>(data) + (int64_t)cid[lane] * dpad;
      if (dpad == 2) {
        const uint2 v = __ldg(reinterpret_cast<const uint2*>(w));
        d = __popc(v.x ^ __float_as_uint(qv[0].x)) + __popc(v.y ^ __float_as_uint(qv[0].y));
      } else {
        d = __popc(__ldg(w) ^ __float_as_uint(qv[0].x));
      }
    }
  } else if (lane < nc) {
    const uint4* row = reinterpret_cast<const uint4*>(data + (int64_t)cid[lane] * dpad);
    uint4 v[NCH];
#pragma unroll
    for (int c = 0; c < NCH; ++c)
      v[c] = (4 * c < dpad) ? __ldg(row + c) : make_uint4(0u, 0u, 0u, 0u);
#pragma unroll
    for (int c = 0; c < NCH; ++c)
      d += __popc(v[c].x ^ __float_as_uint(qv[c].x)) + __popc(v[c].y ^ __float_as_uint(qv[c].y)) +
           __popc(v[c].z ^ __float_as_uint(qv[c].z)) + __popc(v[c].w ^ __float_as_uint(qv[c].w));
  }
  return (float)d;  // exact: d <= 32 * dpad < 2^24
}

template <int NCH, int METRIC, bool UNION = false>
__device__ __forceinline__ float bulk_distance(const float* __restrict__ data, int dpad,
                                               const int* cid, int nc, const float4 (&qv)[NCH],
                                               float* stage, int cosine, int lane) {
  if constexpr (METRIC == MET_HAM) return hamming_distance<NCH>(data, dpad, cid, nc, qv, lane);
  constexpr int R = StageRows<NCH, UNION>::R;
  constexpr int NBUF = StageRows<NCH, UNION>::NBUF;
  constexpr int LR = Log2<R>::value;
  constexpr int G = R < 8 ? R : 8;  // rows per uniform compute group
  constexpr int SR = Stage<NCH>::STRIDE;
  const int d4 = dpad >> 2;
  float mine = 0.0f;
  uint64_t q01[NCH], q23[NCH];
  bool mine_chunk[NCH];  // does this lane own 16 B slice c of a row?
#pragma unroll
  for (int c = 0; c < NCH; ++c) {
    q01[c] = f2pack(qv[c].x, qv[c].y);
    q23[c] = f2pack(qv[c].z, qv[c].w);
    mine_chunk[c] = c * 32 + lane < d4;
  }
  // lane j holds candidate j's id; a row's address for this lane is one
  // IMAD.WIDE: id * rowbytes + (data + 16 B * lane)
  const uint32_t myid = lane < nc ? (uint32_t)cid[lane] : 0u;
  const uint32_t rowbytes = 4u * (uint32_t)dpad;
  const char* lane_base = reinterpret_cast<const char*>(data) + 16 * lane;
  const int rounds = (nc + R - 1) / R;
  const uint32_t stage_s = smem_u32(stage) + 16u * lane;
  auto issue = [&](int k) {
    const uint32_t dst0 = stage_s + (uint32_t)((k % NBUF) * R * SR * 4);
    const int rows = min(R, nc - k * R);
#pragma unroll
    for (int rr = 0; rr < R; ++rr) {
      const uint32_t id = __shfl_sync(FULL, myid, (k * R + rr) & 31);
      const float4* src = reinterpret_cast<const float4*>(lane_base + (uint64_t)id * rowbytes);
#pragma unroll
      for (int c = 0; c < NCH; ++c)
        cp_async16_if(rr < rows && mine_chunk[c], dst0 + (uint32_t)(rr * SR * 4 + 512 * c),
                      src + c * 32);
    }
    cp_async_commit();
  };
  for (int k = 0; k < NBUF && k < rounds; ++k) issue(k);
#if SONG_L2_PREFETCH
  // rows of the later rounds start their DRAM trip now: each such lane asks
  // L2 for its own candidate's row, so round k >= NBUF waits on an L2 hit
  // instead of a second dependent DRAM round trip
  // (rows of >= SONG_BULK_PF_NCH chunks per lane: one bulk L2 prefetch per
  // row; narrower rows: one prefetch per 128 B line — GIST's 3.75 KB rows
  // 2.95 -> 3.27 M QPS with the bulk form, NYTimes' 1 KB rows 6.48 -> 6.69 M,
  // GloVe's 800 B rows unchanged, SIFT's 512 B rows 20.9 -> 19.9 M: kept
  // per line; profiles r03ah / r03ai A/B)
  // Rows of >= 8 chunks per lane keep at most SONG_PF_WINDOW rows prefetched
  // ahead of the staged rounds (a rolling window, advanced one round at a
  // time below): prefetching every later row at once overflows L2 when the
  // rows have no reuse (MNIST8m-shaped 25 GB index).
  constexpr int PFW = NCH >= SONG_PF_WINDOW_NCH ? SONG_PF_WINDOW : 32;
  auto prefetch_rows = [&](int lo, int hi) {  // lanes lo <= lane < hi prefetch their row
    if (lane >= lo && lane < hi && lane < nc) {
      const char* row = reinterpret_cast<const char*>(data) + (uint64_t)myid * rowbytes;
      if (SONG_L2_PREFETCH == 1 || NCH >= SONG_BULK_PF_NCH) {
        asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(row), "r"(rowbytes) : "memory");
      } else {
        for (uint32_t o = 0; o < rowbytes; o += 128)
          asm volatile("prefetch.global.L2 [%0];" ::"l"(row + o));
      }
    }
  };
  prefetch_rows(NBUF * R, NBUF * R + PFW);
#endif
  for (int k = 0; k < rounds; ++k) {
    const int b = k * R;
    const int rows = min(R, nc - b);
    cp_async_wait_pending(min(NBUF - 1, rounds - 1 - k));
    // ---- compute: lane owns its 16 B slices of every staged row
    const float* buf = stage + (size_t)(k % NBUF) * R * SR;
    float part[R];
#pragma unroll
    for (int g = 0; g < R; g += G) {
      if (g < rows) {
#pragma unroll
        for (int r = g; r < g + G; ++r) {
          const float4* row = reinterpret_cast<const float4*>(buf + r * SR) + lane;
          // (slices past dpad stay zero in the stage and in the query: they add 0)
          uint64_t acc = acc4_first<METRIC>(q01[0], q23[0], row[0]);
#pragma unroll
          for (int c = 1; c < NCH; ++c) acc = acc4<METRIC>(acc, q01[c], q23[c], row[c * 32]);
          part[r] = f2sum(acc);
        }
      } else {
#pragma unroll
        for (int r = g; r < g + G; ++r) part[r] = 0.0f;
      }
    }
    // buffer k % NBUF is free again (this lane read only its own slices)
    if (k + NBUF < rounds) issue(k + NBUF);
#if SONG_L2_PREFETCH
    if (PFW < 32 && (k + NBUF + 1) * R + PFW - R < nc)  // slide the window by one round
      prefetch_rows((k + NBUF) * R + PFW, (k + NBUF + 1) * R + PFW);
#endif
    const float tot = transpose_reduce<R>(part, lane);
    const float got = __shfl_sync(FULL, tot, ((lane - b) & (R - 1)) << (5 - LR));
    if (lane >= b && lane < b + R) mine = got;
  }
  if (METRIC == MET_DOT) mine = cosine ? 1.0f - mine : -mine;  // 1 - cos / -<q,x>
  return mine;
}

// Bulk distance, row-team layout (default).  A round stages R rows; each row
// is owned by a team of LPR = 32 / R consecutive lanes and lane g of the team
// copies (cp.async) AND later reads exactly chunks g, g + LPR, g + 2 LPR ... of
// that row, so no lane ever reads another lane's copy (no warp barrier between
// copy and compute), one row address per lane replaces a SHFL + IMAD per row,
// and the reduction is log2(LPR) shuffles instead of a transposed butterfly.
// The query sits in shared memory (qsm, 16 B chunks, zero past dpad) and is
// read with LPR-way broadcast.  Chunk ch of row r is stored at ch ^ swz(r)
// (rows r and r + 1 of an 8-lane LDS.128 phase land in opposite 64 B halves),
// so both the copies and the reads are bank-conflict free.
template <int NCH>
struct Team {
  static constexpr int R = StageRows<NCH>::R;  // rows per round
  static constexpr int LPR = 32 / R;           // lanes per row
  static constexpr int CPL = 32 * NCH / LPR;   // chunks per lane
  __device__ __forceinline__ static int swz(int r) { return LPR == 4 ? ((r & 1) << 2) : 0; }
};

template <int NCH, int METRIC>
__device__ __forceinline__ float bulk_distance_team(const float* __restrict__ data, int dpad,
                                                    const int* cid, int nc, const float* qsm,
                                                    float* stage, int cosine, int lane) {
  using T = Team<NCH>;
  constexpr int R = T::R, LPR = T::LPR, CPL = T::CPL;
  constexpr int SR = Stage<NCH>::STRIDE;  // floats per staged row
  const int d4 = dpad >> 2;
  const int r = lane / LPR;  // row of this lane within a round
  const int g = lane % LPR;  // chunk phase of this lane
  const int sw = T::swz(r);
  const int myc = d4 > g ? (d4 - g + LPR - 1) / LPR : 0;  // my chunks inside the row
  const bool full = myc >= CPL;
  const uint32_t rowbytes = 4u * (uint32_t)dpad;
  const uint32_t st_row = smem_u32(stage) + (uint32_t)(r * SR * 4);
  const float4* q4 = reinterpret_cast<const float4*>(qsm);
  const float4* srow = reinterpret_cast<const float4*>(stage + r * SR);
  constexpr int NBUF = StageRows<NCH>::NBUF;  // rounds in flight
  const int rounds = (nc + R - 1) / R;
  float mine = 0.0f;
  // ---- copy: this lane's chunks of row k*R + r into stage buffer k % NBUF
  auto issue = [&](int k) {
    const int j = k * R + r;
    if (j < nc) {
      const char* src = reinterpret_cast<const char*>(data) + (uint64_t)(uint32_t)cid[j] * rowbytes;
      const uint32_t dst = st_row + (uint32_t)((k % NBUF) * R * SR * 4);
#pragma unroll
      for (int c = 0; c < CPL; ++c) {
        const int ch = g + LPR * c;
        if (full || c < myc)
          asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(dst + (uint32_t)((ch ^ sw) * 16)),
                       "l"(src + ch * 16)
                       : "memory");
      }
    }
    cp_async_commit();
  };
  for (int k = 0; k < NBUF && k < rounds; ++k) issue(k);
  for (int k = 0; k < rounds; ++k) {
    const int j = k * R + r;
    cp_async_wait_pending(min(NBUF - 1, rounds - 1 - k));
    // ---- compute: the same chunks, read back by the lane that copied them
    const float4* buf = srow + (size_t)(k % NBUF) * R * SR / 4;
    float part = 0.0f;
    if (j < nc) {
      uint64_t acc = 0;
#pragma unroll 8
      for (int c = 0; c < CPL; ++c) {
        const int ch = g + LPR * c;
        const float4 x = buf[ch ^ sw];  // (chunks past dpad hold 0, like the query)
        const float4 qq = q4[ch];
        const uint64_t q01 = f2pack(qq.x, qq.y), q23 = f2pack(qq.z, qq.w);
        acc = (c == 0) ? acc4_first<METRIC>(q01, q23, x) : acc4<METRIC>(acc, q01, q23, x);
      }
      part = f2sum(acc);
    }
    if (k + NBUF < rounds) issue(k + NBUF);  // (this lane read only its own chunks)
#pragma unroll
    for (int o = 1; o < LPR; o <<= 1) part += __shfl_xor_sync(FULL, part, o);
    const int b = k * R;
    const float got = __shfl_sync(FULL, part, ((lane - b) & (R - 1)) * LPR);
    if (lane >= b && lane < b + R) mine = got;
  }
  if (METRIC == MET_DOT) mine = cosine ? 1.0f - mine : -mine;  // 1 - cos / -<q,x>
  return mine;
}

// the distance stage used by the kernel: codes -> Hamming; float rows -> the
// lane-slice + transposed butterfly path, or the row-team path with
// SONG_DIST_TEAM (fewer instructions, but measured slower at 1 buffer: see
// profiles/r01_history.md)
template <int NCH, int METRIC, bool UNION = false>
__device__ __forceinline__ float dist_of(const float* __restrict__ data, int dpad, const int* cid,
                                         int nc, const float4 (&qv)[NCH], const float* qsm,
                                         float* stage, int cosine, int lane) {
#ifndef SONG_DIST_TEAM
  return bulk_distance<NCH, METRIC, UNION>(data, dpad, cid, nc, qv, stage, cosine, lane);
#else
  if constexpr (METRIC == MET_HAM) return hamming_distance<NCH>(data, dpad, cid, nc, qv, lane);
  return bulk_distance_team<NCH, METRIC>(data, dpad, cid, nc, qsm, stage, cosine, lane);
#endif
}

// ---------------------------------------------------------- the kernel --
#ifndef SONG_LB_THREADS
#define SONG_LB_THREADS 128
#endif
#ifndef SONG_LB_BLOCKS
#define SONG_LB_BLOCKS 6
#endif
// QR > 0: q / topk in registers (queue_len <= 32*QR); QR == 0: shared memory.
// wide rows (NCH >= 4: d > 256 floats, or 512/1024-bit codes) hold 4-8 float4
// of query per lane: give them 128 registers (4 CTAs/SM) instead of spilling
// shared-memory queues (QR == 0) are held to <= 20 warps per SM by their
// shared memory anyway: 5 CTAs give them 102 registers (the ring moves keep
// 4 keys per lane in flight) instead of spilling at 80
// union in registers: up to this many selected keys are inserted one at a
// time (measured 0 / 2 / 4: SIFT L 16 20.75 / 21.01 / 20.87 M QPS, K = 100
// 6.02 / 6.06 / 6.06 M, NYTimes 6.47 / 6.49 / 6.51 M; profiles r03ae A/B)
// the union in registers reuses the locate probe's empty slot for the insert
// of every candidate (lazy deletion: no tombstones, so the same slots a probe
// would take): K = 100 6.23 -> 6.36 M QPS, NYTimes +0.8 %, SIFT L 16 +0.2 %
// (r03be A/B, bit-exact); W in 8 registers keeps the probing insert (GloVe-IP
// L 160 1.63 vs 1.56 M, r03bg)
#ifndef SONG_SLOT_REUSE
#define SONG_SLOT_REUSE 1
#endif
#ifndef SONG_RUN_INS_MAX
#define SONG_RUN_INS_MAX 2
#endif
// the union with W in registers (QR > 8) needs fewer registers than separate
// q / topk: 7 CTAs (72 registers, 28 warps per SM where shared memory allows)
// measured SIFT1M L 16 20.0 -> 20.6 M QPS (8 CTAs / 64 registers: 20.4 M;
// K = 100 and NYTimes, held by shared memory, unchanged; profiles/r03s_*)
#ifndef SONG_RUN_LB_BLOCKS
#define SONG_RUN_LB_BLOCKS 7
#endif
#ifndef SONG_RUN8_LB_BLOCKS  // W in 8 registers (queue_len 129-256)
#define SONG_RUN8_LB_BLOCKS 7
#endif
template <int NCH, int QR = 1>
struct MinBlocks {
  static constexpr int value =
      NCH >= 4 ? SONG_XWIDE_LB_BLOCKS
               : (QR == 0 ? 5 : QR == 16 ? SONG_RUN8_LB_BLOCKS : QR > 8 ? SONG_RUN_LB_BLOCKS : SONG_LB_BLOCKS);
};
// MS: multi-step probing (a.steps pops per iteration, <= MAX_STEPS; §V)
constexpr int MAX_STEPS = 4;
template <int NCH, int METRIC, int VK, int QR, bool MS = false>
__global__ void __launch_bounds__(SONG_LB_THREADS, MinBlocks<NCH, QR>::value)
    song_search_kernel(const SearchArgs a) {
  extern __shared__ __align__(128) unsigned char smem[];
  constexpr int R = StageRows<NCH, (QR < 0)>::R;
  constexpr bool DEL = (VK == VK_HASH || VK == VK_CUCKOO);  // visited deletion (§IV-E)
  // QR in 1..4: q / topk in registers; QR == 0: separate q and topk tiers in
  // shared memory; QR < 0: reading R17, one bounded list W of q ∪ topk in
  // shared-memory tiers; QR = 8 + r (r = 1, 2, 4): R17's W in r registers per
  // lane (queue_len <= 128)
  constexpr bool RUN = QR > 8;    // R17, W in registers
  constexpr bool UNQ = QR < 0;    // R17, W in shared-memory tiers
  constexpr bool UNI = UNQ || RUN;  // R17 semantics (either storage)
  constexpr bool REG = QR > 0 && !RUN;  // separate q / topk in registers
  constexpr bool GVT = QR == -2;  // R17 with the visited table in global memory
  // the locate probe hands each candidate's insert slot to the insert (the
  // global tables; the union in registers with SONG_SLOT_REUSE)
  constexpr bool SLOT = GVT || (RUN && QR < 16 && SONG_SLOT_REUSE && VK == VK_HASH);
  constexpr int QRr = RUN ? QR - 8 : QR > 0 ? QR : 1;
  const int lane = threadIdx.x & 31;
  const int warp = threadIdx.x >> 5;
  const int L = a.L;
  unsigned char* base = smem + (size_t)warp * a.warp_smem_bytes;
  float* stage = reinterpret_cast<float*>(base);                       // staged rows
  const size_t stage_bytes =  // (Hamming codes are gathered straight into registers)
      METRIC == MET_HAM ? 0 : (size_t)StageRows<NCH, (QR < 0)>::NBUF * R * Stage<NCH>::STRIDE * 4;
  // the query, 16 B chunks (row-team distance path)
  float* qsm = reinterpret_cast<float*>(base + stage_bytes);
  constexpr size_t qsm_bytes = (METRIC == MET_HAM || !kDistTeam) ? 0 : (size_t)NCH * 512;
  int* cid = reinterpret_cast<int*>(base + stage_bytes + qsm_bytes + 16);
  uint64_t* keys32 = reinterpret_cast<uint64_t*>(cid + (MS ? 32 * MAX_STEPS : 32));  // 32 keys
  uint64_t* ev = keys32 + 32;                                           // 32 evicted keys
  // QR == 0 only: q and topk as tiered vectors of ceil(L / 64) blocks
  const int tslots = QR <= 0 ? ((L + 63) >> 6) << 6 : 0;
  // (the evicted-key list only for the Cuckoo filter, the insert slots only
  // for GVT: the other kernels give those bytes to more resident warps)
  int* cslot = reinterpret_cast<int*>(ev + (VK == VK_CUCKOO ? 32 : 0));  // GVT: each candidate's insert slot
  uint64_t* qa = reinterpret_cast<uint64_t*>(cslot + (SLOT ? 32 : 0));  // q (or W, R17)
  uint64_t* tk = qa + tslots;                   // topk (QR == 0 only)
  const int tkslots = QR == 0 ? tslots : 0;
  int* table = GVT ? a.gvis + ((size_t)blockIdx.x * (blockDim.x >> 5) + warp) * ((size_t)1 << a.table_log2)
                  : reinterpret_cast<int*>(                             // 16 B aligned
                        (reinterpret_cast<uintptr_t>(tk + tkslots) + 15) & ~uintptr_t(15));
  // 32-bit words of the shared-memory visited table
  const int twords = VK == VK_HASH    ? (1 << a.table_log2)
                     : VK == VK_BLOOM ? ((1 << a.table_log2) >> 5)
                     : VK == VK_CUCKOO ? (2 << a.table_log2)  // 4 x u16 per bucket
                                       : 0;
  HashSetT<GVT> hs{table, a.table_log2};
  BloomSet bs{reinterpret_cast<uint32_t*>(table), a.table_log2};
  CuckooSet cs{reinterpret_cast<uint16_t*>(table), a.table_log2};
  GHash gh{a.gtab + ((size_t)blockIdx.x * (blockDim.x >> 5) + warp) * ((size_t)1 << a.table_log2),
           a.table_log2, a.gen0};
  const unsigned lt = lanemask_lt();
  if (METRIC != MET_HAM) zero_stage<NCH>(stage, StageRows<NCH, (QR < 0)>::NBUF * R, lane);

  // ---- visited-set operations (§IV-B/D/E) for the four kinds
  auto v_contains = [&](int v, bool act) -> bool {
    if constexpr (VK == VK_HASH) return hs.contains(v, act);
    if constexpr (VK == VK_BLOOM) return bs.contains(v, act);
    if constexpr (VK == VK_GHASH) return gh.contains(v, act);
    if constexpr (VK == VK_CUCKOO) return cs.contains(v, act);
    return false;
  };
  // single-lane insert / erase (entry vertex, topk eviction)
  auto v_insert_lane0 = [&](int v) {
    if constexpr (VK == VK_HASH) hs.insert(v, lane == 0);
    if constexpr (VK == VK_BLOOM) bs.insert(v, lane == 0);
    if constexpr (VK == VK_GHASH) gh.insert(v, lane == 0);
    if constexpr (VK == VK_CUCKOO) {
      if (lane == 0) cs.insert1(v);
      __syncwarp();
    }
  };
  auto v_erase_lane0 = [&](uint64_t k) {
    if constexpr (VK == VK_HASH) hs.erase(key_id(k), k != KEY_MAX && lane == 0 && !a.lazy);
    if constexpr (VK == VK_CUCKOO) {
      if (lane == 0 && k != KEY_MAX) cs.erase1(key_id(k));
      __syncwarp();
    }
  };
  // Cuckoo: erase the evicted keys ev[0..ne) one at a time in decreasing key
  // order (reading R9's eviction order)
  auto cuckoo_erase_sorted_desc = [&](int ne) {
    for (int i = ne - 1; i >= 0; --i) {
      if (lane == 0) cs.erase1(key_id(ev[i]));
      __syncwarp();
    }
  };

  uint32_t gen = a.gen0;
  while (true) {
    int qi = 0;
    if (lane == 0) {
      qi = (int)atomicAdd(a.ticket, 1u);
      if (a.order && (int64_t)qi < a.nq) qi = __ldg(a.order + qi);  // scheduled order
    }
    qi = __shfl_sync(FULL, qi, 0);
    if ((int64_t)qi >= a.nq) break;

    // ---- a1: stage the query in registers (P:269 keeps it on chip)
    float4 qv[NCH];
    bool bad = false;
    const float* qrow = a.queries + (int64_t)qi * a.dim;
    if constexpr (METRIC == MET_HAM) {
      // every lane holds the whole query code (words 4c .. 4c+3 in qv[c]);
      // words past dim are 0, like the index's padding words
#pragma unroll
      for (int c = 0; c < NCH; ++c) {
        const int e = 4 * c;
        qv[c] = make_float4(e + 0 < a.dim ? qrow[e + 0] : 0.f, e + 1 < a.dim ? qrow[e + 1] : 0.f,
                            e + 2 < a.dim ? qrow[e + 2] : 0.f, e + 3 < a.dim ? qrow[e + 3] : 0.f);
      }
    } else
#pragma unroll
    for (int c = 0; c < NCH; ++c) {
      int e = (c * 32 + lane) * 4;
      float v0 = e + 0 < a.dim ? qrow[e + 0] : 0.f;
      float v1 = e + 1 < a.dim ? qrow[e + 1] : 0.f;
      float v2 = e + 2 < a.dim ? qrow[e + 2] : 0.f;
      float v3 = e + 3 < a.dim ? qrow[e + 3] : 0.f;
      bad |= !(isfinite(v0) && isfinite(v1) && isfinite(v2) && isfinite(v3));
      qv[c] = make_float4(v0, v1, v2, v3);
    }
    bad = __any_sync(FULL, bad);
    if (METRIC == MET_DOT && a.cosine) {
      float s = 0.f;
#pragma unroll
      for (int c = 0; c < NCH; ++c)
        s += qv[c].x * qv[c].x + qv[c].y * qv[c].y + qv[c].z * qv[c].z + qv[c].w * qv[c].w;
#pragma unroll
      for (int o = 16; o >= 1; o >>= 1) s += __shfl_xor_sync(FULL, s, o);
      float inv = s > 0.f ? 1.0f / sqrtf(s) : 0.f;
#pragma unroll
      for (int c = 0; c < NCH; ++c) {
        qv[c].x *= inv;
        qv[c].y *= inv;
        qv[c].z *= inv;
        qv[c].w *= inv;
      }
    }
    if constexpr (METRIC != MET_HAM && kDistTeam) {
      // stage the (normalised) query in shared memory: chunk c*32 + lane
      __syncwarp();
#pragma unroll
      for (int c = 0; c < NCH; ++c) reinterpret_cast<float4*>(qsm)[c * 32 + lane] = qv[c];
      __syncwarp();
    }
    int32_t* ids_o = a.ids_out + (int64_t)qi * a.K;
    float* dists_o = a.dists_out + (int64_t)qi * a.K;
    if (bad) {
      for (int i = lane; i < a.K; i += 32) {
        ids_o[i] = -1;
        dists_o[i] = __int_as_float(0x7f800000);
      }
      if (a.counters_out && lane == 0) {
        a.counters_out[2 * (int64_t)qi] = 0;
        a.counters_out[2 * (int64_t)qi + 1] = 0;
      }
      if (lane == 0) atomicOr(a.status, STATUS_BAD_INPUT);
      continue;
    }

    // ---- a2: init — visited = {e}, q = {(d_e, e)}, topk = {} (Alg. 1 line 1)
    if constexpr (VK == VK_HASH)
      hs.clear(lane);
    else
      for (int i = lane; i < twords; i += 32) table[i] = 0;
    if (VK == VK_GHASH) gh.gen = ++gen;  // a fresh generation empties the table
    if (lane == 0) cid[0] = a.entry;
    __syncwarp();
    const float de = dist_of<NCH, METRIC, (QR < 0)>(a.data, a.dpad, cid, 1, qv, qsm, stage, a.cosine, lane);
    const uint64_t ke = make_key(__shfl_sync(FULL, de, 0), a.entry);
    v_insert_lane0(a.entry);
    int used = 1;  // VK_HASH: live + tombstones; VK_GHASH: live
    RegArr<QRr> q, tk_r;
    q.clear();
    tk_r.clear();
    Tier qg{qa, 0, 0}, tg{tk, 0, 0};  // QR <= 0 (qg is W when UNQ)
    int hint = 0;                      // UNQ: index of W's first unpopped key
    if (REG) {
      if (lane == 0) q.v[0] = ke;
    } else if (RUN) {
      if (lane == 0) q.v[0] = (ke & ~0xffffffffull) | ((uint64_t)(uint32_t)a.entry << 1);
    } else {
      if (lane == 0)
        qa[0] = UNQ ? (ke & ~0xffffffffull) | ((uint64_t)(uint32_t)a.entry << 1) : ke;
      qg.size = 1;
      __syncwarp();
    }
    int qsize = 1, tsize = 0;
    int n_dist = 1, n_exp = 0, iters = 0;
    bool capped = false, full = false;
    // adjacency row of the next head, prefetched (lane j holds slot j)
    int adjv = (lane < a.degree) ? __ldg(a.adj + (int64_t)a.entry * a.degree + lane) : -1;
    __syncwarp();

#ifdef SONG_STAGE_TIMING
    unsigned long long st_acc[4] = {0, 0, 0, 0};
    long long st_t = clock64();
#endif
    while (qsize > 0) {
      if (UNQ && hint >= qg.size) break;  // R17: no unpopped key left in W
      int wpos = 0;  // RUN: W's first unpopped key (bit 0 of a W key = popped)
      if constexpr (RUN) {
        wpos = -1;
#pragma unroll
        for (int r = QRr - 1; r >= 0; --r) {
          const unsigned m = __ballot_sync(FULL, (q.v[r] & 1ull) == 0);
          if (m) wpos = r * 32 + __ffs(m) - 1;
        }
        if (wpos < 0) break;  // R17: no unpopped key left in W
      }
      if (iters >= a.max_iters) {
        capped = true;
        break;
      }
      ++iters;
      // ---- a3: pop / terminate / topk update (Alg. 1 lines 3-8)
      uint64_t now, tmax;
      if (REG) {
        now = __shfl_sync(FULL, q.v[0], 0);
        tmax = tk_r.get(L - 1);  // KEY_MAX unless topk is full
      } else if (RUN) {
        now = q.get(wpos);  // W's smallest unpopped key (R17 step 2)
        tmax = KEY_MAX;
      } else if (UNQ) {
        now = qg.at(hint);  // W's smallest unpopped key (R17 step 2)
        tmax = KEY_MAX;
      } else {
        now = qg.at(0);
        tmax = (tsize == L) ? tg.at(L - 1) : KEY_MAX;
      }
      if (tmax < now) break;  // topk full and its max beats now (lines 4-5)
      uint64_t evicted = KEY_MAX;
      // Cuckoo false negatives can re-admit a vertex that is already in topk:
      // topk then stays as it is (the paper's "additional checks to avoid
      // inserting one vertex multiple times"; the oracle's set semantics)
      bool in_topk = false;
      if constexpr (VK == VK_CUCKOO) {
        if (REG) {
#pragma unroll
          for (int r = 0; r < QRr; ++r) in_topk |= __any_sync(FULL, tk_r.v[r] == now);
        } else {
          const int r = tg.rank_warp(now, lane);
          const uint64_t at_r = tg.at(r < tsize ? r : 0);
          in_topk = r < tsize && at_r == now;
        }
      }
      if (REG) {
        if (!in_topk) evicted = tk_r.insert_one(now, L, lane);
        q.pop_front(lane);
      } else if (RUN) {  // now moves from "q" to "topk" inside W
#pragma unroll
        for (int r = 0; r < QRr; ++r) {  // (branch-free below 8 registers: see RegArr::get)
          if constexpr (QRr >= 8) {
            if ((wpos >> 5) == r && lane == (wpos & 31)) q.v[r] |= 1ull;
          } else {
            q.v[r] |= (uint64_t)(((wpos >> 5) == r) & (lane == (wpos & 31)));
          }
        }
      } else if (UNQ) {
        qg.set_flag(hint, lane);  // now moves from "q" to "topk" inside W
        hint = qg.next_unpopped(hint + 1, lane);
      } else {
        qg.pop_front(lane);
        if (!in_topk) evicted = tg.push1(now, L, lane);
      }
      if (!in_topk) tsize = min(tsize + 1, L);
      if (DEL) v_erase_lane0(evicted);  // §IV-E: topk's evicted vertex
      __syncwarp();
      // multi-step probing (§V, R13): up to a.steps pops, each checked
      // against the termination rule with topk as the previous pops left it
      int npop = 1;
      int popid = UNI ? wkey_id(now) : key_id(now);  // lane i < npop: id of the i-th popped vertex
      if constexpr (MS) {
        for (; npop < a.steps && npop < qsize; ++npop) {
          const uint64_t nx = REG ? __shfl_sync(FULL, q.v[0], 0) : qg.at(0);
          const uint64_t tm = REG ? tk_r.get(L - 1) : ((tsize == L) ? tg.at(L - 1) : KEY_MAX);
          if (tm < nx) break;
          uint64_t ev1;
          if (REG) {
            ev1 = tk_r.insert_one(nx, L, lane);
            q.pop_front(lane);
          } else {
            qg.pop_front(lane);
            ev1 = tg.push1(nx, L, lane);
          }
          tsize = min(tsize + 1, L);
          if (DEL) v_erase_lane0(ev1);
          __syncwarp();
          if (lane == npop) popid = key_id(nx);
        }
      }
      const int na = qsize - npop;  // q after the pops

      SONG_ST_MARK(0);
      // ---- a4: candidate locating (§V)
      int v = adjv;
      bool keep = v >= 0;
      if (a.dedup) {
        unsigned grp = __match_any_sync(FULL, v);
        keep = keep && ((grp & lt) == 0);
      }
      // (called by every lane: the probe loops are warp-collective)
      int eslot = -1;
      bool seen;
      if constexpr (SLOT)  // remember where each candidate's insert goes (one probe less)
        seen = hs.contains_slot(v, keep, eslot);
      else
        seen = v_contains(v, keep);
      keep = keep && !seen;
      const unsigned km = __ballot_sync(FULL, keep);
      int nc_all = __popc(km);
      if (keep) cid[__popc(km & lt)] = v;
      if (SLOT && keep) cslot[__popc(km & lt)] = eslot;
      __syncwarp();
      if constexpr (MS) {
        // the other popped rows, in pop order: one candidate list (R13)
        for (int i = 1; i < npop; ++i) {
          const int pid = __shfl_sync(FULL, popid, i);
          int v2 = (lane < a.degree) ? __ldg(a.adj + (int64_t)pid * a.degree + lane) : -1;
          bool k2 = v2 >= 0;
          if (a.dedup) {
            const unsigned grp = __match_any_sync(FULL, v2);
            k2 = k2 && ((grp & lt) == 0);
          }
          bool dup = false;  // already located from an earlier popped row
          for (int j = 0; j < nc_all; ++j) dup |= (cid[j] == v2);
          k2 = k2 && !dup;
          const bool seen2 = v_contains(v2, k2);
          k2 = k2 && !seen2;
          const unsigned m2 = __ballot_sync(FULL, k2);
          if (k2) cid[nc_all + __popc(m2 & lt)] = v2;
          nc_all += __popc(m2);
          __syncwarp();
        }
      }
      n_dist += nc_all;
      n_exp += npop;
      // distance + maintenance over groups of <= 32 candidates (one group
      // unless multi-step probing located more): for the exact hash and the
      // insert-only Bloom filter the result of a batch does not depend on
      // how it is split (the selection threshold is fixed within an iteration
      // and evictions = (q u new) minus its L smallest)
      int na_g = na;
      for (int g0 = 0;; g0 += 32) {
      const int nc = min(32, nc_all - g0);
      const int* cidg = cid + g0;
      const bool last_group = !MS || g0 + 32 >= nc_all;

      SONG_ST_MARK(1);
      // ---- a5: bulk distance computation (§VI)
      const float dist =
          dist_of<NCH, METRIC, (QR < 0)>(a.data, a.dpad, cidg, nc, qv, qsm, stage, a.cosine, lane);

      SONG_ST_MARK(2);
      // ---- a6: maintenance (§IV-C/D/E)
      const int myid = lane < nc ? cidg[lane] : -1;
      uint64_t key = lane < nc ? (UNI ? make_wkey(dist, myid) : make_key(dist, myid)) : KEY_MAX;
      // selected insertion threshold: topk's max once topk is full;
      // R17: W's max once W is full
      const uint64_t thr = RUN   ? ((a.sel && qsize == L) ? q.get(L - 1) : KEY_MAX)
                           : UNQ ? ((a.sel && qg.size == L) ? qg.at(L - 1) : KEY_MAX)
                                 : (a.sel && tsize == L)
                                     ? (REG ? tk_r.get(L - 1) : tg.at(L - 1))
                                     : KEY_MAX;
      // selected insertion: filtered only when worse than ALL of topk
      // (a key equal to topk's max can only arise from a filter false negative)
      const bool sel = (lane < nc) && key <= thr;
      const unsigned smask = __ballot_sync(FULL, sel);
      const int ns = __popc(smask);
      if (!sel) key = KEY_MAX;
      // prefetch the adjacency row of the next head = min(q head, best new key)
      if (last_group) {
        uint64_t qhead = REG   ? __shfl_sync(FULL, q.v[0], 0)
                         : UNQ ? (hint < qg.size ? qg.at(hint) : KEY_MAX)
                               : (na_g > 0 ? qg.at(0) : KEY_MAX);
        if constexpr (RUN) {  // W's first unpopped key after this pop
          qhead = KEY_MAX;
#pragma unroll
          for (int r = QRr - 1; r >= 0; --r) {
            const unsigned m = __ballot_sync(FULL, (q.v[r] & 1ull) == 0);
            const uint64_t h = __shfl_sync(FULL, q.v[r], m ? __ffs(m) - 1 : 0);
            if (m) qhead = h;
          }
        }
        uint64_t nxt = umin64(qhead, warp_min_key(key));
        if (nxt != KEY_MAX && lane < a.degree)
          adjv = __ldg(a.adj + (int64_t)(UNI ? wkey_id(nxt) : key_id(nxt)) * a.degree + lane);
        else
          adjv = -1;
      }
      // visited insert of the selected candidates, in candidate order (R9)
      auto visit_selected = [&]() {
        if constexpr (VK == VK_BLOOM) bs.insert(myid, sel);
        if constexpr (VK == VK_GHASH) {
          gh.insert(myid, sel);
          used += ns;
        }
        if constexpr (VK == VK_CUCKOO) {
          bool dropped = false;
          for (unsigned m = smask; m; m &= m - 1) {
            const int j = __ffs(m) - 1;
            if (lane == j) dropped |= !cs.insert1(myid);
            __syncwarp();
          }
          (void)dropped;  // a dropped fingerprint is a false negative (oracle: drops)
        }
        if constexpr (VK == VK_HASH) {
          // R17 lazy: every candidate is marked visited (a skipped key can
          // never enter W again), so the capacity check counts all of them
          const bool ins = (UNI && a.lazy) ? lane < nc : sel;
          const int nins = (UNI && a.lazy) ? nc : ns;
          bool rebuilt = false;
          if (used + nins > a.rebuild_at) {
            rebuilt = true;
            // tombstones accumulated (eager deletion) or the capacity is reached
            // (lazy deletion, R14): rebuild visited = ids(q) ∪ ids(topk)
            hs.clear(lane);
            __syncwarp();
            if (REG) {
#pragma unroll
              for (int r = 0; r < QRr; ++r) {
                hs.insert(key_id(q.v[r]), q.v[r] != KEY_MAX);
                hs.insert(key_id(tk_r.v[r]), tk_r.v[r] != KEY_MAX);
              }
            } else if (RUN) {  // R17: visited := ids(W)
#pragma unroll
              for (int r = 0; r < QRr; ++r) hs.insert(wkey_id(q.v[r]), q.v[r] != KEY_MAX);
            } else if (UNQ) {  // R17: visited := ids(W)
              for (int i0 = 0; i0 < qg.size; i0 += 32) {
                const uint64_t kw = qg.at(i0 + lane < qg.size ? i0 + lane : 0);  // (all lanes)
                hs.insert(wkey_id(kw), i0 + lane < qg.size);
              }
            } else {
              for (int i0 = 0; i0 < na_g; i0 += 32) {
                const uint64_t kq = qg.at(i0 + lane < na_g ? i0 + lane : 0);  // (all lanes)
                hs.insert(key_id(kq), i0 + lane < na_g);
              }
              for (int i0 = 0; i0 < tsize; i0 += 32) {
                const uint64_t kt = tg.at(i0 + lane < tsize ? i0 + lane : 0);
                hs.insert(key_id(kt), i0 + lane < tsize);
              }
            }
            used = RUN ? qsize : UNQ ? qg.size : na_g + tsize;
            __syncwarp();
          }
          if (SLOT && a.lazy && !rebuilt) {
            // the locate probe left each candidate's slot (the first EMPTY of
            // the bucket its probe ended in): one plain store per candidate,
            // the lowest lane of a shared slot wins, the others probe again
            const int es = ins ? cslot[lane] : -1 - lane;
            const unsigned grp = __match_any_sync(FULL, es);
            const bool win = ins && es >= 0 && (grp & lt) == 0;
            if (win) table[es] = myid;
            __syncwarp();
            const bool took = hs.insert(myid, ins && !win);
            used += __popc(__ballot_sync(FULL, took || win));
          } else {
            const bool took = hs.insert(myid, ins);
            used += __popc(__ballot_sync(FULL, took));
          }
        }
      };
      int qsize_new = min(na_g + ns, L);
      if (RUN) {  // R17, W in registers: merge the selected keys, drop beyond L
        visit_selected();  // (lazy: every candidate is marked visited)
        qsize_new = min(qsize + ns, L);
        if (ns > 0 && ns <= SONG_RUN_INS_MAX) {
          // few selected keys: rank + shift each into W instead of sorting
          // them and running the bitonic merge (the same L smallest stay and
          // the same keys leave: a key that arrives at a full W behind its
          // maximum leaves at once)
          int wsz = qsize;
          for (unsigned m = smask; m; m &= m - 1) {
            const uint64_t kj = __shfl_sync(FULL, key, __ffs(m) - 1);
            uint64_t evk = q.insert_one(kj, L, lane);
            if (wsz < L)
              ++wsz;
            else if (evk == KEY_MAX)
              evk = kj;
            if constexpr (VK == VK_HASH) hs.erase(wkey_id(evk), lane == 0 && evk != KEY_MAX && !a.lazy);
          }
        } else if (ns > 0) {
          if (sel) keys32[__popc(smask & lt)] = key;
          __syncwarp();
          uint64_t k2 = lane < ns ? keys32[lane] : KEY_MAX;
          __syncwarp();
          k2 = sort_prefix(k2, ns, lane);
          const uint64_t sdesc = __shfl_sync(FULL, k2, 31 - lane);  // descending
          uint64_t out;
          merge_into<QRr>(q, sdesc, lane, out);
#pragma unroll
          for (int r = 0; r < QRr; ++r) {
            const bool beyond = r * 32 + lane >= L && q.v[r] != KEY_MAX;
            if constexpr (VK == VK_HASH) hs.erase(wkey_id(q.v[r]), beyond && !a.lazy);  // [del]
            q.v[r] = r * 32 + lane >= L ? KEY_MAX : q.v[r];
          }
          if constexpr (VK == VK_HASH) hs.erase(wkey_id(out), out != KEY_MAX && !a.lazy);
        }
      } else if (REG) {
        if (ns > 0) {  // (ns == 0: q only lost its head, nothing to insert/evict)
          visit_selected();
          // Cuckoo false negatives: a selected key may already be in q
          unsigned qmask = smask;
          if constexpr (VK == VK_CUCKOO) {
            for (unsigned m = smask; m; m &= m - 1) {
              const int j = __ffs(m) - 1;
              const uint64_t kj = __shfl_sync(FULL, key, j);
              bool dup = false;
#pragma unroll
              for (int r = 0; r < QRr; ++r) dup |= __any_sync(FULL, q.v[r] == kj);
              if (dup) qmask &= ~(1u << j);
            }
          }
          const int nq_new = __popc(qmask);
          qsize_new = min(na_g + nq_new, L);
          // compact the selected keys to lanes [0, nq_new), sort only those
          if ((qmask >> lane) & 1u) keys32[__popc(qmask & lt)] = key;
          __syncwarp();
          uint64_t k2 = lane < nq_new ? keys32[lane] : KEY_MAX;
          k2 = sort_prefix(k2, nq_new, lane);
          const uint64_t sdesc = __shfl_sync(FULL, k2, 31 - lane);  // descending
          // merge into q; evict beyond L (§IV-C) and delete from visited (§IV-E)
          uint64_t out;
          merge_into<QRr>(q, sdesc, lane, out);
          int ne = 0;  // number of evicted keys (VK_CUCKOO collects them in ev[])
#pragma unroll
          for (int r = 0; r < QRr; ++r) {
            const bool beyond = r * 32 + lane >= L && q.v[r] != KEY_MAX;
            if constexpr (VK == VK_HASH) hs.erase(key_id(q.v[r]), beyond && !a.lazy);
            if constexpr (VK == VK_CUCKOO) {
              const unsigned bm = __ballot_sync(FULL, beyond);
              if (beyond) ev[ne + __popc(bm & lt)] = q.v[r];
              ne += __popc(bm);
            }
            q.v[r] = r * 32 + lane >= L ? KEY_MAX : q.v[r];
          }
          if constexpr (VK == VK_HASH) hs.erase(key_id(out), out != KEY_MAX && !a.lazy);
          if constexpr (VK == VK_CUCKOO) {
            const bool o = out != KEY_MAX;
            const unsigned bm = __ballot_sync(FULL, o);
            if (o) ev[ne + __popc(bm & lt)] = out;
            ne += __popc(bm);
            __syncwarp();
            // sort the evicted keys ascending, erase from the largest down
            uint64_t e2 = lane < ne ? ev[lane] : KEY_MAX;
            e2 = sort_prefix(e2, ne, lane);
            __syncwarp();
            ev[lane] = e2;
            __syncwarp();
            cuckoo_erase_sorted_desc(ne);
          }
        }
      } else if (UNQ) {  // R17: insert into W, drop its maximum beyond L
        visit_selected();
        __syncwarp();
        if (sel) keys32[__popc(smask & lt)] = key;
        __syncwarp();
        key = lane < ns ? keys32[lane] : KEY_MAX;
        __syncwarp();
        key = sort_prefix(key, ns, lane);
        int ne = 0;
        uint64_t evk = KEY_MAX;  // lane e: the e-th dropped key
        for (int j = 0; j < ns; ++j) {
          const uint64_t x = __shfl_sync(FULL, key, j);
          if (qg.size == L) {
            const uint64_t mx = qg.at(L - 1);
            if (x > mx) {  // x and every later key are dropped at once
              const uint64_t moved = __shfl_sync(FULL, key, (lane - ne + j) & 31);
              if (lane >= ne && lane < ne + ns - j) evk = moved;
              ne += ns - j;
              break;
            }
            if (lane == ne) evk = mx;
            ++ne;
            qg.size = L - 1;
            hint = min(hint, qg.size);
          }
          const int pos = qg.insert(x, lane);
          hint = pos <= hint ? pos : hint;  // a new (unpopped) key before the old first one
        }
        if constexpr (VK == VK_HASH) hs.erase(wkey_id(evk), lane < ne && !a.lazy);  // [del]
        qsize_new = qg.size;
      } else {  // QR == 0: the q ring
        visit_selected();
        __syncwarp();
        // compact the selected keys to lanes [0, ns) and sort only those
        if (sel) keys32[__popc(smask & lt)] = key;
        __syncwarp();
        key = lane < ns ? keys32[lane] : KEY_MAX;
        __syncwarp();
        key = sort_prefix(key, ns, lane);
        int nsq = ns;  // selected keys that enter q
        if constexpr (VK == VK_CUCKOO) {
          // drop keys already in q (Cuckoo false negatives), re-compact
          const int j = qg.rank_lane(key);
          const uint64_t at_j = qg.at(j < na_g ? j : 0);
          const bool dup = lane < ns && j < na_g && at_j == key;
          const unsigned keepm = __ballot_sync(FULL, lane < ns && !dup);
          nsq = __popc(keepm);
          __syncwarp();
          if ((keepm >> lane) & 1u) keys32[__popc(keepm & lt)] = key;
          __syncwarp();
          key = lane < nsq ? keys32[lane] : KEY_MAX;
          __syncwarp();
        }
        if (nsq > 0) {
          // insert the new keys in ascending order; a full q evicts its
          // maximum first (§IV-C) — the evicted set is the largest
          // (na + nsq - L) keys of q and the new ones, as a merge would give
          int ne = 0;
          uint64_t evk = KEY_MAX;  // lane e: the e-th evicted key
          for (int j = 0; j < nsq; ++j) {
            const uint64_t x = __shfl_sync(FULL, key, j);
            if (qg.size == L) {
              const uint64_t mx = qg.at(L - 1);
              if (x > mx) {  // x and every later key are evicted at once
                const uint64_t moved = __shfl_sync(FULL, key, (lane - ne + j) & 31);
                if (lane >= ne && lane < ne + nsq - j) evk = moved;
                ne += nsq - j;
                break;
              }
              if (lane == ne) evk = mx;
              ++ne;
              qg.size = L - 1;
            }
            qg.insert(x, lane);
          }
          if (ne > 0) {
            if constexpr (VK == VK_HASH) hs.erase(key_id(evk), lane < ne && !a.lazy);  // §IV-E
            if constexpr (VK == VK_CUCKOO) {
              // ascending, then erased from the largest down (reading R9)
              const uint64_t srt = sort_prefix(lane < ne ? evk : KEY_MAX, ne, lane);
              ev[lane] = srt;
              __syncwarp();
              cuckoo_erase_sorted_desc(ne);
            }
          }
        }
        qsize_new = qg.size;
      }
      qsize = qsize_new;
      __syncwarp();
      na_g = qsize;
      if (last_group) break;
      }  // candidate groups
      SONG_ST_MARK(3);
      if (VK == VK_GHASH && used > (1 << (a.table_log2 - 1))) {  // keep load <= 1/2
        full = true;
        break;
      }
    }

#ifdef SONG_STAGE_TIMING
    if (lane == 0 && a.stage_cycles)
      for (int k = 0; k < 4; ++k) atomicAdd(a.stage_cycles + k, st_acc[k]);
#endif
    // ---- a7: output the first K of topk (Alg. 1 line 17)
    if (RUN) {  // R17: the first K popped keys of W (all of W at a normal stop)
      int outn = 0;
#pragma unroll
      for (int r = 0; r < QRr; ++r) {
        const uint64_t k = q.v[r];
        const bool pp = k != KEY_MAX && (k & 1ull);
        const unsigned m = __ballot_sync(FULL, pp);
        const int o = outn + __popc(m & lt);
        if (pp && o < a.K) {
          ids_o[o] = wkey_id(k) + a.id_offset;
          dists_o[o] = ord2f((uint32_t)(k >> 32));
        }
        outn += __popc(m);
      }
      for (int i = min(outn, a.K) + lane; i < a.K; i += 32) {
        ids_o[i] = -1;
        dists_o[i] = __int_as_float(0x7f800000);
      }
    } else if (REG) {
#pragma unroll
      for (int r = 0; r < QRr; ++r) {
        const int i = r * 32 + lane;
        if (i < a.K) {
          uint64_t k = tk_r.v[r];
          ids_o[i] = (k != KEY_MAX) ? key_id(k) + a.id_offset : -1;
          dists_o[i] = (k != KEY_MAX) ? ord2f((uint32_t)(k >> 32)) : __int_as_float(0x7f800000);
        }
      }
    } else if (UNQ) {  // R17: the first K popped keys of W (all of W at a normal stop)
      int outn = 0;
      for (int i0 = 0; i0 < qg.size && outn < a.K; i0 += 32) {
        const int i = i0 + lane;
        const uint64_t k = qg.at(i < qg.size ? i : 0);
        const bool pp = i < qg.size && (k & 1ull);
        const unsigned m = __ballot_sync(FULL, pp);
        const int o = outn + __popc(m & lt);
        if (pp && o < a.K) {
          ids_o[o] = wkey_id(k) + a.id_offset;
          dists_o[o] = ord2f((uint32_t)(k >> 32));
        }
        outn += __popc(m);
      }
      for (int i = min(outn, a.K) + lane; i < a.K; i += 32) {
        ids_o[i] = -1;
        dists_o[i] = __int_as_float(0x7f800000);
      }
    } else {
      for (int i0 = 0; i0 < a.K; i0 += 32) {
        const int i = i0 + lane;
        const uint64_t k = tg.at(i < tsize ? i : 0);  // (every lane calls: shuffles)
        if (i < a.K) {
          ids_o[i] = i < tsize ? key_id(k) + a.id_offset : -1;
          dists_o[i] = i < tsize ? ord2f((uint32_t)(k >> 32)) : __int_as_float(0x7f800000);
        }
      }
    }
    if (a.counters_out && lane == 0) {
      a.counters_out[2 * (int64_t)qi] = n_dist;
      a.counters_out[2 * (int64_t)qi + 1] = n_exp;
    }
    if (capped && lane == 0) atomicOr(a.status, STATUS_ITER_CAP);
    if (full && lane == 0) atomicOr(a.status, STATUS_TABLE_FULL);
    __syncwarp();
  }
}

}  // namespace song
