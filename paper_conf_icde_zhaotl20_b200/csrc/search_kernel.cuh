// search_kernel.cuh — the SONG search hot path for sm_100a.
//
// One warp owns one query at a time (persistent: warps pull query tickets from
// an atomic counter, so long and short queries load-balance).  Each iteration
// of Algorithm 1 runs the paper's three stages (§III, Fig. 3)
// warp-cooperatively instead of on "one single thread":
//
//   maintain/pop  q head is read by all lanes; topk insertion is a warp ballot
//                 rank + in-place shift (§IV-C bounded topk, reading A1)
//   locate (§V)   lane j loads adjacency slot j (one coalesced 128 B row),
//                 drops padding, repeats (match.any) and visited ids (parallel
//                 hash probes) and compacts survivors with a ballot
//   distance (§VI) LDG.128 gathers of R candidate rows per batch, every lane a
//                 16 B slice of each row; a transposed butterfly reduces R
//                 partial sums in R-1+(5-log2 R) shuffles (P:455's shfl_down
//                 reduction, batched)
//   maintain      selected insertion (§IV-D) against topk's max, warp bitonic
//                 sort of the <= 32 survivors, visited insert, merge-path merge
//                 into the bounded q (§IV-C) with visited deletion of the
//                 evicted keys (§IV-E)
//
// Priority-queue keys are u64 (orderable(dist) << 32 | id): the (dist, id)
// total order of DESIGN.md reading A3 as a single integer compare.
#pragma once

#include <cstdint>
#include <cuda_runtime.h>

namespace song {

constexpr unsigned FULL = 0xffffffffu;
constexpr int EMPTY = -1;  // hash slot never used
constexpr int TOMB = -2;   // hash slot whose key was deleted (§IV-E)
constexpr uint64_t KEY_MAX = ~0ull;

enum : int { STATUS_BAD_INPUT = 1, STATUS_ITER_CAP = 2 };

struct SearchArgs {
  const float* data;   // [n][dpad], 16 B aligned rows
  const int32_t* adj;  // [n][degree]
  const float* queries;  // [nq][dim] (caller layout, unpadded)
  int32_t* ids_out;      // [nq][K]
  float* dists_out;      // [nq][K]
  int32_t* counters_out; // [nq][2] or nullptr
  unsigned* ticket;      // work counter, zeroed before launch
  int* status;           // sticky STATUS_* bits
  int64_t n;
  int64_t nq;
  int dim, dpad, degree;
  int K, L;
  int table_log2;  // hash: log2 slots; bloom: log2 bits
  int entry, max_iters, id_offset;
  int warp_smem_bytes;
};

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

__device__ __forceinline__ unsigned lanemask_lt() {
  unsigned m;
  asm("mov.u32 %0, %%lanemask_lt;" : "=r"(m));
  return m;
}

__device__ __forceinline__ float4 ldg_f4(const float4* p) {
  float4 r;
  asm volatile("ld.global.nc.L1::no_allocate.v4.f32 {%0,%1,%2,%3}, [%4];"
               : "=f"(r.x), "=f"(r.y), "=f"(r.z), "=f"(r.w)
               : "l"(p));
  return r;
}

// ---------------------------------------------------------------- visited --
// Open-addressing hash in shared memory, linear probing; every lane
// runs its own probe sequence so up to 32 operations proceed in parallel.
struct HashSet {
  int* slot;
  int log2;
  __device__ __forceinline__ unsigned home(int v) const {
    return ((uint32_t)v * 0x9E3779B1u) >> (32 - log2);
  }
  __device__ __forceinline__ bool contains(int v) const {
    unsigned mask = (1u << log2) - 1, h = home(v);
    while (true) {
      int s = slot[h];
      if (s == v) return true;
      if (s == EMPTY) return false;
      h = (h + 1) & mask;
    }
  }
  // returns true when an EMPTY slot was consumed
  __device__ __forceinline__ bool insert(int v) {
    unsigned mask = (1u << log2) - 1, h = home(v);
    while (true) {
      int s = slot[h];
      if (s == EMPTY || s == TOMB) {
        int old = atomicCAS(&slot[h], s, v);
        if (old == s) return s == EMPTY;
        continue;  // lost the race for this slot: re-read it
      }
      h = (h + 1) & mask;
    }
  }
  __device__ __forceinline__ void erase(int v) {
    unsigned mask = (1u << log2) - 1, h = home(v);
    while (true) {
      int s = slot[h];
      if (s == v) {
        slot[h] = TOMB;
        return;
      }
      if (s == EMPTY) return;
      h = (h + 1) & mask;
    }
  }
};

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
  __device__ __forceinline__ bool contains(int v) const {
    uint32_t h1 = fmix32((uint32_t)v), h2 = fmix32((uint32_t)v ^ 0x5bd1e995u) | 1u;
    uint32_t mask = (log2 >= 32) ? 0xffffffffu : ((1u << log2) - 1);
#pragma unroll
    for (int i = 0; i < 7; ++i) {
      uint32_t b = (h1 + (uint32_t)i * h2) & mask;
      if (!((word[b >> 5] >> (b & 31)) & 1u)) return false;
    }
    return true;
  }
  __device__ __forceinline__ void insert(int v) {
    uint32_t h1 = fmix32((uint32_t)v), h2 = fmix32((uint32_t)v ^ 0x5bd1e995u) | 1u;
    uint32_t mask = (log2 >= 32) ? 0xffffffffu : ((1u << log2) - 1);
#pragma unroll
    for (int i = 0; i < 7; ++i) {
      uint32_t b = (h1 + (uint32_t)i * h2) & mask;
      atomicOr(&word[b >> 5], 1u << (b & 31));
    }
  }
};

// ------------------------------------------------------------- utilities --
__device__ __forceinline__ uint64_t bitonic_sort32(uint64_t key, int lane) {
#pragma unroll
  for (int k = 2; k <= 32; k <<= 1) {
#pragma unroll
    for (int j = k >> 1; j > 0; j >>= 1) {
      uint64_t other = __shfl_xor_sync(FULL, key, j);
      bool ascending = (lane & k) == 0;
      bool lower = (lane & j) == 0;
      uint64_t lo = key < other ? key : other;
      uint64_t hi = key < other ? other : key;
      key = (lower == ascending) ? lo : hi;
    }
  }
  return key;
}

// number of elements of sorted a[0..n) strictly below x
__device__ __forceinline__ int count_below(const uint64_t* a, int n, uint64_t x) {
  int lo = 0, hi = n;
  while (lo < hi) {
    int mid = (lo + hi) >> 1;
    if (a[mid] < x)
      lo = mid + 1;
    else
      hi = mid;
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

// ------------------------------------------------------- bulk distance --
// §VI: distances of the nc candidates whose ids are in cid[0..nc) (shared).
// Lane j (< nc) receives candidate j's distance.  NCH = 16 B chunks per lane
// per row (dpad <= 128 * NCH).
template <int NCH, int METRIC>
__device__ __forceinline__ float bulk_distance(const float* __restrict__ data, int dpad,
                                               const int* cid, int nc, const float4 (&qv)[NCH],
                                               int lane) {
  constexpr int R = (NCH >= 8) ? 1 : (8 / NCH);  // rows per batch: 8 LDG.128 in flight
  constexpr int LR = Log2<R>::value;
  const int d4 = dpad >> 2;
  float mine = 0.0f;
  for (int b = 0; b < nc; b += R) {
    float4 x[R][NCH];
#pragma unroll
    for (int r = 0; r < R; ++r) {
      int j = b + r;
      int id = (j < nc) ? cid[j] : -1;
      const float4* row = reinterpret_cast<const float4*>(data + (int64_t)(id < 0 ? 0 : id) * dpad);
#pragma unroll
      for (int c = 0; c < NCH; ++c) {
        int idx = c * 32 + lane;
        if (id >= 0 && idx < d4)
          x[r][c] = ldg_f4(row + idx);
        else
          x[r][c] = make_float4(0.f, 0.f, 0.f, 0.f);
      }
    }
    float part[R];
#pragma unroll
    for (int r = 0; r < R; ++r) {
      float acc = 0.0f;
#pragma unroll
      for (int c = 0; c < NCH; ++c) {
        if (METRIC == 0) {
          float t0 = qv[c].x - x[r][c].x, t1 = qv[c].y - x[r][c].y;
          float t2 = qv[c].z - x[r][c].z, t3 = qv[c].w - x[r][c].w;
          acc = fmaf(t0, t0, acc);
          acc = fmaf(t1, t1, acc);
          acc = fmaf(t2, t2, acc);
          acc = fmaf(t3, t3, acc);
        } else {
          acc = fmaf(qv[c].x, x[r][c].x, acc);
          acc = fmaf(qv[c].y, x[r][c].y, acc);
          acc = fmaf(qv[c].z, x[r][c].z, acc);
          acc = fmaf(qv[c].w, x[r][c].w, acc);
        }
      }
      part[r] = acc;
    }
    float tot = transpose_reduce<R>(part, lane);
    float got = __shfl_sync(FULL, tot, ((lane - b) & (R - 1)) << (5 - LR));
    if (lane >= b && lane < b + R) mine = got;
  }
  if (METRIC == 1) mine = -mine;        // inner product: -<q,x>
  if (METRIC == 2) mine = 1.0f - mine;  // cosine on unit rows: 1 - cos
  return mine;
}

// ---------------------------------------------------------- the kernel --
template <int NCH, int METRIC, bool BLOOM>
__global__ void __launch_bounds__(256) song_search_kernel(const SearchArgs a) {
  extern __shared__ __align__(16) unsigned char smem[];
  const int lane = threadIdx.x & 31;
  const int warp = threadIdx.x >> 5;
  const int L = a.L;
  unsigned char* base = smem + (size_t)warp * a.warp_smem_bytes;
  uint64_t* qa = reinterpret_cast<uint64_t*>(base);  // q, current buffer
  uint64_t* qb = qa + L;                              // q, next buffer
  uint64_t* tk = qb + L;                              // topk, sorted ascending
  uint64_t* stage = tk + L;                           // 32 sorted new keys
  int* cid = reinterpret_cast<int*>(stage + 32);      // 32 candidate ids
  int* table = cid + 32;                              // visited
  const int tslots = BLOOM ? ((1 << a.table_log2) >> 5) : (1 << a.table_log2);
  HashSet hs{table, a.table_log2};
  BloomSet bs{reinterpret_cast<uint32_t*>(table), a.table_log2};
  const unsigned lt = lanemask_lt();

  while (true) {
    int qi = 0;
    if (lane == 0) qi = (int)atomicAdd(a.ticket, 1u);
    qi = __shfl_sync(FULL, qi, 0);
    if ((int64_t)qi >= a.nq) break;

    // ---- a1: stage the query in registers (P:269 keeps it on chip)
    float4 qv[NCH];
    bool bad = false;
    const float* qrow = a.queries + (int64_t)qi * a.dim;
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
    if (METRIC == 2) {
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
    for (int i = lane; i < tslots; i += 32) table[i] = BLOOM ? 0 : EMPTY;
    if (lane == 0) cid[0] = a.entry;
    __syncwarp();
    float de = bulk_distance<NCH, METRIC>(a.data, a.dpad, cid, 1, qv, lane);
    int used = 0;
    if (lane == 0) {
      qa[0] = make_key(de, a.entry);
      if (BLOOM)
        bs.insert(a.entry);
      else
        hs.insert(a.entry);
    }
    used = 1;
    int qsize = 1, tsize = 0;
    int n_dist = 1, n_exp = 0, iters = 0;
    bool capped = false;
    __syncwarp();

    while (qsize > 0) {
      if (iters >= a.max_iters) {
        capped = true;
        break;
      }
      ++iters;
      // ---- a3: pop / terminate / topk update (Alg. 1 lines 3-8)
      const uint64_t now = qa[0];
      const bool full = (tsize == L);
      if (full && tk[L - 1] < now) break;
      const uint64_t evicted = full ? tk[L - 1] : KEY_MAX;
      int pos = 0;
      for (int b0 = 0; b0 < tsize; b0 += 32) {
        int i = b0 + lane;
        pos += __popc(__ballot_sync(FULL, i < tsize && tk[i] < now));
      }
      const int newsize = full ? L : tsize + 1;
      for (int b0 = ((newsize - 1) >> 5) << 5; b0 >= ((pos >> 5) << 5); b0 -= 32) {
        int i = b0 + lane;
        uint64_t val = 0;
        bool w = false;
        if (i > pos && i < newsize) {
          val = tk[i - 1];
          w = true;
        } else if (i == pos) {
          val = now;
          w = true;
        }
        __syncwarp();
        if (w) tk[i] = val;
      }
      tsize = newsize;
      if (!BLOOM && full && lane == 0) hs.erase(key_id(evicted));  // §IV-E
      __syncwarp();
      const uint64_t* A = qa + 1;  // q after the pop
      const int na = qsize - 1;

      // ---- a4: candidate locating (§V)
      const int nowid = key_id(now);
      int v = (lane < a.degree) ? __ldg(a.adj + (int64_t)nowid * a.degree + lane) : -1;
      unsigned grp = __match_any_sync(FULL, v);
      bool keep = (v >= 0) && ((grp & lt) == 0);
      if (keep) keep = BLOOM ? !bs.contains(v) : !hs.contains(v);
      unsigned km = __ballot_sync(FULL, keep);
      const int nc = __popc(km);
      if (keep) cid[__popc(km & lt)] = v;
      __syncwarp();

      // ---- a5: bulk distance computation (§VI)
      float dist = bulk_distance<NCH, METRIC>(a.data, a.dpad, cid, nc, qv, lane);
      n_dist += nc;
      n_exp += 1;

      // ---- a6: maintenance (§IV-C/D/E)
      const int myid = lane < nc ? cid[lane] : -1;
      uint64_t key = lane < nc ? make_key(dist, myid) : KEY_MAX;
      const uint64_t thr = (tsize == L) ? tk[L - 1] : KEY_MAX;
      const bool sel = (lane < nc) && key < thr;  // selected insertion
      const unsigned sm = __ballot_sync(FULL, sel);
      const int ns = __popc(sm);
      if (!sel) key = KEY_MAX;
      if (BLOOM) {
        if (sel) bs.insert(myid);
      } else {
        if (used + ns > ((3 << a.table_log2) >> 2)) {
          // tombstones accumulated: rebuild visited = ids(q) ∪ ids(topk)
          for (int i = lane; i < tslots; i += 32) table[i] = EMPTY;
          __syncwarp();
          for (int i = lane; i < na; i += 32) hs.insert(key_id(A[i]));
          for (int i = lane; i < tsize; i += 32) hs.insert(key_id(tk[i]));
          used = na + tsize;
          __syncwarp();
        }
        bool took = sel ? hs.insert(myid) : false;
        used += __popc(__ballot_sync(FULL, took));
      }
      key = bitonic_sort32(key, lane);
      stage[lane] = key;
      __syncwarp();
      // merge q (A, na) with the selected keys (stage, ns) into qb, keep L
      for (int i = lane; i < na; i += 32) {
        uint64_t x = A[i];
        int p = i + count_below(stage, ns, x);
        if (p < L)
          qb[p] = x;
        else if (!BLOOM)
          hs.erase(key_id(x));
      }
      if (lane < ns) {
        int p = lane + count_below(A, na, key);
        if (p < L)
          qb[p] = key;
        else if (!BLOOM)
          hs.erase(key_id(key));
      }
      qsize = min(na + ns, L);
      uint64_t* t = qa;
      qa = qb;
      qb = t;
      __syncwarp();
    }

    // ---- a7: output the first K of topk (Alg. 1 line 17)
    for (int i = lane; i < a.K; i += 32) {
      if (i < tsize) {
        uint64_t k = tk[i];
        ids_o[i] = key_id(k) + a.id_offset;
        dists_o[i] = ord2f((uint32_t)(k >> 32));
      } else {
        ids_o[i] = -1;
        dists_o[i] = __int_as_float(0x7f800000);
      }
    }
    if (a.counters_out && lane == 0) {
      a.counters_out[2 * (int64_t)qi] = n_dist;
      a.counters_out[2 * (int64_t)qi + 1] = n_exp;
    }
    if (capped && lane == 0) atomicOr(a.status, STATUS_ITER_CAP);
    // restore buffer roles so the next query starts from the block's layout
    qa = reinterpret_cast<uint64_t*>(base);
    qb = qa + L;
    __syncwarp();
  }
}

}  // namespace song
