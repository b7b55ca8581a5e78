// graph_kernel.cuh — fixed-degree proximity-graph construction on the device
// (reading R15: exact-insertion NSW forward lists, capped backward
// lists, HNSW neighbour heuristic with refill).  SONG itself loads pre-built
// NSW graphs; this builds them on the B200 instead of on a CPU.
//
//   knn_prefix_kernel   F(i) = the D smallest keys (d(i,j), j), j < i: a tiled
//                       Gram GEMM (64 x 64 tiles, fp32 FFMA) whose epilogue
//                       merges every tile into per-row top-32 lists in shared
//                       memory (warp bitonic networks); the distance matrix
//                       never reaches HBM
//   reverse_*           B(j) = the D smallest (d(i,j), i) over i with j in F(i):
//                       count -> exclusive scan -> scatter -> per-vertex top-D
//   prune_kernel        C(v) = F(v) u B(v) merged by key; the candidates' Gram
//                       matrix in shared memory; the heuristic walk by one warp
//
// Keys are the search's u64 keys (orderable(dist) << 32 | id), so every order
// is the (dist, id) order of reading A3.  Distances: L2 = |a|^2 + |b|^2 - 2<a,b>
// (exact on integer-valued data such as the SIFT-shaped workload: every term
// is an integer below 2^24), IP = -<a,b>, cosine = 1 - <a,b> on rows
// normalised beforehand.
#pragma once

#include <cuda_runtime.h>

#include <cstdint>

#include "search_kernel.cuh"

namespace song {
namespace graph {

constexpr int GD = 32;       // list width (degree <= 32)
constexpr int BM = 64;       // rows per CTA tile
constexpr int BN = 64;       // columns per tile
constexpr int BK = 16;       // dimensions per shared-memory stage
constexpr int THREADS = 256;

__device__ __forceinline__ float pair_dist(float dot, float na, float nb, int metric) {
  if (metric == 0) return (na + nb) - 2.0f * dot;  // squared L2
  if (metric == 1) return -dot;                    // -<a, b>
  return 1.0f - dot;                               // cosine on normalised rows
}

// merge up to 32 new keys (one per lane, KEY_MAX where none) into the
// ascending list `cur` (lane l holds element l): the 32 smallest of both
__device__ __forceinline__ uint64_t merge_top32(uint64_t cur, uint64_t cand, int lane) {
  cand = bitonic_sort32<true>(cand, lane);   // descending
  uint64_t m = umin64(cur, cand);            // bitonic sequence of the 32 smallest
#pragma unroll
  for (int j = 16; j >= 1; j >>= 1) {
    const uint64_t o = __shfl_xor_sync(FULL, m, j);
    m = ((lane & j) == 0) ? umin64(m, o) : umax64(m, o);
  }
  return m;
}

// row norms (L2) or in-place normalisation of a scratch copy (cosine)
__global__ void row_norms_kernel(float* x, int64_t n, int dim, float* norms, int normalise) {
  const int lane = threadIdx.x & 31;
  for (int64_t r = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5; r < n;
       r += ((int64_t)gridDim.x * blockDim.x) >> 5) {
    float* row = x + r * dim;
    float s = 0.f;
    for (int i = lane; i < dim; i += 32) s = fmaf(row[i], row[i], s);
    for (int o = 16; o >= 1; o >>= 1) s += __shfl_xor_sync(FULL, s, o);
    if (normalise) {
      const float inv = s > 0.f ? 1.0f / sqrtf(s) : 0.f;
      for (int i = lane; i < dim; i += 32) row[i] *= inv;
      s = s > 0.f ? 1.0f : 0.f;
    }
    if (lane == 0) norms[r] = s;
  }
}

// F(i) for the 64 rows of CTA tile ib (tiles in descending size order: the
// triangular prefix makes row tile ib cost ib + 1 column tiles)
__global__ void __launch_bounds__(THREADS) knn_prefix_kernel(const float* __restrict__ x,
                                                              int64_t n, int dim,
                                                              const float* __restrict__ norms,
                                                              int metric, int D,
                                                              uint64_t* __restrict__ fkeys) {
  __shared__ float xs[BK][BM + 4];
  __shared__ float ys[BK][BN + 4];
  __shared__ float tile[BM][BN + 1];  // distances; +inf where j is not an earlier vertex
  __shared__ uint64_t top[BM][GD];
  const int nb = (int)((n + BM - 1) / BM);
  const int ib = nb - 1 - (int)blockIdx.x;
  const int64_t i0 = (int64_t)ib * BM;
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const int tx = tid & 15, ty = tid >> 4;  // 4 columns x 4 rows per thread
  for (int e = tid; e < BM * GD; e += THREADS) top[e / GD][e % GD] = KEY_MAX;
  const int64_t jend = min(n, i0 + BM);  // columns j < i <= i0 + 63
  for (int64_t j0 = 0; j0 < jend; j0 += BN) {
    float acc[4][4];
#pragma unroll
    for (int a = 0; a < 4; ++a)
#pragma unroll
      for (int b = 0; b < 4; ++b) acc[a][b] = 0.f;
    for (int k0 = 0; k0 < dim; k0 += BK) {
#pragma unroll
      for (int t = 0; t < (BM * BK) / THREADS; ++t) {
        const int e = t * THREADS + tid;
        const int rr = e >> 4, kk = e & 15;
        const int k = k0 + kk;
        const int64_t gi = i0 + rr, gj = j0 + rr;
        xs[kk][rr] = (gi < n && k < dim) ? __ldg(x + gi * dim + k) : 0.f;
        ys[kk][rr] = (gj < n && k < dim) ? __ldg(x + gj * dim + k) : 0.f;
      }
      __syncthreads();
#pragma unroll
      for (int kk = 0; kk < BK; ++kk) {
        const float4 a4 = *reinterpret_cast<const float4*>(&xs[kk][4 * ty]);
        const float4 b4 = *reinterpret_cast<const float4*>(&ys[kk][4 * tx]);
        const float av[4] = {a4.x, a4.y, a4.z, a4.w};
        const float bv[4] = {b4.x, b4.y, b4.z, b4.w};
#pragma unroll
        for (int a = 0; a < 4; ++a)
#pragma unroll
          for (int b = 0; b < 4; ++b) acc[a][b] = fmaf(av[a], bv[b], acc[a][b]);
      }
      __syncthreads();
    }
    // keys of the tile; j >= i (not an earlier vertex) and j >= n excluded
#pragma unroll
    for (int a = 0; a < 4; ++a) {
      const int64_t gi = i0 + 4 * ty + a;
      const float ni = gi < n ? norms[gi] : 0.f;
#pragma unroll
      for (int b = 0; b < 4; ++b) {
        const int64_t gj = j0 + 4 * tx + b;
        tile[4 * ty + a][4 * tx + b] =
            (gi < n && gj < gi) ? pair_dist(acc[a][b], ni, norms[gj], metric) : __int_as_float(0x7f800000);
      }
    }
    __syncthreads();
    // merge into the rows' top lists: warp w owns rows w, w + 8, ...
    for (int r = warp; r < BM; r += THREADS / 32) {
      uint64_t cur = top[r][lane];
      const uint64_t thr = __shfl_sync(FULL, cur, D - 1);  // current D-th best
      const int64_t gi = i0 + r;
      const float d0 = tile[r][lane], d1 = tile[r][lane + 32];
      const bool v0 = j0 + lane < gi, v1 = j0 + lane + 32 < gi;  // (inf is a valid distance key)
      const uint64_t c0 = v0 ? make_key(d0, (int)(j0 + lane)) : KEY_MAX;
      const uint64_t c1 = v1 ? make_key(d1, (int)(j0 + lane + 32)) : KEY_MAX;
      const bool h0 = c0 < thr, h1 = c1 < thr;
      if (__any_sync(FULL, h0)) cur = merge_top32(cur, h0 ? c0 : KEY_MAX, lane);
      if (__any_sync(FULL, h1)) cur = merge_top32(cur, h1 ? c1 : KEY_MAX, lane);
      top[r][lane] = cur;
    }
    __syncthreads();
  }
  for (int r = warp; r < BM; r += THREADS / 32) {
    const int64_t gi = i0 + r;
    if (gi < n && lane < D) fkeys[gi * D + lane] = top[r][lane];
  }
}

// backward lists: count / scatter / select
__global__ void reverse_count_kernel(const uint64_t* __restrict__ fkeys, int64_t nedges,
                                     int* __restrict__ cnt) {
  for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < nedges;
       e += (int64_t)gridDim.x * blockDim.x) {
    const uint64_t k = fkeys[e];
    if (k != KEY_MAX) atomicAdd(&cnt[key_id(k)], 1);
  }
}

__global__ void reverse_scatter_kernel(const uint64_t* __restrict__ fkeys, int64_t nedges, int D,
                                       const int64_t* __restrict__ off, int* __restrict__ cursor,
                                       uint64_t* __restrict__ inc) {
  for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < nedges;
       e += (int64_t)gridDim.x * blockDim.x) {
    const uint64_t k = fkeys[e];
    if (k == KEY_MAX) continue;
    const int j = key_id(k);
    const int i = (int)(e / D);
    const int pos = atomicAdd(&cursor[j], 1);
    inc[off[j] + pos] = (k & 0xffffffff00000000ull) | (uint32_t)i;  // (d(i,j), i)
  }
}

__global__ void reverse_select_kernel(const uint64_t* __restrict__ inc,
                                      const int64_t* __restrict__ off, const int* __restrict__ cnt,
                                      int64_t n, int D, uint64_t* __restrict__ bkeys) {
  const int lane = threadIdx.x & 31;
  for (int64_t j = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5; j < n;
       j += ((int64_t)gridDim.x * blockDim.x) >> 5) {
    const int64_t o = off[j];
    const int c = cnt[j];
    uint64_t cur = KEY_MAX;
    for (int b = 0; b < c; b += 32) {
      const uint64_t k = (b + lane < c) ? inc[o + b + lane] : KEY_MAX;
      const uint64_t thr = __shfl_sync(FULL, cur, D - 1);
      const bool h = k < thr;
      if (__any_sync(FULL, h)) cur = merge_top32(cur, h ? k : KEY_MAX, lane);
    }
    if (lane < D) bkeys[j * D + lane] = cur;
  }
}

// candidates, their Gram matrix and the heuristic: one 128-thread CTA per vertex
constexpr int PT = 128;
constexpr int PC = 2 * GD;  // <= 64 candidates

__global__ void __launch_bounds__(PT) prune_kernel(const float* __restrict__ x, int64_t n, int dim,
                                                   const float* __restrict__ norms, int metric,
                                                   int D, const uint64_t* __restrict__ fkeys,
                                                   const uint64_t* __restrict__ bkeys,
                                                   int32_t* __restrict__ adj) {
  __shared__ uint64_t cand[PC];
  __shared__ int cid[PC];
  __shared__ float cs[BK][PC + 4];
  __shared__ float pd[PC][PC + 1];
  __shared__ int ncand;
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const int rg = tid >> 4, cg = tid & 15;  // 8 rows x 4 columns of the Gram per thread
  for (int64_t v = blockIdx.x; v < n; v += gridDim.x) {
    // ---- C(v) = F(v) u B(v) ascending: a bitonic merge of 2 x 32 keys
    if (warp == 0) {
      uint64_t a0 = lane < D ? fkeys[v * D + lane] : KEY_MAX;             // ascending
      uint64_t a1 = (31 - lane) < D ? bkeys[v * D + (31 - lane)] : KEY_MAX;  // descending
      {
        const uint64_t lo = umin64(a0, a1), hi = umax64(a0, a1);
        a0 = lo;
        a1 = hi;
      }
#pragma unroll
      for (int j = 16; j >= 1; j >>= 1) {
        const uint64_t o0 = __shfl_xor_sync(FULL, a0, j), o1 = __shfl_xor_sync(FULL, a1, j);
        const bool low = (lane & j) == 0;
        a0 = low ? umin64(a0, o0) : umax64(a0, o0);
        a1 = low ? umin64(a1, o1) : umax64(a1, o1);
      }
      // C(v) as a set of vertices: drop v itself and every repeat of an id
      // after its first (smallest-key) occurrence — F(v) and B(v) overlap
      // when the forward lists are not earlier-only (kNN lists given to
      // song_build_graph_from_forward); a no-op for the builders' own lists
      const int i0 = a0 != KEY_MAX ? key_id(a0) : -1, i1 = a1 != KEY_MAX ? key_id(a1) : -1;
      cid[lane] = i0;
      cid[lane + 32] = i1;
      __syncwarp();
      bool k0 = i0 >= 0 && i0 != (int)v, k1 = i1 >= 0 && i1 != (int)v;
      for (int t = 0; t < PC; ++t) {
        const int o = cid[t];
        k0 = k0 && !(t < lane && o == i0);
        k1 = k1 && !(t < lane + 32 && o == i1);
      }
      const unsigned m0 = __ballot_sync(FULL, k0), m1 = __ballot_sync(FULL, k1);
      const unsigned lt = lanemask_lt();
      __syncwarp();
      if (k0) {
        cand[__popc(m0 & lt)] = a0;
        cid[__popc(m0 & lt)] = i0;
      }
      if (k1) {
        cand[__popc(m0) + __popc(m1 & lt)] = a1;
        cid[__popc(m0) + __popc(m1 & lt)] = i1;
      }
      const int c = __popc(m0) + __popc(m1);
      __syncwarp();
      if (lane >= c) {
        cand[lane] = KEY_MAX;
        cid[lane] = 0;
      }
      if (lane + 32 >= c) {
        cand[lane + 32] = KEY_MAX;
        cid[lane + 32] = 0;
      }
      if (lane == 0) ncand = c;
    }
    __syncthreads();
    const int nc = ncand;
    // ---- Gram matrix of the candidates (dims staged 16 at a time)
    float g[8][4];
#pragma unroll
    for (int a = 0; a < 8; ++a)
#pragma unroll
      for (int b = 0; b < 4; ++b) g[a][b] = 0.f;
    for (int k0 = 0; k0 < dim; k0 += BK) {
      for (int e = tid; e < PC * BK; e += PT) {
        const int c = e >> 4, kk = e & 15;
        const int k = k0 + kk;
        cs[kk][c] = (c < nc && k < dim) ? __ldg(x + (int64_t)cid[c] * dim + k) : 0.f;
      }
      __syncthreads();
#pragma unroll
      for (int kk = 0; kk < BK; ++kk) {
        const float4 r0 = *reinterpret_cast<const float4*>(&cs[kk][8 * rg]);
        const float4 r1 = *reinterpret_cast<const float4*>(&cs[kk][8 * rg + 4]);
        const float4 c4 = *reinterpret_cast<const float4*>(&cs[kk][4 * cg]);
        const float av[8] = {r0.x, r0.y, r0.z, r0.w, r1.x, r1.y, r1.z, r1.w};
        const float bv[4] = {c4.x, c4.y, c4.z, c4.w};
#pragma unroll
        for (int a = 0; a < 8; ++a)
#pragma unroll
          for (int b = 0; b < 4; ++b) g[a][b] = fmaf(av[a], bv[b], g[a][b]);
      }
      __syncthreads();
    }
#pragma unroll
    for (int a = 0; a < 8; ++a)
#pragma unroll
      for (int b = 0; b < 4; ++b) {
        const int ra = 8 * rg + a, cb = 4 * cg + b;
        float d = 0.f;
        if (ra < nc && cb < nc)
          d = pair_dist(g[a][b], norms[cid[ra]], norms[cid[cb]], metric);
        pd[ra][cb] = d;
      }
    __syncthreads();
    // ---- the heuristic walk (warp 0): keep t if d(t, k) > d(t, v) for every kept k
    if (warp == 0) {
      int kept = -1;      // lane l < nkept: candidate index of the l-th kept
      int nkept = 0;
      uint64_t takenlo = 0;  // bit t: candidate t kept
      for (int t = 0; t < nc && nkept < D; ++t) {
        const float dt = ord2f((uint32_t)(cand[t] >> 32));
        const bool bad = lane < nkept && !(pd[t][kept] > dt);
        if (!__any_sync(FULL, bad)) {
          if (lane == nkept) kept = t;
          ++nkept;
          takenlo |= 1ull << t;
        }
      }
      for (int t = 0; t < nc && nkept < D; ++t) {  // refill in candidate order
        if (!((takenlo >> t) & 1ull)) {
          if (lane == nkept) kept = t;
          ++nkept;
        }
      }
      if (lane < D) adj[v * D + lane] = lane < nkept ? cid[kept] : -1;
    }
    __syncthreads();
  }
}

}  // namespace graph
}  // namespace song
