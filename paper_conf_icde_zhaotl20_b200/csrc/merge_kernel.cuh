// merge_kernel.cuh — G-way top-K merge of per-shard results ("shard the
// data for each GPU, build a graph index for each shard, perform graph search
// on each GPU and merge the results").
//
// One warp per query.  Every input row is already sorted by the (dist, id)
// key, so an element's rank in the merged order is the sum over shards of the
// number of keys below it (binary search per shard); elements with rank < K
// scatter straight to their output slot.  Keys are unique (global ids differ
// across shards), so ranks are a permutation: exact and deterministic.
#pragma once

#include <cstdint>
#include <cuda_runtime.h>

namespace song {

__device__ __forceinline__ uint64_t merge_key(const int32_t* ids, const float* dists, int64_t i) {
  int id = ids[i];
  if (id < 0) return ~0ull;
  float d = dists[i] + 0.0f;
  uint32_t u = __float_as_uint(d);
  uint32_t o = (u & 0x80000000u) ? ~u : (u | 0x80000000u);
  return ((uint64_t)o << 32) | (uint32_t)id;
}

__global__ void song_merge_kernel(const int32_t* __restrict__ ids_in,
                                  const float* __restrict__ dists_in, int G, int64_t nq,
                                  int Kin, int K, int32_t* __restrict__ ids_out,
                                  float* __restrict__ dists_out) {
  const int lane = threadIdx.x & 31;
  const int64_t q = (int64_t)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5);
  if (q >= nq) return;
  for (int i = lane; i < K; i += 32) {
    ids_out[q * K + i] = -1;
    dists_out[q * K + i] = __int_as_float(0x7f800000);
  }
  __syncwarp();
  const int total = G * Kin;
  for (int e = lane; e < total; e += 32) {
    const int g = e / Kin;
    const int64_t src = ((int64_t)g * nq + q) * Kin + (e % Kin);
    const uint64_t k = merge_key(ids_in, dists_in, src);
    if (k == ~0ull) continue;
    int rank = e % Kin;  // keys below k in its own (sorted, unique) shard row
    for (int h = 0; h < G && rank < K; ++h) {
      if (h == g) continue;
      const int64_t row = ((int64_t)h * nq + q) * Kin;
      int lo = 0, hi = Kin;
      while (lo < hi) {
        int mid = (lo + hi) >> 1;
        if (merge_key(ids_in, dists_in, row + mid) < k)
          lo = mid + 1;
        else
          hi = mid;
      }
      rank += lo;
    }
    if (rank < K) {
      ids_out[q * K + rank] = ids_in[src];
      dists_out[q * K + rank] = dists_in[src] + 0.0f;
    }
  }
}

}  // namespace song
