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

namespace song {

// One-shot gather + merge over peer memory (dataset sharding, fused):
// every rank's search wrote its [nq][Kin] (ids, dists) rows into a buffer the
// other ranks can address (symmetric memory over NVLink / NVSwitch).  This
// kernel (one per rank, on the stream after that rank's search) first tells
// every peer that its rows are complete — a release store of `epoch` into
// slot `rank` of each peer's signal pad — then waits until every peer's slot
// of its OWN pad holds >= epoch (acquire loads), and merges straight from
// the peers' buffers: the all-gather is the merge's own loads, no staging
// copy and no separate collective.  Without pads (sig == nullptr) the caller
// guarantees visibility (one-GPU emulation, or an external barrier).
__device__ __forceinline__ void st_release_sys(uint32_t* p, uint32_t v) {
  asm volatile("st.release.sys.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ uint32_t ld_acquire_sys(const uint32_t* p) {
  uint32_t v;
  asm volatile("ld.acquire.sys.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}

__device__ __forceinline__ uint64_t peer_key(const int32_t* ids, const float* dists, int64_t i) {
  const int id = ids[i];
  if (id < 0) return ~0ull;
  const uint32_t u = __float_as_uint(dists[i] + 0.0f);
  const uint32_t o = (u & 0x80000000u) ? ~u : (u | 0x80000000u);
  return ((uint64_t)o << 32) | (uint32_t)id;
}

__global__ void song_merge_peers_kernel(const int32_t* const* __restrict__ ids_p,
                                        const float* const* __restrict__ dists_p,
                                        uint32_t* const* __restrict__ sig, int rank, int G,
                                        int64_t nq, int Kin, int K, uint32_t epoch,
                                        int32_t* __restrict__ ids_out,
                                        float* __restrict__ dists_out) {
  if (sig) {
    if ((int)threadIdx.x < G) {
      __threadfence_system();
      st_release_sys(sig[threadIdx.x] + rank, epoch);  // "my rows are complete"
      const uint32_t* mine = sig[rank] + threadIdx.x;
      while ((int)(ld_acquire_sys(mine) - epoch) < 0) {
      }
    }
    __syncthreads();
  }
  const int lane = threadIdx.x & 31;
  const int64_t q = (int64_t)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5);
  if (q >= nq) return;
  for (int i = lane; i < K; i += 32) {
    ids_out[q * K + i] = -1;
    dists_out[q * K + i] = __int_as_float(0x7f800000);
  }
  __syncwarp();
  // an element's merged rank = its position in its own (sorted, unique) row
  // + the number of smaller keys in each other row (binary search)
  for (int e = lane; e < G * Kin; e += 32) {
    const int g = e / Kin;
    const int64_t src = q * Kin + (e % Kin);
    const uint64_t k = peer_key(ids_p[g], dists_p[g], src);
    if (k == ~0ull) continue;
    int r = e % Kin;
    for (int h = 0; h < G && r < K; ++h) {
      if (h == g) continue;
      const int32_t* hi_ids = ids_p[h];
      const float* hi_d = dists_p[h];
      int lo = 0, hi = Kin;
      while (lo < hi) {
        const int mid = (lo + hi) >> 1;
        if (peer_key(hi_ids, hi_d, q * Kin + mid) < k)
          lo = mid + 1;
        else
          hi = mid;
      }
      r += lo;
    }
    if (r < K) {
      ids_out[q * K + r] = ids_p[g][src];
      dists_out[q * K + r] = dists_p[g][src] + 0.0f;
    }
  }
}

}  // namespace song
