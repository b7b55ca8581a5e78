// schedule.cuh — outlier-first ticket order for the persistent search grid
// (song_search_params.schedule).
//
// A batch of independent queries is issued to a fixed number of resident warps
// (148 SMs x 24 warps); with a few queries per warp, the step ends when the last
// warp's last query ends, and a long query drawn late sets the step time.
// Longest-expected-first list scheduling removes most of that tail.  The
// expected length comes from one number per query: its squared distance from the
// centroid of the indexed rows (far-out queries need the longest searches: on
// the SIFT1M-shaped batch it orders the step 9.4M -> 10.4M QPS, an oracle that
// knows every query's expansion count 11.5M; tools/order_probe.py).
//
// Results do not depend on the order: every query owns its q / topk / visited
// structures and writes only its own output rows.
//
//   centroid_partial_kernel + centroid_final_kernel   (once, at index creation)
//       deterministic two-level column sums of the (normalised) rows
//   order_keys_kernel      one warp per query: key = |q - c|^2 (cosine: q
//                          normalised first), bin = SCHED_BINS - 1 - (float bits
//                          >> 19) (16 bins per octave, descending), count[bin]++
//   order_scatter_kernel   per CTA: exclusive scan of the 4096 counts, then
//                          order[off[bin] + cursor[bin]++] = query
#pragma once

#include <cuda_runtime.h>

#include <cstdint>

namespace song {

constexpr int SCHED_BINS = 4096;
constexpr int CENTROID_BLOCKS = 296;

// block b sums rows [b*chunk, (b+1)*chunk) of column j into part[b][j]
__global__ void centroid_partial_kernel(const float* __restrict__ data, int64_t n, int dpad,
                                        int64_t chunk, float* __restrict__ part) {
  const int64_t r0 = (int64_t)blockIdx.x * chunk;
  const int64_t r1 = r0 + chunk < n ? r0 + chunk : n;
  for (int j = threadIdx.x; j < dpad; j += blockDim.x) {
    float s = 0.f;
    for (int64_t r = r0; r < r1; ++r) s += data[r * dpad + j];
    part[(int64_t)blockIdx.x * dpad + j] = s;
  }
}

__global__ void centroid_final_kernel(const float* __restrict__ part, int nparts, int dpad,
                                      int64_t n, float* __restrict__ c) {
  for (int j = threadIdx.x; j < dpad; j += blockDim.x) {
    double s = 0.0;
    for (int b = 0; b < nparts; ++b) s += part[(int64_t)b * dpad + j];
    c[j] = (float)(s / (double)n);
  }
}

__global__ void order_keys_kernel(const float* __restrict__ q, int64_t nq, int dim,
                                  const float* __restrict__ c, int cosine,
                                  unsigned* __restrict__ count, uint16_t* __restrict__ qbin) {
  const int lane = threadIdx.x & 31;
  const int64_t warps = (int64_t)gridDim.x * (blockDim.x >> 5);
  for (int64_t i = (int64_t)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5); i < nq;
       i += warps) {
    const float* row = q + i * dim;
    float ss = 0.f, qc = 0.f, cc = 0.f;
    for (int j = lane; j < dim; j += 32) {
      const float x = row[j], y = c[j];
      ss += x * x;
      qc += x * y;
      cc += y * y;
    }
#pragma unroll
    for (int o = 16; o >= 1; o >>= 1) {
      ss += __shfl_xor_sync(0xffffffffu, ss, o);
      qc += __shfl_xor_sync(0xffffffffu, qc, o);
      cc += __shfl_xor_sync(0xffffffffu, cc, o);
    }
    if (lane == 0) {
      // |s q - c|^2 = s^2 |q|^2 - 2 s <q, c> + |c|^2, s = 1 / |q| for cosine
      const float sc = (cosine && ss > 0.f) ? rsqrtf(ss) : 1.f;
      float key = sc * sc * ss - 2.f * sc * qc + cc;
      key = key > 0.f ? key : 0.f;  // (also maps NaN to 0)
      const unsigned bits = __float_as_uint(key) >> 19;  // < 4096 for key >= 0
      const int bin = SCHED_BINS - 1 - (int)bits;
      atomicAdd(count + bin, 1u);
      qbin[i] = (uint16_t)bin;
    }
  }
}

__global__ void __launch_bounds__(256) order_scatter_kernel(int64_t nq,
                                                            const unsigned* __restrict__ count,
                                                            unsigned* __restrict__ cursor,
                                                            const uint16_t* __restrict__ qbin,
                                                            int32_t* __restrict__ order) {
  __shared__ unsigned off[SCHED_BINS];
  __shared__ unsigned part[256];
  constexpr int PER = SCHED_BINS / 256;
  const int t = threadIdx.x;
  unsigned local[PER];
  uint4 c4[PER / 4];  // the thread's 16 counts in 4 vector loads (one round trip)
#pragma unroll
  for (int k = 0; k < PER / 4; ++k) c4[k] = reinterpret_cast<const uint4*>(count)[t * (PER / 4) + k];
  unsigned s = 0;
#pragma unroll
  for (int k = 0; k < PER / 4; ++k) {
    local[4 * k + 0] = s;
    s += c4[k].x;
    local[4 * k + 1] = s;
    s += c4[k].y;
    local[4 * k + 2] = s;
    s += c4[k].z;
    local[4 * k + 3] = s;
    s += c4[k].w;
  }
  // exclusive scan of the 256 partial sums: within warps by shuffles, then
  // across the 8 warp totals
  const int lane = t & 31, w = t >> 5;
  unsigned inc = s;
#pragma unroll
  for (int d = 1; d < 32; d <<= 1) {
    const unsigned v = __shfl_up_sync(0xffffffffu, inc, d);
    if (lane >= d) inc += v;
  }
  if (lane == 31) part[w] = inc;
  __syncthreads();
  unsigned wbase = 0;
  for (int k = 0; k < w; ++k) wbase += part[k];
  const unsigned base = wbase + inc - s;
#pragma unroll
  for (int k = 0; k < PER; ++k) off[t * PER + k] = base + local[k];
  __syncthreads();
  for (int64_t i = (int64_t)blockIdx.x * 256 + t; i < nq; i += (int64_t)gridDim.x * 256) {
    const int b = qbin[i];
    order[off[b] + atomicAdd(cursor + b, 1u)] = (int32_t)i;
  }
}

}  // namespace song
