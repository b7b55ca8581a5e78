// rp_kernel.cuh — 1-bit random projection encoder (§VII).
//
// codes[i] bit j = [<x_i, r_j> > 0] (reading R11), packed LSB-first
// into h / 32 uint32 words ("the bit vector can be stored as several
// 32-bit unsigned integers").  The projection X R^T is a dense contraction
// (n x dim x h); it runs here as a register-tiled fp32 FFMA GEMM with the sign
// test and the bit packing fused into the epilogue, so only the codes (h / 8
// bytes per point) are ever written — the projections never reach HBM.
//
// Why fp32 CUDA cores and not tcgen05: each output is a sign decision, so the
// precision of the accumulation decides integers (the code bits).  fp32 keeps
// the decision within rounding of the oracle's fp64 (exactly equal on the
// workload's integer pixels and 1/64-step R, which tests certify); the tensor
// cores' tf32 / bf16 operand rounding would move it by ~1e-3 relative.  The
// encoder runs once per index (and per query batch, ~1 GFLOP for 10K MNIST
// queries at h = 128), off the search's critical path.
#pragma once

#include <cuda_runtime.h>

#include <cstdint>

namespace song {

constexpr int RP_TM = 128;     // points per CTA tile
constexpr int RP_TN = 64;      // bits per CTA tile (two code words)
constexpr int RP_TK = 16;      // dimensions per shared-memory stage
constexpr int RP_THREADS = 256;

// X [n][ldx] fp32 (dim used), R [h][dim] fp32, codes [n][ldc] words (the first
// h/32 written).
// grid = (ceil(n / 128), ceil(h / 64)); h % 32 == 0.
__global__ void __launch_bounds__(RP_THREADS) rp_encode_kernel(const float* __restrict__ X,
                                                                int64_t n, int dim, int64_t ldx,
                                                                const float* __restrict__ R, int h,
                                                                uint32_t* __restrict__ codes,
                                                                int64_t ldc) {
  __shared__ float xs[RP_TK][RP_TM + 4];  // k-major: xs[k][point]
  __shared__ float rs[RP_TK][RP_TN + 4];  // k-major: rs[k][bit]
  const int tid = threadIdx.x;
  const int tx = tid & 15;   // bit group: bits 4*tx .. 4*tx+3 of the tile
  const int ty = tid >> 4;   // point group: points 8*ty .. 8*ty+7 of the tile
  const int64_t p0 = (int64_t)blockIdx.x * RP_TM;
  const int b0 = blockIdx.y * RP_TN;
  float acc[8][4];
#pragma unroll
  for (int i = 0; i < 8; ++i)
#pragma unroll
    for (int j = 0; j < 4; ++j) acc[i][j] = 0.f;

  for (int k0 = 0; k0 < dim; k0 += RP_TK) {
    // stage X: 128 points x 16 dims, 8 per thread (16 consecutive dims of a
    // row per 16 threads: 64 B segments)
#pragma unroll
    for (int t = 0; t < 8; ++t) {
      const int e = t * RP_THREADS + tid;
      const int pr = e >> 4, kk = e & 15;
      const int64_t p = p0 + pr;
      const int k = k0 + kk;
      xs[kk][pr] = (p < n && k < dim) ? __ldg(X + p * ldx + k) : 0.f;
    }
    // stage R: 64 bits x 16 dims, 4 per thread
#pragma unroll
    for (int t = 0; t < 4; ++t) {
      const int e = t * RP_THREADS + tid;
      const int br = e >> 4, kk = e & 15;
      const int b = b0 + br;
      const int k = k0 + kk;
      rs[kk][br] = (b < h && k < dim) ? __ldg(R + (int64_t)b * dim + k) : 0.f;
    }
    __syncthreads();
#pragma unroll
    for (int kk = 0; kk < RP_TK; ++kk) {
      const float4 xa = *reinterpret_cast<const float4*>(&xs[kk][8 * ty]);
      const float4 xb = *reinterpret_cast<const float4*>(&xs[kk][8 * ty + 4]);
      const float4 r4 = *reinterpret_cast<const float4*>(&rs[kk][4 * tx]);
      const float xv[8] = {xa.x, xa.y, xa.z, xa.w, xb.x, xb.y, xb.z, xb.w};
      const float rv[4] = {r4.x, r4.y, r4.z, r4.w};
#pragma unroll
      for (int i = 0; i < 8; ++i)
#pragma unroll
        for (int j = 0; j < 4; ++j) acc[i][j] = fmaf(xv[i], rv[j], acc[i][j]);
    }
    __syncthreads();
  }
  // epilogue: sign -> nibble -> OR over the 8 lanes that share a code word
  // (lanes 0-7 and 8-15 of each 16-lane half-warp: tx = lane & 15)
  const int words = h >> 5;
#pragma unroll
  for (int i = 0; i < 8; ++i) {
    uint32_t nib = 0;
#pragma unroll
    for (int j = 0; j < 4; ++j) nib |= (acc[i][j] > 0.f ? 1u : 0u) << j;
    uint32_t w = nib << (4 * (tx & 7));
    w |= __shfl_xor_sync(0xffffffffu, w, 1);
    w |= __shfl_xor_sync(0xffffffffu, w, 2);
    w |= __shfl_xor_sync(0xffffffffu, w, 4);
    const int64_t p = p0 + 8 * ty + i;
    const int word = (b0 >> 5) + (tx >> 3);
    if ((tx & 7) == 0 && p < n && word < words) codes[p * ldc + word] = w;
  }
}

}  // namespace song
