// knn_tc.cuh — the NSW forward lists of reading R15 on the 5th-generation
// tensor cores: F(i) = the D smallest (d(i, j), j) over j < i.
//
// One CTA per 128-row block (heaviest blocks first: block ib has ib + 1
// column tiles of the triangular prefix), warp-specialised:
//   warp 0      TMA producer: 128 x 32-float chunks of the row block (A) and of
//               the column block (B), SWIZZLE_128B, into an NSTAGE ring
//   warp 1      TMEM allocator + MMA issuer: tcgen05.mma.kind::tf32, M = N =
//               128, K = 8 per instruction, D = A B^T accumulated in TMEM
//               (two 128-column accumulators: the MMA of tile t + 1 overlaps
//               the epilogue of tile t)
//   warps 2-5   epilogue: tcgen05.ld of the thread's row (128 columns), the
//               distance, and a per-row sorted top-32 list in shared memory
//               (insertion only below the row's current D-th key)
// The distance matrix never leaves the SM.  tf32 products are exact and fp32
// sums of them exact below 2^24, so on tf32-representable data (integers up to
// 2^11, e.g. the SIFT- and MNIST-shaped pixels) every distance equals the
// oracle's; song_build_graph uses this path only for such data (else the fp32
// FFMA tile path of graph_kernel.cuh).
#pragma once

#include <cuda.h>
#include <cuda_runtime.h>

#include <cstdint>

#include "graph_kernel.cuh"

namespace song {
namespace graph {
namespace tc {

constexpr int TM = 128, TN = 128, TK = 32;   // tile rows, tile columns, floats per chunk
constexpr int NSTAGE = 5;
constexpr int CHUNK_BYTES = TM * TK * 4;     // 16 KB (A and B chunks alike)
constexpr int STAGE_BYTES = 2 * CHUNK_BYTES;
constexpr int TOPW = GD + 1;                 // padded top-list row (u64)
constexpr int THREADS = 192;
constexpr size_t SMEM_BYTES = 1024 /*align*/ + (size_t)NSTAGE * STAGE_BYTES +
                              (size_t)TM * TOPW * 8 + 256;

__device__ __forceinline__ uint32_t su32(const void* p) {
  return (uint32_t)__cvta_generic_to_shared(p);
}
__device__ __forceinline__ void mbar_init(uint64_t* b, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(su32(b)), "r"(count));
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t* b, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(su32(b)), "r"(bytes)
               : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint64_t* b) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(su32(b)) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* b, uint32_t parity) {
  asm volatile(
      "{\n\t.reg .pred P1;\n\tLAB_WAIT:\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n\t"
      "@P1 bra DONE;\n\tbra LAB_WAIT;\n\tDONE:\n\t}" ::"r"(su32(b)),
      "r"(parity)
      : "memory");
}
__device__ __forceinline__ void tma_load_2d(void* dst, const CUtensorMap* map, uint64_t* bar,
                                            int c0, int c1) {
  asm volatile(
      "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes"
      " [%0], [%1, {%3, %4}], [%2];" ::"r"(su32(dst)),
      "l"(reinterpret_cast<uint64_t>(map)), "r"(su32(bar)), "r"(c0), "r"(c1)
      : "memory");
}
// K-major SWIZZLE_128B UMMA smem descriptor: LBO = 16 B (ignored), SBO = 1024 B
// (8-row groups), version 1 (sm_100), layout type 2 (SWIZZLE_128B)
__device__ __forceinline__ uint64_t umma_desc(uint32_t saddr) {
  return (uint64_t)((saddr >> 4) & 0x3FFF) | (1ull << 16) | (64ull << 32) | (1ull << 46) |
         (2ull << 61);
}
// kind::tf32 instruction descriptor: D f32, A/B tf32, both K-major, N = 128, M = 128
constexpr uint32_t IDESC = (1u << 4) | (2u << 7) | (2u << 10) | ((uint32_t)(TN >> 3) << 17) |
                           ((uint32_t)(TM >> 4) << 24);

__device__ __forceinline__ void mma_tf32(uint32_t dtmem, uint64_t adesc, uint64_t bdesc,
                                         uint32_t accumulate) {
  asm volatile(
      "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
      "tcgen05.mma.cta_group::1.kind::tf32 [%0], %1, %2, %3, p;\n\t}" ::"r"(dtmem),
      "l"(adesc), "l"(bdesc), "r"(IDESC), "r"(accumulate));
}
__device__ __forceinline__ void mma_commit(uint64_t* bar) {
  asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(
                   su32(bar))
               : "memory");
}

// 32 consecutive accumulator columns of this thread's TMEM lane
__device__ __forceinline__ void tmem_ld32(uint32_t taddr, float (&v)[32]) {
  uint32_t r[32];
  asm volatile(
      "tcgen05.ld.sync.aligned.32x32b.x32.b32 {%0, %1, %2, %3, %4, %5, %6, %7, %8, %9, %10, %11, "
      "%12, %13, %14, %15, %16, %17, %18, %19, %20, %21, %22, %23, %24, %25, %26, %27, %28, %29, "
      "%30, %31}, [%32];"
      : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]),
        "=r"(r[7]), "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]),
        "=r"(r[14]), "=r"(r[15]), "=r"(r[16]), "=r"(r[17]), "=r"(r[18]), "=r"(r[19]),
        "=r"(r[20]), "=r"(r[21]), "=r"(r[22]), "=r"(r[23]), "=r"(r[24]), "=r"(r[25]),
        "=r"(r[26]), "=r"(r[27]), "=r"(r[28]), "=r"(r[29]), "=r"(r[30]), "=r"(r[31])
      : "r"(taddr));
#pragma unroll
  for (int i = 0; i < 32; ++i) v[i] = __uint_as_float(r[i]);
}

__global__ void __launch_bounds__(THREADS, 1)
    knn_prefix_tc_kernel(const __grid_constant__ CUtensorMap xmap, int64_t n, int dim,
                         const float* __restrict__ norms, int metric, int D,
                         uint64_t* __restrict__ fkeys) {
  extern __shared__ unsigned char smem_raw[];
  unsigned char* smem = reinterpret_cast<unsigned char*>(
      (reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  unsigned char* stages = smem;                                      // NSTAGE x (A | B)
  uint64_t* top = reinterpret_cast<uint64_t*>(smem + (size_t)NSTAGE * STAGE_BYTES);
  uint64_t* bars = top + TM * TOPW;                                  // full, empty, tfull, tempty
  uint64_t* full = bars;
  uint64_t* empty = bars + NSTAGE;
  uint64_t* tfull = bars + 2 * NSTAGE;
  uint64_t* tempty = tfull + 2;
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(tempty + 2);

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int nb = (int)((n + TM - 1) / TM);
  const int ib = nb - 1 - (int)blockIdx.x;
  const int64_t i0 = (int64_t)ib * TM;
  const int ntiles = ib + 1;                  // column tiles j0 = 0, 128, ..., i0
  const int nk = (dim + TK - 1) / TK;

  if (threadIdx.x == 0) {
    for (int s = 0; s < NSTAGE; ++s) {
      mbar_init(&full[s], 1);
      mbar_init(&empty[s], 1);
    }
    for (int a = 0; a < 2; ++a) {
      mbar_init(&tfull[a], 1);
      mbar_init(&tempty[a], 128);
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (warp == 1) {  // 2 accumulators x 128 fp32 columns
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(
                     su32(tmem_slot)),
                 "r"(256));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  for (int e = threadIdx.x; e < TM * TOPW; e += THREADS) top[e] = KEY_MAX;
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
  const uint32_t tmem = *tmem_slot;

  if (warp == 0) {
    if (lane == 0) {  // ---- TMA producer
      int s = 0;
      uint32_t ph = 0;
      for (int t = 0; t < ntiles; ++t) {
        for (int kc = 0; kc < nk; ++kc) {
          mbar_wait(&empty[s], ph ^ 1);
          unsigned char* st = stages + (size_t)s * STAGE_BYTES;
          mbar_expect_tx(&full[s], STAGE_BYTES);
          tma_load_2d(st, &xmap, &full[s], kc * TK, (int)i0);
          tma_load_2d(st + CHUNK_BYTES, &xmap, &full[s], kc * TK, t * TN);
          if (++s == NSTAGE) {
            s = 0;
            ph ^= 1;
          }
        }
      }
    }
  } else if (warp == 1) {
    if (lane == 0) {  // ---- MMA issuer
      int s = 0;
      uint32_t ph = 0;
      for (int t = 0; t < ntiles; ++t) {
        const int acc = t & 1;
        mbar_wait(&tempty[acc], ((t >> 1) & 1) ^ 1);
        asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
        const uint32_t d = tmem + (uint32_t)(acc * TN);
        for (int kc = 0; kc < nk; ++kc) {
          mbar_wait(&full[s], ph);
          asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
          const uint32_t a = su32(stages + (size_t)s * STAGE_BYTES);
          const uint32_t b = a + CHUNK_BYTES;
#pragma unroll
          for (int k = 0; k < TK / 8; ++k)  // UMMA_K = 8 tf32 = 32 B along the swizzled row
            mma_tf32(d, umma_desc(a + 32 * k), umma_desc(b + 32 * k), (kc | k) != 0);
          mma_commit(&empty[s]);  // the stage is free once these MMAs have read it
          if (++s == NSTAGE) {
            s = 0;
            ph ^= 1;
          }
        }
        mma_commit(&tfull[acc]);  // the accumulator is complete
      }
    }
  } else {
    // ---- epilogue: thread = one row of the block (TMEM lane = row)
    const int q = warp & 3;                 // TMEM lane quarter this warp may access
    const int row = 32 * q + lane;
    const int64_t gi = i0 + row;
    const bool live = gi < n;
    const float ni = live ? norms[gi] : 0.f;
    uint64_t* mytop = top + (size_t)row * TOPW;
    uint64_t thr = KEY_MAX;                 // the row's current D-th key
    for (int t = 0; t < ntiles; ++t) {
      const int acc = t & 1;
      mbar_wait(&tfull[acc], (t >> 1) & 1);
      asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
      const int64_t j0 = (int64_t)t * TN;
      for (int c0 = 0; c0 < TN; c0 += 32) {
        float v[32];
        tmem_ld32(tmem + ((uint32_t)(32 * q) << 16) + (uint32_t)(acc * TN + c0), v);
        asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
        if (c0 + 32 == TN) {  // every column read: hand the accumulator back
          asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
          mbar_arrive(&tempty[acc]);
        }
        if (live && j0 + c0 < gi) {
        const float4* nj4 = reinterpret_cast<const float4*>(norms + j0 + c0);
#pragma unroll
        for (int c = 0; c < 32; c += 4) {
          const float4 nj = __ldg(nj4 + c / 4);
          const float njv[4] = {nj.x, nj.y, nj.z, nj.w};
#pragma unroll
          for (int u = 0; u < 4; ++u) {
            const int64_t j = j0 + c0 + c + u;
            const uint64_t key = make_key(pair_dist(v[c + u], ni, njv[u], metric), (int)j);
            if (j < gi && key < thr) {
              // sorted insertion into the row's list (rare once the list is warm)
              int p = D - 1;
              while (p > 0 && mytop[p - 1] > key) {
                mytop[p] = mytop[p - 1];
                --p;
              }
              mytop[p] = key;
              thr = mytop[D - 1];
            }
          }
        }
        }
      }
    }
    if (live)
      for (int p = 0; p < D; ++p) fkeys[gi * D + p] = mytop[p];
  }
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  if (warp == 1) {
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(256));
  }
}

}  // namespace tc
}  // namespace graph
}  // namespace song
