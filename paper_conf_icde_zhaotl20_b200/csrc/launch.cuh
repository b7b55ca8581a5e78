// launch.cuh — kernel dispatch (template instantiation lives in
// launch_nch<N>.cu so the 128 kernel variants compile in parallel).
#pragma once

#include <algorithm>

#include "song_internal.h"

namespace song {

// global visited tables for the HASH_GLOBAL kinds: one table of 2^table_log2
// u64 slots per launched warp; generations make clearing unnecessary
inline int prepare_global_tables(song_index* ix, SearchArgs& a, int64_t warps_total,
                          cudaStream_t st) {
  const size_t need = (size_t)warps_total * ((size_t)1 << a.table_log2) * sizeof(uint64_t);
  if (need > ix->gtab_bytes) {
    CUDA_TRY(cudaStreamSynchronize(st));
    cudaFree(ix->d_gtab);
    ix->d_gtab = nullptr;
    ix->gtab_bytes = 0;
    CUDA_TRY(cudaMalloc(&ix->d_gtab, need));
    ix->gtab_bytes = need;
    CUDA_TRY(cudaMemsetAsync(ix->d_gtab, 0, need, st));  // generation 0 is never used
    ix->gen_next = 1;
  }
  if (ix->gen_next + (uint64_t)a.nq + 1 >= 0xffffffffull) {
    CUDA_TRY(cudaMemsetAsync(ix->d_gtab, 0, ix->gtab_bytes, st));
    ix->gen_next = 1;
  }
  a.gtab = ix->d_gtab;
  a.gen0 = (uint32_t)ix->gen_next;
  ix->gen_next += (uint64_t)a.nq + 1;  // each warp uses gen0 + 1 + (its query count)
  return SONG_OK;
}

template <int NCH, int METRIC, int VK, int QR, bool MS>
int launch_t(song_index* ix, SearchArgs a, int warps, int blocks_per_sm, int num_sms,
             cudaStream_t st) {
  auto kern = song_search_kernel<NCH, METRIC, VK, QR, MS>;
  const size_t smem = (size_t)a.warp_smem_bytes * warps;
  CUDA_TRY(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
  int fit = 0;
  CUDA_TRY(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&fit, kern, warps * 32, smem));
  if (fit < 1) return fail(SONG_EUNSUPPORTED, "search kernel does not fit an SM (%zu B smem)", smem);
  int bps = blocks_per_sm > 0 ? std::min(blocks_per_sm, fit) : fit;
  int64_t want = (a.nq + warps - 1) / warps;
  int64_t grid = std::min<int64_t>((int64_t)bps * num_sms, want);
  if (VK == VK_GHASH) {
    int rc = prepare_global_tables(ix, a, grid * warps, st);
    if (rc) return rc;
  }
  if (QR == -2) {  // per-warp visited tables in global memory (cleared by the kernel)
    const size_t need = (size_t)grid * warps * ((size_t)4 << a.table_log2);
    if (need > ix->gvis_bytes) {
      CUDA_TRY(cudaStreamSynchronize(st));
      cudaFree(ix->d_gvis);
      ix->d_gvis = nullptr;
      ix->gvis_bytes = 0;
      CUDA_TRY(cudaMalloc(&ix->d_gvis, need));
      ix->gvis_bytes = need;
    }
    a.gvis = ix->d_gvis;
  }
  CUDA_TRY(cudaMemsetAsync(a.ticket, 0, sizeof(unsigned), st));
  kern<<<(unsigned)grid, warps * 32, smem, st>>>(a);
  CUDA_TRY(cudaGetLastError());
  return SONG_OK;
}

template <int NCH, int METRIC, int VK, bool MS = false>
int launch_q(song_index* ix, const SearchArgs& a, int qr, int warps, int bps, int sms,
             cudaStream_t st) {
  switch (qr) {
    case 1: return launch_t<NCH, METRIC, VK, 1, MS>(ix, a, warps, bps, sms, st);
    case 2: return launch_t<NCH, METRIC, VK, 2, MS>(ix, a, warps, bps, sms, st);
    case 4: return launch_t<NCH, METRIC, VK, 4, MS>(ix, a, warps, bps, sms, st);
    case 9:   // reading R17 with W in 1, 2 or 4 registers per lane (queue_len <= 128)
    case 10:
    case 12:
    case 16:
      if constexpr (VK == VK_HASH && !MS) {
        if (qr == 9) return launch_t<NCH, METRIC, VK, 9, false>(ix, a, warps, bps, sms, st);
        if (qr == 10) return launch_t<NCH, METRIC, VK, 10, false>(ix, a, warps, bps, sms, st);
#if SONG_RUN_MAX_L > 128
        if (qr == 16) return launch_t<NCH, METRIC, VK, 16, false>(ix, a, warps, bps, sms, st);
#endif
        return launch_t<NCH, METRIC, VK, 12, false>(ix, a, warps, bps, sms, st);
      } else {
        return fail(SONG_EUNSUPPORTED, "the bounded-union queue needs visited HASH, steps 1");
      }
    case -1:  // reading R17 (one bounded list of q ∪ topk): the hash visited set only
    case -2:  // ... with the visited table in global memory
      if constexpr (VK == VK_HASH && !MS) {
        if (qr == -2) return launch_t<NCH, METRIC, VK, -2, false>(ix, a, warps, bps, sms, st);
        return launch_t<NCH, METRIC, VK, -1, false>(ix, a, warps, bps, sms, st);
      } else {
        return fail(SONG_EUNSUPPORTED, "the bounded-union queue needs visited HASH, steps 1");
      }
    default: return launch_t<NCH, METRIC, VK, 0, MS>(ix, a, warps, bps, sms, st);
  }
}

template <int NCH, int METRIC>
int launch_v(song_index* ix, const SearchArgs& a, int vk, int qr, int warps, int bps,
             int sms, cudaStream_t st) {
  using namespace song;
  // multi-step probing (a.steps > 1, §V): hash-sel-del and Bloom only
  if (a.steps > 1) {
    if (vk == VK_BLOOM) return launch_q<NCH, METRIC, VK_BLOOM, true>(ix, a, qr, warps, bps, sms, st);
    if (vk == VK_HASH) return launch_q<NCH, METRIC, VK_HASH, true>(ix, a, qr, warps, bps, sms, st);
    return fail(SONG_EUNSUPPORTED, "multi-step probing supports the hash and Bloom visited sets");
  }
  switch (vk) {
    case VK_BLOOM: return launch_q<NCH, METRIC, VK_BLOOM>(ix, a, qr, warps, bps, sms, st);
    case VK_GHASH: return launch_q<NCH, METRIC, VK_GHASH>(ix, a, qr, warps, bps, sms, st);
    case VK_CUCKOO: return launch_q<NCH, METRIC, VK_CUCKOO>(ix, a, qr, warps, bps, sms, st);
    default: return launch_q<NCH, METRIC, VK_HASH>(ix, a, qr, warps, bps, sms, st);
  }
}

template <int NCH>
int launch_m(song_index* ix, const SearchArgs& a, int metric, int vk, int qr, int warps,
             int bps, int sms, cudaStream_t st) {
  if (metric == SONG_L2) return launch_v<NCH, MET_L2>(ix, a, vk, qr, warps, bps, sms, st);
  if (metric == SONG_HAMMING) {
    // codes: the two shared-memory visited sets of §IV (hash-sel-del, Bloom)
    if (vk == VK_BLOOM) return launch_q<NCH, MET_HAM, VK_BLOOM>(ix, a, qr, warps, bps, sms, st);
    if (vk == VK_HASH) return launch_q<NCH, MET_HAM, VK_HASH>(ix, a, qr, warps, bps, sms, st);
    return fail(SONG_EUNSUPPORTED, "Hamming indexes support the hash and Bloom visited sets");
  }
  return launch_v<NCH, MET_DOT>(ix, a, vk, qr, warps, bps, sms, st);
}

}  // namespace song
