// song_internal.h — definitions shared by the library's translation units
// (song_api.cu and launch_nch<N>.cu).  Not part of the public ABI.
#pragma once

#include <cuda_runtime.h>

#include <cstdint>
#include <string>

#include "search_kernel.cuh"
#include "song.h"

struct song_index {
  int device = 0;
  int num_sms = 0;
  int64_t n = 0;
  int dim = 0, dpad = 0, degree = 0, metric = 0;
  float* d_data = nullptr;
  int32_t* d_adj = nullptr;
  unsigned* d_ticket = nullptr;
  int* d_status = nullptr;
  int dedup = 1;                       // some adjacency row repeats an id
  uint64_t* d_gtab = nullptr;          // global visited tables (HASH_GLOBAL kinds)
  size_t gtab_bytes = 0;
  uint64_t gen_next = 1;               // next generation base for d_gtab
  int* d_gvis = nullptr;               // R17 global visited tables (QR == -2)
  size_t gvis_bytes = 0;
  cudaStream_t stream = nullptr;       // owned; used by song_search
  cudaStream_t last_stream = nullptr;  // stream of the last search
  cudaEvent_t last_done = nullptr;     // recorded after the last search's kernels
  // scratch for the host-buffer entry point
  float* d_q = nullptr;
  int32_t* d_ids = nullptr;
  float* d_dists = nullptr;
  size_t cap_q = 0, cap_out = 0;
  // SONG_HAMMING (§VII): dim / dpad count 32-bit code words
  int code_bits = 0;
  int rp_dim = 0;                      // length of float queries (0: codes only)
  float* d_R = nullptr;                // [code_bits][rp_dim] random vectors
  uint32_t* d_qcodes = nullptr;        // scratch: encoded query batch
  size_t cap_qcodes = 0;
  // outlier-first schedule (song_search_params.schedule)
  float* d_centroid = nullptr;         // [dpad] mean of the (normalised) rows
  unsigned* d_bins = nullptr;          // [2][SCHED_BINS] counts, cursors
  int32_t* d_order = nullptr;          // [nq] ticket -> query
  uint16_t* d_qbin = nullptr;          // [nq] bin of each query
  size_t cap_order = 0;
  int* h_status = nullptr;             // pinned: song_search's status read-back
  unsigned long long* d_stage = nullptr;  // SONG_STAGE_TIMING builds: [4] cycles
  // song_search_pipelined: a second lane (its own work counter, status, order
  // scratch, buffers and compute stream; the rows, graph, centroid and R are
  // this index's), copy streams, and per-lane events
  song_index* twin = nullptr;
  bool is_twin = false;
  cudaStream_t h2d = nullptr, d2h = nullptr;
  cudaEvent_t ev_h2d = nullptr, ev_done = nullptr, ev_out = nullptr;
};

// the bounded union (reading R17) keeps W in registers up to this queue_len
// (128: 4 u64 per lane; 256: 8), in shared-memory tiers above.  256: GloVe-IP
// at L 160 1.61 -> 1.63 M QPS once the wide-row prefetches were bulk (r03ap;
// 1.61 -> 1.56 M before, r03u)
#ifndef SONG_RUN_MAX_L
#define SONG_RUN_MAX_L 256
#endif

namespace song {
int fail(int code, const char* fmt, ...);
// non-owning search index over device rows (the batched graph builder, R16):
// xv [n][dpad] rows (normalised for cosine), adj [n][degree]; the view never
// frees them
int make_search_view(const float* xv, int64_t n, int dim, int degree, int metric, int32_t* adj,
                     song_index** out);
// search the view restricted to its first m rows (entry 0; ids < m)
int search_view(song_index* view, int64_t m, const song_search_params* p, const float* q,
                int64_t nq, int32_t* ids, float* dists, cudaStream_t st);
int view_status(song_index* view, int* status, cudaStream_t st);
void free_search_view(song_index* view);
}  // namespace song

#define CUDA_TRY(expr)                                                                  \
  do {                                                                                  \
    cudaError_t e_ = (expr);                                                            \
    if (e_ != cudaSuccess)                                                              \
      return song::fail(e_ == cudaErrorMemoryAllocation ? SONG_ENOMEM : SONG_ECUDA,     \
                        "%s: %s (%s:%d)", #expr, cudaGetErrorString(e_), __FILE__,     \
                        __LINE__);                                                      \
  } while (0)
