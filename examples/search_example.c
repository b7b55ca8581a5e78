/* search_example.c — libsong.so used from plain C through include/song.h
 * (no Python, no torch): build an index from host arrays, search a batch
 * with host buffers, stream batches through song_search_pipelined, and check
 * the answer against brute force.
 *
 *   gcc -O2 -I include examples/search_example.c \
 *       -L paper_conf_icde_zhaotl20_b200 -lsong -Wl,-rpath,$PWD/paper_conf_icde_zhaotl20_b200 \
 *       -o /tmp/search_example && /tmp/search_example
 *
 * Data: n points on a d-dimensional integer grid with a ring + random-chord
 * graph (every vertex reachable from entry 0); with queue_len >= n the search
 * visits every reachable vertex, so its top K is the exact top K (Alg. 1 with
 * a full queue) and must equal brute force.  Exit status 0 = ok. */
#include <math.h>
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>

#include "song.h"

#define CHECK(call)                                                          \
  do {                                                                       \
    int rc_ = (call);                                                        \
    if (rc_ != SONG_OK) {                                                    \
      fprintf(stderr, "%s -> %d: %s\n", #call, rc_, song_last_error());      \
      return 1;                                                              \
    }                                                                        \
  } while (0)

static uint32_t rng = 12345u;
static uint32_t next_u32(void) {
  rng = rng * 1664525u + 1013904223u;
  return rng >> 8;
}

int main(void) {
  const int64_t n = 1500, nq = 64, nbatch = 3;
  const int32_t dim = 12, degree = 8, K = 5, L = 1536;
  float* x = malloc(sizeof(float) * n * dim);
  float* q = malloc(sizeof(float) * nbatch * nq * dim);
  int32_t* adj = malloc(sizeof(int32_t) * n * degree);
  int32_t* ids = malloc(sizeof(int32_t) * nbatch * nq * K);
  float* dists = malloc(sizeof(float) * nbatch * nq * K);
  for (int64_t i = 0; i < n * dim; ++i) x[i] = (float)(next_u32() % 16);
  for (int64_t i = 0; i < nbatch * nq * dim; ++i) q[i] = (float)(next_u32() % 16);
  for (int64_t v = 0; v < n; ++v) {
    adj[v * degree + 0] = (int32_t)((v + 1) % n);  /* ring: all reachable from 0 */
    for (int j = 1; j < degree; ++j) adj[v * degree + j] = (int32_t)(next_u32() % n);
  }

  printf("%s\n", song_version());
  song_index* idx = NULL;
  CHECK(song_index_create(x, n, dim, adj, degree, SONG_L2, &idx));
  song_index_info info;
  CHECK(song_index_get_info(idx, &info));
  printf("index: n=%lld dim=%d (padded %d) degree=%d, %lld B of vectors on device %d\n",
         (long long)info.n, info.dim, info.dim_padded, info.degree,
         (long long)info.vector_bytes, info.device);

  /* one batch, host buffers: HtoD + search + DtoH inside the call */
  CHECK(song_search(idx, q, nq, K, L, ids, dists));
  /* a stream of batches: copies overlap the searches */
  song_search_params p;
  song_default_params(&p, K, L);
  int32_t* ids_p = malloc(sizeof(int32_t) * nbatch * nq * K);
  float* dists_p = malloc(sizeof(float) * nbatch * nq * K);
  CHECK(song_search_pipelined(idx, &p, q, nbatch, nq, ids_p, dists_p));

  int bad = 0;
  for (int64_t b = 0; b < nbatch; ++b) {
    for (int64_t i = 0; i < nq; ++i) {
      const float* qi = q + (b * nq + i) * dim;
      /* brute force: the K smallest (squared L2, id) pairs */
      float bd[8];
      int32_t bi[8];
      for (int k = 0; k < K; ++k) {
        bd[k] = INFINITY;
        bi[k] = -1;
      }
      for (int64_t v = 0; v < n; ++v) {
        float d = 0.f;
        for (int c = 0; c < dim; ++c) {
          const float t = qi[c] - x[v * dim + c];
          d += t * t;
        }
        int k = K;
        while (k > 0 && (d < bd[k - 1] || (d == bd[k - 1] && v < bi[k - 1]))) --k;
        if (k < K) {
          memmove(bd + k + 1, bd + k, sizeof(float) * (K - 1 - k));
          memmove(bi + k + 1, bi + k, sizeof(int32_t) * (K - 1 - k));
          bd[k] = d;
          bi[k] = (int32_t)v;
        }
      }
      for (int k = 0; k < K; ++k) {
        const int64_t o = (b * nq + i) * K + k;
        if (ids_p[o] != bi[k] || dists_p[o] != bd[k]) ++bad;
        if (b == 0 && (ids[o] != bi[k] || dists[o] != bd[k])) ++bad;
      }
    }
  }
  CHECK(song_index_destroy(idx));
  printf("%lld queries, %s\n", (long long)(nbatch * nq), bad ? "MISMATCH" : "exact top-K ok");
  free(x), free(q), free(adj), free(ids), free(dists), free(ids_p), free(dists_p);
  return bad ? 2 : 0;
}
