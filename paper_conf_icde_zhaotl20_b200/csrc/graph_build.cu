// graph_build.cu — song_build_graph (include/song.h): the device graph builder
// of DESIGN.md reading R15 over the kernels of graph_kernel.cuh.
#include <cuda_runtime.h>

#include <cub/device/device_scan.cuh>

#include <algorithm>

#include "graph_kernel.cuh"
#include "song.h"
#include "song_internal.h"

namespace {
using song::fail;

struct Scratch {
  void* p[10] = {};
  int k = 0;
  ~Scratch() {
    for (int i = 0; i < k; ++i) cudaFree(p[i]);
  }
  template <class T>
  cudaError_t get(T** out, size_t bytes) {
    cudaError_t e = cudaMalloc(reinterpret_cast<void**>(out), bytes > 0 ? bytes : 1);
    if (e == cudaSuccess) p[k++] = *out;
    return e;
  }
};

__global__ void i64_from_u64_kernel(const unsigned long long* a, int64_t* b, int64_t n) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n;
       i += (int64_t)gridDim.x * blockDim.x)
    b[i] = (int64_t)a[i];
}

__global__ void count_u64_kernel(const uint64_t* __restrict__ fkeys, int64_t nedges,
                                 unsigned long long* cnt) {
  for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < nedges;
       e += (int64_t)gridDim.x * blockDim.x) {
    const uint64_t k = fkeys[e];
    if (k != song::KEY_MAX) atomicAdd(&cnt[song::key_id(k)], 1ull);
  }
}

__global__ void narrow_kernel(const unsigned long long* a, int* b, int64_t n) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n;
       i += (int64_t)gridDim.x * blockDim.x)
    b[i] = (int)a[i];
}
}  // namespace

#define G_TRY(expr)                                                                   \
  do {                                                                                \
    cudaError_t e_ = (expr);                                                          \
    if (e_ != cudaSuccess)                                                            \
      return fail(e_ == cudaErrorMemoryAllocation ? SONG_ENOMEM : SONG_ECUDA,         \
                  "song_build_graph: %s: %s", #expr, cudaGetErrorString(e_));         \
  } while (0)

extern "C" int song_build_graph(const float* vectors, int64_t n, int32_t dim, song_metric metric,
                                int32_t degree, int32_t* adjacency_out, void* stream) {
  using namespace song::graph;
  if (!vectors || !adjacency_out) return fail(SONG_EINVAL, "NULL argument");
  if (n < 1 || dim < 1 || degree < 1) return fail(SONG_EINVAL, "n, dim and degree must be >= 1");
  if (n > 0x7fffffffll) return fail(SONG_EUNSUPPORTED, "n must fit int32 ids");
  if (degree > SONG_MAX_DEGREE)
    return fail(SONG_EUNSUPPORTED, "degree %d > %d", degree, SONG_MAX_DEGREE);
  if (metric < SONG_L2 || metric > SONG_COSINE)
    return fail(SONG_EINVAL, "metric %d: the builder takes SONG_L2, SONG_IP or SONG_COSINE",
                (int)metric);
  cudaStream_t st = (cudaStream_t)stream;
  const int D = degree;
  const int64_t nedges = n * (int64_t)D;
  Scratch s;
  float* norms = nullptr;
  float* xs = nullptr;
  uint64_t *fkeys = nullptr, *bkeys = nullptr, *inc = nullptr;
  unsigned long long* cnt = nullptr;
  int64_t* off = nullptr;
  int *cursor = nullptr, *cnt32 = nullptr;
  G_TRY(s.get(&norms, n * sizeof(float)));
  const float* x = vectors;
  if (metric == SONG_COSINE) {  // normalise a scratch copy (1 - cos)
    G_TRY(s.get(&xs, (size_t)n * dim * sizeof(float)));
    G_TRY(cudaMemcpyAsync(xs, vectors, (size_t)n * dim * sizeof(float), cudaMemcpyDeviceToDevice, st));
    x = xs;
  }
  G_TRY(s.get(&fkeys, nedges * sizeof(uint64_t)));
  G_TRY(s.get(&bkeys, nedges * sizeof(uint64_t)));
  G_TRY(s.get(&inc, nedges * sizeof(uint64_t)));
  G_TRY(s.get(&cnt, n * sizeof(unsigned long long)));
  G_TRY(s.get(&off, (n + 1) * sizeof(int64_t)));
  G_TRY(s.get(&cursor, n * sizeof(int)));
  G_TRY(s.get(&cnt32, n * sizeof(int)));
  const int met = metric == SONG_L2 ? 0 : metric == SONG_IP ? 1 : 2;
  const int blocks = (int)std::min<int64_t>((n + 7) / 8, 65535);
  row_norms_kernel<<<blocks, 256, 0, st>>>(const_cast<float*>(x), n, dim, norms,
                                           metric == SONG_COSINE);
  G_TRY(cudaGetLastError());
  // 1. forward lists
  const int64_t nb = (n + BM - 1) / BM;
  knn_prefix_kernel<<<(unsigned)nb, THREADS, 0, st>>>(x, n, dim, norms, met, D, fkeys);
  G_TRY(cudaGetLastError());
  // 2. backward lists
  G_TRY(cudaMemsetAsync(cnt, 0, n * sizeof(unsigned long long), st));
  G_TRY(cudaMemsetAsync(cursor, 0, n * sizeof(int), st));
  const int eb = (int)std::min<int64_t>((nedges + 255) / 256, 148 * 32);
  count_u64_kernel<<<eb, 256, 0, st>>>(fkeys, nedges, cnt);
  G_TRY(cudaGetLastError());
  i64_from_u64_kernel<<<eb, 256, 0, st>>>(cnt, off, n);
  narrow_kernel<<<eb, 256, 0, st>>>(cnt, cnt32, n);
  G_TRY(cudaGetLastError());
  size_t tmp_bytes = 0;
  G_TRY(cub::DeviceScan::ExclusiveSum(nullptr, tmp_bytes, off, off, n, st));
  void* tmp = nullptr;
  G_TRY(s.get(&tmp, tmp_bytes));
  G_TRY(cub::DeviceScan::ExclusiveSum(tmp, tmp_bytes, off, off, n, st));
  reverse_scatter_kernel<<<eb, 256, 0, st>>>(fkeys, nedges, D, off, cursor, inc);
  G_TRY(cudaGetLastError());
  reverse_select_kernel<<<blocks, 256, 0, st>>>(inc, off, cnt32, n, D, bkeys);
  G_TRY(cudaGetLastError());
  // 3. + 4. candidates and the heuristic
  const int pb = (int)std::min<int64_t>(n, 148 * 16);
  prune_kernel<<<pb, PT, 0, st>>>(x, n, dim, norms, met, D, fkeys, bkeys, adjacency_out);
  G_TRY(cudaGetLastError());
  G_TRY(cudaStreamSynchronize(st));  // the scratch is freed on return
  return SONG_OK;
}
