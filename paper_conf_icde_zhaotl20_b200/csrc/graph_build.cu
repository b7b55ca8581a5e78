// graph_build.cu — song_build_graph (include/song.h): the device graph builder
// of DESIGN.md reading R15 over the kernels of graph_kernel.cuh.
#include <cuda_runtime.h>

#include <cub/device/device_scan.cuh>
#include <cudaTypedefs.h>

#include <algorithm>
#include <cstdlib>
#include <cstring>

#include "graph_kernel.cuh"
#include "knn_tc.cuh"
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
// TMA descriptor of X [n][dim] fp32: 32-float x 128-row boxes, SWIZZLE_128B
// (the layout the UMMA descriptors of knn_tc.cuh expect)
int make_xmap(CUtensorMap* map, const float* x, int64_t n, int dim) {
  static PFN_cuTensorMapEncodeTiled_v12000 encode = nullptr;
  if (!encode) {
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", reinterpret_cast<void**>(&encode),
                                cudaEnableDefault, &q) != cudaSuccess ||
        q != cudaDriverEntryPointSuccess || !encode)
      return fail(SONG_ECUDA, "cuTensorMapEncodeTiled is unavailable");
  }
  cuuint64_t dims[2] = {(cuuint64_t)dim, (cuuint64_t)n};
  cuuint64_t strides[1] = {(cuuint64_t)dim * 4};
  cuuint32_t box[2] = {(cuuint32_t)song::graph::tc::TK, (cuuint32_t)song::graph::tc::TM};
  cuuint32_t estr[2] = {1, 1};
  CUresult r = encode(map, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, const_cast<float*>(x), dims,
                      strides, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE,
                      CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                      CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) return fail(SONG_ECUDA, "cuTensorMapEncodeTiled failed (%d)", (int)r);
  return SONG_OK;
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
  G_TRY(s.get(&norms, (n + 256) * sizeof(float)));  // (+ tail: tile-wide norm loads)
  G_TRY(cudaMemsetAsync(norms, 0, (n + 256) * sizeof(float), st));
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
  // 1. forward lists: tensor cores (tcgen05, tf32) when that is exact for the
  // data (every value tf32-representable, rows 16 B aligned), else fp32 FFMA
  bool use_tc = dim % 4 == 0 && metric != SONG_COSINE;
  const char* force = std::getenv("SONG_GRAPH_PATH");  // "simt" / "tc" (tests, A/B)
  if (use_tc && !(force && std::strcmp(force, "tc") == 0)) {
    int* d_flag = nullptr;
    G_TRY(s.get(&d_flag, sizeof(int)));
    G_TRY(cudaMemsetAsync(d_flag, 0, sizeof(int), st));
    song::graph::tc::tf32_exact_kernel<<<592, 256, 0, st>>>(x, n * (int64_t)dim, d_flag);
    G_TRY(cudaGetLastError());
    int not_exact = 0;
    G_TRY(cudaMemcpyAsync(&not_exact, d_flag, sizeof(int), cudaMemcpyDeviceToHost, st));
    G_TRY(cudaStreamSynchronize(st));
    use_tc = !not_exact;
  }
  if (force && std::strcmp(force, "simt") == 0) use_tc = false;
  if (use_tc) {
    namespace tc = song::graph::tc;
    CUtensorMap xmap;
    int rc = make_xmap(&xmap, x, n, dim);
    if (rc) return rc;
    G_TRY(cudaFuncSetAttribute(tc::knn_prefix_tc_kernel,
                               cudaFuncAttributeMaxDynamicSharedMemorySize,
                               (int)tc::SMEM_BYTES));
    const int64_t nbt = (n + tc::TM - 1) / tc::TM;
    tc::knn_prefix_tc_kernel<<<(unsigned)nbt, tc::THREADS, tc::SMEM_BYTES, st>>>(
        xmap, n, dim, norms, met, D, fkeys);
    G_TRY(cudaGetLastError());
  } else {
    const int64_t nb = (n + BM - 1) / BM;
    knn_prefix_kernel<<<(unsigned)nb, THREADS, 0, st>>>(x, n, dim, norms, met, D, fkeys);
    G_TRY(cudaGetLastError());
  }
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
