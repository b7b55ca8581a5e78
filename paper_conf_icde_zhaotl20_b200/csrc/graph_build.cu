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
  void* p[24] = {};
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

// one pass over the builder's input rows: non-finite values (rejected),
// whether every value is an integer, and the largest |value| (bits of a
// non-negative float compare like ints) — the tensor-core Gram is taken only
// when it is provably exact (forward_exact)
struct RowScan {
  unsigned long long nonfinite;
  int non_integer;
  unsigned max_abs_bits;
};

__global__ void scan_rows_kernel(const float* __restrict__ x, int64_t m, RowScan* out) {
  unsigned long long bad = 0;
  int nonint = 0;
  unsigned mx = 0;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < m;
       i += (int64_t)gridDim.x * blockDim.x) {
    const float v = x[i];
    if (!isfinite(v)) {
      ++bad;
      continue;
    }
    nonint |= rintf(v) != v;
    mx = max(mx, __float_as_uint(fabsf(v)));
  }
  if (bad) atomicAdd(&out->nonfinite, bad);
  if (__syncthreads_or(nonint) && threadIdx.x == 0) atomicOr(&out->non_integer, 1);
  for (int o = 16; o >= 1; o >>= 1) mx = max(mx, __shfl_xor_sync(0xffffffffu, mx, o));
  if ((threadIdx.x & 31) == 0 && mx) atomicMax(&out->max_abs_bits, mx);
}

// forward-list ids given by the caller: in [-1, n)
__global__ void check_ids_kernel(const int32_t* __restrict__ ids, int64_t m, int64_t n,
                                 unsigned long long* bad) {
  unsigned long long b = 0;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < m;
       i += (int64_t)gridDim.x * blockDim.x)
    b += (ids[i] < -1 || ids[i] >= n);
  if (b) atomicAdd(bad, b);
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

namespace {
using song::fail;

// graph of rows [0, n) from the forward lists fkeys[0, n): R15 steps 2-4
struct Finish {
  uint64_t *bkeys = nullptr, *inc = nullptr;
  unsigned long long* cnt = nullptr;
  int64_t* off = nullptr;
  int *cursor = nullptr, *cnt32 = nullptr;
  void* tmp = nullptr;
  size_t tmp_bytes = 0;
  cudaError_t alloc(Scratch& s, int64_t n, int D, cudaStream_t st) {
    const int64_t nedges = n * (int64_t)D;
    cudaError_t e;
    if ((e = s.get(&bkeys, nedges * sizeof(uint64_t)))) return e;
    if ((e = s.get(&inc, nedges * sizeof(uint64_t)))) return e;
    if ((e = s.get(&cnt, n * sizeof(unsigned long long)))) return e;
    if ((e = s.get(&off, (n + 1) * sizeof(int64_t)))) return e;
    if ((e = s.get(&cursor, n * sizeof(int)))) return e;
    if ((e = s.get(&cnt32, n * sizeof(int)))) return e;
    if ((e = cub::DeviceScan::ExclusiveSum(nullptr, tmp_bytes, off, off, n, st))) return e;
    return s.get(&tmp, tmp_bytes);
  }
};

int finish_graph(const float* x, int64_t n, int dim, int met, int D, const float* norms,
                 const uint64_t* fkeys, Finish& f, int32_t* adjacency_out, cudaStream_t st) {
  using namespace song::graph;
  const int64_t nedges = n * (int64_t)D;
  // 2. backward lists
  G_TRY(cudaMemsetAsync(f.cnt, 0, n * sizeof(unsigned long long), st));
  G_TRY(cudaMemsetAsync(f.cursor, 0, n * sizeof(int), st));
  const int eb = (int)std::min<int64_t>((nedges + 255) / 256, 148 * 32);
  count_u64_kernel<<<eb, 256, 0, st>>>(fkeys, nedges, f.cnt);
  G_TRY(cudaGetLastError());
  i64_from_u64_kernel<<<eb, 256, 0, st>>>(f.cnt, f.off, n);
  narrow_kernel<<<eb, 256, 0, st>>>(f.cnt, f.cnt32, n);
  G_TRY(cudaGetLastError());
  size_t tb = f.tmp_bytes;
  G_TRY(cub::DeviceScan::ExclusiveSum(f.tmp, tb, f.off, f.off, n, st));
  reverse_scatter_kernel<<<eb, 256, 0, st>>>(fkeys, nedges, D, f.off, f.cursor, f.inc);
  G_TRY(cudaGetLastError());
  const int blocks = (int)std::min<int64_t>((n + 7) / 8, 65535);
  reverse_select_kernel<<<blocks, 256, 0, st>>>(f.inc, f.off, f.cnt32, n, D, f.bkeys);
  G_TRY(cudaGetLastError());
  // 3. + 4. candidates and the heuristic
  const int pb = (int)std::min<int64_t>(n, 148 * 16);
  prune_kernel<<<pb, PT, 0, st>>>(x, n, dim, norms, met, D, fkeys, f.bkeys, adjacency_out);
  G_TRY(cudaGetLastError());
  return SONG_OK;
}

// R15 step 1 on rows [0, n): tensor cores (tcgen05, tf32) only when that is
// provably exact — every value an integer with dim * max|x|^2 < 2^24, so every
// product and partial sum is an integer below 2^24 and any summation order
// gives the same fp32 result as the FFMA tiles and the oracle — else FFMA
int forward_exact(const float* x, int64_t n, int dim, int met, bool cosine, int D,
                  const float* norms, const RowScan& scan, uint64_t* fkeys, Scratch& s,
                  cudaStream_t st) {
  using namespace song::graph;
  float mx;
  std::memcpy(&mx, &scan.max_abs_bits, sizeof mx);
  bool use_tc = dim % 4 == 0 && !cosine && (reinterpret_cast<uintptr_t>(x) & 15) == 0 &&
                !scan.non_integer && (double)dim * mx * mx < 16777216.0;
  const char* force = std::getenv("SONG_GRAPH_PATH");  // "simt" / "tc" (tests, A/B)
  if (force && std::strcmp(force, "tc") == 0)
    use_tc = dim % 4 == 0 && !cosine && (reinterpret_cast<uintptr_t>(x) & 15) == 0;
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
  return SONG_OK;
}

// scan the input rows (rejecting non-finite values: song.h, SONG_EINVAL)
int scan_rows(const float* vectors, int64_t n, int dim, Scratch& s, RowScan* out,
              cudaStream_t st) {
  RowScan* d = nullptr;
  G_TRY(s.get(&d, sizeof(RowScan)));
  G_TRY(cudaMemsetAsync(d, 0, sizeof(RowScan), st));
  scan_rows_kernel<<<592, 256, 0, st>>>(vectors, n * (int64_t)dim, d);
  G_TRY(cudaGetLastError());
  G_TRY(cudaMemcpyAsync(out, d, sizeof(RowScan), cudaMemcpyDeviceToHost, st));
  G_TRY(cudaStreamSynchronize(st));
  if (out->nonfinite)
    return fail(SONG_EINVAL, "%llu non-finite vector values", out->nonfinite);
  return SONG_OK;
}

int check_build_args(const float* vectors, int64_t n, int32_t dim, song_metric metric,
                     int32_t degree, int32_t* adjacency_out) {
  if (!vectors || !adjacency_out) return fail(SONG_EINVAL, "NULL argument");
  if (n < 1 || dim < 1 || degree < 1) return fail(SONG_EINVAL, "n, dim and degree must be >= 1");
  if (n > 0x7fffffffll) return fail(SONG_EUNSUPPORTED, "n must fit int32 ids");
  if (degree > SONG_MAX_DEGREE)
    return fail(SONG_EUNSUPPORTED, "degree %d > %d", degree, SONG_MAX_DEGREE);
  if (metric < SONG_L2 || metric > SONG_COSINE)
    return fail(SONG_EINVAL, "metric %d: the builder takes SONG_L2, SONG_IP or SONG_COSINE",
                (int)metric);
  return SONG_OK;
}

// row norms (and the normalised scratch copy for cosine: 1 - cos)
int prepare_rows(const float* vectors, int64_t n, int dim, song_metric metric, Scratch& s,
                 float** norms, const float** x, cudaStream_t st) {
  using namespace song::graph;
  G_TRY(s.get(norms, (n + 256) * sizeof(float)));  // (+ tail: tile-wide norm loads)
  G_TRY(cudaMemsetAsync(*norms, 0, (n + 256) * sizeof(float), st));
  *x = vectors;
  if (metric == SONG_COSINE) {
    float* xs = nullptr;
    G_TRY(s.get(&xs, (size_t)n * dim * sizeof(float)));
    G_TRY(cudaMemcpyAsync(xs, vectors, (size_t)n * dim * sizeof(float), cudaMemcpyDeviceToDevice, st));
    *x = xs;
  }
  const int blocks = (int)std::min<int64_t>((n + 7) / 8, 65535);
  row_norms_kernel<<<blocks, 256, 0, st>>>(const_cast<float*>(*x), n, dim, *norms,
                                           metric == SONG_COSINE);
  G_TRY(cudaGetLastError());
  return SONG_OK;
}

// search results [nq][D] (ids, dists) -> forward keys (reading R16 step 2)
__global__ void keys_from_results_kernel(const int32_t* __restrict__ ids,
                                         const float* __restrict__ dists, int64_t cnt,
                                         uint64_t* __restrict__ fkeys) {
  for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < cnt;
       e += (int64_t)gridDim.x * blockDim.x) {
    const int id = ids[e];
    fkeys[e] = id >= 0 ? song::make_key(dists[e], id) : song::KEY_MAX;
  }
}

// reading R18: row v = the first `take` ids of first[v], then the ids of
// second[v], then the rest of first[v] — each id once (first occurrence),
// -1 skipped, truncated to degree, -1 padded.  One warp per row, lane j =
// slot j of each input row.
__global__ void merge_rows_kernel(const int32_t* __restrict__ first,
                                  const int32_t* __restrict__ second, int64_t n, int degree,
                                  int take, int32_t* __restrict__ out) {
  const int lane = threadIdx.x & 31;
  unsigned lt;
  asm("mov.u32 %0, %%lanemask_lt;" : "=r"(lt));
  for (int64_t v = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5; v < n;
       v += ((int64_t)gridDim.x * blockDim.x) >> 5) {
    const int a = lane < degree ? first[v * degree + lane] : -1;
    const int b = lane < degree ? second[v * degree + lane] : -1;
    // the candidate sequence: a[0..take), b[0..D), a[take..D)
    int nk = 0;        // ids kept so far (warp-uniform)
    int mine = -1;     // lane j < nk: the j-th kept id
    auto take_from = [&](int id, bool in) {
      bool keep = in && id >= 0;
      // first occurrence inside this group
      const unsigned grp = __match_any_sync(0xffffffffu, keep ? id : -1 - lane);
      keep = keep && (grp & lt) == 0;
      // not kept before
      for (int j = 0; j < nk; ++j) {  // (the shuffle outside the &&: every lane calls it)
        const int kj = __shfl_sync(0xffffffffu, mine, j);
        keep = keep && kj != id;
      }
      const unsigned m = __ballot_sync(0xffffffffu, keep);
      const int pos = nk + __popc(m & lt);
      // lane pos receives id: every lane with keep sends to lane pos
      for (unsigned mm = m; mm; mm &= mm - 1) {
        const int src = __ffs(mm) - 1;
        const int idv = __shfl_sync(0xffffffffu, id, src);
        const int p = nk + __popc(m & ((1u << src) - 1));
        if (lane == p) mine = idv;
      }
      nk = min(32, nk + __popc(m));
    };
    take_from(a, lane < take);
    take_from(b, true);
    take_from(a, lane >= take);
    if (lane < degree) out[v * degree + lane] = lane < nk ? mine : -1;
  }
}

}  // namespace

extern "C" int song_graph_merge_rows(const int32_t* first, const int32_t* second, int64_t n,
                                     int32_t degree, int32_t take_first, int32_t* out,
                                     void* stream) {
  if (!first || !second || !out) return fail(SONG_EINVAL, "NULL argument");
  if (n < 1 || degree < 1) return fail(SONG_EINVAL, "n and degree must be >= 1");
  if (degree > SONG_MAX_DEGREE) return fail(SONG_EUNSUPPORTED, "degree %d > %d", degree, SONG_MAX_DEGREE);
  if (take_first < 0 || take_first > degree)
    return fail(SONG_EINVAL, "take_first %d outside [0, degree]", take_first);
  const int blocks = (int)std::min<int64_t>((n + 7) / 8, 148 * 64);
  merge_rows_kernel<<<blocks, 256, 0, (cudaStream_t)stream>>>(first, second, n, degree, take_first, out);
  G_TRY(cudaGetLastError());
  return SONG_OK;
}

extern "C" int song_build_graph(const float* vectors, int64_t n, int32_t dim, song_metric metric,
                                int32_t degree, int32_t* adjacency_out, void* stream) {
  int rc = check_build_args(vectors, n, dim, metric, degree, adjacency_out);
  if (rc) return rc;
  cudaStream_t st = (cudaStream_t)stream;
  const int D = degree;
  const int met = metric == SONG_L2 ? 0 : metric == SONG_IP ? 1 : 2;
  Scratch s;
  float* norms = nullptr;
  const float* x = nullptr;
  uint64_t* fkeys = nullptr;
  RowScan scan;
  if ((rc = scan_rows(vectors, n, dim, s, &scan, st))) return rc;
  if ((rc = prepare_rows(vectors, n, dim, metric, s, &norms, &x, st))) return rc;
  G_TRY(s.get(&fkeys, n * (int64_t)D * sizeof(uint64_t)));
  // 1. forward lists
  if ((rc = forward_exact(x, n, dim, met, metric == SONG_COSINE, D, norms, scan, fkeys, s, st)))
    return rc;
  // 2. - 4.
  Finish f;
  G_TRY(f.alloc(s, n, D, st));
  if ((rc = finish_graph(x, n, dim, met, D, norms, fkeys, f, adjacency_out, st))) return rc;
  G_TRY(cudaStreamSynchronize(st));  // the scratch is freed on return
  return SONG_OK;
}

extern "C" int song_build_graph_batched(const float* vectors, int64_t n, int32_t dim,
                                        song_metric metric, int32_t degree, int32_t prefix,
                                        int32_t queue_len, int32_t batch_shift,
                                        int32_t* adjacency_out, void* stream) {
  int rc = check_build_args(vectors, n, dim, metric, degree, adjacency_out);
  if (rc) return rc;
  if (prefix < 1) return fail(SONG_EINVAL, "prefix %d < 1", prefix);
  if (queue_len < degree || queue_len > SONG_MAX_QUEUE_LEN)
    return fail(SONG_EINVAL, "queue_len %d outside [degree, %d]", queue_len, SONG_MAX_QUEUE_LEN);
  if (batch_shift < 0 || batch_shift > 16) return fail(SONG_EINVAL, "batch_shift %d outside [0, 16]", batch_shift);
  cudaStream_t st = (cudaStream_t)stream;
  const int D = degree;
  const int met = metric == SONG_L2 ? 0 : metric == SONG_IP ? 1 : 2;
  Scratch s;
  float* norms = nullptr;
  const float* x = nullptr;
  uint64_t* fkeys = nullptr;
  RowScan scan;
  if ((rc = scan_rows(vectors, n, dim, s, &scan, st))) return rc;
  if ((rc = prepare_rows(vectors, n, dim, metric, s, &norms, &x, st))) return rc;
  G_TRY(s.get(&fkeys, n * (int64_t)D * sizeof(uint64_t)));
  // 1. exact forward lists of the prefix (R15 step 1)
  const int64_t m0 = std::min<int64_t>(n, prefix);
  if ((rc = forward_exact(x, m0, dim, met, metric == SONG_COSINE, D, norms, scan, fkeys, s, st)))
    return rc;
  Finish f;
  G_TRY(f.alloc(s, n, D, st));
  if (m0 < n) {
    // the search's view of the rows: [n][dpad] (16 B rows; normalised for cosine)
    const int dpad = (dim + 3) & ~3;
    const float* xv = x;
    if (dpad != dim) {
      float* xp = nullptr;
      G_TRY(s.get(&xp, (size_t)n * dpad * sizeof(float)));
      G_TRY(cudaMemsetAsync(xp, 0, (size_t)n * dpad * sizeof(float), st));
      G_TRY(cudaMemcpy2DAsync(xp, dpad * sizeof(float), x, dim * sizeof(float), dim * sizeof(float),
                              n, cudaMemcpyDeviceToDevice, st));
      xv = xp;
    }
    const int64_t CH = 1 << 22;  // queries per search launch
    int32_t* ids = nullptr;
    float* dists = nullptr;
    G_TRY(s.get(&ids, CH * D * sizeof(int32_t)));
    G_TRY(s.get(&dists, CH * D * sizeof(float)));
    song_search_params p;
    song_default_params(&p, D, queue_len);
    song_index* view = nullptr;
    if ((rc = song::make_search_view(xv, n, dim, D, (int)metric, adjacency_out, &view))) return rc;
    int64_t m = m0;
    while (m < n && rc == SONG_OK) {
      const int64_t b = std::min<int64_t>(n - m, std::max<int64_t>(1, m >> batch_shift));
      // G_m = R15 steps 2-4 on F of rows [0, m), into adjacency rows [0, m)
      if ((rc = finish_graph(x, m, dim, met, D, norms, fkeys, f, adjacency_out, st))) break;
      // every row of the batch searches G_m: F(i) = its top D (ids < m)
      for (int64_t c0 = m; c0 < m + b && rc == SONG_OK; c0 += CH) {
        const int64_t nc = std::min<int64_t>(CH, m + b - c0);
        rc = song::search_view(view, m, &p, vectors + c0 * dim, nc, ids, dists, st);
        if (rc) break;
        const int kb = (int)std::min<int64_t>((nc * D + 255) / 256, 148 * 32);
        keys_from_results_kernel<<<kb, 256, 0, st>>>(ids, dists, nc * D, fkeys + c0 * D);
        if (cudaGetLastError() != cudaSuccess) rc = fail(SONG_ECUDA, "keys_from_results launch");
      }
      m += b;
    }
    int status = 0;
    if (rc == SONG_OK) rc = song::view_status(view, &status, st);
    song::free_search_view(view);
    if (rc) return rc;
    if (status) return fail(SONG_ECUDA, "batch search status %d", status);
  }
  // 3. the graph on all rows
  if ((rc = finish_graph(x, n, dim, met, D, norms, fkeys, f, adjacency_out, st))) return rc;
  G_TRY(cudaStreamSynchronize(st));
  return SONG_OK;
}

extern "C" int song_build_graph_from_forward(const float* vectors, int64_t n, int32_t dim,
                                             song_metric metric, int32_t degree,
                                             const int32_t* fwd_ids, const float* fwd_dists,
                                             int32_t* adjacency_out, void* stream) {
  int rc = check_build_args(vectors, n, dim, metric, degree, adjacency_out);
  if (rc) return rc;
  if (!fwd_ids || !fwd_dists) return fail(SONG_EINVAL, "NULL forward lists");
  cudaStream_t st = (cudaStream_t)stream;
  const int D = degree;
  const int met = metric == SONG_L2 ? 0 : metric == SONG_IP ? 1 : 2;
  Scratch s;
  float* norms = nullptr;
  const float* x = nullptr;
  uint64_t* fkeys = nullptr;
  RowScan scan;
  if ((rc = scan_rows(vectors, n, dim, s, &scan, st))) return rc;
  {
    unsigned long long* d_bad = nullptr;
    G_TRY(s.get(&d_bad, sizeof *d_bad));
    G_TRY(cudaMemsetAsync(d_bad, 0, sizeof *d_bad, st));
    check_ids_kernel<<<592, 256, 0, st>>>(fwd_ids, n * (int64_t)D, n, d_bad);
    G_TRY(cudaGetLastError());
    unsigned long long bad = 0;
    G_TRY(cudaMemcpyAsync(&bad, d_bad, sizeof bad, cudaMemcpyDeviceToHost, st));
    G_TRY(cudaStreamSynchronize(st));
    if (bad) return fail(SONG_EINVAL, "%llu forward-list ids outside [-1, n)", bad);
  }
  if ((rc = prepare_rows(vectors, n, dim, metric, s, &norms, &x, st))) return rc;
  G_TRY(s.get(&fkeys, n * (int64_t)D * sizeof(uint64_t)));
  const int kb = (int)std::min<int64_t>((n * D + 255) / 256, 148 * 32);
  keys_from_results_kernel<<<kb, 256, 0, st>>>(fwd_ids, fwd_dists, n * D, fkeys);
  G_TRY(cudaGetLastError());
  Finish f;
  G_TRY(f.alloc(s, n, D, st));
  if ((rc = finish_graph(x, n, dim, met, D, norms, fkeys, f, adjacency_out, st))) return rc;
  G_TRY(cudaStreamSynchronize(st));
  return SONG_OK;
}
