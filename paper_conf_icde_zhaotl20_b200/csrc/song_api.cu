// song_api.cu — the C ABI of include/song.h over the sm_100a kernels.
//
// Index layout in HBM: vectors [n][dpad] fp32 with dpad =
// round_up(dim, 4) so every row starts on a 16 B boundary (LDG.128 gathers);
// adjacency [n][degree] int32, -1 padded (fixed-degree storage).
#include <cuda_runtime.h>

#include <algorithm>
#include <cmath>
#include <cstdarg>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <string>

#include "merge_kernel.cuh"
#include "rp_kernel.cuh"
#include "schedule.cuh"
#include "search_kernel.cuh"
#include "mq_kernel.cuh"
#include "song.h"

#include "song_internal.h"

namespace song {
thread_local std::string g_err;

int fail(int code, const char* fmt, ...) {
  char buf[512];
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(buf, sizeof buf, fmt, ap);
  va_end(ap);
  g_err = buf;
  return code;
}
}  // namespace song

namespace song {
// launch_m<NCH> lives in launch_nch<NCH>.cu (one translation unit per NCH,
// compiled in parallel)
template <int NCH>
int launch_m(song_index* ix, const SearchArgs& a, int metric, int vk, int qr, int warps, int bps,
             int sms, cudaStream_t st);
}  // namespace song

namespace {
using song::fail;
using song::launch_m;
using song::g_err;


int next_pow2_log2(int64_t x) {
  int l = 0;
  while ((1ll << l) < x) ++l;
  return l;
}

// Validation (create_device): counts adjacency ids outside [-1, n) and
// non-finite vector values.
__global__ void validate_kernel(const float* __restrict__ v, int64_t nv,
                                const int32_t* __restrict__ adj, int64_t na, int64_t n,
                                unsigned long long* bad) {
  unsigned long long local = 0;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < nv;
       i += (int64_t)gridDim.x * blockDim.x)
    local += !isfinite(v[i]);
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < na;
       i += (int64_t)gridDim.x * blockDim.x) {
    int32_t a = adj[i];
    local += (a < -1 || a >= n);
  }
  if (local) atomicAdd(bad, local);
}

// Does any adjacency row list an id twice?  (If not, the search kernel skips
// the in-row de-duplication of reading A7.)
__global__ void dup_check_kernel(const int32_t* __restrict__ adj, int64_t n, int degree,
                                 int* any_dup) {
  const int lane = threadIdx.x & 31;
  for (int64_t r = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5; r < n;
       r += ((int64_t)gridDim.x * blockDim.x) >> 5) {
    int v = lane < degree ? adj[r * degree + lane] : -1;
    unsigned lt;
    asm("mov.u32 %0, %%lanemask_lt;" : "=r"(lt));
    unsigned grp = __match_any_sync(0xffffffffu, v);
    bool dup = v >= 0 && (grp & lt) != 0;
    if (__any_sync(0xffffffffu, dup) && lane == 0) atomicOr(any_dup, 1);
  }
}

// Cosine: rows are L2-normalised once at index creation so the search
// computes 1 - <q̂, x̂> with one dot product; zero rows stay zero (distance 1).
__global__ void normalize_rows_kernel(float* data, int64_t n, int dpad) {
  const int lane = threadIdx.x & 31;
  for (int64_t r = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5; r < n;
       r += ((int64_t)gridDim.x * blockDim.x) >> 5) {
    float* row = data + r * dpad;
    float s = 0.f;
    for (int i = lane; i < dpad; i += 32) s += row[i] * row[i];
    for (int o = 16; o >= 1; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
    float inv = s > 0.f ? 1.0f / sqrtf(s) : 0.f;
    for (int i = lane; i < dpad; i += 32) row[i] *= inv;
  }
}

int dpad_of(int dim, int metric) {
  return (metric == SONG_HAMMING && (dim == 1 || dim == 2)) ? dim : (dim + 3) & ~3;
}

int alloc_index(song_index* ix, int64_t n, int32_t dim, int32_t degree, song_metric metric) {
  CUDA_TRY(cudaGetDevice(&ix->device));
  CUDA_TRY(cudaDeviceGetAttribute(&ix->num_sms, cudaDevAttrMultiProcessorCount, ix->device));
  ix->n = n;
  ix->dim = dim;
  // float rows: 16 B multiples; codes: 1, 2 or a multiple of 4 words, so
  // h = 32 / 64 take exactly h / 8 bytes per point (Table IV)
  ix->dpad = dpad_of(dim, (int)metric);
  ix->degree = degree;
  ix->metric = (int)metric;
  CUDA_TRY(cudaMalloc(&ix->d_data, (size_t)n * ix->dpad * sizeof(float)));
  CUDA_TRY(cudaMalloc(&ix->d_adj, (size_t)n * degree * sizeof(int32_t)));
  CUDA_TRY(cudaMalloc(&ix->d_ticket, sizeof(unsigned)));
  CUDA_TRY(cudaMalloc(&ix->d_status, sizeof(int)));
  CUDA_TRY(cudaMemset(ix->d_status, 0, sizeof(int)));
  CUDA_TRY(cudaStreamCreateWithFlags(&ix->stream, cudaStreamNonBlocking));
  ix->last_stream = ix->stream;
  return SONG_OK;
}

void free_index(song_index* ix) {
  if (!ix) return;
  if (ix->twin) free_index(ix->twin);
  if (ix->is_twin) {  // the rows, graph, centroid and R belong to the owner
    ix->d_data = nullptr;
    ix->d_adj = nullptr;
    ix->d_centroid = nullptr;
    ix->d_R = nullptr;
  }
  if (ix->h2d) cudaStreamDestroy(ix->h2d);
  if (ix->d2h) cudaStreamDestroy(ix->d2h);
  if (ix->ev_h2d) cudaEventDestroy(ix->ev_h2d);
  if (ix->ev_done) cudaEventDestroy(ix->ev_done);
  if (ix->ev_out) cudaEventDestroy(ix->ev_out);
  cudaFree(ix->d_data);
  cudaFree(ix->d_adj);
  cudaFree(ix->d_ticket);
  cudaFree(ix->d_status);
  cudaFree(ix->d_q);
  cudaFree(ix->d_ids);
  cudaFree(ix->d_dists);
  cudaFree(ix->d_gtab);
  cudaFree(ix->d_gvis);
  cudaFree(ix->d_R);
  cudaFree(ix->d_centroid);
  cudaFreeHost(ix->h_status);
  cudaFree(ix->d_bins);
  cudaFree(ix->d_order);
  cudaFree(ix->d_qbin);
  cudaFree(ix->d_qcodes);
  cudaFree(ix->d_stage);
  if (ix->stream) cudaStreamDestroy(ix->stream);
  if (ix->last_done) cudaEventDestroy(ix->last_done);
  delete ix;
}

int check_create_args(const void* vectors, int64_t n, int32_t dim, const void* adjacency,
                      int32_t degree, song_metric metric, song_index** out) {
  if (!out) return fail(SONG_EINVAL, "out is NULL");
  *out = nullptr;
  if (!vectors || !adjacency) return fail(SONG_EINVAL, "vectors/adjacency is NULL");
  if (n < 1 || dim < 1 || degree < 1) return fail(SONG_EINVAL, "n, dim and degree must be >= 1");
  if (n > 0x7fffffffll) return fail(SONG_EUNSUPPORTED, "n must fit int32 ids");
  if (metric < SONG_L2 || metric > SONG_COSINE)
    return fail(SONG_EINVAL, "metric %d: float indexes take SONG_L2, SONG_IP or SONG_COSINE "
                             "(SONG_HAMMING indexes come from song_index_create_codes/_rp)",
                (int)metric);
  if (degree > SONG_MAX_DEGREE) return fail(SONG_EUNSUPPORTED, "degree %d > %d", degree, SONG_MAX_DEGREE);
  if (dim > SONG_MAX_DIM) return fail(SONG_EUNSUPPORTED, "dim %d > %d", dim, SONG_MAX_DIM);
  return SONG_OK;
}

#ifndef SONG_HASH_FACTOR
#define SONG_HASH_FACTOR 8
#endif
#ifndef SONG_HASH_FACTOR_WIDE  // 64 < L <= 128 (QR = 4)
#define SONG_HASH_FACTOR_WIDE 4
#endif
#ifndef SONG_HASH_REBUILD_NUM  // rebuild at NUM/16 occupancy
#define SONG_HASH_REBUILD_NUM 4
#endif
// per-warp shared memory of the search kernel
struct Shape {
  int lazy = 0;
  int table_log2;
  int rebuild_at;
  int warp_bytes;
  int qr;  // register queue width (L <= 32*qr), 0 = shared-memory tiers, -1 = union (R17)
  int qk;  // QueueKind
  int gvis;  // 1: the visited table in global memory (R17, QR == -2)
  int nch;
  int warps;  // warps per CTA
};

// slots of the shared-memory visited hash: >= F (2L + 32), the live-key bound;
// shared-memory queues (L > 128) take F = 4/3 — the least table whose 3/4
// still holds the bound (measured: at L = 1280 the 32 KB table of F = 2 held
// 3 warps per SM, the 16 KB one holds 5)
#ifndef SONG_HASH_BIG_NUM
#define SONG_HASH_BIG_NUM 4
#endif
#ifndef SONG_HASH_BIG_DEN
#define SONG_HASH_BIG_DEN 3
#endif
// the bounded union (reading R17) holds <= L + 32 live ids; its table is
// sized F_u (L + 32), F_u = NUM / DEN
#ifndef SONG_HASH_UNION_NUM
#define SONG_HASH_UNION_NUM 8
#endif
#ifndef SONG_HASH_UNION_DEN
#define SONG_HASH_UNION_DEN 3
#endif
// wide rows (NCH >= 2: > 128 floats, a 4 KB+ stage per warp) take F = 4 for
// L <= 64: shared memory, not recomputation, is their limit (NYTimes-shaped
// L = 56: 5.94 M -> 6.39 M QPS; SIFT-shaped rows keep 8: 19.6 M vs 18.4 M,
// profiles/r03hf_*)
#ifndef SONG_HASH_FACTOR_WIDEROW
#define SONG_HASH_FACTOR_WIDEROW 4
#endif
// queue_kind AUTO picks the union with W in registers for queue_len in
// [SONG_RUN_AUTO_MIN_L, 128] (above 128 the union is the default anyway).
// Measured against separate register q / topk at equal table sizes
// (profiles/r03q_*): SIFT1M L 16 19.6 -> 20.0 M QPS, K = 100 at L 100
// 5.49 -> 6.00 M, NYTimes L 56 6.39 -> 6.42 M: the pop no longer shifts q
// and no topk insertion runs (W keeps popped keys in place, flagged)
#ifndef SONG_RUN_AUTO_MIN_L
#define SONG_RUN_AUTO_MIN_L 1
#endif
// rows wider than 256 floats (GIST-shaped, 8 chunks per lane) keep F = 8: their
// 8-row stage (30 KB per warp) sets residency anyway, and a smaller table only
// adds recomputation (GIST L = 24: 2.67 M (F 4) -> 2.86 M QPS, profiles/r03p_*)
#ifndef SONG_HASH_FACTOR_XWIDE
#define SONG_HASH_FACTOR_XWIDE 8
#endif
int nch_of(int dpad, bool hamming) {
  int n = hamming ? (dpad + 3) / 4 : (dpad + 127) / 128;
  return n <= 1 ? 1 : n <= 2 ? 2 : n <= 4 ? 4 : 8;
}

int hash_log2_slots(int L, bool uni = false, int nch = 1) {
  // (queue_len <= 128: the union with W in registers takes the table of the
  // separate register queues — live ids <= L + 32 there, so the load halves
  // and lazy deletion rebuilds less often; F (L + 32) slots with F = 8/3, 3
  // or 4 measured slower (more recomputation: K = 100 6.01 -> 5.68 M at F 3,
  // NYTimes 6.42 -> 6.27 M at F 4, SIFT L 16 20.5 -> 19.7 M at F 4;
  // profiles/r03q_*, r03ad A/B)
  if (uni && L > 128)
    return next_pow2_log2((SONG_HASH_UNION_NUM * (L + 32ll) + SONG_HASH_UNION_DEN - 1) /
                          SONG_HASH_UNION_DEN);

  const long long live = 2ll * L + 32;
  if (L > 128) return next_pow2_log2((SONG_HASH_BIG_NUM * live + SONG_HASH_BIG_DEN - 1) / SONG_HASH_BIG_DEN);
  const long long F = L > 64 ? SONG_HASH_FACTOR_WIDE
                     : nch >= 4 ? SONG_HASH_FACTOR_XWIDE
                     : nch >= 2 ? SONG_HASH_FACTOR_WIDEROW : SONG_HASH_FACTOR;
  return next_pow2_log2(F * live);
}

// the queue structure of a search: registers (L <= 128, separate q / topk),
// shared-memory tiers (separate q / topk), or the bounded union (R17)
enum QueueKind { QK_REGS = 0, QK_SEPARATE = 1, QK_UNION = 2 };
int queue_kind_of(int L, int vk, const song_search_params* p) {
  const bool union_ok = vk == song::VK_HASH && p->steps <= 1;
  if (p->queue_kind == SONG_QUEUE_UNION && union_ok) return QK_UNION;
  if (L <= 128 && L >= SONG_RUN_AUTO_MIN_L && p->queue_kind == SONG_QUEUE_AUTO && union_ok)
    return QK_UNION;
  if (L <= 128) return QK_REGS;
  if (p->queue_kind == SONG_QUEUE_AUTO && union_ok) return QK_UNION;
  return QK_SEPARATE;
}

Shape search_shape(int L, int vk, const song_search_params* p, int dpad, bool hamming) {
  const int steps = p->steps;
  Shape s;
  if (p->queries_per_warp > 0) {  // Fig. 8's packing kernel (mq_kernel.cuh)
    s.table_log2 = hash_log2_slots(L, false, nch_of(dpad, hamming));
    s.rebuild_at = (1 << s.table_log2) / 4;  // tombstones: rebuild at 1/4 load
    s.lazy = 0;
    s.qr = 0;
    s.qk = QK_SEPARATE;
    s.gvis = 0;
    s.nch = nch_of(dpad, hamming);
    s.warps = 4;
    s.warp_bytes = p->queries_per_warp * song::mq_layout(L, dpad, s.table_log2).total;
    return s;
  }
  int tbytes = 0;
  s.rebuild_at = 0;
  if (vk == song::VK_BLOOM) {
    s.table_log2 = p->bloom_log2_bits > 0 ? p->bloom_log2_bits : next_pow2_log2(80ll * L);
    if (s.table_log2 < 5) s.table_log2 = 5;
    tbytes = (1 << s.table_log2) / 8;
  } else if (vk == song::VK_GHASH) {
    s.table_log2 = p->table_log2 > 0 ? p->table_log2 : std::max(14, next_pow2_log2(64ll * L));
    tbytes = 0;  // global memory
  } else if (vk == song::VK_CUCKOO) {
    // reading R10 default: 4 slots per key of the live bound 2L + 32
    s.table_log2 = p->table_log2 > 0 ? p->table_log2 : next_pow2_log2(4ll * (2 * L + 32)) - 2;
    tbytes = (4 << s.table_log2) * 2;
  } else if (queue_kind_of(L, vk, p) == QK_UNION) {
    // R17: live keys <= |W| + 32 new ones <= L + 32; lazy by default
    s.table_log2 = hash_log2_slots(L, true, nch_of(dpad, hamming));
    s.lazy = p->visited_cap >= 0;
    s.rebuild_at = s.lazy && p->visited_cap > 0 ? p->visited_cap : (3 << s.table_log2) / 4;
    tbytes = (1 << s.table_log2) * 4;
  } else {
    // live keys <= |q| + |topk| + 32 new ones <= 2L + 32.  Register-queue
    // sizes get >= 8x (L <= 64) or 4x (L <= 128: a 16 KB table would cut
    // residency to 10 warps/SM, measured 2.7M -> 3.9M QPS at K = 100) that many slots and rebuild at 1/4 occupancy (about one
    // probe per operation); shared-memory queues (L > 128) get >= 2x and
    // rebuild at 3/4 to bound shared memory.
    const bool big = L > 128;
    s.table_log2 = hash_log2_slots(L, false, nch_of(dpad, hamming));
    s.rebuild_at = big ? (3 << s.table_log2) / 4 : (SONG_HASH_REBUILD_NUM << s.table_log2) / 16;
    // lazy deletion (R14): visited holds up to C live ids, no tombstones
    s.lazy = p->visited_cap >= 0 && p->steps <= 1;
    if (s.lazy)
      s.rebuild_at = p->visited_cap > 0 ? p->visited_cap
                                        : (big ? (3 << s.table_log2) / 4 : (5 << s.table_log2) / 8);
    tbytes = (1 << s.table_log2) * 4;
  }
  // float rows: NCH = 16 B chunks per lane (128 floats per chunk row);
  // Hamming codes: NCH = 16 B chunks per code (4 words), no row stage
  s.nch = nch_of(dpad, hamming);
  const int qk = queue_kind_of(L, vk, p);
  s.qk = qk;
  const int regs = L <= 32 ? 1 : L <= 64 ? 2 : L <= 128 ? 4 : 8;
  // QR codes of the kernel: 1/2/4 registers, 0 tiers, -1 union in tiers,
  // 8 + regs the union with W in registers (queue_len <= 128)
  s.qr = qk == QK_UNION ? (L <= SONG_RUN_MAX_L ? 8 + regs : -1) : qk == QK_SEPARATE ? 0 : regs;
#ifndef SONG_UNION_WIDE_ROWS
#define SONG_UNION_WIDE_ROWS 4
#endif
  const int rows = s.nch >= 2 ? (s.qr < 0 ? SONG_UNION_WIDE_ROWS : s.nch >= 4 ? SONG_XWIDE_ROWS : SONG_WIDE_ROWS)
                              : SONG_STAGE_ROWS;  // StageRows<NCH, UNION>::R
  const int stage_bytes = hamming ? 0 : SONG_STAGE_BUFS * rows * 512 * s.nch;  // Stage<NCH>::STRIDE
  const int cid_ints = steps > 1 ? 32 * song::MAX_STEPS : 32;  // located candidates
  const int qsm_bytes = (hamming || !song::kDistTeam) ? 0 : 512 * s.nch;  // query in smem
  // stage, query, 16 B, candidate ids, 32 keys, 32 evicted keys (Cuckoo only),
  // [32 insert slots: the union with global tables, added below], tiers, table
  s.warp_bytes = stage_bytes + qsm_bytes + 16 + cid_ints * 4 + 32 * 8 +
                 (vk == song::VK_CUCKOO ? 32 * 8 : 0) +
                 (SONG_SLOT_REUSE && s.qr > 8 && s.qr < 16 && vk == song::VK_HASH ? 32 * 4 : 0) +
                 (s.qr <= 0 ? (s.qr == 0 ? 2 : 1) * (((L + 63) / 64) * 64) * 8 + 8 : 0) +
                 tbytes;
  s.warp_bytes = (s.warp_bytes + 127) & ~127;
  s.gvis = 0;
  if (s.qr == -1) {
    // R17 at large queue_len: the visited table moves to global memory (L2)
    // when that holds >= 1.5x the resident warps per SM (the union kernels
    // use <= 80 registers: at most 24 warps per SM)
    auto resident = [](int wb) { return std::min(24, (int)((227 * 1024) / (wb + 256))); };
    const int wb0 = ((s.warp_bytes - tbytes + 32 * 4) + 127) & ~127;  // + the insert slots
    if (2 * resident(wb0) >= 3 * resident(s.warp_bytes)) {
      s.gvis = 1;
      s.qr = -2;
      s.warp_bytes = wb0;
    }
  }
  // CTA size (1 warp = 1 query): 4 warps unless shared memory is the limit
  s.warps = p->warps_per_block > 0 ? p->warps_per_block : 4;
  while (s.warps > 1 && (size_t)s.warp_bytes * s.warps > 200 * 1024) s.warps >>= 1;
  if (p->warps_per_block <= 0) {
    // shared-memory-bound queue lengths: the CTA size that keeps the most warps
    // resident (227 KB per SM; e.g. 73 KB per warp at L = 1536: 1-warp CTAs
    // hold 3 warps per SM where 2-warp CTAs hold 2)
    const size_t sm = 227 * 1024;
    int best = 0;
    for (int w = 4; w >= 1; w >>= 1) {
      const size_t cta = (size_t)s.warp_bytes * w + 1024;  // + the per-CTA reservation
      const int res = cta <= sm ? (int)(sm / cta) * w : 0;
      if (res > best) {
        best = res;
        s.warps = w;
      }
    }
  }
  return s;
}


// the checks that need no index (song_search_plan_get and every search)
int check_params_common(const song_search_params* p, int metric) {
  if (p->K < 1) return fail(SONG_EINVAL, "K must be >= 1");
  if (p->queue_len < p->K) return fail(SONG_EINVAL, "queue_len %d < K %d", p->queue_len, p->K);
  if (p->queue_len > SONG_MAX_QUEUE_LEN)
    return fail(SONG_EUNSUPPORTED, "queue_len %d > %d", p->queue_len, SONG_MAX_QUEUE_LEN);
  if (p->visited < SONG_VISITED_HASH || p->visited > SONG_VISITED_CUCKOO)
    return fail(SONG_EINVAL, "unknown visited kind %d", p->visited);
  if (p->table_log2 < 0 || p->table_log2 > 24)
    return fail(SONG_EUNSUPPORTED, "table_log2 %d outside [0, 24]", p->table_log2);
  if (p->bloom_log2_bits < 0 || p->bloom_log2_bits > 24)
    return fail(SONG_EUNSUPPORTED, "bloom_log2_bits %d outside [0, 24]", p->bloom_log2_bits);
  if (p->warps_per_block < 0 || p->warps_per_block > SONG_LB_THREADS / 32)
    return fail(SONG_EINVAL, "warps_per_block %d outside [0, %d]", p->warps_per_block, SONG_LB_THREADS / 32);
  if (p->max_iters < 0 || p->blocks_per_sm < 0) return fail(SONG_EINVAL, "negative launch parameter");
  if (p->steps < 0) return fail(SONG_EINVAL, "steps %d < 0", p->steps);
  if (p->visited_cap < -1) return fail(SONG_EINVAL, "visited_cap %d < -1", p->visited_cap);
  if (p->queue_kind < SONG_QUEUE_AUTO || p->queue_kind > SONG_QUEUE_UNION)
    return fail(SONG_EINVAL, "unknown queue_kind %d", p->queue_kind);
  if (p->queue_kind == SONG_QUEUE_UNION && (p->visited != SONG_VISITED_HASH || p->steps > 1))
    return fail(SONG_EUNSUPPORTED, "the bounded-union queue needs visited HASH and steps <= 1");

  if (p->schedule < SONG_SCHEDULE_AUTO || p->schedule > SONG_SCHEDULE_OUTLIER_FIRST)
    return fail(SONG_EINVAL, "unknown schedule %d", p->schedule);
  if (p->queries_per_warp != 0 && p->queries_per_warp != 1 && p->queries_per_warp != 2 &&
      p->queries_per_warp != 4)
    return fail(SONG_EINVAL, "queries_per_warp %d not in {0, 1, 2, 4}", p->queries_per_warp);
  if (p->queries_per_warp > 0 &&
      (p->visited != SONG_VISITED_HASH || p->visited_cap != -1 || p->steps > 1 ||
       p->queue_kind == SONG_QUEUE_UNION || p->queue_len > 128 || metric == SONG_HAMMING))
    return fail(SONG_EUNSUPPORTED,
                "queries_per_warp > 0 needs visited HASH, visited_cap -1, steps <= 1, queue_kind "
                "AUTO or SEPARATE, queue_len <= 128 and a float index");
  if (p->steps > SONG_MAX_STEPS)
    return fail(SONG_EUNSUPPORTED, "steps %d > %d", p->steps, SONG_MAX_STEPS);
  if (p->steps > 1 && ((p->visited != SONG_VISITED_HASH && p->visited != SONG_VISITED_BLOOM) ||
                       metric == SONG_HAMMING))
    return fail(SONG_EUNSUPPORTED, "multi-step probing needs visited HASH or BLOOM on a float index");
  if (metric == SONG_HAMMING && p->visited != SONG_VISITED_HASH && p->visited != SONG_VISITED_BLOOM)
    return fail(SONG_EUNSUPPORTED, "Hamming indexes support the hash and Bloom visited sets");
  if ((p->visited == SONG_VISITED_HASH_GLOBAL || p->visited == SONG_VISITED_HASH_GLOBAL_SEL) &&
      p->table_log2 > 0 && (1 << (p->table_log2 - 1)) < SONG_MAX_DEGREE + 1)
    // one iteration inserts up to 32 ids after a load check at 1/2: a smaller
    // table could fill up inside an iteration and its probes would never end
    return fail(SONG_EUNSUPPORTED, "table_log2 %d: the global visited table needs >= 2^7 slots",
                p->table_log2);
  return SONG_OK;
}

// an explicit lazy capacity must lie in [live bound, 3/4 of the table]
int check_cap(const song_search_params* p, int dpad, int metric) {
  if (p->visited_cap > 0 && p->visited == SONG_VISITED_HASH) {
    const bool uni = queue_kind_of(p->queue_len, song::VK_HASH, p) == QK_UNION;
    const int slots =
        1 << hash_log2_slots(p->queue_len, uni, nch_of(dpad, metric == SONG_HAMMING));
    const int lo = uni ? p->queue_len + 32 : 2 * p->queue_len + 32;
    if (p->visited_cap < lo || p->visited_cap > 3 * (slots / 4))
      return fail(SONG_EINVAL, "visited_cap %d outside [%d, 3/4 of %d slots]", p->visited_cap,
                  lo, slots);
  }
  return SONG_OK;
}

int check_params(const song_index* ix, const song_search_params* p) {
  int rc = check_params_common(p, ix->metric);
  if (rc) return rc;
  rc = check_cap(p, ix->dpad, ix->metric);
  if (rc) return rc;
  if (p->entry < 0 || p->entry >= ix->n) return fail(SONG_EINVAL, "entry %d out of range", p->entry);
  return SONG_OK;
}

// searches of one index share d_ticket / d_status and the order / query-code
// scratch: a search on another stream waits for the previous one (song.h,
// Concurrency)
int order_after_last(song_index* ix, cudaStream_t st) {
  if (st != ix->last_stream && ix->last_done) CUDA_TRY(cudaStreamWaitEvent(st, ix->last_done, 0));
  ix->last_stream = st;
  return SONG_OK;
}

// index-free part of a search's plan: the visited kind, the data-structure
// sizes and the launch shape
int vk_of(const song_search_params* p) {
  switch (p->visited) {
    case SONG_VISITED_BLOOM: return song::VK_BLOOM;
    case SONG_VISITED_HASH_GLOBAL:
    case SONG_VISITED_HASH_GLOBAL_SEL: return song::VK_GHASH;
    case SONG_VISITED_CUCKOO: return song::VK_CUCKOO;
    default: return song::VK_HASH;
  }
}

int plan_shape(const song_search_params* p, int dpad, int metric, Shape* out) {
  *out = search_shape(p->queue_len, vk_of(p), p, dpad, metric == SONG_HAMMING);
  if ((size_t)out->warp_bytes * out->warps > 227 * 1024)
    return fail(SONG_EUNSUPPORTED, "queue_len %d needs %d B of shared memory per warp",
                p->queue_len, out->warp_bytes);
  return SONG_OK;
}

// outlier-first ticket order of a float query batch q [nq][dim] into ix->d_order
int prepare_order(song_index* ix, const float* q, int64_t nq, cudaStream_t st) {
  if ((size_t)nq > ix->cap_order) {
    CUDA_TRY(cudaStreamSynchronize(st));
    cudaFree(ix->d_order);
    cudaFree(ix->d_qbin);
    ix->d_order = nullptr;
    ix->d_qbin = nullptr;
    ix->cap_order = 0;
    CUDA_TRY(cudaMalloc(&ix->d_order, (size_t)nq * sizeof(int32_t)));
    CUDA_TRY(cudaMalloc(&ix->d_qbin, (size_t)nq * sizeof(uint16_t)));
    ix->cap_order = (size_t)nq;
  }
  if (!ix->d_bins) CUDA_TRY(cudaMalloc(&ix->d_bins, 2 * song::SCHED_BINS * sizeof(unsigned)));
  CUDA_TRY(cudaMemsetAsync(ix->d_bins, 0, 2 * song::SCHED_BINS * sizeof(unsigned), st));
  const int kb = (int)std::min<int64_t>((nq + 7) / 8, (int64_t)ix->num_sms * 8);
  song::order_keys_kernel<<<kb, 256, 0, st>>>(q, nq, ix->dim, ix->d_centroid,
                                              ix->metric == SONG_COSINE, ix->d_bins, ix->d_qbin);
  CUDA_TRY(cudaGetLastError());
  const int sb = (int)std::min<int64_t>((nq + 255) / 256, (int64_t)ix->num_sms);
  song::order_scatter_kernel<<<sb, 256, 0, st>>>(nq, ix->d_bins, ix->d_bins + song::SCHED_BINS,
                                                 ix->d_qbin, ix->d_order);
  CUDA_TRY(cudaGetLastError());
  return SONG_OK;
}

// Fig. 8's packing kernel: G = queries_per_warp queries per warp (mq_kernel.cuh)
template <int G, int METRIC>
int launch_mq_t(song_index* ix, const song::MqArgs& m, cudaStream_t st) {
  auto kern = song::song_search_mq_kernel<G, METRIC>;
  const size_t smem = (size_t)m.team_smem_bytes * G * 4;  // 4 warps per CTA
  if (smem > 227 * 1024) return fail(SONG_EUNSUPPORTED, "packing kernel needs %zu B per CTA", smem);
  CUDA_TRY(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
  int fit = 0;
  CUDA_TRY(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&fit, kern, 128, smem));
  if (fit < 1) return fail(SONG_EUNSUPPORTED, "packing kernel does not fit an SM");
  const int64_t want = (m.nq + 4 * G - 1) / (4 * G);
  const int64_t grid = std::min<int64_t>((int64_t)fit * ix->num_sms, want);
  CUDA_TRY(cudaMemsetAsync(m.ticket, 0, sizeof(unsigned), st));
  kern<<<(unsigned)grid, 128, smem, st>>>(m);
  CUDA_TRY(cudaGetLastError());
  return SONG_OK;
}

int enqueue_mq(song_index* ix, const song_search_params* p, const Shape& sh,
               const song::SearchArgs& a, cudaStream_t st) {
  song::MqArgs m;
  m.data = a.data;
  m.adj = a.adj;
  m.queries = a.queries;
  m.ids_out = a.ids_out;
  m.dists_out = a.dists_out;
  m.counters_out = a.counters_out;
  m.ticket = a.ticket;
  m.order = nullptr;
  m.status = a.status;
  m.nq = a.nq;
  m.dim = a.dim;
  m.dpad = a.dpad;
  m.degree = a.degree;
  m.K = a.K;
  m.L = a.L;
  m.table_log2 = sh.table_log2;
  m.rebuild_at = sh.rebuild_at;
  m.entry = p->entry;
  m.max_iters = p->max_iters > 0 ? p->max_iters : (1 << 30);
  m.id_offset = p->id_offset;
  m.cosine = ix->metric == SONG_COSINE;
  m.dedup = ix->dedup;
  m.team_smem_bytes = sh.warp_bytes / p->queries_per_warp;
  int rc = order_after_last(ix, st);
  if (rc) return rc;
  const bool l2 = ix->metric == SONG_L2;
  switch (p->queries_per_warp) {
    case 1: rc = l2 ? launch_mq_t<1, song::MET_L2>(ix, m, st) : launch_mq_t<1, song::MET_DOT>(ix, m, st); break;
    case 2: rc = l2 ? launch_mq_t<2, song::MET_L2>(ix, m, st) : launch_mq_t<2, song::MET_DOT>(ix, m, st); break;
    default: rc = l2 ? launch_mq_t<4, song::MET_L2>(ix, m, st) : launch_mq_t<4, song::MET_DOT>(ix, m, st); break;
  }
  if (rc) return rc;
  if (!ix->last_done) CUDA_TRY(cudaEventCreateWithFlags(&ix->last_done, cudaEventDisableTiming));
  CUDA_TRY(cudaEventRecord(ix->last_done, st));
  return SONG_OK;
}

int enqueue_search(song_index* ix, const song_search_params* p, const float* q, int64_t nq,
                   int32_t* ids, float* dists, int32_t* counters, cudaStream_t st) {
  song::SearchArgs a;
  a.data = ix->d_data;
  a.adj = ix->d_adj;
  a.queries = q;
  a.ids_out = ids;
  a.dists_out = dists;
  a.counters_out = counters;
  a.ticket = ix->d_ticket;
  a.order = nullptr;
  a.status = ix->d_status;
  a.n = ix->n;
  a.nq = nq;
  a.dim = ix->dim;
  a.dpad = ix->dpad;
  a.degree = ix->degree;
  a.K = p->K;
  a.L = p->queue_len;
  a.cosine = ix->metric == SONG_COSINE;
  a.dedup = ix->dedup;
  int vk = song::VK_HASH;
  a.sel = 1;
  switch (p->visited) {
    case SONG_VISITED_BLOOM: vk = song::VK_BLOOM; break;
    case SONG_VISITED_HASH_GLOBAL: vk = song::VK_GHASH; a.sel = 0; break;
    case SONG_VISITED_HASH_GLOBAL_SEL: vk = song::VK_GHASH; break;
    case SONG_VISITED_CUCKOO: vk = song::VK_CUCKOO; break;
    default: break;
  }
  a.gtab = nullptr;
  a.gen0 = 0;
  a.stage_cycles = nullptr;
  a.gvis = nullptr;
#ifdef SONG_STAGE_TIMING
  if (!ix->d_stage) {
    CUDA_TRY(cudaMalloc(&ix->d_stage, 4 * sizeof(unsigned long long)));
    CUDA_TRY(cudaMemset(ix->d_stage, 0, 4 * sizeof(unsigned long long)));
  }
  a.stage_cycles = ix->d_stage;
#endif
  if (ix->metric == SONG_HAMMING && vk != song::VK_HASH && vk != song::VK_BLOOM)
    return fail(SONG_EUNSUPPORTED, "Hamming indexes support the hash and Bloom visited sets");
  Shape sh = search_shape(p->queue_len, vk, p, ix->dpad, ix->metric == SONG_HAMMING);
  if (p->queries_per_warp > 0) return enqueue_mq(ix, p, sh, a, st);
  a.table_log2 = sh.table_log2;
  a.rebuild_at = sh.rebuild_at;
  a.lazy = sh.lazy;
  a.warp_smem_bytes = sh.warp_bytes;
  a.entry = p->entry;
  a.max_iters = p->max_iters > 0 ? p->max_iters : (1 << 30);
  a.id_offset = p->id_offset;
  a.steps = p->steps > 1 ? p->steps : 1;
  const int warps = sh.warps;
  if ((size_t)sh.warp_bytes * warps > 227 * 1024)
    return fail(SONG_EUNSUPPORTED, "queue_len %d needs %d B of shared memory per warp",
                p->queue_len, sh.warp_bytes);
  // searches of one index share d_ticket / d_status / the order scratch: a
  // search on another stream waits for the previous one (song.h, Concurrency)
  int orc = order_after_last(ix, st);
  if (orc) return orc;
  // ticket order (song_search_params.schedule): outlier-first needs the centroid
  // (float indexes) and pays when the batch outnumbers the resident warps
  const bool outlier_first =
      ix->d_centroid && nq > 1 &&
      (p->schedule == SONG_SCHEDULE_OUTLIER_FIRST ||
       (p->schedule == SONG_SCHEDULE_AUTO && nq > (int64_t)ix->num_sms * 24));
  if (outlier_first) {
    int rc = prepare_order(ix, q, nq, st);
    if (rc) return rc;
    a.order = ix->d_order;
  }
  const int m = ix->metric, qr = sh.qr, bps = p->blocks_per_sm, sms = ix->num_sms;
  int rc;
  switch (sh.nch) {
    case 1: rc = launch_m<1>(ix, a, m, vk, qr, warps, bps, sms, st); break;
    case 2: rc = launch_m<2>(ix, a, m, vk, qr, warps, bps, sms, st); break;
    case 4: rc = launch_m<4>(ix, a, m, vk, qr, warps, bps, sms, st); break;
    default: rc = launch_m<8>(ix, a, m, vk, qr, warps, bps, sms, st); break;
  }
  if (rc) return rc;
  if (!ix->last_done) CUDA_TRY(cudaEventCreateWithFlags(&ix->last_done, cudaEventDisableTiming));
  CUDA_TRY(cudaEventRecord(ix->last_done, st));
  return SONG_OK;
}

int finish_create(song_index* ix, cudaStream_t st) {
  {
    int* d_dup = nullptr;
    CUDA_TRY(cudaMalloc(&d_dup, sizeof(int)));
    CUDA_TRY(cudaMemsetAsync(d_dup, 0, sizeof(int), st));
    int blocks = (int)std::min<int64_t>((ix->n + 7) / 8, 65535);
    dup_check_kernel<<<blocks, 256, 0, st>>>(ix->d_adj, ix->n, ix->degree, d_dup);
    int dup = 1;
    cudaError_t e = cudaGetLastError();
    if (e == cudaSuccess) e = cudaMemcpyAsync(&dup, d_dup, sizeof(int), cudaMemcpyDeviceToHost, st);
    if (e == cudaSuccess) e = cudaStreamSynchronize(st);
    cudaFree(d_dup);
    if (e != cudaSuccess) return fail(SONG_ECUDA, "dup check: %s", cudaGetErrorString(e));
    ix->dedup = dup;
  }
  if (ix->metric == SONG_COSINE) {
    int blocks = (int)std::min<int64_t>((ix->n + 7) / 8, 65535);
    normalize_rows_kernel<<<blocks, 256, 0, st>>>(ix->d_data, ix->n, ix->dpad);
    CUDA_TRY(cudaGetLastError());
  }
  if (ix->metric != SONG_HAMMING) {  // centroid for the outlier-first schedule
    const int64_t chunk = (ix->n + song::CENTROID_BLOCKS - 1) / song::CENTROID_BLOCKS;
    const int nparts = (int)((ix->n + chunk - 1) / chunk);
    float* part = nullptr;
    CUDA_TRY(cudaMalloc(&part, (size_t)nparts * ix->dpad * sizeof(float)));
    CUDA_TRY(cudaMalloc(&ix->d_centroid, (size_t)ix->dpad * sizeof(float)));
    song::centroid_partial_kernel<<<nparts, 128, 0, st>>>(ix->d_data, ix->n, ix->dpad, chunk, part);
    song::centroid_final_kernel<<<1, 256, 0, st>>>(part, nparts, ix->dpad, ix->n, ix->d_centroid);
    cudaError_t e = cudaGetLastError();
    if (e == cudaSuccess) e = cudaStreamSynchronize(st);
    cudaFree(part);
    if (e != cudaSuccess) return fail(SONG_ECUDA, "centroid: %s", cudaGetErrorString(e));
  }
  CUDA_TRY(cudaStreamSynchronize(st));
  return SONG_OK;
}

int check_bits(int32_t bits) {
  if (bits < 32 || bits % 32) return fail(SONG_EINVAL, "bits %d is not a positive multiple of 32", bits);
  if (bits > SONG_MAX_CODE_BITS) return fail(SONG_EUNSUPPORTED, "bits %d > %d", bits, SONG_MAX_CODE_BITS);
  return SONG_OK;
}

// §VII encoder launch: X [n][ldx] -> codes [n][ldc] words (first bits/32 used)
int launch_rp(const float* X, int64_t n, int dim, int64_t ldx, const float* R, int bits,
              uint32_t* codes, int64_t ldc, cudaStream_t st) {
  const int64_t tiles = (n + song::RP_TM - 1) / song::RP_TM;
  if (tiles > 0x7fffffffll) return fail(SONG_EUNSUPPORTED, "n too large for one encode launch");
  dim3 grid((unsigned)tiles, (unsigned)((bits + song::RP_TN - 1) / song::RP_TN));
  song::rp_encode_kernel<<<grid, song::RP_THREADS, 0, st>>>(X, n, dim, ldx, R, bits, codes, ldc);
  CUDA_TRY(cudaGetLastError());
  return SONG_OK;
}

// encode a float query batch of a song_index_create_rp index into ix->d_qcodes
int encode_queries(song_index* ix, const float* q, int64_t nq, cudaStream_t st) {
  const size_t need = (size_t)nq * ix->dim * sizeof(uint32_t);
  if (need > ix->cap_qcodes) {
    CUDA_TRY(cudaStreamSynchronize(st));
    cudaFree(ix->d_qcodes);
    ix->d_qcodes = nullptr;
    ix->cap_qcodes = 0;
    CUDA_TRY(cudaMalloc(&ix->d_qcodes, need));
    ix->cap_qcodes = need;
  }
  return launch_rp(q, nq, ix->rp_dim, ix->rp_dim, ix->d_R, ix->code_bits, ix->d_qcodes, ix->dim,
                   st);
}

int check_adjacency_host(const int32_t* adjacency, int64_t n, int32_t degree) {
  for (int64_t i = 0; i < n * (int64_t)degree; ++i)
    if (adjacency[i] < -1 || adjacency[i] >= n)
      return fail(SONG_EINVAL, "adjacency[%lld] = %d outside [-1, %lld)", (long long)i,
                  adjacency[i], (long long)n);
  return SONG_OK;
}

// common part of the two SONG_HAMMING creators: a zeroed [n][dpad]-word code
// array (padding words stay 0 on both sides of every XOR) and the adjacency
int alloc_codes_index(int64_t n, int32_t bits, const int32_t* adjacency, int32_t degree,
                      song_index** out, song_index** made) {
  if (!out) return fail(SONG_EINVAL, "out is NULL");
  *out = nullptr;
  if (!adjacency) return fail(SONG_EINVAL, "adjacency is NULL");
  if (n < 1 || degree < 1) return fail(SONG_EINVAL, "n and degree must be >= 1");
  if (n > 0x7fffffffll) return fail(SONG_EUNSUPPORTED, "n must fit int32 ids");
  if (degree > SONG_MAX_DEGREE) return fail(SONG_EUNSUPPORTED, "degree %d > %d", degree, SONG_MAX_DEGREE);
  int rc = check_bits(bits);
  if (rc) return rc;
  rc = check_adjacency_host(adjacency, n, degree);
  if (rc) return rc;
  song_index* ix = new song_index();
  rc = alloc_index(ix, n, bits / 32, degree, SONG_HAMMING);
  if (rc) {
    free_index(ix);
    return rc;
  }
  ix->code_bits = bits;
  cudaError_t e = cudaMemsetAsync(ix->d_data, 0, (size_t)n * ix->dpad * 4, ix->stream);
  if (e == cudaSuccess)
    e = cudaMemcpyAsync(ix->d_adj, adjacency, (size_t)n * degree * sizeof(int32_t),
                        cudaMemcpyHostToDevice, ix->stream);
  if (e != cudaSuccess) {
    free_index(ix);
    return fail(SONG_ECUDA, "index upload: %s", cudaGetErrorString(e));
  }
  *made = ix;
  return SONG_OK;
}

}  // namespace

namespace song {
int make_search_view(const float* xv, int64_t n, int dim, int degree, int metric, int32_t* adj,
                     song_index** out) {
  song_index* ix = new song_index();
  cudaError_t e = cudaGetDevice(&ix->device);
  if (e == cudaSuccess)
    e = cudaDeviceGetAttribute(&ix->num_sms, cudaDevAttrMultiProcessorCount, ix->device);
  if (e == cudaSuccess) e = cudaMalloc(&ix->d_ticket, sizeof(unsigned));
  if (e == cudaSuccess) e = cudaMalloc(&ix->d_status, sizeof(int));
  if (e == cudaSuccess) e = cudaMemset(ix->d_status, 0, sizeof(int));
  ix->n = n;
  ix->dim = dim;
  ix->dpad = (dim + 3) & ~3;
  ix->degree = degree;
  ix->metric = metric;
  ix->d_data = const_cast<float*>(xv);
  ix->d_adj = adj;
  ix->dedup = 1;
  if (e != cudaSuccess) {
    free_search_view(ix);
    return fail(e == cudaErrorMemoryAllocation ? SONG_ENOMEM : SONG_ECUDA, "search view: %s",
                cudaGetErrorString(e));
  }
  *out = ix;
  return SONG_OK;
}

int search_view(song_index* view, int64_t m, const song_search_params* p, const float* q,
                int64_t nq, int32_t* ids, float* dists, cudaStream_t st) {
  view->n = m;
  return enqueue_search(view, p, q, nq, ids, dists, nullptr, st);
}

int view_status(song_index* view, int* status, cudaStream_t st) {
  CUDA_TRY(cudaMemcpyAsync(status, view->d_status, sizeof(int), cudaMemcpyDeviceToHost, st));
  CUDA_TRY(cudaStreamSynchronize(st));
  return SONG_OK;
}

void free_search_view(song_index* view) {
  if (!view) return;
  view->d_data = nullptr;  // not owned
  view->d_adj = nullptr;
  cudaFree(view->d_ticket);
  cudaFree(view->d_status);
  cudaFree(view->d_gtab);
  cudaFree(view->d_gvis);
  cudaFree(view->d_order);
  cudaFree(view->d_qbin);
  cudaFree(view->d_bins);
  delete view;
}
}  // namespace song

extern "C" {

int song_rp_encode(const float* vectors, int64_t n, int32_t dim, const float* R, int32_t bits,
                   uint32_t* codes, void* stream) {
  if (!vectors || !R || !codes) return fail(SONG_EINVAL, "NULL argument");
  if (n < 1 || dim < 1) return fail(SONG_EINVAL, "n and dim must be >= 1");
  int rc = check_bits(bits);
  if (rc) return rc;
  return launch_rp(vectors, n, dim, dim, R, bits, codes, bits / 32, (cudaStream_t)stream);
}

int song_index_create_codes(const uint32_t* codes, int64_t n, int32_t bits,
                            const int32_t* adjacency, int32_t degree, song_index** out) {
  if (!codes) {
    if (out) *out = nullptr;
    return fail(SONG_EINVAL, "codes is NULL");
  }
  song_index* ix = nullptr;
  int rc = alloc_codes_index(n, bits, adjacency, degree, out, &ix);
  if (rc) return rc;
  const int words = bits / 32;
  cudaError_t e = cudaMemcpy2DAsync(ix->d_data, ix->dpad * 4, codes, words * 4, words * 4, n,
                                    cudaMemcpyHostToDevice, ix->stream);
  if (e == cudaSuccess) e = cudaStreamSynchronize(ix->stream);
  if (e != cudaSuccess) {
    free_index(ix);
    return fail(SONG_ECUDA, "codes upload: %s", cudaGetErrorString(e));
  }
  ix->dedup = 1;
  rc = finish_create(ix, ix->stream);
  if (rc) {
    free_index(ix);
    return rc;
  }
  *out = ix;
  return SONG_OK;
}

int song_index_create_rp(const float* vectors, int64_t n, int32_t dim, const float* R,
                         int32_t bits, const int32_t* adjacency, int32_t degree,
                         song_index** out) {
  if (!vectors || !R) {
    if (out) *out = nullptr;
    return fail(SONG_EINVAL, "vectors/R is NULL");
  }
  if (dim < 1) return fail(SONG_EINVAL, "dim must be >= 1");
  if (bits >= 32 && bits % 32 == 0)
    for (int64_t i = 0; i < (int64_t)bits * dim; ++i)
      if (!std::isfinite(R[i])) return fail(SONG_EINVAL, "R[%lld] is not finite", (long long)i);
  song_index* ix = nullptr;
  int rc = alloc_codes_index(n, bits, adjacency, degree, out, &ix);
  if (rc) return rc;
  ix->rp_dim = dim;
  cudaStream_t st = ix->stream;
  // the vectors need not fit in device memory — stream them through a
  // double-buffered device chunk (<= 256 MiB each) and keep only the codes
  int64_t chunk = std::max<int64_t>(1, std::min<int64_t>(n, (256ll << 20) / (4ll * dim)));
  if (const char* env = std::getenv("SONG_RP_CHUNK_ROWS"))  // tests: force many chunks
    chunk = std::max<int64_t>(1, std::min<int64_t>(chunk, std::atoll(env)));
  float* d_chunk[2] = {nullptr, nullptr};
  unsigned long long* d_bad = nullptr;
  cudaEvent_t done[2] = {nullptr, nullptr};
  auto cleanup = [&]() {
    cudaStreamSynchronize(st);
    cudaFree(d_chunk[0]);
    cudaFree(d_chunk[1]);
    cudaFree(d_bad);
    if (done[0]) cudaEventDestroy(done[0]);
    if (done[1]) cudaEventDestroy(done[1]);
  };
  cudaError_t e = cudaMalloc(&ix->d_R, (size_t)bits * dim * 4);
  if (e == cudaSuccess) e = cudaMalloc(&d_chunk[0], (size_t)chunk * dim * 4);
  if (e == cudaSuccess && chunk < n) e = cudaMalloc(&d_chunk[1], (size_t)chunk * dim * 4);
  if (e == cudaSuccess) e = cudaMalloc(&d_bad, sizeof *d_bad);
  if (e == cudaSuccess) e = cudaMemsetAsync(d_bad, 0, sizeof *d_bad, st);
  if (e == cudaSuccess) e = cudaEventCreateWithFlags(&done[0], cudaEventDisableTiming);
  if (e == cudaSuccess) e = cudaEventCreateWithFlags(&done[1], cudaEventDisableTiming);
  if (e == cudaSuccess)
    e = cudaMemcpyAsync(ix->d_R, R, (size_t)bits * dim * 4, cudaMemcpyHostToDevice, st);
  for (int64_t s0 = 0, k = 0; e == cudaSuccess && s0 < n; s0 += chunk, ++k) {
    const int64_t rows = std::min(chunk, n - s0);
    float* buf = d_chunk[k & 1];
    e = cudaEventSynchronize(done[k & 1]);  // the encode that last read buf is finished
    if (e == cudaSuccess)
      e = cudaMemcpyAsync(buf, vectors + s0 * dim, (size_t)rows * dim * 4, cudaMemcpyHostToDevice, st);
    if (e != cudaSuccess) break;
    validate_kernel<<<592, 256, 0, st>>>(buf, rows * dim, nullptr, 0, n, d_bad);
    rc = launch_rp(buf, rows, dim, dim, ix->d_R, bits,
                   reinterpret_cast<uint32_t*>(ix->d_data) + s0 * ix->dpad, ix->dpad, st);
    if (rc) {
      cleanup();
      free_index(ix);
      return rc;
    }
    e = cudaEventRecord(done[k & 1], st);
  }
  unsigned long long bad = 0;
  if (e == cudaSuccess) e = cudaMemcpyAsync(&bad, d_bad, sizeof bad, cudaMemcpyDeviceToHost, st);
  if (e == cudaSuccess) e = cudaStreamSynchronize(st);
  cleanup();
  if (e != cudaSuccess) {
    free_index(ix);
    return fail(e == cudaErrorMemoryAllocation ? SONG_ENOMEM : SONG_ECUDA, "rp index: %s",
                cudaGetErrorString(e));
  }
  if (bad) {
    free_index(ix);
    return fail(SONG_EINVAL, "%llu non-finite vector values", bad);
  }
  rc = finish_create(ix, st);
  if (rc) {
    free_index(ix);
    return rc;
  }
  *out = ix;
  return SONG_OK;
}


int song_search_plan_get(const song_search_params* p, int32_t dim, int32_t metric,
                         song_search_plan* out) {
  if (!p || !out) return fail(SONG_EINVAL, "NULL argument");
  std::memset(out, 0, sizeof *out);
  if (dim < 1) return fail(SONG_EINVAL, "dim must be >= 1");
  if (metric < SONG_L2 || metric > SONG_HAMMING) return fail(SONG_EINVAL, "metric %d", metric);
  if (metric != SONG_HAMMING && dim > SONG_MAX_DIM)
    return fail(SONG_EUNSUPPORTED, "dim %d > %d", dim, SONG_MAX_DIM);
  if (metric == SONG_HAMMING && dim * 32 > SONG_MAX_CODE_BITS)
    return fail(SONG_EUNSUPPORTED, "%d code words > %d bits", dim, SONG_MAX_CODE_BITS);
  int rc = check_params_common(p, metric);
  if (rc) return rc;
  rc = check_cap(p, dpad_of(dim, metric), metric);
  if (rc) return rc;
  Shape sh;
  rc = plan_shape(p, dpad_of(dim, metric), metric, &sh);
  if (rc) return rc;
  const int vk = vk_of(p);
  out->visited_log2 = sh.table_log2;
  out->visited_cap = vk != song::VK_HASH ? 0 : sh.lazy ? sh.rebuild_at : -1;
  out->queue_regs = sh.qr > 8 ? sh.qr - 8 : sh.qr > 0 ? sh.qr : 0;
  out->queue_kind = sh.qk;
  out->visited_global = sh.gvis;
  out->row_chunks = sh.nch;
  out->smem_per_warp = sh.warp_bytes;
  out->warps_per_block = sh.warps;
  return SONG_OK;
}

void song_default_params(song_search_params* p, int32_t K, int32_t queue_len) {
  if (!p) return;
  std::memset(p, 0, sizeof *p);
  p->K = K;
  p->queue_len = queue_len;
  p->visited = SONG_VISITED_HASH;
}

int song_index_create(const float* vectors, int64_t n, int32_t dim, const int32_t* adjacency,
                      int32_t degree, song_metric metric, song_index** out) {
  int rc = check_create_args(vectors, n, dim, adjacency, degree, metric, out);
  if (rc) return rc;
  for (int64_t i = 0; i < n * (int64_t)degree; ++i)
    if (adjacency[i] < -1 || adjacency[i] >= n)
      return fail(SONG_EINVAL, "adjacency[%lld] = %d outside [-1, %lld)", (long long)i,
                  adjacency[i], (long long)n);
  for (int64_t i = 0; i < n * (int64_t)dim; ++i)
    if (!std::isfinite(vectors[i]))
      return fail(SONG_EINVAL, "vectors[%lld] is not finite", (long long)i);
  song_index* ix = new song_index();
  rc = alloc_index(ix, n, dim, degree, metric);
  if (rc) {
    free_index(ix);
    return rc;
  }
  cudaError_t e = cudaMemsetAsync(ix->d_data, 0, (size_t)n * ix->dpad * sizeof(float), ix->stream);
  if (e == cudaSuccess)
    e = cudaMemcpy2DAsync(ix->d_data, ix->dpad * sizeof(float), vectors, dim * sizeof(float),
                          dim * sizeof(float), n, cudaMemcpyHostToDevice, ix->stream);
  if (e == cudaSuccess)
    e = cudaMemcpyAsync(ix->d_adj, adjacency, (size_t)n * degree * sizeof(int32_t),
                        cudaMemcpyHostToDevice, ix->stream);
  if (e != cudaSuccess) {
    free_index(ix);
    return fail(SONG_ECUDA, "index upload: %s", cudaGetErrorString(e));
  }
  rc = finish_create(ix, ix->stream);
  if (rc) {
    free_index(ix);
    return rc;
  }
  *out = ix;
  return SONG_OK;
}

int song_index_create_device(const float* vectors, int64_t n, int32_t dim,
                             const int32_t* adjacency, int32_t degree, song_metric metric,
                             void* stream, song_index** out) {
  int rc = check_create_args(vectors, n, dim, adjacency, degree, metric, out);
  if (rc) return rc;
  cudaStream_t st = (cudaStream_t)stream;
  unsigned long long* d_bad = nullptr;
  CUDA_TRY(cudaMalloc(&d_bad, sizeof *d_bad));
  CUDA_TRY(cudaMemsetAsync(d_bad, 0, sizeof *d_bad, st));
  validate_kernel<<<1184, 256, 0, st>>>(vectors, n * (int64_t)dim, adjacency, n * (int64_t)degree,
                                        n, d_bad);
  unsigned long long bad = 0;
  cudaError_t e = cudaGetLastError();
  if (e == cudaSuccess) e = cudaMemcpyAsync(&bad, d_bad, sizeof bad, cudaMemcpyDeviceToHost, st);
  if (e == cudaSuccess) e = cudaStreamSynchronize(st);
  cudaFree(d_bad);
  if (e != cudaSuccess) return fail(SONG_ECUDA, "validation: %s", cudaGetErrorString(e));
  if (bad) return fail(SONG_EINVAL, "%llu invalid adjacency ids / non-finite values", bad);
  song_index* ix = new song_index();
  rc = alloc_index(ix, n, dim, degree, metric);
  if (rc) {
    free_index(ix);
    return rc;
  }
  e = cudaMemsetAsync(ix->d_data, 0, (size_t)n * ix->dpad * sizeof(float), st);
  if (e == cudaSuccess)
    e = cudaMemcpy2DAsync(ix->d_data, ix->dpad * sizeof(float), vectors, dim * sizeof(float),
                          dim * sizeof(float), n, cudaMemcpyDeviceToDevice, st);
  if (e == cudaSuccess)
    e = cudaMemcpyAsync(ix->d_adj, adjacency, (size_t)n * degree * sizeof(int32_t),
                        cudaMemcpyDeviceToDevice, st);
  if (e != cudaSuccess) {
    free_index(ix);
    return fail(SONG_ECUDA, "index copy: %s", cudaGetErrorString(e));
  }
  rc = finish_create(ix, st);
  if (rc) {
    free_index(ix);
    return rc;
  }
  *out = ix;
  return SONG_OK;
}

int song_index_destroy(song_index* idx) {
  if (!idx) return SONG_OK;
  cudaStreamSynchronize(idx->last_stream);
  free_index(idx);
  return SONG_OK;
}

int song_index_get_info(const song_index* ix, song_index_info* info) {
  if (!ix || !info) return fail(SONG_EINVAL, "NULL argument");
  info->n = ix->n;
  info->dim = ix->dim;
  info->dim_padded = ix->dpad;
  info->degree = ix->degree;
  info->metric = ix->metric;
  info->vector_bytes = ix->n * (int64_t)ix->dpad * 4;
  info->graph_bytes = ix->n * (int64_t)ix->degree * 4;
  info->device = ix->device;
  info->num_sms = ix->num_sms;
  info->code_bits = ix->code_bits;
  info->reserved = 0;
  if (ix->metric == SONG_HAMMING) info->dim = ix->rp_dim;
  return SONG_OK;
}

int song_search_ex(song_index* ix, const song_search_params* p, const float* queries, int64_t nq,
                   int32_t* ids_out, float* dists_out, int32_t* counters_out, void* stream) {
  if (!ix || !p || !queries || !ids_out || !dists_out) return fail(SONG_EINVAL, "NULL argument");
  if (nq < 1) return fail(SONG_EINVAL, "nq must be >= 1");
  if (nq > 0x7fffffffll) return fail(SONG_EUNSUPPORTED, "nq must fit int32");
  int rc = check_params(ix, p);
  if (rc) return rc;
  if (ix->metric == SONG_HAMMING) {
    if (!ix->d_R)
      return fail(SONG_EINVAL, "this index holds codes without R: use song_search_codes_ex");
    rc = order_after_last(ix, (cudaStream_t)stream);
    if (rc) return rc;
    rc = encode_queries(ix, queries, nq, (cudaStream_t)stream);
    if (rc) return rc;
    queries = reinterpret_cast<const float*>(ix->d_qcodes);
  }
  return enqueue_search(ix, p, queries, nq, ids_out, dists_out, counters_out,
                        (cudaStream_t)stream);
}

int song_search_codes_ex(song_index* ix, const song_search_params* p, const uint32_t* qcodes,
                         int64_t nq, int32_t* ids_out, float* dists_out, int32_t* counters_out,
                         void* stream) {
  if (!ix || !p || !qcodes || !ids_out || !dists_out) return fail(SONG_EINVAL, "NULL argument");
  if (ix->metric != SONG_HAMMING) return fail(SONG_EINVAL, "not a SONG_HAMMING index");
  if (nq < 1) return fail(SONG_EINVAL, "nq must be >= 1");
  if (nq > 0x7fffffffll) return fail(SONG_EUNSUPPORTED, "nq must fit int32");
  int rc = check_params(ix, p);
  if (rc) return rc;
  return enqueue_search(ix, p, reinterpret_cast<const float*>(qcodes), nq, ids_out, dists_out,
                        counters_out, (cudaStream_t)stream);
}

static int status_code(int st) {
  if (st & song::STATUS_BAD_INPUT) return fail(SONG_EINVAL, "a query had a non-finite value");
  if (st & song::STATUS_ITER_CAP) return fail(SONG_EITERCAP, "a query reached max_iters");
  if (st & song::STATUS_TABLE_FULL)
    return fail(SONG_EUNSUPPORTED, "a query filled half of its global visited table; raise "
                                   "table_log2");
  return SONG_OK;
}

int song_index_last_status(song_index* ix) {
  if (!ix) return fail(SONG_EINVAL, "NULL index");
  CUDA_TRY(cudaStreamSynchronize(ix->last_stream));
  int st = 0;
  CUDA_TRY(cudaMemcpy(&st, ix->d_status, sizeof st, cudaMemcpyDeviceToHost));
  CUDA_TRY(cudaMemset(ix->d_status, 0, sizeof st));
  return status_code(st);
}

}  // extern "C"

namespace {
// device buffers of the host-buffer entry points (grown, never shrunk)
int ensure_io(song_index* ix, size_t qbytes, size_t obytes) {
  if (qbytes > ix->cap_q) {
    cudaFree(ix->d_q);
    ix->d_q = nullptr;
    ix->cap_q = 0;
    CUDA_TRY(cudaMalloc(&ix->d_q, qbytes));
    ix->cap_q = qbytes;
  }
  if (obytes > ix->cap_out) {
    cudaFree(ix->d_ids);
    cudaFree(ix->d_dists);
    ix->d_ids = nullptr;
    ix->d_dists = nullptr;
    ix->cap_out = 0;
    CUDA_TRY(cudaMalloc(&ix->d_ids, obytes));
    CUDA_TRY(cudaMalloc(&ix->d_dists, obytes));
    ix->cap_out = obytes;
  }
  return SONG_OK;
}

int make_events(song_index* ix) {
  if (!ix->ev_h2d) CUDA_TRY(cudaEventCreateWithFlags(&ix->ev_h2d, cudaEventDisableTiming));
  if (!ix->ev_done) CUDA_TRY(cudaEventCreateWithFlags(&ix->ev_done, cudaEventDisableTiming));
  if (!ix->ev_out) CUDA_TRY(cudaEventCreateWithFlags(&ix->ev_out, cudaEventDisableTiming));
  return SONG_OK;
}

// the second lane of song_search_pipelined: shares the owner's rows, graph,
// centroid and R (read-only in every kernel), owns the rest
int ensure_twin(song_index* ix) {
  if (ix->twin) return SONG_OK;
  song_index* t = new song_index();
  t->is_twin = true;
  t->device = ix->device;
  t->num_sms = ix->num_sms;
  t->n = ix->n;
  t->dim = ix->dim;
  t->dpad = ix->dpad;
  t->degree = ix->degree;
  t->metric = ix->metric;
  t->d_data = ix->d_data;
  t->d_adj = ix->d_adj;
  t->dedup = ix->dedup;
  t->code_bits = ix->code_bits;
  t->rp_dim = ix->rp_dim;
  t->d_R = ix->d_R;
  t->d_centroid = ix->d_centroid;
  cudaError_t e = cudaMalloc(&t->d_ticket, sizeof(unsigned));
  if (e == cudaSuccess) e = cudaMalloc(&t->d_status, sizeof(int));
  if (e == cudaSuccess) e = cudaMemset(t->d_status, 0, sizeof(int));
  if (e == cudaSuccess) e = cudaStreamCreateWithFlags(&t->stream, cudaStreamNonBlocking);
  if (e != cudaSuccess) {  // no half-made lane is ever attached to the index
    free_index(t);
    return fail(e == cudaErrorMemoryAllocation ? SONG_ENOMEM : SONG_ECUDA, "second lane: %s",
                cudaGetErrorString(e));
  }
  t->last_stream = t->stream;
  ix->twin = t;  // freed with the owner from here on
  return SONG_OK;
}
// host batches streamed through two lanes: chunk b = queries [b * chunk,
// min(total, (b + 1) * chunk)); its HtoD runs on the copy stream once its
// lane's previous search has read the lane's query buffer, its search on the
// lane's compute stream, its DtoH on the other copy stream (song.h,
// song_search_pipelined).  Params are checked by the caller.
int run_pipeline(song_index* ix, const song_search_params* p, const float* queries,
                 int64_t nchunks, int64_t chunk, int64_t total, int32_t* ids_out,
                 float* dists_out) {
  const int qdim = ix->metric == SONG_HAMMING ? ix->rp_dim : ix->dim;
  const size_t qrow = (size_t)qdim * sizeof(float), orow = (size_t)p->K * sizeof(int32_t);
  const int nl = nchunks > 1 ? 2 : 1;
  int rc;
  if (nl == 2) {
    rc = ensure_twin(ix);
    if (rc) return rc;
  }
  song_index* lane[2] = {ix, ix->twin};
  if (!ix->h2d) CUDA_TRY(cudaStreamCreateWithFlags(&ix->h2d, cudaStreamNonBlocking));
  if (!ix->d2h) CUDA_TRY(cudaStreamCreateWithFlags(&ix->d2h, cudaStreamNonBlocking));
  for (int l = 0; l < nl; ++l) {
    rc = ensure_io(lane[l], chunk * qrow, chunk * orow);
    if (!rc) rc = make_events(lane[l]);
    if (rc) return rc;
    // after every search enqueued earlier on the index (any stream)
    if (ix->last_done) CUDA_TRY(cudaStreamWaitEvent(lane[l]->stream, ix->last_done, 0));
    lane[l]->last_stream = lane[l]->stream;
  }
  // the copy streams too: a lane's buffers may still be read by an earlier call
  if (ix->last_done) {
    CUDA_TRY(cudaStreamWaitEvent(ix->h2d, ix->last_done, 0));
    CUDA_TRY(cudaStreamWaitEvent(ix->d2h, ix->last_done, 0));
  }
  const char* qh = reinterpret_cast<const char*>(queries);
  char* ih = reinterpret_cast<char*>(ids_out);
  char* dh = reinterpret_cast<char*>(dists_out);
  for (int64_t b = 0; b < nchunks; ++b) {
    song_index* L = lane[b % nl];
    cudaStream_t st = L->stream;
    const int64_t q0 = b * chunk, nq = std::min(total, q0 + chunk) - q0;
    // HtoD of chunk b once the lane's previous search (b - nl) has read d_q
    if (b >= nl) CUDA_TRY(cudaStreamWaitEvent(ix->h2d, L->ev_done, 0));
    CUDA_TRY(cudaMemcpyAsync(L->d_q, qh + q0 * qrow, nq * qrow, cudaMemcpyHostToDevice, ix->h2d));
    CUDA_TRY(cudaEventRecord(L->ev_h2d, ix->h2d));
    CUDA_TRY(cudaStreamWaitEvent(st, L->ev_h2d, 0));
    // the lane's outputs once the DtoH of chunk b - nl has read them
    if (b >= nl) CUDA_TRY(cudaStreamWaitEvent(st, L->ev_out, 0));
    const float* dq = L->d_q;
    if (ix->metric == SONG_HAMMING) {
      rc = encode_queries(L, L->d_q, nq, st);
      if (rc) return rc;
      dq = reinterpret_cast<const float*>(L->d_qcodes);
    }
    rc = enqueue_search(L, p, dq, nq, L->d_ids, L->d_dists, nullptr, st);
    if (rc) return rc;
    CUDA_TRY(cudaEventRecord(L->ev_done, st));
    CUDA_TRY(cudaStreamWaitEvent(ix->d2h, L->ev_done, 0));
    CUDA_TRY(cudaMemcpyAsync(ih + q0 * orow, L->d_ids, nq * orow, cudaMemcpyDeviceToHost, ix->d2h));
    CUDA_TRY(cudaMemcpyAsync(dh + q0 * orow, L->d_dists, nq * orow, cudaMemcpyDeviceToHost, ix->d2h));
    CUDA_TRY(cudaEventRecord(L->ev_out, ix->d2h));
  }
  // the last DtoH waits for the last search, which follows every earlier one
  // on its lane; the other lane's last search precedes its own DtoH on d2h
  CUDA_TRY(cudaStreamSynchronize(ix->d2h));
  int st_all = 0;
  for (int l = 0; l < nl; ++l) {
    int s = 0;
    CUDA_TRY(cudaMemcpy(&s, lane[l]->d_status, sizeof s, cudaMemcpyDeviceToHost));
    CUDA_TRY(cudaMemset(lane[l]->d_status, 0, sizeof s));
    st_all |= s;
  }
  ix->last_stream = ix->stream;
  return status_code(st_all);
}
}  // namespace

extern "C" {

int song_search(song_index* ix, const float* queries, int64_t nq, int32_t K, int32_t queue_len,
                int32_t* ids_out, float* dists_out) {
  if (!ix || !queries || !ids_out || !dists_out) return fail(SONG_EINVAL, "NULL argument");
  if (nq < 1) return fail(SONG_EINVAL, "nq must be >= 1");
  song_search_params p;
  song_default_params(&p, K, queue_len);
  int rc = check_params(ix, &p);
  if (rc) return rc;
  if (ix->metric == SONG_HAMMING && !ix->d_R)
    return fail(SONG_EINVAL, "this index holds codes without R: use song_search_codes_ex");
  const int qdim = ix->metric == SONG_HAMMING ? ix->rp_dim : ix->dim;
  const size_t qbytes = (size_t)nq * qdim * sizeof(float);
  const size_t obytes = (size_t)nq * K * sizeof(int32_t);
  rc = ensure_io(ix, qbytes, obytes);
  if (rc) return rc;
  cudaStream_t st = ix->stream;
  rc = order_after_last(ix, st);
  if (rc) return rc;
  CUDA_TRY(cudaMemcpyAsync(ix->d_q, queries, qbytes, cudaMemcpyHostToDevice, st));
  const float* dq = ix->d_q;
  if (ix->metric == SONG_HAMMING) {
    rc = encode_queries(ix, ix->d_q, nq, st);
    if (rc) return rc;
    dq = reinterpret_cast<const float*>(ix->d_qcodes);
  }
  rc = enqueue_search(ix, &p, dq, nq, ix->d_ids, ix->d_dists, nullptr, st);
  if (rc) return rc;
  CUDA_TRY(cudaMemcpyAsync(ids_out, ix->d_ids, obytes, cudaMemcpyDeviceToHost, st));
  CUDA_TRY(cudaMemcpyAsync(dists_out, ix->d_dists, obytes, cudaMemcpyDeviceToHost, st));
  // the status word rides the same stream (one synchronisation per call)
  if (!ix->h_status) CUDA_TRY(cudaMallocHost(&ix->h_status, sizeof(int)));
  CUDA_TRY(cudaMemcpyAsync(ix->h_status, ix->d_status, sizeof(int), cudaMemcpyDeviceToHost, st));
  CUDA_TRY(cudaMemsetAsync(ix->d_status, 0, sizeof(int), st));
  CUDA_TRY(cudaStreamSynchronize(st));
  return status_code(*ix->h_status);
}

int song_search_pipelined(song_index* ix, const song_search_params* p, const float* queries,
                          int64_t nbatch, int64_t nq, int32_t* ids_out, float* dists_out) {
  if (!ix || !p || !queries || !ids_out || !dists_out) return fail(SONG_EINVAL, "NULL argument");
  if (nbatch < 1 || nq < 1) return fail(SONG_EINVAL, "nbatch and nq must be >= 1");
  if (nq > 0x7fffffffll) return fail(SONG_EUNSUPPORTED, "nq must fit int32");
  if (ix->is_twin) return fail(SONG_EINVAL, "not an index handle");
  int rc = check_params(ix, p);
  if (rc) return rc;
  if (ix->metric == SONG_HAMMING && !ix->d_R)
    return fail(SONG_EINVAL, "this index holds codes without R: use song_search_codes_ex");
  return run_pipeline(ix, p, queries, nbatch, nq, nbatch * nq, ids_out, dists_out);
}

int song_merge_topk(const int32_t* ids_in, const float* dists_in, int32_t G, int64_t nq,
                    int32_t Kin, int32_t K, int32_t* ids_out, float* dists_out, void* stream) {
  if (!ids_in || !dists_in || !ids_out || !dists_out) return fail(SONG_EINVAL, "NULL argument");
  if (G < 1 || nq < 1 || Kin < 1 || K < 1) return fail(SONG_EINVAL, "sizes must be >= 1");
  if (K > 1024 || Kin > 1024) return fail(SONG_EUNSUPPORTED, "K and Kin must be <= 1024");
  const int warps = 8;
  int64_t blocks = (nq + warps - 1) / warps;
  song::song_merge_kernel<<<(unsigned)blocks, warps * 32, 0, (cudaStream_t)stream>>>(
      ids_in, dists_in, G, nq, Kin, K, ids_out, dists_out);
  CUDA_TRY(cudaGetLastError());
  return SONG_OK;
}

int song_stage_cycles(song_index* ix, uint64_t* cycles_out, int32_t reset) {
  if (!ix || !cycles_out) return fail(SONG_EINVAL, "NULL argument");
#ifdef SONG_STAGE_TIMING
  CUDA_TRY(cudaStreamSynchronize(ix->last_stream));
  if (!ix->d_stage) {
    for (int k = 0; k < 4; ++k) cycles_out[k] = 0;
    return SONG_OK;
  }
  CUDA_TRY(cudaMemcpy(cycles_out, ix->d_stage, 4 * sizeof(uint64_t), cudaMemcpyDeviceToHost));
  if (reset) CUDA_TRY(cudaMemset(ix->d_stage, 0, 4 * sizeof(uint64_t)));
  return SONG_OK;
#else
  (void)reset;
  for (int k = 0; k < 4; ++k) cycles_out[k] = 0;
  return fail(SONG_EUNSUPPORTED, "this libsong.so was built without SONG_STAGE_TIMING");
#endif
}

int song_merge_topk_peers(const int32_t* const* ids_peers, const float* const* dists_peers,
                          uint32_t* const* signal_peers, int32_t rank, int32_t G, int64_t nq,
                          int32_t Kin, int32_t K, uint32_t epoch, int32_t* ids_out,
                          float* dists_out, void* stream) {
  if (!ids_peers || !dists_peers || !ids_out || !dists_out) return fail(SONG_EINVAL, "NULL argument");
  if (G < 1 || G > 256 || nq < 1 || Kin < 1 || K < 1)
    return fail(SONG_EINVAL, "G must be in [1, 256], nq, Kin, K >= 1");
  if (K > 1024 || Kin > 1024) return fail(SONG_EUNSUPPORTED, "K and Kin must be <= 1024");
  if (signal_peers && (rank < 0 || rank >= G || epoch == 0))
    return fail(SONG_EINVAL, "rank %d outside [0, %d) or epoch 0", rank, G);
  const int warps = 8;
  const int64_t blocks = (nq + warps - 1) / warps;
  const int threads = std::max(warps * 32, ((G + 31) / 32) * 32);
  song::song_merge_peers_kernel<<<(unsigned)blocks, threads, 0, (cudaStream_t)stream>>>(
      ids_peers, dists_peers, signal_peers, rank, G, nq, Kin, K, epoch, ids_out, dists_out);
  CUDA_TRY(cudaGetLastError());
  return SONG_OK;
}

const char* song_last_error(void) { return g_err.c_str(); }

const char* song_version(void) { return "song-b200 0.1 sm_100a"; }

}  // extern "C"
