/* song.h — C ABI of the B200-native SONG search library (libsong.so).
 *
 * SONG: Approximate Nearest Neighbor Search on GPU (Zhao, Tan, Li; ICDE 2020).
 * "P:<n>" cites /root/reference/PAPER.md line n.
 *
 * The library runs the paper's batched best-first graph search (Algorithm 1,
 * P:41-49) decoupled into candidate locating (§V), bulk distance
 * computation (§VI) and data-structure maintenance (§IV)
 * with a bounded priority queue (§IV-C), selected insertion (§IV-D,
 * P:425-431), visited deletion (§IV-E) and a shared-memory
 * open-addressing hash or Bloom-filter visited set.  Every
 * step runs in sm_100a kernels; there is no CPU fallback.
 *
 * Conventions for every entry point:
 *  - returns SONG_OK (0) on success or a negative song_status;
 *    song_last_error() then holds a thread-local message;
 *  - "host" pointers are ordinary CPU memory (pinned or pageable);
 *    "device" pointers are CUDA global memory on the index's device;
 *  - all matrices are dense row-major; ids are int32, vectors fp32;
 *  - the library never takes ownership of caller buffers.
 *
 * Semantics (DESIGN.md §3 lists every reading of the paper):
 *  - entry vertex = params.entry (default 0; "default starting point");
 *  - adjacency entries lie in [-1, n); -1 is padding (fixed-degree rows);
 *  - distances: SONG_L2 = squared Euclidean, SONG_IP = -<q,x>,
 *    SONG_COSINE = 1 - <q,x>/(|q||x|); zero-norm vectors give 1;
 *  - ties are broken by id: every order is on the key (dist, id);
 *  - outputs are the first K of topk in ascending (dist, id) order; if fewer
 *    than K vertices are reached, the rest is (-1, +INF) (Alg. 1 line 17);
 *  - q and topk both hold at most queue_len = L >= K entries (readings A1, A2).
 */
#ifndef SONG_H_
#define SONG_H_

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct song_index song_index; /* opaque; owns its device copies */

/* SONG_HAMMING: the index holds h-bit codes of the 1-bit random projection
 * (§VII) and the distance is the Hamming distance (number of
 * differing bits, returned as an exact integer-valued float).  Such indexes
 * are made only by song_index_create_codes / song_index_create_rp. */
typedef enum { SONG_L2 = 0, SONG_IP = 1, SONG_COSINE = 2, SONG_HAMMING = 3 } song_metric;

typedef enum {
  SONG_OK = 0,
  SONG_EINVAL = -1,       /* bad argument: NULL, sizes < 1, K > queue_len, id out of
                             range, non-finite input value */
  SONG_ENOMEM = -2,       /* device or host allocation failed */
  SONG_ECUDA = -3,        /* a CUDA runtime call or kernel failed */
  SONG_EUNSUPPORTED = -4, /* a size above the compiled maxima (degree > 32,
                             dim > 1024, queue_len > SONG_MAX_QUEUE_LEN,
                             shared-memory budget exceeded) */
  SONG_EITERCAP = -5      /* a query reached params.max_iters expansions */
  /* (SONG_EUNSUPPORTED is also the sticky status of a query whose global
     visited table filled up; raise params.table_log2) */
} song_status;

typedef enum {
  SONG_VISITED_HASH = 0,            /* shared-memory open addressing, selected insertion +
                                       visited deletion ("hashtable-sel-del", Fig. 7)
                                       — the default and the fast path */
  SONG_VISITED_BLOOM = 1,           /* shared-memory Bloom filter, selected insertion, no
                                       deletion ("bloomfilter") */
  SONG_VISITED_HASH_GLOBAL = 2,     /* exact hash in global memory, no selected insertion,
                                       no deletion ("hashtable", Fig. 7) */
  SONG_VISITED_HASH_GLOBAL_SEL = 3, /* as 2 with selected insertion ("hashtable-sel") */
  SONG_VISITED_CUCKOO = 4           /* shared-memory Cuckoo filter, selected insertion +
                                       visited deletion ("cuckoofilter"; DESIGN.md
                                       reading R10) */
} song_visited_kind;

#define SONG_MAX_DEGREE 32
#define SONG_MAX_DIM 1024
#define SONG_MAX_QUEUE_LEN 2048
#define SONG_MAX_CODE_BITS 1024
#define SONG_MAX_STEPS 4

typedef struct song_search_params {
  int32_t K;               /* results per query, 1 <= K <= queue_len */
  int32_t queue_len;       /* L: capacity of q and of topk (§IV-C) */
  int32_t visited;         /* song_visited_kind */
  int32_t bloom_log2_bits; /* Bloom size m = 2^bloom_log2_bits bits; 0 = default
                              2^ceil(log2(80 L)) (reading A11) */
  int32_t entry;           /* starting vertex id, 0 <= entry < n */
  int32_t max_iters;       /* expansion cap per query (0 = 1<<30); a query that
                              reaches it is flagged, see song_search_ex */
  int32_t warps_per_block; /* launch shape: 0 = library default (4); at most 4 */
  int32_t blocks_per_sm;   /* launch shape: 0 = as many as fit */
  int32_t id_offset;       /* added to every returned id (dataset sharding, P:471:
                              shard-local ids become global ids); default 0 */
  int32_t table_log2;      /* capacity of the visited table: HASH_GLOBAL(_SEL): log2
                              slots per warp (default max(14, ceil(log2(64 L)))); a
                              query that fills half of it stops with SONG_EUNSUPPORTED
                              status; CUCKOO: log2 buckets of 4 (default: 4 slots per
                              live key bound 2L+32); ignored otherwise; 0 = default */
  int32_t steps;           /* multi-step probing (§V, reading R13): up to
                              `steps` vertices popped per iteration into one candidate
                              list; 0 or 1 = Algorithm 1's single pop; at most
                              SONG_MAX_STEPS; > 1 needs visited HASH or BLOOM and a
                              float index (else SONG_EUNSUPPORTED) */
  int32_t visited_cap;     /* SONG_VISITED_HASH deletion schedule (§IV-E, DESIGN.md
                              reading R14).  0 = lazy deletion with the default capacity
                              C: separate q / topk (queue_kind SEPARATE) C = 5S/8 for
                              queue_len <= 128, 3S/4 above, where S = 2^ceil(log2(F (2L +
                              32))) table slots, F = 8 (L <= 64; 4 for rows of 129-256
                              floats), 4 (L <= 128) or 4/3; the union (queue_kind UNION,
                              the default for visited HASH, steps 1): see queue_kind
                              (song_search_plan_get reports the C in effect); > 0 =
                              lazy with C = visited_cap (2L + 32 <= C <= 3S/4, or
                              L + 32 <= C for the union; else SONG_EINVAL); -1 = eager deletion (every evicted vertex
                              erased at once, the paper's literal schedule).  Lazy: the
                              erasures are applied together (visited := ids(q) ∪
                              ids(topk)) when the selected candidates of an iteration
                              would grow visited past C — same results, fewer recomputed
                              distances.  steps > 1 always uses eager deletion.  Ignored
                              by the other visited kinds. */
  int32_t schedule;        /* order in which the batch's queries are issued to the
                              persistent grid (a scheduling choice: every query's ids,
                              distances and counters are independent of it).
                              SONG_SCHEDULE_AUTO (0, default) = outlier-first for float
                              indexes when nq exceeds the grid's resident warps, else
                              batch order; SONG_SCHEDULE_BATCH = batch order;
                              SONG_SCHEDULE_OUTLIER_FIRST = descending squared distance
                              from the index centroid (longest-expected-first list
                              scheduling: far-out queries search longest),
                              in 4096 log-spaced key bins.  Codes indexes always use
                              batch order. */
  int32_t queue_kind;      /* how q and topk are held (results never depend on it).
                              SONG_QUEUE_AUTO (0, default): with visited HASH and steps
                              <= 1 the bounded union (W in 1, 2, 4 or 8 registers per
                              lane for queue_len <= 256, in shared memory above); otherwise
                              separate q and topk, in registers for queue_len <= 128,
                              in shared memory above.
                              SONG_QUEUE_SEPARATE: q and topk as the paper keeps them
                              (§IV-C), each bounded at L.  SONG_QUEUE_UNION (DESIGN.md
                              reading R17): ONE list of the L best keys of q ∪ topk,
                              each marked popped or not — the next pop is its first
                              unpopped key, the search stops when none is left; the
                              hash then holds <= L + 32 live ids (lazy capacity C in
                              [L + 32, 3S/4], default 3S/4, S = 2^ceil(log2(8 (L + 32)
                              / 3)) above queue_len 128 and the separate queues' S up
                              to 128) and a vertex dropped from the list is recomputed if
                              met again (counters differ, results do not).  UNION needs
                              visited HASH and steps <= 1 (else SONG_EUNSUPPORTED). */
  int32_t queries_per_warp; /* Fig. 8's multi-query packing (§V).
                              0 (default) = the production kernel (one query per warp,
                              every stage warp-cooperative).  1, 2 or 4 = the packing
                              kernel: that many queries per warp, each searched by its
                              own team of 32 / queries_per_warp lanes with team-scoped
                              collectives and its own shared-memory q, topk (sorted
                              arrays) and exact hash; the paper's literal schedule
                              (separate q / topk, selected insertion, eager deletion).
                              Needs visited HASH, visited_cap -1, steps <= 1,
                              queue_kind AUTO or SEPARATE, queue_len <= 128 and a float
                              index (else SONG_EUNSUPPORTED); results equal the other
                              kernels', counters equal the eager schedule's.  It issues
                              the batch in batch order (schedule is ignored). */
} song_search_params;

#define SONG_QUEUE_AUTO 0
#define SONG_QUEUE_SEPARATE 1
#define SONG_QUEUE_UNION 2

#define SONG_SCHEDULE_AUTO 0
#define SONG_SCHEDULE_BATCH 1
#define SONG_SCHEDULE_OUTLIER_FIRST 2

typedef struct song_index_info {
  int64_t n;               /* points */
  int32_t dim;             /* dimensions */
  int32_t dim_padded;      /* row stride in floats (multiple of 4: 16 B rows) */
  int32_t degree;          /* adjacency slots per vertex */
  int32_t metric;          /* song_metric */
  int64_t vector_bytes;    /* n * dim_padded * 4 */
  int64_t graph_bytes;     /* n * degree * 4 (Table III) */
  int32_t device;          /* CUDA device ordinal */
  int32_t num_sms;         /* SMs on that device */
  int32_t code_bits;       /* SONG_HAMMING: h bits per code (dim_padded is then the
                              row stride in 32-bit words, vector_bytes the codes'
                              bytes, Table IV, and dim the length of the float
                              queries song_search accepts: the original dimension for
                              an index made by song_index_create_rp, else 0); else 0 */
  int32_t reserved;        /* 0 (keeps the struct free of implicit padding) */
} song_index_info;

/* Fill p with the library defaults for (K, queue_len). Never fails. */
void song_default_params(song_search_params* p, int32_t K, int32_t queue_len);

/* What song_search_ex would run for `params` on an index of `dim` dimensions
 * and `metric` (SONG_HAMMING: dim = code words, bits / 32) — the resolved
 * data-structure sizes and launch shape.  Pure host computation: it never
 * touches a device, so it is callable without a GPU.  This is the single
 * source of the library's defaults (tests, bench and tools read the lazy
 * deletion capacity and the visited-table size from here rather than
 * re-deriving them). */
typedef struct song_search_plan {
  int32_t visited_log2;    /* SONG_VISITED_HASH, _HASH_GLOBAL(_SEL): log2 table slots;
                              BLOOM: log2 bits m (reading A11); CUCKOO: log2 buckets of
                              4 fingerprints (reading R10) */
  int32_t visited_cap;     /* SONG_VISITED_HASH: the capacity C of lazy deletion in effect
                              (reading R14, or R17's when queue_kind is 2; the oracle's
                              lazy_cap), or -1 for eager
                              deletion (visited_cap = -1 or steps > 1); 0 for the other
                              kinds */
  int32_t queue_regs;      /* q and topk held in registers, queue_regs u64 per lane
                              (queue_len <= 32 * queue_regs); 0 = shared-memory queues */
  int32_t row_chunks;      /* 16 B chunks per lane of a staged row (NCH) */
  int32_t smem_per_warp;   /* shared-memory bytes per warp */
  int32_t warps_per_block; /* CTA size of the persistent grid (1 warp = 1 query) */
  int32_t queue_kind;      /* 0 registers, 1 separate shared-memory q and topk, 2 the
                              bounded union of reading R17 (song_search_params.queue_kind) */
  int32_t visited_global;  /* 1: the hash visited table of each warp lives in global
                              memory (L2) instead of shared memory — chosen for the
                              bounded union when it lets >= 1.5x the warps reside on an
                              SM; 0 otherwise */
} song_search_plan;

/* Errors: SONG_EINVAL (NULL, bad params as song_search_ex would report them,
 * except the entry range, which needs the index), SONG_EUNSUPPORTED (the
 * sizes above the compiled maxima, shared-memory budget exceeded). */
int song_search_plan_get(const song_search_params* params, int32_t dim, int32_t metric,
                         song_search_plan* out);

/* Create an index on the current CUDA device from HOST arrays (§IV-A, P:267,
 * graph and data are persisted in global memory before any query).
 *   vectors   [n][dim] fp32, host; copied (rows padded to 16 B; for
 *             SONG_COSINE rows are L2-normalised on the device).
 *   adjacency [n][degree] int32, host; copied.  Entries in [-1, n).
 *   out       receives the handle; *out is NULL on error.
 * Errors: SONG_EINVAL (NULL, n < 1, dim < 1, degree < 1, id out of range,
 * non-finite vector value), SONG_EUNSUPPORTED (degree > 32, dim > 1024),
 * SONG_ENOMEM, SONG_ECUDA. */
int song_index_create(const float* vectors, int64_t n, int32_t dim,
                      const int32_t* adjacency, int32_t degree, song_metric metric,
                      song_index** out);

/* As song_index_create, but vectors and adjacency are DEVICE pointers on the
 * current device (validated on the device); stream is a cudaStream_t or NULL
 * (legacy default stream).  The call returns after the copies complete. */
int song_index_create_device(const float* vectors, int64_t n, int32_t dim,
                             const int32_t* adjacency, int32_t degree, song_metric metric,
                             void* stream, song_index** out);

/* Release the index and its device memory.  NULL is a no-op (returns 0). */
int song_index_destroy(song_index* idx);

int song_index_get_info(const song_index* idx, song_index_info* info);

/* Search nq queries with HOST buffers (Alg. 1 over a batch); blocking.
 *   queries   [nq][dim] fp32 host; ids_out [nq][K] int32 host;
 *   dists_out [nq][K] fp32 host.  Uses song_default_params(K, queue_len).
 * The HtoD copy of the queries, the kernel and the DtoH copy of the results all
 * happen inside this call (Fig. 10's HtoD / kernel / DtoH).
 * Errors: SONG_EINVAL (NULL, nq < 1, K < 1, queue_len < K, non-finite query),
 * SONG_EUNSUPPORTED (queue_len too large), SONG_EITERCAP, SONG_ECUDA. */
int song_search(song_index* idx, const float* queries, int64_t nq, int32_t K,
                int32_t queue_len, int32_t* ids_out, float* dists_out);

/* Search a STREAM of nbatch query batches held in HOST memory (the batched
 * throughput setting of §VIII, with Fig. 10's HtoD / kernel / DtoH per
 * batch); blocking.
 *   queries   [nbatch][nq][dim] fp32 host (dim = song_index_info.dim);
 *   ids_out   [nbatch][nq][K] int32 host; dists_out [nbatch][nq][K] fp32 host.
 * Batch b's results are exactly those of song_search_ex(params) on batch b
 * alone (every query is searched independently; the ticket order never
 * changes results).  The call keeps two batches in flight on two device
 * buffer sets with their own work counters: the HtoD copy of batch b + 1 and
 * the DtoH copy of batch b - 1 run on copy streams under the search of batch
 * b, and batch b + 1's search kernel takes the SMs batch b's persistent grid
 * releases in its tail (two compute streams).  Page-locked host buffers
 * (cudaHostAlloc, torch pin_memory) let the copies overlap; pageable ones
 * give the same results with serialised copies.  Ordered after any search
 * previously enqueued on the index.  Errors: as song_search (SONG_EINVAL also
 * for nbatch < 1); the sticky status covers every batch. */
int song_search_pipelined(song_index* idx, const song_search_params* params,
                          const float* queries, int64_t nbatch, int64_t nq,
                          int32_t* ids_out, float* dists_out);

/* Search with DEVICE buffers on a caller stream; asynchronous (returns after
 * enqueueing).  counters_out, if not NULL, receives [nq][2] int32
 * (distance computations, expansions) per query — the algorithmic work that
 * defines the roofline bytes.  A query with a non-finite value gets ids -1;
 * one that reaches max_iters returns its partial topk; both are reported by
 * song_index_last_status().
 * Concurrency: the searches of one index share its work counter and status
 * word, so the library orders them: a search enqueued on a stream other than
 * the previous search's waits (cudaStreamWaitEvent) for that search to finish
 * on the device.  Searches of distinct indexes run concurrently.  Host calls
 * on one index must not race (one host thread at a time per index).
 * Errors detectable before launch: SONG_EINVAL, SONG_EUNSUPPORTED, SONG_ECUDA. */
int song_search_ex(song_index* idx, const song_search_params* params,
                   const float* queries, int64_t nq, int32_t* ids_out, float* dists_out,
                   int32_t* counters_out, void* stream);

/* Synchronise the index's last stream and return the sticky status of the
 * searches since the previous call (SONG_OK, SONG_EINVAL for a non-finite
 * query, SONG_EITERCAP); clears it. */
int song_index_last_status(song_index* idx);

/* G-way merge of per-shard results ("perform graph search on each GPU
 * and merge the results").  DEVICE buffers:
 *   ids_in [G][nq][Kin] int32 global ids, dists_in [G][nq][Kin] fp32, each row
 *   sorted ascending by (dist, id), -1 padded;
 *   ids_out [nq][K], dists_out [nq][K]: the K smallest (dist, id) keys.
 * Asynchronous on stream.  Errors: SONG_EINVAL, SONG_EUNSUPPORTED (K > 1024). */
int song_merge_topk(const int32_t* ids_in, const float* dists_in, int32_t G, int64_t nq,
                    int32_t Kin, int32_t K, int32_t* ids_out, float* dists_out,
                    void* stream);

/* The same merge fused with the gather over peer memory (dataset sharding on
 * one node): each of the G ranks searched its shard into a [nq][Kin]
 * ids / dists buffer the other ranks can address (e.g. torch symmetric memory
 * over NVLink / NVSwitch), rows sorted by (dist, global id), -1 padded.
 *   ids_peers, dists_peers  DEVICE arrays of G DEVICE pointers: rank g's rows;
 *   signal_peers            DEVICE array of G DEVICE pointers to each rank's
 *                           signal pad (>= G uint32, zero-initialised once and
 *                           reserved for this call), or NULL;
 *   rank                    this rank (0 <= rank < G);
 *   epoch                   > every epoch used before with these pads;
 *   ids_out, dists_out      DEVICE [nq][K] on this rank: the K smallest keys.
 * With pads, the kernel (enqueued on `stream` after this rank's search) first
 * stores `epoch` into slot `rank` of every peer's pad (release, system
 * scope), then waits for every peer's slot of its own pad (acquire) and
 * merges straight from the peers' buffers: no staging copy, no separate
 * all-gather.  Every rank must make the call with the same G, nq, Kin, epoch.
 * Without pads the caller guarantees the peers' rows are complete and
 * visible (one-GPU emulation, or after its own barrier).  Asynchronous.
 * Errors: SONG_EINVAL (NULL, sizes, rank/epoch), SONG_EUNSUPPORTED (K or Kin
 * > 1024). */
int song_merge_topk_peers(const int32_t* const* ids_peers, const float* const* dists_peers,
                          uint32_t* const* signal_peers, int32_t rank, int32_t G, int64_t nq,
                          int32_t Kin, int32_t K, uint32_t epoch, int32_t* ids_out,
                          float* dists_out, void* stream);

/* ---- 1-bit random projection (§VII "Out-of-GPU-memory datasets") ----
 * "For two data vectors u, v ... we generate a random vector r with entries in
 * iid standard normal ... With h independent random vectors, each data point
 * is mapped into an h-bit vector. The hamming distance between the
 * bit-vectors becomes an good estimate of the similarity".
 * Code layout (reading R11): bit j = [<x, r_j> > 0] (a zero
 * projection gives 0), stored in 32-bit word j / 32 at bit j % 32; a code is
 * h / 32 words ("h can be set as a multiple of 32").  R is [h][dim]
 * fp32 row-major (row j = r_j), drawn by the caller. */

/* Encode n DEVICE vectors [n][dim] fp32 with DEVICE R [bits][dim] into DEVICE
 * codes [n][bits/32] uint32 (dense rows).  fp32 accumulation; asynchronous on
 * stream.  Errors: SONG_EINVAL (NULL, n < 1, dim < 1, bits not a positive
 * multiple of 32), SONG_EUNSUPPORTED (bits > SONG_MAX_CODE_BITS), SONG_ECUDA. */
int song_rp_encode(const float* vectors, int64_t n, int32_t dim, const float* R, int32_t bits,
                   uint32_t* codes, void* stream);

/* Create a SONG_HAMMING index from HOST codes [n][bits/32] uint32 and HOST
 * adjacency [n][degree] int32 (both copied).  Queries then go through
 * song_search_codes_ex.  Errors as song_index_create, plus SONG_EINVAL for
 * bits not a positive multiple of 32, SONG_EUNSUPPORTED for bits >
 * SONG_MAX_CODE_BITS. */
int song_index_create_codes(const uint32_t* codes, int64_t n, int32_t bits,
                            const int32_t* adjacency, int32_t degree, song_index** out);

/* Create a SONG_HAMMING index from HOST vectors [n][dim] fp32 that need not fit
 * in device memory: the vectors are streamed to the device in chunks,
 * encoded with HOST R [bits][dim] (copied; kept by the index) and only the
 * codes stay resident.  adjacency is HOST [n][degree] int32 (the graph built on
 * the original vectors).  song_search / song_search_ex then take float
 * queries [nq][dim], encoded on the device with the same R before the search.
 * Errors as song_index_create_codes, plus SONG_EINVAL for a non-finite vector
 * or R value. */
int song_index_create_rp(const float* vectors, int64_t n, int32_t dim, const float* R,
                         int32_t bits, const int32_t* adjacency, int32_t degree,
                         song_index** out);

/* Search a SONG_HAMMING index with DEVICE query codes [nq][bits/32] uint32;
 * otherwise as song_search_ex (same params, outputs, counters and errors;
 * params.visited must be SONG_VISITED_HASH or SONG_VISITED_BLOOM, else
 * SONG_EUNSUPPORTED).  Returned distances are Hamming distances. */
int song_search_codes_ex(song_index* idx, const song_search_params* params,
                         const uint32_t* query_codes, int64_t nq, int32_t* ids_out,
                         float* dists_out, int32_t* counters_out, void* stream);

/* ---- graph construction (reading R15) ----
 * All three builders first scan the rows on the device: a non-finite value is
 * SONG_EINVAL.  Step 1's distance tiles run on the tensor cores (tcgen05
 * kind::tf32) only when that is exact — every value an integer, dim *
 * max|x|^2 < 2^24, rows 16 B aligned — and on fp32 FFMA tiles otherwise.
 *
 * SONG searches pre-built NSW graphs; this builds one on the
 * device: forward lists F(i) = the `degree` nearest earlier vertices (exact
 * insertion NSW), backward lists B(j) = the `degree` nearest i with j in F(i),
 * candidates F(v) u B(v) by (dist, id), HNSW neighbour heuristic with refill,
 * -1 padding.  Distances are the search's (L2 squared, -<a,b>, 1 - cos).
 *   vectors       DEVICE [n][dim] fp32 (not modified)
 *   adjacency_out DEVICE [n][degree] int32 (caller-allocated)
 * Blocking on stream (scratch ~ 24 n degree bytes is allocated and freed).
 * Errors: SONG_EINVAL (NULL, sizes < 1, metric), SONG_EUNSUPPORTED (degree >
 * SONG_MAX_DEGREE, n >= 2^31), SONG_ENOMEM, SONG_ECUDA. */
int song_build_graph(const float* vectors, int64_t n, int32_t dim, song_metric metric,
                     int32_t degree, int32_t* adjacency_out, void* stream);

/* ---- batched-insertion graph construction (reading R16) ----
 * The scale-out builder (R15's exact forward lists cost O(n^2)): rows
 * [0, prefix) get R15's exact forward lists; then, batch by batch, rows
 * [m, m + max(1, m >> batch_shift)) search the graph G_m built (R15 steps 2-4)
 * from the forward lists of rows [0, m) — Algorithm 1 from entry 0 with
 * K = degree and queue_len, this library's own search — and take its top
 * `degree` as their forward lists; the graph is R15 steps 2-4 on every row.
 * With prefix >= n it equals song_build_graph.
 *   vectors       DEVICE [n][dim] fp32 (not modified)
 *   adjacency_out DEVICE [n][degree] int32 (caller-allocated; also holds G_m
 *                 while the batches run)
 * Blocking on stream; scratch ~ 24 n degree bytes (+ n dpad floats when dim %
 * 4 != 0 or cosine).  Errors: as song_build_graph; SONG_EINVAL for prefix < 1,
 * queue_len outside [degree, SONG_MAX_QUEUE_LEN], batch_shift outside [0, 16]
 * or non-finite vectors. */
int song_build_graph_batched(const float* vectors, int64_t n, int32_t dim, song_metric metric,
                             int32_t degree, int32_t prefix, int32_t queue_len,
                             int32_t batch_shift, int32_t* adjacency_out, void* stream);

/* R15 steps 2-4 (backward lists, candidates, HNSW heuristic with refill) on
 * caller-given forward lists: fwd_ids / fwd_dists DEVICE [n][degree] (each row
 * ascending by (dist, id), -1 past its entries, distances in the search's
 * definition), e.g. kNN lists from another builder or a refinement search.
 * The lists need not be earlier-only: the candidates C(v) = F(v) u B(v) are
 * taken as a set of vertices (v itself dropped, an id in both lists kept once
 * at its smaller key).  Same arguments, scratch and errors as
 * song_build_graph, + SONG_EINVAL for NULL lists or an id outside [-1, n)
 * (checked on the device before any work). */
int song_build_graph_from_forward(const float* vectors, int64_t n, int32_t dim,
                                  song_metric metric, int32_t degree, const int32_t* fwd_ids,
                                  const float* fwd_dists, int32_t* adjacency_out, void* stream);

/* Instrumentation builds only (compiled with -DSONG_STAGE_TIMING, e.g.
 * `python -m paper_conf_icde_zhaotl20_b200._build --define SONG_STAGE_TIMING
 * --out libsong_stages.so`; never the product library): the SM cycles the
 * searches of this index spent per stage since the last reset, summed over
 * warps — cycles_out[0] pop / terminate / topk update (Alg. 1 lines 3-8),
 * [1] candidate locating (§V), [2] bulk distance computation (§VI), [3]
 * maintenance (§IV) — the in-kernel split of Fig. 10.
 * Synchronises the index's last stream; reset != 0 zeroes the counters.
 * Errors: SONG_EINVAL (NULL), SONG_EUNSUPPORTED (a build without the
 * instrumentation; cycles_out is zeroed). */
int song_stage_cycles(song_index* idx, uint64_t* cycles_out, int32_t reset);

/* Reading R18 (graphs for the inner-product metric): row v of out = the first
 * `take_first` ids of first[v], then the ids of second[v], then the rest of
 * first[v] — each id once (its first occurrence), -1 skipped, truncated to
 * `degree`, -1 padded.  With first = the IP graph (song_build_graph, SONG_IP)
 * and second = the angular graph (song_build_graph_batched, SONG_COSINE) this
 * keeps each vertex's best inner-product links and fills the row with
 * direction-preserving ones, which the IP search navigates far better than
 * either graph alone (R18).
 *   first, second, out  DEVICE [n][degree] int32 (out may not alias the inputs)
 * Asynchronous on stream.  Errors: SONG_EINVAL (NULL, n < 1, degree < 1,
 * take_first outside [0, degree]), SONG_EUNSUPPORTED (degree > 32). */
int song_graph_merge_rows(const int32_t* first, const int32_t* second, int64_t n,
                          int32_t degree, int32_t take_first, int32_t* out, void* stream);

/* Thread-local message of the last failing call ("" if none). */
const char* song_last_error(void);

/* Library version string, e.g. "song-b200 0.1 sm_100a". */
const char* song_version(void);

#ifdef __cplusplus
}
#endif

#endif /* SONG_H_ */
