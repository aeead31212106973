/*
 * ganns.h -- C ABI of the B200-native GANNS search / GGraphCon NSW construction
 * library (libganns.so).  Yu, Wen, Zhang, Qin, Zhang, Lin, "GPU-accelerated
 * Proximity Graph Approximate Nearest Neighbor Search and Construction",
 * ICDE 2022.  "P:NNN" = line NNN of the paper text.
 *
 * Conventions for every entry point
 *  - Plain C types only.  `stream` is a cudaStream_t passed as void* (NULL =
 *    the legacy default stream).  Device pointers are CUDA global memory on the
 *    graph's device; host pointers are ordinary (optionally pinned) memory.
 *  - Vectors are fp32, row-major, rows of d floats, 16-byte aligned, d % 4 == 0.
 *  - Ids are int32 vertex numbers = row index in `points` = insertion order
 *    (P:260).  -1 marks an empty slot.
 *  - Every function returns a ganns_status (0 = OK, < 0 = error) and never
 *    throws or aborts; ganns_last_error() describes the last failure of the
 *    calling thread.  On error no output is guaranteed to be written.
 *  - Asynchronous on `stream` unless stated ("syncs").
 *  - Results are deterministic: the same inputs give bit-identical outputs on
 *    every run, stream and GPU count.
 */
#ifndef GANNS_H
#define GANNS_H

#include <stddef.h>
#include <stdint.h>

#if defined(__GNUC__)
#define GANNS_API __attribute__((visibility("default")))
#else
#define GANNS_API
#endif

#ifdef __cplusplus
extern "C" {
#endif

/* Distance delta(q, x) (Table I: "Euclidean" and "Cosine Similarity").
 *  GANNS_L2     squared Euclidean sum_j (q_j - x_j)^2 (same ranking as Euclidean)
 *  GANNS_IP     -<q, x>
 *  GANNS_COSINE 1 - <q, x> / ||q||; the caller passes unit-normalised `points`.
 *               Inside ganns_build, COSINE orders candidates by -<x_v, x_u>
 *               (identical ranking for unit rows, symmetric in u and v). */
typedef enum { GANNS_L2 = 0, GANNS_IP = 1, GANNS_COSINE = 2 } ganns_metric;

typedef enum {
    GANNS_OK = 0,
    GANNS_EINVAL = -1,   /* argument outside the documented domain */
    GANNS_ENOMEM = -2,   /* device or host allocation failed */
    GANNS_ECUDA = -3,    /* a CUDA runtime error (message has the CUDA string) */
    GANNS_ENOTSUP = -4,  /* valid but unsupported combination */
    GANNS_EIO = -5       /* file could not be read / written / has a bad header */
} ganns_status;

/* Opaque graph handle, library-owned.  Holds the fixed-degree adjacency
 * int32 nbr[n][d_max] in device memory (Def. 2: directed, out-lists
 * bounded by d_max; P:197 graph kept in GPU global memory) and its metadata.
 * It does NOT hold or copy the point vectors: every search must pass the same
 * `points` the graph was built from (a precondition that cannot be checked). */
typedef struct ganns_graph ganns_graph;

/* Parameters of Algorithm 2.  Zero-initialise for defaults. */
typedef struct {
    int d_min;          /* forward edges per vertex (Alg. 2 input P:316); 0 -> degree/2 */
    int l_build;        /* candidate-array length of the build searches; 0 -> 64   */
    int e_build;        /* explore budget of the build searches; 0 -> l_build      */
    int64_t group_size; /* |P_i| of the partition (Alg. 2 line 1); 0 -> auto        */
    int max_rounds;     /* 0 -> all t Phase-2 rounds; > 0 -> at most that many (parity hook) */
    int stop_after_phase1; /* != 0: return the union of local graphs (parity hook)         */
    uint64_t *stats;    /* host, nullable, [4]: search iterations, distance computations,
                           searches, rounds -- filled when ganns_build returns             */
    int l_local;        /* list length of the Phase-1 searches on the local graphs (lines
                           4-5); 0 -> l_build; else in [d_min, l_build]; their explore
                           budget is min(e_build, l_local) (R-C13: the paper leaves both
                           lengths open).  Ignored by ganns_build_hnsw.                    */
} ganns_build_params;

/* Extra search parameters.  Zero-initialise for defaults. */
typedef struct {
    int e;              /* explore budget: only N[0..e) is eligible; 0 -> l        */
    int64_t entry;      /* start vertex v_s; 0 (default) = vertex 0, R-C4           */
    uint32_t *stats;    /* device, nullable, [nq][3] per query: iterations, distance
                           computations (entry + every valid neighbour), T entries
                           merged into N (kept among the first l)                   */
    uint32_t *descent_stats; /* device, nullable, [nq][2] (HNSW searches only): iterations and
                           distance computations of the greedy descent through the upper
                           layers (R-H1), summed over the layers; ignored by the NSW calls */
} ganns_search_params;

/* ganns_build -- GGraphCon NSW construction, Algorithm 2 (§IV-B
 * P:253-297).  Phase 1 builds one local NSW per group by sequential insertion
 * (P:266-281), Phase 2 merges groups 1..t into G_0 round by round,
 * every search being the GANNS search of ganns_search with (l_build, e_build).
 *   points  device, [n][d] fp32, read only, must stay alive for later searches
 *   n       number of points, d_min < n < 2^31
 *   d       dimension, d % 4 == 0, 4 <= d <= 1024
 *   metric  ganns_metric
 *   degree  d_max, 2 <= degree <= 128
 *   p       nullable (all defaults)
 *   out     receives a new graph on the current device.  Syncs `stream`.
 * Scratch (build-form adjacency with distances, G', E, offsets) is allocated
 * and freed inside the call. */
GANNS_API int ganns_build(const float *points, int64_t n, int d, int metric, int degree,
                const ganns_build_params *p, void *stream, ganns_graph **out);

/* ---------------------------------------------------------------- staged build
 * Algorithm 2 one step at a time, for a construction split over several working
 * units (the paper's Remarks: "each working unit ... builds one local
 * graph" and the searches of an iteration are independent).  Every rank holds
 * the same points and a full replica of the graph state; a rank runs Phase 1 for
 * its share of the groups and the Phase-2 searches for its share of each round's
 * vertices; the caller exchanges the results (ganns_build_rows, the F blocks)
 * and every rank applies the same round, so the replicas stay bit-identical to
 * ganns_build with the same parameters (python: dist.build_distributed).
 *
 * ganns_build_begin  -- validate (exactly as ganns_build) and allocate the state
 *   and the graph rows on the current device; returns the state in *out.
 *   p->max_rounds / stop_after_phase1 / stats are ignored (the caller drives the
 *   rounds; ganns_build_finish returns the counters).
 * ganns_build_info   -- group size s (R-C14), number of groups t + 1,
 *   d_min, d_max.  Group g holds vertices [g*s, min((g+1)*s, n)).
 * ganns_build_phase1 -- Alg. 2 lines 2-8 for groups [g0, g1) (a group's
 *   insertions touch only its own rows); async on `stream`.
 * ganns_build_rows   -- copy the build-form rows of vertices [v0, v1) out of
 *   (to_state = 0) or into (to_state = 1) the state: device buffers ids / dists
 *   [v1-v0][d_max] (row-major, -1 / +inf padded) and pids / pdists [v1-v0][d_min]
 *   (N').  Importing whole groups marks them ready for Phase 2.
 * ganns_build_round_search -- Alg. 2 lines 10-17 of round i (1 <= i <= t) for
 *   the vertices [v0, v1) of P_i: writes each v's new forward row F (the first
 *   d_min of Search(G_0, v) u v.N' by (dist, id), R-C16) to f_ids / f_dists
 *   (device, [v1-v0][d_min], -1 / +inf padded).  Requires Phase 1 of groups
 *   0..i and rounds 1..i-1 applied.  Reads the state only.
 * ganns_build_round_apply -- the rest of round i from the F of ALL of P_i
 *   (f_ids / f_dists [|P_i|][d_min], in vertex order): rows of P_i <- F (R-C15),
 *   E from F (line 17), GatherScatter and the per-vertex merges (lines 19-22).
 *   Rounds must be applied in order 1, 2, ..., t.
 * ganns_build_finish -- syncs `stream`; *out receives the graph (same as
 *   ganns_build's), stats (nullable, host [4]) the build counters (search
 *   iterations, distance computations, searches run on THIS rank, rounds); the
 *   state is freed.
 * ganns_build_abort  -- frees a state and its graph (NULL is a no-op).
 * Errors: GANNS_EINVAL for out-of-range groups / vertices / rounds, rounds out of
 *   order, or a round before its groups are ready; otherwise as ganns_build. */
typedef struct ganns_build_state ganns_build_state;
GANNS_API int ganns_build_begin(const float *points, int64_t n, int d, int metric, int degree,
                                const ganns_build_params *p, void *stream,
                                ganns_build_state **out);
GANNS_API int ganns_build_info(const ganns_build_state *s, int64_t *group_size,
                               int64_t *ngroups, int *d_min, int *d_max);
GANNS_API int ganns_build_phase1(ganns_build_state *s, int64_t g0, int64_t g1, void *stream);
GANNS_API int ganns_build_rows(ganns_build_state *s, int64_t v0, int64_t v1, int32_t *ids,
                               float *dists, int32_t *pids, float *pdists, int to_state,
                               void *stream);
GANNS_API int ganns_build_round_search(ganns_build_state *s, int64_t i, int64_t v0, int64_t v1,
                                       int32_t *f_ids, float *f_dists, void *stream);
GANNS_API int ganns_build_round_apply(ganns_build_state *s, int64_t i, const int32_t *f_ids,
                                      const float *f_dists, void *stream);
GANNS_API int ganns_build_finish(ganns_build_state *s, void *stream, uint64_t *stats,
                                 ganns_graph **out);
GANNS_API void ganns_build_abort(ganns_build_state *s);

/* ganns_search -- batched GANNS search (§III-B): for each query,
 * the k approximate nearest neighbours (Def. 1) found with a
 * candidate array of length l (lazy update) and the lazy check.
 *   g         graph
 *   points    device [n][d], the vectors the graph was built from
 *   queries   device [nq][d]
 *   nq        >= 0 (0 is a no-op)
 *   k         1 <= k <= l, k < n
 *   l         k <= l <= 1024 (any value; not restricted to powers of two, R-C7)
 *   out_ids   device [nq][k] int32, ascending (dist, id); -1 if fewer reachable (R-C8)
 *   out_dists device [nq][k] fp32, +inf where out_ids is -1 */
GANNS_API int ganns_search(const ganns_graph *g, const float *points, const float *queries, int64_t nq,
                 int k, int l, int32_t *out_ids, float *out_dists, void *stream);

/* ganns_search_ex -- ganns_search with explore budget e, entry vertex and
 * per-query statistics (p nullable = ganns_search). */
GANNS_API int ganns_search_ex(const ganns_graph *g, const float *points, const float *queries,
                    int64_t nq, int k, int l, const ganns_search_params *p,
                    int32_t *out_ids, float *out_dists, void *stream);

/* ganns_search_host -- end-to-end search from HOST buffers (P:218 remark):
 * queries_host [nq][d] is copied in, results are copied back to out_ids_host /
 * out_dists_host [nq][k].  The batch is split in chunks pipelined over the
 * library's copy/compute streams (H2D of chunk i+1 overlaps the search of
 * chunk i and the D2H of chunk i-1).  Host buffers should be pinned
 * (cudaHostAlloc / cudaHostRegister) for overlap.  Syncs. */
GANNS_API int ganns_search_host(const ganns_graph *g, const float *points, const float *queries_host,
                      int64_t nq, int k, int l, const ganns_search_params *p,
                      int32_t *out_ids_host, float *out_dists_host, void *stream);

/* ganns_search_host_async -- one batch end to end from HOST buffers, enqueued on
 * `stream` without synchronising (the streamed multi-batch pipeline, P:218:
 * "the data transfer can be overlapped with the search using CUDA streams").
 * On `stream`, in order: H2D queries_host -> queries_dev, the search
 * (= ganns_search_ex), D2H ids_dev / dists_dev -> out_ids_host / out_dists_host.
 * Alternating two streams over consecutive batches overlaps one batch's copies
 * and drain tail with the next batch's search.
 *   queries_host   host [nq][d] fp32, pinned (cudaHostAlloc / cudaHostRegister)
 *   queries_dev    device scratch [nq][d] fp32, 16-B aligned
 *   ids_dev, dists_dev  device scratch [nq][k]
 *   out_ids_host, out_dists_host  host [nq][k], pinned
 * Ownership: every buffer is the caller's; none may be reused or freed until
 * `stream` has passed this call (e.g. cudaStreamSynchronize).  Errors as
 * ganns_search_ex; EINVAL for NULL buffers.  Does not sync. */
GANNS_API int ganns_search_host_async(const ganns_graph *g, const float *points,
                                      const float *queries_host, int64_t nq, int k, int l,
                                      const ganns_search_params *p, float *queries_dev,
                                      int32_t *ids_dev, float *dists_dev, int32_t *out_ids_host,
                                      float *out_dists_host, void *stream);

/* ganns_merge_topk -- K6: merge W per-shard top-k lists into the global top-k
 * (multi-GPU base-set sharding).  For each query the k smallest
 * (dist, global id) over all shards.  All pointers device.
 *   shard_ids   [W][nq][k] int32 GLOBAL ids (-1 = empty), shard_dists [W][nq][k]
 *   out_ids / out_dists [nq][k]. */
GANNS_API int ganns_merge_topk(const int32_t *shard_ids, const float *shard_dists, int W, int64_t nq,
                     int k, int32_t *out_ids, float *out_dists, void *stream);

/* ganns_offset_ids -- add `offset` to every id >= 0 of ids[count] (device),
 * turning shard-local ids into global ids. */
GANNS_API int ganns_offset_ids(int32_t *ids, int64_t count, int64_t offset, void *stream);

/* ganns_graph_from_adjacency -- import an adjacency array (tests, oracle graphs).
 *   nbr_host  host [n][d_max] int32; each row: distinct ids in [0, n), -1 padded
 *             (rows with a repeated id are rejected: EINVAL)
 *   d, metric metadata (the graph does not store vectors)
 *   device    CUDA device ordinal for the copy.  Syncs. */
GANNS_API int ganns_graph_from_adjacency(const int32_t *nbr_host, int64_t n, int d_max, int d,
                               int metric, int device, ganns_graph **out);

/* ganns_graph_adjacency -- copy the adjacency to host out_host [n][d_max].  Syncs. */
GANNS_API int ganns_graph_adjacency(const ganns_graph *g, int32_t *out_host);

/* ganns_graph_device_ptr -- device pointer to the adjacency [n][d_max] (borrowed). */
GANNS_API int ganns_graph_device_ptr(const ganns_graph *g, const int32_t **nbr);

/* ganns_graph_info -- any output pointer may be NULL. */
GANNS_API int ganns_graph_info(const ganns_graph *g, int64_t *n, int *d, int *d_max, int *metric);

/* ganns_graph_save / ganns_graph_load -- file = 32-byte header
 * ("GANNSG01", n, d, d_max, metric) + int32 [n][d_max].  Syncs. */
GANNS_API int ganns_graph_save(const ganns_graph *g, const char *path);
GANNS_API int ganns_graph_load(const char *path, int device, ganns_graph **out);

/* ganns_graph_free -- NULL is a no-op. */
GANNS_API void ganns_graph_free(ganns_graph *g);

/* ---------------------------------------------------------------- HNSW
 * HNSW extension of Algorithm 2 (Section IV-D).  Layer j holds the
 * points whose level >= j (levels are drawn by the caller -- the random
 * selection of P:369 -- and passed in).  (1) ids are shuffled: points sorted by
 * level descending, ties by id (perm[new] = old), so layer j is the shuffled-id
 * prefix [0, n_j); (2) layers are built top-down with Algorithm 2 on their
 * prefix; a Phase-2 search enters layer j at the vertex reached by a greedy
 * descent (GANNS search with l = e = 1) of the finished layers above, if that
 * vertex is already merged, else at vertex 0; (3) layer 0 is relabelled to the
 * original ids (a plain ganns_graph); the upper layers stay in shuffled ids.
 * Search = greedy descent of the upper layers, then the GANNS search on layer 0
 * from the vertex reached. */
typedef struct ganns_hnsw ganns_hnsw;

/* ganns_build_hnsw -- as ganns_build (p->max_rounds and p->stop_after_phase1 are
 * ignored; p->l_local applies to every layer's Phase 1, R-C13), plus
 *   levels_host  host int8 [n], level of every point, 0 <= level < 16.
 * Syncs.  The index keeps a device copy of the rows of the upper-layer points. */
GANNS_API int ganns_build_hnsw(const float *points, int64_t n, int d, int metric, int degree,
                               const int8_t *levels_host, const ganns_build_params *p,
                               void *stream, ganns_hnsw **out);

/* ganns_hnsw_search -- ganns_search_ex on the HNSW index; p->entry is ignored
 * (each query enters layer 0 where its descent ends).  d <= 256: one kernel (the
 * descent runs inside K1); d > 256: an entry kernel, then K1. */
GANNS_API int ganns_hnsw_search(const ganns_hnsw *h, const float *points, const float *queries,
                                int64_t nq, int k, int l, const ganns_search_params *p,
                                int32_t *out_ids, float *out_dists, void *stream);

/* ganns_hnsw_search_host_async -- ganns_search_host_async on the HNSW index
 * (H2D, ganns_hnsw_search, D2H on `stream`; same buffers, ownership and errors). */
GANNS_API int ganns_hnsw_search_host_async(const ganns_hnsw *h, const float *points,
                                           const float *queries_host, int64_t nq, int k, int l,
                                           const ganns_search_params *p, float *queries_dev,
                                           int32_t *ids_dev, float *dists_dev,
                                           int32_t *out_ids_host, float *out_dists_host,
                                           void *stream);

/* ganns_hnsw_info -- number of layers; layer_n (nullable) receives n_j for j < nlayers. */
GANNS_API int ganns_hnsw_info(const ganns_hnsw *h, int *nlayers, int64_t *layer_n);

/* ganns_hnsw_layer -- copy layer j's adjacency to host out [n_j][d_max]: layer 0
 * in original ids, layers >= 1 in shuffled ids.  Syncs. */
GANNS_API int ganns_hnsw_layer(const ganns_hnsw *h, int layer, int32_t *out_host);

/* ganns_hnsw_perm -- copy perm[n] (shuffled id -> original id) to host.  Syncs. */
GANNS_API int ganns_hnsw_perm(const ganns_hnsw *h, int32_t *out_host);

/* ganns_hnsw_base -- layer 0 as a ganns_graph (borrowed; valid until ganns_hnsw_free). */
GANNS_API int ganns_hnsw_base(const ganns_hnsw *h, const ganns_graph **base);

/* ganns_hnsw_free -- NULL is a no-op. */
GANNS_API void ganns_hnsw_free(ganns_hnsw *h);

/* ---------------------------------------------------------------- KNN graph
 * ganns_build_knn -- KNN graph (every list = K nearest, k = d_min = d_max)
 * by neighbours-of-neighbours iterations (Section IV-D, after
 * NN-Descent [9]): from the random lists init_host, each iteration joins every
 * pair of a vertex's neighbours (its list and its reverse list, capped at the K
 * nearest) and every list keeps its K nearest distinct candidates; stops when no
 * list changes or after max_iters iterations.
 *   init_host   host int32 [n][K]: distinct ids != row, no -1 (e.g. random)
 *   K           1 <= K <= 32, K < n
 *   out         graph [n][K] ascending by (dist, id); iters_out / changed_last
 *               (nullable): iterations run, lists changed in the last one.
 * Proposal buffer: n * 2K * (2K - 1) entries of 12 bytes (ENOMEM if it does not fit). Syncs. */
GANNS_API int ganns_build_knn(const float *points, int64_t n, int d, int metric, int K,
                              const int32_t *init_host, int max_iters, void *stream,
                              ganns_graph **out, int *iters_out, int64_t *changed_last);

/* ganns_last_error -- thread-local message of the last failing call ("" if none). */
GANNS_API const char *ganns_last_error(void);

/* ganns_kernel_launches -- number of kernels this library launched in this
 * process so far (bench evidence for "gpu_launches"). */
GANNS_API uint64_t ganns_kernel_launches(void);

/* ganns_profile_read -- per-phase cycle counters of the search loop (the
 * analogue of the paper's time breakdowns, Fig. 7 / Fig. 10), summed
 * over every search (batched search and build) on the current device since the last
 * reset: out[0..5] = cycles in candidate locating, neighbourhood exploration,
 * bulk distance, lazy check, sort, merge (lane 0's clock64 at the phase
 * boundaries), out[6] = iterations, out[7] = searches.  Syncs the device; reset != 0
 * zeroes the counters.  GANNS_ENOTSUP unless the library was built with
 * -DGANNS_PROFILE=1 (tools/build_variants.sh prof -DGANNS_PROFILE=1). */
GANNS_API int ganns_profile_read(uint64_t *out, int reset);

/* ganns_profile_read_n -- the same counters, `count` (0..16) of them: out[0..7] as
 * above; inside the bulk distance out[8] = cycles from the start of a TMA round to
 * its last issue, out[9] = cycles waiting on the round's mbarrier, out[10] = TMA
 * rounds; out[11] = explorations whose adjacency row the speculative load of the
 * second unexplored entry had already fetched; out[12] / out[13] = the largest loop
 * cycles / iterations of a single search (maxima).  GANNS_EINVAL if count is out of range. */
GANNS_API int ganns_profile_read_n(uint64_t *out, int count, int reset);

#ifdef __cplusplus
}
#endif
#endif /* GANNS_H */
