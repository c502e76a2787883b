/* hec.h — C-ABI of libhec: the B200 (sm_100a) hot path of iterated Heavy Edge
 * Coarsening (HEC), Gilbert, Acer, Boman, Madduri, Rajamanickam, IPDPS 2021.
 *
 * PAPER.md references are to /root/reference/PAPER.md (line numbers "L…").
 * The three north-star entry points follow the paper's Algorithm 1 (L37-53):
 *   hec_find_mapping   FINDCOARSEMAPPING with HEC (Alg 3 L99-130; parallel Alg 4
 *                      L168-225): M[1..n], n_c  (L103)
 *   build_coarse_graph CONSTRUCTCOARSEGRAPH (Alg 6): G(V_c, E_c, W_c) in CSR
 *   coarsen_hierarchy  Alg 1 with cutoff C and the discard rule of L367
 *
 * Conventions:
 *   - 0-based ids (the paper is 1-based, L280).  Vertex ids, labels, columns and
 *     edge/vertex weights are int32; row offsets are int64 (R7).
 *   - Pointers inside hec_graph and all array arguments documented "device" are
 *     CUDA device pointers; "host" arguments are host pointers.
 *   - All work is stream-ordered on the context's stream.  Calls that must know a
 *     size on the host (n_c, nnz_c) synchronise that stream once to read it.
 *   - Inputs are never written.  Outputs allocated by the library are owned by the
 *     returned handle and released with the matching *_free call.
 *   - Every function returns HEC_OK (0) or a negative HEC_E* code; on error no
 *     output handle is returned and hec_last_error() (thread-local) describes it.
 *   - Results are deterministic and bit-exact with the plain sequential
 *     definition (Alg 3 under the visit order of hec_prio, coarse ids by ascending
 *     root id, coarse rows with ascending columns and summed integer weights).
 */
#ifndef HEC_H
#define HEC_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#if defined(_WIN32)
#define HEC_API __declspec(dllexport)
#else
#define HEC_API __attribute__((visibility("default")))
#endif

/* ------------------------------------------------------------------ errors */
enum {
  HEC_OK = 0,
  HEC_EINVAL = -1,    /* bad argument or (validate=1) malformed graph */
  HEC_ENOMEM = -2,    /* device allocation failed */
  HEC_ECUDA = -3,     /* CUDA runtime / kernel error */
  HEC_EOVERFLOW = -4  /* a coarse weight or vertex weight exceeds INT32_MAX */
};
/* Why coarsen_hierarchy stopped (Alg 1 loop test L46 + L367). */
enum {
  HEC_STOP_CUTOFF = 0,     /* n_l <= C */
  HEC_STOP_DISCARD = 1,    /* next level would drop below discard_below: not built */
  HEC_STOP_STALL = 2,      /* n_c == n (only possible with all vertices isolated) */
  HEC_STOP_MAX_LEVELS = 3  /* level cap reached */
};

/* Thread-local, static storage; valid until the next failing call on the thread. */
HEC_API const char *hec_last_error(void);

/* ------------------------------------------------------------------- graph */
/* Borrowed CSR view of an undirected graph G(V,E,W):
 * each undirected edge stored in both endpoint rows, no self-loops, no parallel
 * edges, weights > 0 and symmetric, columns strictly ascending within a row. */
typedef struct {
  int64_t n;               /* |V| (0 <= n < 2^31)                                  */
  int64_t nnz;             /* directed entries = 2m                                 */
  const int64_t *row_ptr;  /* device [n+1], row_ptr[0]=0, non-decreasing, [n]=nnz  */
  const int32_t *col;      /* device [nnz]                                          */
  const int32_t *wgt;      /* device [nnz], > 0, W(u,v) == W(v,u)                   */
  const int32_t *vwgt;     /* device [n] vertex weights > 0, or NULL = all ones     */
} hec_graph;

/* --------------------------------------------------------------- context */
typedef struct CUstream_st *hec_stream_t; /* == cudaStream_t */
/* Optional device allocator (e.g. a framework caching allocator).  Must return
 * 256-byte aligned device memory usable on `stream`, or NULL on failure. */
typedef void *(*hec_alloc_fn)(size_t bytes, hec_stream_t stream, void *user);
typedef void (*hec_free_fn)(void *ptr, hec_stream_t stream, void *user);

typedef struct hec_ctx hec_ctx;

/* Create a context bound to the current CUDA device and `stream` (NULL = the
 * legacy default stream).  alloc/free NULL => cudaMallocAsync/cudaFreeAsync on
 * the device's default pool.  The context owns a grow-only device workspace
 * reused across calls (no per-call allocation once warm). */
HEC_API int hec_ctx_create(hec_stream_t stream, hec_alloc_fn alloc, hec_free_fn free,
                           void *user, hec_ctx **out);
HEC_API void hec_ctx_destroy(hec_ctx *ctx);
/* validate=1: every call first checks R1 on the device (O(nnz)): offsets
 * monotone, columns in range/strictly ascending/no self-loop, weights > 0,
 * symmetric structure and weights; a violation returns HEC_EINVAL. */
HEC_API int hec_ctx_set_validate(hec_ctx *ctx, int validate);
HEC_API int hec_ctx_set_stream(hec_ctx *ctx, hec_stream_t stream);

/* Per-call statistics of the most recent hec_find_mapping/coarsen_hierarchy
 * level processed by this context. */
typedef struct {
  int32_t rounds;          /* resolution rounds of the last mapping */
  int32_t fallback;        /* 1 if the round cap was hit and the residual was finished sequentially */
  int64_t n_c;             /* coarse vertices of the last mapping */
  int64_t nnz_c;           /* coarse entries of the last construction */
  int64_t huge_rows;       /* rows routed to the skewed-degree path in the last construction */
  int64_t dense_rows;      /* of which used the dense accumulator */
} hec_stats;
HEC_API int hec_ctx_last_stats(const hec_ctx *ctx, hec_stats *out);

/* ------------------------------------------------- north-star call 1: mapping */
/* Visit-order priority of vertex u at level l (the paper's
 * GENPERM "random order", L61, L104):
 *   s_l = splitmix64(seed + l);  prio_l(u) = (splitmix64(s_l ^ u) >> 32) << 32 | u
 * Host helper so callers can reproduce the order. */
HEC_API uint64_t hec_prio(uint64_t seed, int level, int64_t u);

/* HEC fine-to-coarse mapping of g (Alg 3 semantics, computed by the parallel
 * heavy-neighbour scan + deterministic resolution rounds):
 *   H[u]  = heaviest neighbour, ties -> smallest id, isolated -> u   (L116, L184)
 *   visit order ascending hec_prio(seed, level, u)
 *   M     = device int32[n] caller-allocated; coarse ids 0..n_c-1 ordered by the
 *           aggregate's root (the vertex an aggregate was created at) ascending
 *   *n_c  = host int64, number of aggregates.
 * Synchronises the stream once (to read n_c).  n == 0 gives n_c = 0. */
HEC_API int hec_find_mapping(hec_ctx *ctx, const hec_graph *g, uint64_t seed, int level,
                             int32_t *M, int64_t *n_c);

/* Same with explicit device priorities prio[n] (uint64, pairwise distinct: the
 * visit order is ascending prio).  Test hook for hand-drawn visit orders. */
HEC_API int hec_find_mapping_prio(hec_ctx *ctx, const hec_graph *g, const uint64_t *prio,
                                  int32_t *M, int64_t *n_c);

/* The paper's other FINDCOARSEMAPPING methods, same
 * contract as hec_find_mapping (M device int32[n], *n_c host, one sync):
 *   HEC_MAP_HEC   Alg 3 (the default of every other call)
 *   HEC_MAP_HEC3  Alg 5 (L248-273): mutual heavy neighbours collapse onto the
 *                 smaller id, vertices with in-degree > 0 in the heavy-neighbour
 *                 pseudoforest are roots, the others inherit; order-free (seed
 *                 and level are ignored)
 *   HEC_MAP_HEM   Alg 2 (L73-97): heavy-edge matching in the hec_prio visit
 *                 order, the heaviest *unmatched* neighbour (ties -> smallest
 *                 id), identical to the sequential algorithm (root = the
 *                 visiting vertex); coarsening ratio <= 2 (L61)
 * Coarse ids ascend with the aggregates' roots (FINDUNIQANDRELABEL, reading Z3). */
enum { HEC_MAP_HEC = 0, HEC_MAP_HEC3 = 1, HEC_MAP_HEM = 2 };
HEC_API int hec_find_mapping_method(hec_ctx *ctx, const hec_graph *g, int method, uint64_t seed, int level,
                                    int32_t *M, int64_t *n_c);
/* Same with explicit device priorities (test hook, as hec_find_mapping_prio). */
HEC_API int hec_find_mapping_method_prio(hec_ctx *ctx, const hec_graph *g, int method, const uint64_t *prio,
                                         int32_t *M, int64_t *n_c);

/* --------------------------------------------- north-star call 2: construction */
typedef struct hec_csr_owned hec_csr_owned; /* device CSR owned by the library */

/* Coarse graph G_c = P A P^T without the diagonal (L141, L280):
 *   W_c(a,b) = sum_{M[u]=a} sum_{v in N(u), M[v]=b} W(u,v) for a != b,
 *   rows ascending by b, vwgt_c(a) = sum_{M[u]=a} vwgt(u).
 * M: device int32[n] with values in [0, n_c), every label used.
 * Returns HEC_EOVERFLOW if a sum exceeds INT32_MAX.  Synchronises once (nnz_c). */
HEC_API int build_coarse_graph(hec_ctx *ctx, const hec_graph *g, const int32_t *M,
                               int64_t n_c, hec_csr_owned **out);
/* The construction methods (Alg 6); all
 * give the same canonical G_c, only the work differs:
 *   HEC_BUILD_HASH     per-row shared-memory hash merge + order-preserving
 *                      bucket rank (the default of every other call)
 *   HEC_BUILD_SORT     sort-based DEDUPWITHWTS (register bitonic pieces,
 *                      shared-memory bucket sort) for every row
 *   HEC_BUILD_ONE_END  degree-based one-end storage: an entry is kept only in
 *                      the row of its end with the smaller C' (the count of a
 *                      row's non-self fine entries, l.1-5; ties: smaller coarse
 *                      id, reading Z7), then GraphConsWithTrans (l.22)
 *   HEC_BUILD_AUTO     ONE_END when max degree / average degree > 10 (L324,
 *                      reading Z15), else HASH */
enum { HEC_BUILD_HASH = 0, HEC_BUILD_SORT = 1, HEC_BUILD_ONE_END = 2, HEC_BUILD_AUTO = 3 };
HEC_API int build_coarse_graph_ex(hec_ctx *ctx, const hec_graph *g, const int32_t *M, int64_t n_c, int method,
                                  hec_csr_owned **out);
/* Borrow the owned CSR as a hec_graph (valid until hec_csr_free). */
HEC_API int hec_csr_view(const hec_csr_owned *csr, hec_graph *view);
HEC_API void hec_csr_free(hec_csr_owned *csr);

/* ---------------------------------------------- north-star call 3: hierarchy */
typedef struct hec_hierarchy hec_hierarchy;

/* Alg 1: l = 0; while n_l > cutoff and l < max_levels:
 *   (M, n') = hec_find_mapping(G_l, seed, level = l);
 *   if n' < discard_below: stop (DISCARD; G_{l+1} not built)   (L367, reading Z11/Z12)
 *   if n' == n_l: stop (STALL)
 *   G_{l+1} = build_coarse_graph(G_l, M, n'); l++
 * Output levels i = 1..l hold G_i and M_i (M_i maps G_{i-1} -> G_i).
 * discard_below <= 0 selects the paper's 10; max_levels <= 0 selects 200. */
HEC_API int coarsen_hierarchy(hec_ctx *ctx, const hec_graph *g0, int64_t cutoff, uint64_t seed,
                              int64_t discard_below, int max_levels, hec_hierarchy **out);
/* coarsen_hierarchy with the mapping method (HEC_MAP_*) and the construction
 * method (HEC_BUILD_*) of every level chosen (coarsen_hierarchy ==
 * coarsen_hierarchy_ex(..., HEC_MAP_HEC, HEC_BUILD_HASH, ...)). */
HEC_API int coarsen_hierarchy_ex(hec_ctx *ctx, const hec_graph *g0, int64_t cutoff, uint64_t seed,
                                 int64_t discard_below, int max_levels, int map_method, int build_method,
                                 hec_hierarchy **out);
HEC_API int hec_hierarchy_levels(const hec_hierarchy *h);
/* i in [1, levels]: view of G_i, device pointer to M_i (length n_{i-1}), n_{i-1}. */
HEC_API int hec_hierarchy_level(const hec_hierarchy *h, int i, hec_graph *g_i,
                                const int32_t **M_i, int64_t *n_fine);
HEC_API int hec_hierarchy_stop_reason(const hec_hierarchy *h);
/* n' of the discarded mapping when stop_reason == HEC_STOP_DISCARD, else -1. */
HEC_API int64_t hec_hierarchy_discarded_n_c(const hec_hierarchy *h);
/* Resolution rounds used at level i (1-based), or -1. */
HEC_API int hec_hierarchy_rounds(const hec_hierarchy *h, int i);
HEC_API void hec_hierarchy_free(hec_hierarchy *h);

/* ------------------------------------------- consumer: spectral bisection */
/* Multilevel spectral bisection on a hierarchy (PAPER.md
 * §III-C): on every level, coarsest first, power iteration for the
 * Fiedler vector of the graph Laplacian L = D - A (x <- (sigma I - L) x with
 * sigma = 2 max weighted degree, projected off the constant vector and
 * normalised; fp64), stopped when ||x_{k+1} - x_k||_2 < tol or after max_iter;
 * interpolation x_fine[u] = x_coarse[M[u]]; then part 0 = the n/2 vertices with
 * the smallest (x, id) (no imbalance, L330).  The coarsest start vector is
 * x0[u] = (splitmix64(seed ^ u) >> 11) 2^-53 - 1/2.
 *   g0: the hierarchy's input graph; h from coarsen_hierarchy on g0.
 *   part: device uint8[n0] (0 / 1); x: device double[n0] or NULL (the finest
 *   iterate); *cut (host): weight of the cut edges; iters (host, optional):
 *   int64[levels + 1], iterations per level from the coarsest. */
typedef struct {
  int64_t max_iter;  /* per level; <= 0 selects 1000 */
  double tol;        /* < 0 selects 1e-10 (L367); 0 runs max_iter iterations */
  uint64_t seed;
} hec_spectral_opts;
HEC_API int hec_spectral_bisection(hec_ctx *ctx, const hec_graph *g0, const hec_hierarchy *h,
                                   const hec_spectral_opts *opts, uint8_t *part, double *x, int64_t *cut,
                                   int64_t *iters);

/* ------------------------------------------------------------ profiling */
/* When enabled, every phase of the hot path is bracketed by CUDA events on the
 * context stream; hec_ctx_profile() synchronises, then reports per phase the
 * summed device time, number of calls and the algorithmic bytes (compulsory
 * traffic: each input read once, each output written once).
 * Phases: "heavy" (a1), "rounds" (a3), "relabel" (a4+a5), "bucket" (a7),
 * "expand", "rows_skew", "rows" (a8/a9), "place" (a10), "gather" (the
 * all-gathers of the multi-GPU calls), and inside
 * coarsen_hierarchy one "level" phase per level l spanning its mapping and
 * construction, with SURVEY §8(d)'s compulsory bytes
 *   B_l = 16 nnz + 8 nnz_c + 28 n + 12 n_c   (built level)
 *   B_l = 8 nnz + 12 n                       (discarded level: mapping only).
 * Entries are accumulated per (phase, level). */
typedef struct {
  char name[24];
  double ms;         /* summed device time */
  int64_t calls;
  double bytes;      /* summed algorithmic bytes */
  int32_t level;     /* coarsen_hierarchy level index l (fine graph G_l), -1 outside a hierarchy */
} hec_phase_time;
HEC_API int hec_ctx_set_profiling(hec_ctx *ctx, int on);
/* Clears the accumulated phase times and the launch counter. */
HEC_API int hec_ctx_profile_reset(hec_ctx *ctx);
/* Writes up to max entries; *count receives the number of phases. */
HEC_API int hec_ctx_profile(hec_ctx *ctx, hec_phase_time *out, int max, int *count);
/* Number of libhec kernel launches since the last reset. */
HEC_API int64_t hec_ctx_launches(const hec_ctx *ctx);

/* ------------------------------------------------------- debug / test hooks */
/* Heavy-neighbour array only (a1): H device int32[n]. */
HEC_API int hec_debug_heavy(hec_ctx *ctx, const hec_graph *g, int32_t *H);
/* Root flags after the resolution rounds (a3): root device uint8[n] (1 = root);
 * *rounds (host) receives the number of rounds.  prio NULL => hec_prio(seed, level). */
HEC_API int hec_debug_roots(hec_ctx *ctx, const hec_graph *g, const uint64_t *prio,
                            uint64_t seed, int level, uint8_t *root, int *rounds);

/* ----------------------------------------------- multi-GPU calls (§8(e)) */
/* One process per GPU; every rank holds the whole input graph (replicated,
 * e.g. generated or loaded on each rank) and calls the same function with the
 * same arguments.  The only exchange step is an all-gather of equal-size byte
 * blocks, supplied by the caller (NCCL through torch.distributed on a GPU box,
 * gloo in tests), so the library needs no NCCL link of its own:
 *   allgather(send, recv, bytes, stream, user): rank r's `bytes` bytes at
 *   device pointer `send` land at recv + r * bytes on every rank, ordered on
 *   `stream` (the context's); returns 0, or non-zero on failure (the library
 *   call then returns HEC_ECUDA).
 * Uneven pieces are padded to the largest one.  Results are bit-identical to
 * the single-GPU calls (tests/test_gpu_dist.py). */
typedef int (*hec_allgather_fn)(const void *send, void *recv, size_t bytes, hec_stream_t stream, void *user);
typedef struct {
  int32_t rank, world;          /* 0 <= rank < world */
  hec_allgather_fn allgather;
  void *user;
} hec_comm;

/* hec_find_mapping partitioned over the ranks: heavy neighbours of the rank's
 * fine-vertex slice (the mapping's only edge stream, a1) -> all-gather H; the
 * resolution rounds and the relabel (vertex-only, cheap) run on every rank;
 * M of the slice -> all-gather M.  M (device int32[n]) is complete on every
 * rank on return. */
HEC_API int hec_find_mapping_dist(hec_ctx *ctx, const hec_graph *g, uint64_t seed, int level,
                                  const hec_comm *comm, int32_t *M, int64_t *n_c);
/* build_coarse_graph partitioned by coarse-row range (
 * construction input "G, n, m, M, n_c" of Alg 6): the
 * ranks split the coarse rows into contiguous ranges of about equal
 * member-edge volume (identical on every rank), each builds its rows, the
 * slices' entry counts are all-gathered and every rank derives the global row
 * offsets.  gather_full = 1: the slices (row offsets, columns, weights, vertex
 * weights) are all-gathered and every rank receives the whole G_c, stitched in
 * C; gather_full = 0: *out holds the rank's slice only -- a CSR of rows
 * [row_begin, row_end) with local row offsets -- placed by hec_csr_dist_slice. */
HEC_API int build_coarse_graph_dist(hec_ctx *ctx, const hec_graph *g, const int32_t *M, int64_t n_c,
                                    const hec_comm *comm, int gather_full, hec_csr_owned **out);
/* Placement of a slice from build_coarse_graph_dist(gather_full = 0): its rows
 * [*row_begin, *row_end) of G_c, its first entry at global position
 * *entry_offset, *nnz_total entries in all slices.  A whole graph reports
 * [0, n_c), 0, nnz_c. */
HEC_API int hec_csr_dist_slice(const hec_csr_owned *csr, int64_t *row_begin, int64_t *row_end,
                               int64_t *entry_offset, int64_t *nnz_total);
/* coarsen_hierarchy with every level whose fine graph has at least
 * partition_min_nnz entries mapped and built by hec_find_mapping_dist and
 * build_coarse_graph_dist(gather_full = 1); smaller levels run on every rank
 * locally (no exchange: the construction of small graphs is launch-bound).
 * Every rank receives the whole hierarchy, identical to coarsen_hierarchy.
 * partition_min_nnz <= 0 partitions every level. */
HEC_API int coarsen_hierarchy_dist(hec_ctx *ctx, const hec_graph *g0, int64_t cutoff, uint64_t seed,
                                   int64_t discard_below, int max_levels, const hec_comm *comm,
                                   int64_t partition_min_nnz, hec_hierarchy **out);

/* ------------------------------------------- multi-GPU building blocks (§8(e)) */
/* The partitioned hierarchy level (one process per GPU; the collectives are the
 * caller's, e.g. torch.distributed over NCCL):
 *   1. hec_heavy_range on the rank's fine-vertex slice, all-gather H;
 *   2. hec_mapping_from_heavy (rounds + relabel are replicated, cheap, vertex-
 *      only), M written for the rank's slice, all-gather M;
 *   3. hec_balance_rows: every rank derives the same coarse-row ranges;
 *   4. hec_build_rows_count on the rank's coarse rows, all-gather the counts;
 *   5. hec_build_rows_write at the slice's global entry offset.
 * Every result is identical to the single-GPU calls (bit-exact). */

/* H[u] for u in [u_begin, u_end) only (same definition as hec_debug_heavy);
 * H is a device int32[n] array indexed by global vertex id. */
HEC_API int hec_heavy_range(hec_ctx *ctx, const hec_graph *g, int64_t u_begin, int64_t u_end,
                            int32_t *H);
/* Mapping from a complete heavy-neighbour array H (device int32[n]): the
 * resolution rounds and the relabel run over all vertices; M (device int32[n])
 * is written for [u_begin, u_end) only.  *n_c (host) as hec_find_mapping. */
HEC_API int hec_mapping_from_heavy(hec_ctx *ctx, const hec_graph *g, const int32_t *H,
                                   uint64_t seed, int level, int64_t u_begin, int64_t u_end,
                                   int32_t *M, int64_t *n_c);
/* Split the coarse rows into `parts` contiguous ranges of about equal member-
 * edge volume (sum of fine degrees of the members): host bounds[parts+1],
 * bounds[0] = 0, bounds[parts] = n_c. */
HEC_API int hec_balance_rows(hec_ctx *ctx, const hec_graph *g, const int32_t *M, int64_t n_c,
                             int parts, int64_t *bounds);
/* Build coarse rows [a_begin, a_end) of G_c (the same rows build_coarse_graph
 * produces).  counts (device int64[a_end-a_begin], may be NULL) receives the
 * row lengths, *nnz_slice (host) their sum.  The slice is kept in ctx until
 * hec_build_rows_write (no other libhec call on ctx in between). */
HEC_API int hec_build_rows_count(hec_ctx *ctx, const hec_graph *g, const int32_t *M, int64_t n_c,
                                 int64_t a_begin, int64_t a_end, int64_t *counts,
                                 int64_t *nnz_slice);
/* Write the pending slice: row_ptr_c[0..rows] = offset + local offsets (device
 * int64[rows+1]), col_c/wgt_c[0..nnz_slice) and vwgt_c[0..rows) (device int32);
 * pass pointers already advanced to the slice's global position. */
HEC_API int hec_build_rows_write(hec_ctx *ctx, int64_t offset, int64_t *row_ptr_c, int32_t *col_c,
                                 int32_t *wgt_c, int32_t *vwgt_c);

#ifdef __cplusplus
}
#endif
#endif /* HEC_H */
