/*
 * hdb.h -- C-ABI of the B200-native HYBRID-DBSCAN hot path.
 *
 * Gowanlock, Rude, Blair, Li, Pankratius, "Clustering Throughput Optimization
 * on the GPU", IPDPS Workshops 2017.  Citations "P:n" are line numbers of the
 * paper text (reference PAPER.md), with the section / algorithm they fall in.
 *
 * The four calls of the method (north star):
 *   (1) hdb_grid_build      -- build a grid of cell width eps over 2-D points
 *                              (Sec. IV, Fig. 1 P:376-437;
 *                              ConstructIndex, Alg. 4 line 5 P:665).
 *   (2) hdb_neighbor_table  -- the eps-neighbour table T for (points, eps)
 *                              (Sec. III; GPUCalcGlobal Alg. 2
 *                              P:463-489; batching Sec. VI P:677-823;
 *                              ConstructNeighborTable Alg. 4 line 8).
 *   (3) hdb_dbscan          -- DBSCAN(eps, minpts) on that table
 *                              (Alg. 1 P:196-249 with NeighborSearch replaced
 *                              by a lookup in T; Alg. 4 line 9).
 *   (4) hdb_sweep           -- re-cluster over a sweep of (eps, minpts)
 *                              reusing one table per eps (variants V, P:333-336;
 *                              reuse P:603-605; pipelining
 *                              P:1089-1097).
 *
 * Conventions (apply to every call):
 *  - Points are interleaved (x, y) rows of double (HDB_F64) or float
 *    (HDB_F32); point ids are 0-based input row indices, so n < 2^32 - 1.
 *  - Neighbour predicate (the paper gives none beyond dist <= eps, P:147-148;
 *    DESIGN.md reading R1/R2): q in N_eps(p) <=> fl(fl(dx*dx) + fl(dy*dy))
 *    <= fl(eps*eps), dx = fl(x_p - x_q), dy = fl(y_p - y_q), IEEE
 *    round-to-nearest-even in the input precision, no FMA.  eps is converted
 *    once to the input precision.  Every list contains the point itself.
 *  - Status: every call returns hdb_status (0 == HDB_OK).  On failure *out
 *    (where present) is set to NULL, no partial output is published, and
 *    hdb_last_error() returns a thread-local message.
 *  - Ownership: the caller owns all inputs; the library copies what it needs
 *    and keeps no caller pointer after return.  Grids and tables are library
 *    owned and released only by their *_free call; views are borrowed and
 *    valid until that free.  Output arrays (labels, ...) are caller allocated.
 *  - Threading: calls on one hdb_ctx are serialised internally; hdb_dbscan
 *    on a (const, immutable) table is re-entrant, so several minpts variants
 *    may run concurrently on one table.
 *  - n == 0 is valid and yields empty outputs.
 */
#ifndef HDB_H
#define HDB_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
    HDB_OK = 0,
    HDB_EINVAL = -1,    /* NULL pointer with n > 0, non-finite coordinate, eps not finite or <= 0,
                           minpts == 0, unknown dtype, table not host-resident where required   */
    HDB_ERANGE = -2,    /* n >= 2^32-1, extent/eps > 2^30, or grid cell count over the limit      */
    HDB_ENOMEM = -3,    /* device/host allocation failed, or 4*P bytes exceed host_budget_bytes
                           (detected from the exact count, before any pair is written)            */
    HDB_ECUDA = -4,     /* CUDA runtime failure (message in hdb_last_error)                       */
    HDB_EINTERNAL = -5  /* internal invariant violated                                            */
} hdb_status;

typedef enum { HDB_F64 = 0, HDB_F32 = 1 } hdb_dtype;

typedef struct hdb_ctx hdb_ctx;     /* devices, streams, device + pinned memory pools (opaque) */
typedef struct hdb_grid hdb_grid;   /* device-resident sorted points + eps-grid (opaque)       */
typedef struct hdb_table hdb_table; /* eps-neighbour table T, host- or device-resident (opaque) */

/* Options.  Always initialise with hdb_opts_default() and then override. */
typedef struct {
    const int* devices;         /* CUDA device ordinals; NULL / n_devices == 0 => current device. Queries
                                   are sharded across them; the table is one host table. */
    int n_devices;
    double sample_fraction;     /* f of the result-size estimator, default 0.01            */
    double alpha;               /* over-estimation factor, default 0.05             */
    int n_streams;              /* D2H streams, default 3                                  */
    uint64_t batch_pairs;       /* b_b override in pairs; 0 = the paper's buffer rule      */
    int sort_lists;             /* 1 => every neighbour list ascending (canonical)                     */
    uint64_t host_budget_bytes; /* 0 = unlimited; else HDB_ENOMEM when 4*P exceeds it                  */
    int shard_rank;             /* process-level query sharding (torchrun mode): this process          */
    int shard_count;            /*   computes shard shard_rank of shard_count; 0 => unsharded          */
    int search_kernel;          /* 0 = default: dense device-resident whole tables take the single
                                   pass (count + reserve + write in one kernel) when the grid's
                                   candidate tests per query or the sampled pairs per query say
                                   dense, everything else the count -> scan -> write passes;
                                   other values select kernel variants:
                                   1 = exact-f64-only tests, 2 = write pass recomputes the tests,
                                   3 = no dense/sparse split, 4 = single-pass device table
                                   (sampled-estimate capacity), 7 / 8 = the paper's GPUCalcGlobal
                                   (Alg. 2) / GPUCalcShared (Alg. 3) with an atomic key/value result
                                   set sorted by key (device-resident whole tables; the Table II
                                   baseline)                                               */
    int host_threads;           /* threads for host-side work (T assembly, DBSCAN); 0 = all cores      */
    int cell_split;             /* k >= 1: grid cells of width eps/k, (2k+1)^2-cell stencil (fewer
                                   candidate tests on dense data); 0 = auto (k from a sampled cell
                                   occupancy); 1 = the paper's eps cells;
                                   k <= 6 (HDB_EINVAL above)                                         */
    int sweep_on_device;        /* hdb_sweep only: 0 = the paper's hybrid split (tables D2H, host
                                   DBSCAN pipelined with the next table's build);
                                   1 = tables stay in HBM and DBSCAN runs on the GPU (NEXT-4);
                                   labels are identical either way                                    */
} hdb_opts;

/* Borrowed view of a table T (T_i^min/T_i^max ranges into B).
 * For original point id p: its list is nbrs[begin[p] .. begin[p] + count[p]).
 * Lists are in the order the search produced them unless sort_lists was set
 * or hdb_table_canonicalize was called (then ascending ids, rows in id order). */
typedef struct {
    uint64_t n;                 /* number of points                                          */
    uint64_t npairs;            /* P = sum of |N_eps(p)| (self pairs included)               */
    const uint64_t* begin;      /* [n]  by original id                                       */
    const uint32_t* count;      /* [n]  |N_eps(p)|                                           */
    const uint32_t* nbrs;       /* [npairs] original ids (the paper's value buffer B)        */
    int on_device;              /* 0: host pointers; 1: device pointers on `device`          */
    int device;
    uint64_t first_query;       /* sharded tables: rows [first_query, end_query) of the      */
    uint64_t end_query;         /*   cell-sorted query order are present; else 0, n          */
    double eps;
    hdb_dtype dtype;
} hdb_table_view;

/* Borrowed view of a grid (Fig. 1, re-laid out: A is the sorted
 * position -> original id map; G keeps only the NON-EMPTY cells, as ascending
 * keys h = cy*nx + cx with half-open start offsets into A).
 * All pointers are DEVICE pointers on `device`. */
typedef struct {
    uint64_t n;
    double eps;
    hdb_dtype dtype;
    double xmin, ymin, xmax, ymax;   /* bounding box of the data (reading R10)               */
    double cell_w;                   /* w = eps_F * (1 + 2^-19) (reading R9)                  */
    uint32_t nx, ny;                 /* cells per axis; cell key h = cy * nx + cx             */
    uint64_t n_cells;                /* nx * ny (cells of the full grid, most may be empty)   */
    uint64_t n_nonempty;             /* non-empty cells (Table II's block count)   */
    uint64_t n_groups;               /* query groups (<= 32 queries of one cell)              */
    int device;
    const void* xy_sorted;           /* [n] double2 / float2 in cell order                    */
    const uint32_t* ids;             /* [n] A: sorted position -> original id                 */
    const uint64_t* cell_keys;       /* [n_nonempty] key h of each non-empty cell, ascending  */
    const uint32_t* cell_start;      /* [n_nonempty + 1] G: non-empty cell c holds the sorted
                                        positions [cell_start[c], cell_start[c+1])            */
} hdb_grid_view;

/* Per-call statistics of the last hdb_neighbor_table* / hdb_grid_build on a context. */
typedef struct {
    uint64_t n, npairs, n_cells, n_nonempty, n_groups;
    uint64_t sample_size;        /* |sample| of the estimator                          */
    uint64_t sample_pairs;       /* e_b                                                            */
    uint64_t est_pairs;          /* a_b = e_b / f                                                  */
    uint64_t planned_batch_pairs;/* b_b from the buffer rule or batch_pairs            */
    uint64_t planned_batches;    /* n_b from Eq. 1                                     */
    uint64_t n_batches;          /* batches actually run (cut on exact counts)                     */
    uint64_t max_batch_pairs;
    uint64_t candidate_tests;    /* distance tests performed by one search pass                    */
    uint64_t bytes_h2d, bytes_d2h;
    uint64_t pool_grows;         /* pinned / device buffer growths beyond the estimate             */
    int n_streams, n_devices;
    uint32_t kernel_launches;    /* kernels launched by the last call                              */
    uint32_t write_launches;     /* launches of the neighbour write kernel                         */
    double ms_grid;              /* device time of the grid build (CUDA events)                    */
    double ms_sample, ms_count, ms_scan;
    double ms_write_kernel;      /* summed device time of the write-kernel launches (CUDA events)  */
    double ms_table_wall;        /* host wall time of the whole table call                         */
    int single_pass;             /* 1: the last device-resident table was built in one pass (count +
                                    reserve + emit per query group, rows in reservation order);
                                    ms_write_kernel is that kernel's time, ms_count = ms_scan = 0    */
    double ms_sort;              /* search_kernel 7 / 8 (the paper's kernels): device time of the sort
                                    of the key/value result set by key + the T ranges (Alg. 4 line 7-8);
                                    ms_write_kernel is then the search kernel's time                   */
    uint64_t n_sparse_queries;   /* queries of the grid's sparse groups, handled thread-per-query (the
                                    dense/sparse hybrid); 0 = none       */
    int query_lanes;             /* 1: those are the SMALL groups' queries, taken one per lane by the
                                    query-lane single pass (k_qlanes; the
                                    default for point sets beyond the L2, HDB_QLANES=0/1 forces it) */
} hdb_stats;

/* ---- context ------------------------------------------------------------- */
void        hdb_opts_default(hdb_opts* opts);
hdb_status  hdb_ctx_create(const hdb_opts* opts /* NULL = defaults */, hdb_ctx** out);
void        hdb_ctx_destroy(hdb_ctx* ctx);   /* all grids/tables of ctx must be freed first */
/* Enqueue the grid build and device-resident table work of the FIRST device
 * on `cuda_stream` (a cudaStream_t; NULL = the context's own stream). */
hdb_status  hdb_ctx_set_stream(hdb_ctx* ctx, void* cuda_stream);
hdb_status  hdb_stats_get(const hdb_ctx* ctx, hdb_stats* out);

/* ---- (1) grid ---------------------------------------------------------- */
/* xy: n interleaved rows, host or device memory (detected); dtype selects the
 * precision.  Builds on every device of ctx (each holds the full point set
 * and its grid). */
hdb_status  hdb_grid_build(hdb_ctx* ctx, const void* xy, uint64_t n, hdb_dtype dtype,
                           double eps, hdb_grid** out);
void        hdb_grid_free(hdb_grid* grid);
hdb_status  hdb_grid_view_get(const hdb_grid* grid, hdb_grid_view* out);   /* first device */
/* Copy the first device's grid arrays to caller buffers (any may be NULL):
 * ids[n] (A), cell_keys[n_nonempty], cell_start[n_nonempty+1] (G),
 * xy_sorted[2n] of the grid's dtype. */
hdb_status  hdb_grid_copy_to_host(const hdb_grid* grid, uint32_t* ids, uint64_t* cell_keys, uint32_t* cell_start,
                                  void* xy_sorted);

/* ---- (2) neighbour table ----------------------------------------------- */
/* Host-resident T: count -> scan -> batched write kernels on n_streams streams,
 * each batch DMA'd straight into the host table (pinned pool of ctx). */
hdb_status  hdb_neighbor_table(hdb_ctx* ctx, const hdb_grid* grid, hdb_table** out);
/* Device-resident T (first device, or this process's shard): no D2H.  begin /
 * count are by original id as for host tables; the rows' placement in nbrs is
 * the production order -- cell-sorted for the count -> scan -> write passes,
 * reservation order for the single pass that dense whole tables take with
 * search_kernel 0 -- so begin[] is not monotone in id.
 * Dense whole tables are sized by the grid's candidate tests (an upper bound on
 * the pairs; HDB_ENOMEM only if that bound cannot be allocated and the exact
 * two-pass path cannot either). */
hdb_status  hdb_neighbor_table_device(hdb_ctx* ctx, const hdb_grid* grid, hdb_table** out);
/* Wrap a copy of a host CSR as a table (for reuse / tests): begin/count by id. */
hdb_status  hdb_table_from_host(uint64_t n, const uint64_t* begin, const uint32_t* count,
                                const uint32_t* nbrs, uint64_t npairs, hdb_table** out);
hdb_status  hdb_table_view_get(const hdb_table* table, hdb_table_view* out);
/* Copy a host- or device-resident table into caller buffers (any may be NULL):
 * begin[n], count[n], nbrs[npairs] -- same layout as the view. */
hdb_status  hdb_table_copy_to_host(const hdb_table* table, uint64_t* begin, uint32_t* count, uint32_t* nbrs);
/* Host tables only: rows in id order (begin[p] = sum of earlier counts) and
 * each list ascending. */
hdb_status  hdb_table_canonicalize(hdb_table* table);
void        hdb_table_free(hdb_table* table);

/* ---- (3) DBSCAN on a host table ------------------------------------------ */
/* core(p) <=> count[p] >= minpts (count includes p); clusters are
 * the components of the core-core eps-graph numbered 0.. by increasing
 * minimum core id; a non-core point with a core neighbour (border) takes the
 * cluster of smallest number among its core neighbours' clusters; others are
 * noise (-1).  This is exactly Alg. 1 run over p = 0..n-1 (R4-R7).
 * labels[n] required; is_core[n] and n_clusters optional (NULL).
 * n_threads: 0 = the table's default (opts.host_threads of its ctx, else all
 * cores); 1 = sequential BFS; > 1 = parallel union-find (same labels). */
hdb_status  hdb_dbscan(const hdb_table* table, uint32_t minpts, int32_t* labels,
                       uint8_t* is_core, uint32_t* n_clusters);
hdb_status  hdb_dbscan_ex(const hdb_table* table, uint32_t minpts, int n_threads,
                          int32_t* labels, uint8_t* is_core, uint32_t* n_clusters);

/* ---- (4) sweep ----------------------------------------------------------- */
/* For each eps[i] (one grid + one table, built while the host clusters the
 * previous table) and each minpts[j] (concurrent):
 * labels[(i * n_minpts + j) * n + p], n_clusters[i * n_minpts + j].
 * xy: host or device memory (as hdb_grid_build).  labels: caller-allocated,
 * host memory, or -- with opts.sweep_on_device = 1 -- host or device memory
 * (HDB_EINVAL otherwise); n_clusters: host memory or NULL.  With
 * sweep_on_device = 1 each table stays in HBM and DBSCAN runs on the GPU
 * (NEXT-4); the labels are identical to the hybrid path's. */
hdb_status  hdb_sweep(hdb_ctx* ctx, const void* xy, uint64_t n, hdb_dtype dtype,
                      const double* eps, uint32_t n_eps, const uint32_t* minpts, uint32_t n_minpts,
                      int32_t* labels, uint32_t* n_clusters);

/* ---- host-side planning helpers (Sec. VI), exposed for tests ------------- */
/* Buffer rule and Eq. 1: given the total estimate
 * a_b, alpha and the stream count, returns b_b (pairs per stream buffer) and
 * n_b = ceil((1 + alpha) a_b / b_b). */
hdb_status  hdb_plan_batches(double est_pairs, double alpha, int n_streams,
                             double* b_b, uint64_t* n_b);
/* Fig. 2 strided assignment: the 0-based point index
 * processed by global thread gid of batch l (0-based) out of n_b batches. */
uint64_t    hdb_strided_point(uint64_t gid, uint64_t l, uint64_t n_b);
/* Split `n_items` weighted items into `parts` contiguous ranges of near-equal
 * weight; cuts[parts+1].  Used for batch cuts and query shards. */
hdb_status  hdb_balanced_cuts(const uint64_t* prefix /* [n_items+1] inclusive prefix of weights */,
                              uint64_t n_items, uint32_t parts, uint64_t* cuts);

const char* hdb_last_error(void);
const char* hdb_version(void);
/* Total kernels this process has launched through the library (monotone). */
uint64_t    hdb_kernel_launches(void);

#ifdef __cplusplus
}
#endif
#endif /* HDB_H */
