/*
 * dts.h -- C ABI of libdts.so, a B200-native (sm_100a) distance threshold
 * search over 4-D (t, x, y, z) trajectory line segments.
 *
 * Operation (Gowanlock & Casanova, §III "Problem statement"):
 * given an entry database D of line segments, a query set Q of line segments
 * and a distance d, return every triple (q, l, [t_start, t_end]) such that query
 * segment q and entry segment l are within Euclidean distance d of each other
 * in (x, y, z) during the closed time interval [t_start, t_end].  The index
 * (temporal bins, §IV-B.1, and a flattened spatial grid, §IV-A.1)
 * only prunes candidates; every result is decided by the refinement
 * compare() of Alg. 1 l.14, whose reading is fixed in DESIGN.md
 * §"Readings" (strict temporal overlap, closed distance inequality, linear
 * interpolation along each segment, fp64 arithmetic).
 *
 * Conventions shared by every entry point:
 *  - Segments are 64-byte records in the order of dts_segment below, stored
 *    contiguously (array of structs, row i = segment id i).  The id reported
 *    for a segment is its position in the array passed (reading c6).
 *  - Results are sorted by (query_id, entry_id), contain no duplicates, and
 *    are byte-identical across reruns and independent of dts_index_params
 *    (reading c7).
 *  - Functions returning dts_status never throw and never abort; on error
 *    every output pointer is set to NULL / 0, nothing is leaked, and
 *    dts_last_error() returns a message (thread-local, valid until the next
 *    call on the same thread).
 *  - "device" arguments are CUDA device pointers on the index's device;
 *    "host" arguments are ordinary (pageable or pinned) host pointers.
 *  - cuda_stream is a cudaStream_t (NULL = the legacy default stream).  All
 *    entry points are synchronous with respect to the host on return.
 */
#ifndef DTS_H
#define DTS_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
    DTS_OK = 0,
    DTS_EINVAL = -1,      /* invalid argument or invalid segment data            */
    DTS_ENOMEM = -2,      /* device or pinned host allocation failed             */
    DTS_ECUDA = -3,       /* CUDA runtime error (message in dts_last_error)      */
    DTS_ENOTSUP = -4,     /* no sm_100 device / unsupported configuration        */
    DTS_EINTERNAL = -5    /* internal invariant violated (a bug)                 */
} dts_status;

/* One trajectory line segment: spatiotemporal start and end point. */
typedef struct {
    double t_start, x_start, y_start, z_start;
    double t_end, x_end, y_end, z_end;
} dts_segment;

/* One result triple (q, l, [t_start, t_end]) of P:L32; 24 bytes.
 * t_start <= t_end, both absolute times inside the two segments' common
 * temporal extent.  A tangency at exactly d gives t_start == t_end. */
typedef struct {
    uint32_t query_id;    /* position in Q as passed, plus query_id_base */
    uint32_t entry_id;    /* position in D as passed                     */
    double t_start;
    double t_end;
} dts_result;

/* Candidate generator of an index.  All three return the same results; they
 * differ only in which candidates are refined. */
typedef enum {
    DTS_METHOD_GRID = 0,        /* temporal bins x flattened spatial grid, each entry
                                   filed once by its MBB midpoint (default)           */
    DTS_METHOD_TEMPORAL = 1,    /* GPUTemporal (P:L72-P:L80): every entry of the bins
                                   overlapping the query, the range E_k              */
    DTS_METHOD_SUBBIN = 2       /* GPUSpatioTemporal (P:L82-P:L120): per-dimension
                                   spatial subbins of each temporal bin, id arrays
                                   X, Y, Z in (subbin, bin) order, the dimension with
                                   the fewest entries chosen per query, temporal
                                   fallback when the query spans several subbins in
                                   every dimension                                    */
} dts_method;

/* Index construction parameters; zero means "choose automatically". */
typedef struct {
    int      device;            /* CUDA ordinal                                        */
    uint32_t temporal_bins;     /* m of P:L76; 0 = bin width = max segment duration    */
    uint32_t cells_per_dim;     /* grid resolution cap per axis; 0 = from extents     */
    double   d_hint;            /* typical search distance, sizes grid cells; 0 = none */
    uint64_t mem_budget_bytes;  /* device bytes the index may use (0 = no limit).  When
                                   dts_build_index's estimate for D (~310 B per entry)
                                   exceeds it, D is split by t_start into temporal
                                   shards kept in pinned host memory, each indexed on
                                   the device in turn at search time; results are the
                                   same.  Ignored by
                                   dts_build_index_device (D is already resident).   */
    uint32_t method;            /* dts_method                                          */
    uint32_t subbins;           /* v of P:L87 per dimension (SUBBIN); 0 = 16, always
                                   capped so a subbin is wider than the largest
                                   entry extent in that dimension             */
    const uint32_t* entry_ids;  /* optional: id reported for row i of D (a shard of a
                                   larger database reports global ids); host memory
                                   for dts_build_index, device memory for
                                   dts_build_index_device; NULL = i                   */
    const uint32_t* entry_traj; /* optional: trajectory id of row i of D ("a
                                   segment id and a trajectory id"), needed by
                                   exclude_same_trajectory; same memory kind as D     */
} dts_index_params;

/* Options of the *_ex searches (pointer fields: host memory for dts_search_ex,
 * device memory for dts_search_device_ex; all may be NULL / 0). */
typedef struct {
    uint32_t query_id_base;     /* added to row indices when query_ids is NULL        */
    const uint32_t* query_ids;  /* reported id of row i of Q (increasing)             */
    const uint32_t* query_traj; /* trajectory id of row i of Q                        */
    uint32_t exclude_same_trajectory;  /* nonzero: drop pairs whose query and entry
                                   trajectory ids are equal -- "any OTHER stellar
                                   trajectory" of the application; needs
                                   query_traj and an index built with entry_traj     */
} dts_search_options;

/* One trajectory-level result (the stars within d of another star and
 * the time intervals in which this happens): the union of the segment-level
 * intervals of one (query trajectory, entry trajectory) pair, split into its
 * maximal connected pieces. */
typedef struct {
    uint32_t query_traj;
    uint32_t entry_traj;
    double t_start;
    double t_end;
} dts_traj_result;

/* Per-search statistics (optional output of the *_ex entry points). */
typedef struct {
    uint64_t candidates;        /* candidate (query, entry) pairs refined per pass      */
    uint64_t cell_lookups;      /* (bin, cell) probes issued per pass                   */
    uint64_t results;           /* results returned                                     */
    uint32_t max_results_per_query;
    uint32_t time_kernels;      /* in: 1 = record CUDA-event phase times below and read
                                   them before returning; 2 = record them only (read
                                   later by dts_search_read_times, so that the call
                                   returns as soon as its results are ready); 3 = as 2,
                                   pass 1 (ms_count) only: two events instead of six */
    float    ms_prep;           /* query keys + sort                                    */
    float    ms_count;          /* pass 1 (fused candidate streaming + refine, count)   */
    float    ms_scan;           /* exclusive scan of per-query counts                   */
    float    ms_scatter;        /* pass 2 (fused streaming + refine, scatter)           */
    float    ms_canon;          /* per-query sort by entry id                           */
    uint32_t timer_slot;        /* out (time_kernels == 2): the call's event set        */
    uint32_t tile_queries;      /* out: queries per warp tile of pass 1                 */
    float    work_estimate;     /* out: expected candidates per query (grid method)     */
} dts_search_stats;

/* The phase times of a search made with time_kernels == 2: fills ms_* of
 * *stats from the event set named by stats->timer_slot (waits for those
 * events).  Event sets live per calling thread and device, 1024 of them
 * recycled in call order: call from the searching thread, with its device
 * current, within 1024 timed searches.  DTS_EINVAL for a recycled or unknown
 * slot. */
dts_status dts_search_read_times(dts_search_stats* stats);

typedef struct dts_index dts_index;   /* opaque; owns the device copy of D + index */

/* Build the index over n host segments D (copied; caller keeps ownership).
 * n == 0 builds an empty index.  Errors: DTS_EINVAL for NULL D with n > 0,
 * n >= 2^32, non-finite coordinates or times, t_end < t_start, or a segment
 * whose speed overflows fp64; DTS_ENOMEM; DTS_ECUDA; DTS_ENOTSUP. */
dts_status dts_build_index(const dts_segment* D, size_t n,
                           const dts_index_params* params,      /* NULL = defaults */
                           dts_index** out_index);

/* Same, from device memory: D_dev points to n dts_segment records in device
 * memory of params->device, 16-byte aligned.  Validation errors are returned
 * synchronously; the last build kernels may still run on cuda_stream when
 * the call returns (stream-ordered, like a kernel launch), so D_dev and the
 * params' device arrays must stay valid until the stream reaches that point
 * (later work on the stream, or dts_index_get_info, which waits for it).
 * Searches on other streams wait for the build by themselves, after their
 * query preparation (which needs only the grid chosen at build time), so that
 * preparation overlaps the build's tail. Not retained. */
dts_status dts_build_index_device(const dts_segment* D_dev, size_t n,
                                  const dts_index_params* params,
                                  void* cuda_stream, dts_index** out_index);

/* Search nq host query segments Q (copied) at distance d >= 0 (finite).
 * On success *out_results is library-allocated pinned host memory holding
 * *out_count results (NULL / 0 when there are none); release it with
 * dts_free_results.  query_id_base is added to every reported query id
 * (callers that shard Q).  Errors: DTS_EINVAL (NULL with nq > 0, nq >= 2^32,
 * bad d, invalid query segments, query_id_base + nq > 2^32), DTS_ENOMEM,
 * DTS_ECUDA. */
dts_status dts_search(const dts_index* index,
                      const dts_segment* Q, size_t nq, double d,
                      uint32_t query_id_base, void* cuda_stream,
                      dts_result** out_results, size_t* out_count);

/* dts_search with options (host pointers in opts, may be NULL) and stats. */
dts_status dts_search_ex(const dts_index* index,
                         const dts_segment* Q, size_t nq, double d,
                         const dts_search_options* opts, void* cuda_stream,
                         dts_result** out_results, size_t* out_count,
                         dts_search_stats* stats);                /* may be NULL */

/* Device-resident search: Q_dev holds nq segments in device memory
 * (16-byte aligned); results are returned in library-owned device memory
 * (*out_results_dev, NULL when empty), freed with dts_free_results_device. */
dts_status dts_search_device(const dts_index* index,
                             const dts_segment* Q_dev, size_t nq, double d,
                             uint32_t query_id_base, void* cuda_stream,
                             dts_result** out_results_dev, size_t* out_count,
                             dts_search_stats* stats);            /* may be NULL */

/* dts_search_device with options (device pointers in opts, may be NULL).
 * With opts->query_ids the id reported for row i of Q_dev is query_ids[i];
 * they must be increasing for the output to stay in canonical order (e.g. the
 * rows of a larger query set routed to one shard of D). */
dts_status dts_search_device_ex(const dts_index* index,
                                const dts_segment* Q_dev, size_t nq, double d,
                                const dts_search_options* opts, void* cuda_stream,
                                dts_result** out_results_dev, size_t* out_count,
                                dts_search_stats* stats);         /* may be NULL */

/* Count-only search (P:L32's result set, counted, not materialised): the
 * number of results of every query of Q (host, copied) at distance d, with
 * the same options as dts_search_ex (query_ids / query_id_base do not
 * matter for counting).  counts: host array of nq uint32 (may be NULL);
 * *total: the sum.  Runs the candidate generation and fp64 refinement of the
 * search without keeping any hit, so it works for
 * any result size (S2 at d = 5: 7.5e9 results, the paper's largest).
 * Errors as dts_search_ex.  Synchronous. */
dts_status dts_search_count(const dts_index* index, const dts_segment* Q, size_t nq, double d,
                            const dts_search_options* opts, void* cuda_stream,
                            uint32_t* counts, uint64_t* total, dts_search_stats* stats);

/* dts_search_count on device Q (16-byte aligned); counts_dev: device array of
 * nq uint32 (may be NULL); option pointers in device memory. */
dts_status dts_search_count_device(const dts_index* index, const dts_segment* Q_dev, size_t nq,
                                   double d, const dts_search_options* opts, void* cuda_stream,
                                   uint32_t* counts_dev, uint64_t* total,
                                   dts_search_stats* stats);

/* Receives one chunk of results (library-owned pinned memory, valid only
 * during the call); return 0 to continue, nonzero to stop the search. */
typedef int (*dts_result_callback)(const dts_result* results, size_t count, void* user);

/* Streamed search of host Q for result sets larger than device or host
 * memory -- the paper processes Q incrementally when its result buffer
 * fills: a count pass, then contiguous query-id chunks of
 * at most chunk_results results (0 = auto, from free device memory; a single
 * query with more results is one chunk) are searched and handed to callback
 * in canonical (query_id, entry_id) order, so the concatenation of all
 * chunks is exactly dts_search_ex's output.  Options as dts_search_ex (host
 * pointers).  stats->results = results delivered.  Errors as dts_search_ex;
 * DTS_EINVAL for a NULL callback.  Synchronous; the callback runs on the
 * calling thread. */
dts_status dts_search_stream(const dts_index* index, const dts_segment* Q, size_t nq, double d,
                             const dts_search_options* opts, uint64_t chunk_results,
                             dts_result_callback callback, void* user, void* cuda_stream,
                             dts_search_stats* stats);

/* Trajectory-level results from segment-level ones, all in device memory:
 * every result (q, l, [t_s, t_e]) is mapped to (query_traj[q], entry_traj[l])
 * (query_traj indexed by reported query id, n_query_ids entries; entry_traj by
 * entry id, n_entry_ids entries); the intervals of each trajectory pair are
 * merged into their union's maximal connected pieces (closed intervals that
 * touch merge).  Output sorted by (query_traj, entry_traj, t_start) in
 * library-owned device memory (dts_free_results_device). */
dts_status dts_merge_trajectories_device(const dts_result* results_dev, size_t n,
                                         const uint32_t* query_traj, size_t n_query_ids,
                                         const uint32_t* entry_traj, size_t n_entry_ids,
                                         void* cuda_stream,
                                         dts_traj_result** out_dev, size_t* out_count);

/* Per-query candidate counts ("per-query candidate count
 * estimate (for balancing)"; the partitioned search of P:L17 / P:L34 over
 * independent queries).  For every query of Q_dev (nq segments in
 * device memory of the index's device, 16-byte aligned) the candidate
 * generation of the search (bins, stencil cells, row probes of the index) is
 * run and the lengths of its candidate runs are summed: exactly the
 * (query, entry) pairs dts_search at distance d would refine for it (the
 * `candidates` statistic, per query).  No candidate record is read.
 * costs_dev (device memory, ceil(nq / block) uint64, written, not
 * accumulated) receives the sums over blocks of `block` consecutive queries
 * (block = 1: per query).  A caller sharding Q over ranks splits the prefix
 * sum of these costs evenly (dist.py).  Invalid query segments count 0 (the
 * search reports them).  Errors: DTS_EINVAL (NULL with nq > 0, block == 0,
 * bad d, nq >= 2^32, misaligned Q_dev), DTS_ECUDA.  Synchronous on return. */
dts_status dts_query_costs_device(const dts_index* index, const dts_segment* Q_dev, size_t nq,
                                  double d, uint32_t block, void* cuda_stream,
                                  uint64_t* costs_dev);

/* The same estimate from every stride-th query (queries 0, stride, 2 stride
 * ...), each counted stride times: 1/stride of the work, for balancing a
 * shard split when the exact counts cost too much (stride = 1 is
 * dts_query_costs_device).  Measured on C4's 1/8 share (125 k queries):
 * exact 0.10 ms; DTS_EINVAL also for stride == 0. */
dts_status dts_query_costs_sampled_device(const dts_index* index, const dts_segment* Q_dev,
                                          size_t nq, double d, uint32_t block, uint32_t stride,
                                          void* cuda_stream, uint64_t* costs_dev);

/* Sort n results in device memory into canonical (query_id, entry_id) order,
 * in place (e.g. after concatenating the outputs of shards of D). */
dts_status dts_canonicalize_device(dts_result* results_dev, size_t n, void* cuda_stream);

void dts_free_results(dts_result* results);          /* NULL is a no-op */
void dts_free_results_device(void* results);         /* NULL is a no-op; also for dts_traj_result */
void dts_free_index(dts_index* index);               /* NULL is a no-op */

/* Introspection of a built index (for tests and benchmarks). */
typedef struct {
    uint64_t n;                 /* entries                                   */
    uint64_t cells;             /* non-empty (bin, cell) keys                */
    uint32_t bins;              /* m                                         */
    uint32_t grid[3];           /* cells per axis                            */
    double   bin_width;         /* b of P:L76                                */
    double   cell_width[3];
    double   max_extent[3];     /* max |x_end - x_start| etc.        */
    double   max_duration;
    float    ms_build;          /* device time of the last build (CUDA events) */
    uint32_t method;            /* dts_method of the index                   */
    uint32_t subbins[3];        /* v per dimension (SUBBIN), else 0          */
    uint64_t subbin_ids[3];     /* length of the X, Y, Z id arrays (SUBBIN)  */
    float    ms_phase[5];       /* device time of the last build's phases (CUDA
                                   events on the build stream): bounds, keys,
                                   radix sort, gather (+ bins, cell count),
                                   hash insert                               */
    uint32_t build_flags;       /* bit 0: grid from a strided sample of D and
                                   one fused read of D for exact bounds, keys
                                   and sort histograms (phase "bounds" is then
                                   the sample, "keys" the fused pass)        */
    uint32_t hash_kind;         /* cell table: 1 = one 32-byte slot per block
                                   of 8 consecutive cell keys (the only kind) */
    uint64_t hash_items;        /* slots in use (blocks)                     */
    uint64_t hash_bytes;        /* table size in bytes                       */
    uint32_t shards;            /* temporal shards on the host (mem_budget_bytes
                                   exceeded), 0 for an index resident on the device */
    uint64_t outlier_rows;      /* entries filed as copies along their path (extent
                                   or duration above 8x the mean; grid method) */
    uint64_t outlier_copies;    /* their copies (n counts them)               */
} dts_index_info;

dts_status dts_index_get_info(const dts_index* index, dts_index_info* info);

/* Number of kernels this library has launched in the process so far. */
uint64_t dts_kernel_launches(void);

const char* dts_last_error(void);
const char* dts_version(void);

#ifdef __cplusplus
}
#endif
#endif /* DTS_H */
