/*
 * sj.h -- C ABI of the B200-native eps-grid similarity self-join (libsj.so).
 *
 * Method: Gallet & Gowanlock, "Load Imbalance Mitigation Optimizations for
 * GPU-Accelerated Similarity Joins", IPDPSW 2019.  Citations are
 * PAPER.md line numbers ("P:L") plus the section / algorithm they fall in.
 *
 * The operation (§II-A): for a dataset D of n points in `dim` dimensions,
 * return every ordered pair (i, j), i != j, with dist(p_i, p_j) <= eps.  The
 * predicate is evaluated exactly as s(i,j) <= fl(eps*eps), where
 * s = fl(...fl(fl(t_0*t_0) + fl(t_1*t_1)) + ...), t_d = fl(p_i[d] - p_j[d]),
 * IEEE binary64 round-to-nearest, dimension order, no FMA (DESIGN.md readings
 * c1, c2).  Self pairs are excluded; exact duplicates i != j are pairs (c3).
 * Both (i, j) and (j, i) are returned (mirrored emission, c4).
 *
 * The hot path behind these calls: eps-grid index with a radix
 * sort of point->cell ids, per-cell workload,
 * SortByWL, an atomic WorkQueue over D', k threads per
 * query point with the LID-UNICOMP cell pattern (P:172-185,
 * Alg. 3), warp-shuffle cooperation and batched result emission with a
 * 1 % batch estimator.
 *
 * Threading: a handle is not thread-safe; distinct handles are independent.
 * Every call runs on the CUDA device that was current when the handle was
 * created.
 *
 * Stream ordering: the library runs on streams of its own.  Every call that reads or
 * writes caller memory (sj_create*, sj_self_join, sj_neighbor_csr, sj_export_index,
 * sj_create_from_index) first makes them wait for the work queued so far on the
 * caller's stream -- the legacy default stream, or the one named with sj_set_stream
 * -- so device inputs written asynchronously by the caller are complete before they
 * are read.  Completion: sj_self_join, sj_neighbor_csr, sj_export_index and
 * sj_create_from_index return after their GPU work ended.  sj_create / sj_create_ex /
 * sj_create_part return once the caller's points (and ids) are no longer read; the
 * build's last kernels may still run on the handle's stream, every later call on the
 * handle is ordered after them, and an asynchronous error of theirs surfaces at the
 * next call (SJ_SYNC_BUILD=1 in the environment makes the build fully synchronous).
 */
#ifndef SJ_H
#define SJ_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define SJ_ABI_VERSION 3

typedef struct sj_handle sj_handle;

/* Return codes. */
enum sj_status {
    SJ_OK = 0,       /* join complete; *count pairs written by this call            */
    SJ_MORE = 1,     /* out_pairs filled to cap; call sj_self_join again to continue */
    SJ_EINVAL = -1,  /* bad argument (NULL, dim, n, eps, non-finite coordinate, ...) */
    SJ_ENOMEM = -2,  /* device or pinned host allocation failed                     */
    SJ_ECUDA = -3,   /* CUDA runtime error (no device, launch failure, ...)         */
    SJ_EGRID = -4,   /* grid too large: some nc_d >= 2^30 or prod nc_d >= 2^64     */
    SJ_ESTATE = -5   /* handle is in the error state after an earlier failure       */
};

/* Options for sj_set_option (set them before the sj_self_join they should affect). */
enum sj_option {
    SJ_OPT_K = 1,              /* threads per query point k in {1,2,4,8,16,32}; default 8 */
    SJ_OPT_BATCH_PAIRS = 2,    /* b_s, pairs per batch buffer; default 1e8                        */
    SJ_OPT_STREAMS = 3,        /* CUDA streams for batches, 1..8; default 3                       */
    SJ_OPT_SAMPLE_PPM = 4,     /* estimator sample of D' in parts per million; default 10000 = 1%*/
    SJ_OPT_GRAB = 5,           /* WorkQueue chunks one warp dequeues per atomic (1..1024); default 4 for
                                  1-D..3-D (one same-address atomic per chunk congests its L2 slice,
                                  measured), 1 for 4-D+ (heavy chunks: balance at the queue's end)   */
    SJ_OPT_COUNT_CALCS = 6,    /* 1 = instrument the join with a distance-calculation counter; default 0 */
    SJ_OPT_BLOCKS_PER_SM = 7,  /* persistent-grid CTAs per SM; 0 = occupancy maximum (default)           */
    SJ_OPT_FAST_PATH = 8,      /* 1 = device output written in place when it fits (default); 0 = always
                                  stage per batch (the paper's scheme)                             */
    SJ_OPT_EXACT = 9,          /* 1 = exact two-pass sizing: a count pass records every
                                  WorkQueue chunk's pairs, their scan gives each chunk its output slots,
                                  batches are cut at exact sizes <= b_s and the fill pass writes each
                                  chunk at its own offset -- no estimator, no overflow retries, and the
                                  output ORDER is deterministic.  0 = the paper's 1% estimator (P:71,
                                  P:200) with atomic placement (default)                                 */
    SJ_OPT_QUEUE = 10,         /* 1 = WorkQueue: warps dequeue D' chunks with an atomic
                                  counter, batches are contiguous ranges of D', the estimator samples
                                  the first 1% of D' (default).  0 = SortByWL only
                                  (P:187-192): warp w statically takes chunks w, w + #warps, ... of D'
                                  (no atomics), staged batches are the strided D'_l = {chunk v :
                                  v mod nbBatches = l} (Fig. 1) and the estimator samples
                                  every (1/1%)-th chunk of the whole queue.  The pair set is
                                  the same either way                                                    */
    SJ_OPT_OUT_BLOCKS = 11     /* in-place output allocation: 0 = one atomic on the output counter per
                                  warp flush; 1 = blocks of 4096 pairs per warp (one atomic per block),
                                  the gaps the warps' last blocks leave closed by a compaction pass;
                                  2 = blocks when the caller's buffer holds >= 3e8 pairs (default): a
                                  single counter taking every flush of a large result congests its L2
                                  slice and doubles the join (measured)                  */
};

/* Cell access patterns (sj_create_ex).  The paper's variants, Table II:
 *   SJ_PATTERN_LID_UNICOMP -- neighbour cells with a higher linear id, mirrored emission
 *                             (Alg. 3); the default and the hot path;
 *   SJ_PATTERN_GCG         -- GPUCALCGLOBAL's full 3^n neighbourhood, one pair per
 *                             distance calculation (Alg. 1): twice the calculations;
 *   SJ_PATTERN_UNICOMP     -- the odd-coordinate pattern of [18] (Alg. 2), mirrored.
 * All three return the same pair set. */
enum sj_pattern { SJ_PATTERN_LID_UNICOMP = 0, SJ_PATTERN_GCG = 1, SJ_PATTERN_UNICOMP = 2 };

/* Order of the query queue D' (sj_create_ex):
 *   SJ_ORDER_WORKLOAD -- SortByWL: cells by non-increasing workload; default;
 *   SJ_ORDER_CELL     -- cells in linear-id order (no sort by workload);
 *   SJ_ORDER_INPUT    -- the input order of the points (the unsorted D of GPUCALCGLOBAL). */
enum sj_order { SJ_ORDER_WORKLOAD = 0, SJ_ORDER_CELL = 1, SJ_ORDER_INPUT = 2 };

/* Statistics of the handle (sj_get_stats).  Times are CUDA-event milliseconds. */
typedef struct sj_stats {
    uint64_t n;               /* points                                              */
    uint32_t dim;             /* dimensionality                                      */
    uint32_t key_bits;        /* significant bits of the linear cell id              */
    uint64_t n_cells;         /* M, non-empty cells (|B|)                      */
    uint64_t fwd_runs;        /* forward runs: per cell, the non-empty LID-UNICOMP
                                 neighbour cells of one grid row form one contiguous
                                 run of the lid-ordered points        */
    uint64_t dist_calcs;      /* D_alg: distance calculations of the LID-UNICOMP
                                 pattern, sum_A [C(m_A,2) + m_A * sum_fwd m_B]       */
    uint64_t calcs_measured;  /* instrumented counter of the last join (0 if off)    */
    uint64_t pairs;           /* ordered pairs of the last completed join            */
    uint64_t est_pairs;       /* batch estimator's estimate                  */
    uint32_t batches;         /* nbBatches of the last join                          */
    uint32_t retries;         /* overflow re-runs of the last join                   */
    uint32_t join_launches;   /* join kernel launches of the last join               */
    uint32_t k;               /* threads per query point used                        */
    uint64_t max_cell_load;   /* largest per-point workload W                */
    double ms_build;          /* sj_create: upload .. SortByWL (device span)         */
    double ms_estimate;       /* estimator kernel                                    */
    double ms_join;           /* join kernels: device span first start .. last end   */
    double ms_join_sum;       /* join kernels: sum of per-launch durations           */
    double ms_transfer;       /* copies of staged batches to the caller's buffer     */
    double ms_total;          /* last sj_self_join call, device span                 */
    uint32_t fast_path;       /* 1 if the last join wrote the caller's device buffer in place */
    uint32_t nc[8];           /* cells per dimension                                 */
    uint64_t n_chunks;        /* WorkQueue chunks of D'                              */
    uint32_t tiled_min;       /* smallest cell (points) that gets shared-memory tiles */
    uint32_t pattern;         /* enum sj_pattern of the index                        */
    uint32_t order;           /* enum sj_order of the index                          */
    uint32_t est_fused;       /* 1 if the estimator (a9) ran fused into the in-place join */
    uint32_t lookup_hash;     /* a6's lid -> cell lookup: 0 dense table over prod nc_d cells,
                                 1 open-addressing hash of the non-empty cells (sparse grids) */
} sj_stats;

/* Build the eps-grid index of `n` points of dimension `dim` (row-major AoS,
 * points[i*dim + d]) with threshold `eps`.
 *   points : host (pageable or pinned) or device pointer on the current device;
 *            read only during the call -- the library copies it (caller keeps ownership).
 *   n      : 1 <= n < 2^32.      dim : 1 <= dim <= 8 (the paper uses 2..6).
 *   eps    : finite, > 0.
 * Runs steps a1..a8 of DESIGN.md §1 (upload+validate, bounding box, cell
 * linearisation, radix sort, compaction, forward neighbours, workload, SortByWL).
 * Returns once the caller's points are no longer read (they may be freed or overwritten);
 * the build's last kernels may still be running on the handle's stream -- every other call
 * on the handle is ordered after them (set SJ_SYNC_BUILD=1 for a fully synchronous build).
 * Returns NULL on error (see sj_last_error): NaN/Inf coordinate or bad argument
 * (SJ_EINVAL), grid overflow (SJ_EGRID), allocation (SJ_ENOMEM), CUDA (SJ_ECUDA); an
 * asynchronous CUDA error of the build's last kernels surfaces at the next call instead. */
sj_handle *sj_create(const double *points, uint64_t n, int dim, double eps);

/* sj_create with an explicit cell pattern (enum sj_pattern) and queue order (enum sj_order),
 * for the paper's ablations (Tables III-V).  sj_create(...) == sj_create_ex(..., 0, 0).
 * SJ_EINVAL for an unknown pattern or order. */
sj_handle *sj_create_ex(const double *points, uint64_t n, int dim, double eps, int pattern, int order);

/* A spatial PARTITION of a larger self-join (data beyond one GPU's memory, or
 * several GPUs without replication).  The caller cuts the global grid (cell side
 * w = eps(1+2^-20), origin = the global per-dimension minimum) into slabs of whole cell columns
 * along dimension 0 and gives each partition
 *   points[0 .. n_query)  : its own points -- the QUERIES of this handle,
 *   points[n_query .. n)  : its halo -- the points of the FIRST cell column of the next slab,
 *                           candidates only (the LID-UNICOMP forward cells of a cell, P:174,
 *                           Alg. 3, never lie more than one column ahead in dimension 0);
 *   ids                   : the global id of every point (uint32[n], host or device), written
 *                           into the output instead of input positions; NULL = positions;
 *   origin                : host double[dim], the global grid origin (every coordinate must be
 *                           >= it, else SJ_EINVAL), so all partitions' cells align.
 * sj_self_join on the handle returns exactly the ordered pairs of the global join that this
 * partition's queries own (both directions): the partitions' results are disjoint and
 * their union is the global result.  Pattern LID-UNICOMP, order SortByWL.  A cell holding both
 * query and halo points (a cut through a cell column) is rejected with SJ_EINVAL.  NULL on error. */
sj_handle *sj_create_part(const double *points, const uint32_t *ids, uint64_t n, uint64_t n_query, int dim,
                          double eps, const double *origin);

/* Run (or continue) the self-join.
 *   out_pairs : caller-owned uint32[2*cap], interleaved (i, j) of 0-based input ids,
 *               host (pinned or pageable) or device memory; a device buffer must be
 *               16-byte aligned.  Order is unspecified; each unordered neighbour pair
 *               appears as (i, j) and (j, i); (i, i) never appears.
 *   cap       : capacity in pairs.
 *   count     : receives the number of pairs written by THIS call.
 * out_pairs == NULL && cap == 0 : count-only; *count = total pairs, nothing written.
 * Returns SJ_OK when the join is complete, SJ_MORE when cap was filled and pairs
 * remain (call again with the same or another buffer to receive the next ones).
 * A call after SJ_OK restarts the join; the pair SET is deterministic.
 * Errors: SJ_EINVAL (NULL count, out_pairs NULL with cap > 0, misaligned device
 * buffer), SJ_ECUDA, SJ_ENOMEM; after an error the handle answers SJ_ESTATE. */
int sj_self_join(sj_handle *h, uint32_t *out_pairs, uint64_t cap, uint64_t *count);

/* Device-resident CSR neighbour lists (the clustering consumers of a
 * self-join): row i holds the input ids j != i with s(i, j) <= fl(eps^2), i.e.
 * nbrs[row_off[i] .. row_off[i+1]) -- the same pair set as sj_self_join, grouped by i.
 * Needs a handle created with SJ_PATTERN_GCG (sj_create_ex): with the full 3^n
 * neighbourhood (Alg. 1) every query point evaluates all of its own candidates,
 * so it owns its row and the two passes (degrees -> exclusive scan -> fill) need no
 * atomics; and the whole queue (slice world 1).
 *   row_off : uint64[n+1] (host or device), or NULL; receives the exclusive scan of the
 *             degrees, row_off[n] = total.
 *   nbrs    : uint32[cap] (host or device), or NULL with cap == 0 (offsets only).
 *   total   : receives the number of ordered pairs (sum of the degrees).
 * Row contents follow the neighbourhood traversal order (deterministic, not sorted).
 * Returns SJ_OK; SJ_EINVAL for NULL total, a handle of another pattern or slice, a
 * join continuation in progress (SJ_MORE pending), or cap < total (row_off and *total
 * are filled first, nbrs untouched; the handle stays usable); SJ_ECUDA / SJ_ENOMEM. */
int sj_neighbor_csr(sj_handle *h, uint64_t *row_off, uint32_t *nbrs, uint64_t cap, uint64_t *total);

/* Free every device / pinned resource of the handle.  NULL-safe. */
void sj_destroy(sj_handle *h);

/* Text of the last error raised on the calling thread ("" if none). */
const char *sj_last_error(void);

/* Set an option (enum sj_option).  Returns SJ_OK or SJ_EINVAL (unknown option /
 * out-of-range value).  Takes effect at the next sj_self_join that (re)starts. */
int sj_set_option(sj_handle *h, int opt, int64_t value);

/* Restrict this handle to the queue slice of `rank` out of `world` replicas
 * (multi-GPU): D' is cut into WorkQueue chunks (at most 32
 * positions, never straddling a cell of >= 8 points) and chunk c belongs to rank
 * c mod world.  Slices of all ranks are disjoint and cover D'; each slice's pairs
 * are disjoint (every unordered pair is evaluated by exactly one query point).
 * world = 1 restores the whole queue. */
int sj_set_slice(sj_handle *h, int rank, int world);

/* Copy the statistics of the handle into *s. */
int sj_get_stats(const sj_handle *h, sj_stats *s);

/* Serialise the built index (header + device arrays) into one contiguous blob
 * for an NCCL broadcast.  dst: device or host pointer of cap bytes, or NULL to
 * only query the size in *bytes.  Format "SJIDX004" (this library version only). */
int sj_export_index(const sj_handle *h, void *dst, uint64_t cap, uint64_t *bytes);

/* Create a handle from a blob produced by sj_export_index (device or host
 * pointer, possibly on another GPU / process).  NULL on error. */
sj_handle *sj_create_from_index(const void *blob, uint64_t bytes);

/* The caller's CUDA stream (a cudaStream_t) for the ordering rule above, for the calling
 * thread; NULL = the legacy default stream (the initial value).  The Python binding passes
 * torch's current stream before every call. */
void sj_set_stream(void *stream);

/* Zero-copy variant of sj_create_from_index for a blob in device memory of the current device
 * (256-byte aligned, e.g. the output of an NCCL broadcast): the handle's index arrays ARE the
 * blob's -- nothing is allocated or copied -- so the caller keeps the blob alive and unchanged
 * until sj_destroy.  The blob is validated as in sj_create_from_index.  NULL on error. */
sj_handle *sj_create_from_index_view(const void *blob, uint64_t bytes);

/* ABI version (SJ_ABI_VERSION). */
int sj_abi_version(void);

/* Number of CUDA kernels libsj.so has launched in this process (diagnostics). */
uint64_t sj_kernel_launches(void);

/* ---- slab partition of a multi-GPU join -------------------
 * The device-side arithmetic of cutting the global grid into slabs of whole dimension-0 cell
 * columns; the caller only runs the collectives between the calls (all-reduce MIN/MAX of the
 * bounds, all-reduce SUM of the histogram, all_to_all of the packed rows), then builds its
 * partition with sj_create_part.  Column of a point: c = floor(fl(fl(x_0 - origin_0) / w)),
 * w = fl(eps (1 + 2^-20)) -- the build's own cell arithmetic (readings c5, c6), so a cut never
 * splits a cell.  These calls run on the caller's stream (sj_set_stream) and return after
 * their GPU work ended.  points: n x dim row-major doubles on the current device; 0 <= n < 2^32. */

/* Local per-dimension bounds: mn[d] / mx[d] (host double[dim]) = min / max of points[:, d]
 * (+inf / -inf when n = 0).  SJ_EINVAL for a non-finite coordinate or bad arguments. */
int sj_part_bounds(const double *points, uint64_t n, int dim, double *mn, double *mx);

/* Number of dimension-0 cell columns of the global grid: c(max0) + 1 for the global origin0 and
 * maximum max0 (host arithmetic, the same binary64 operations).  SJ_EINVAL, or SJ_EGRID when the
 * column count reaches 2^30 (reading c5's bound). */
int64_t sj_part_columns(double origin0, double max0, double eps);

/* Column histogram of the local points: hist (device uint64[ncol], overwritten) counts the
 * points of every column.  SJ_EINVAL if a point lies below origin0 or in a column >= ncol. */
int sj_part_histogram(const double *points, uint64_t n, int dim, double origin0, double eps, uint64_t ncol,
                      uint64_t *hist);

/* Routes and packs the local points for the all-to-all, given the GLOBAL histogram (device
 * uint64[ncol], the sum over the ranks).  Column c is owned by rank
 * min(world - 1, floor(start_c * world / total)), start_c = the points of columns < c: slabs of
 * whole columns balanced by points.  own_pts / own_ids (device, n rows of dim doubles / uint32)
 * receive every point, grouped by owner rank ascending, input order inside a rank;
 * own_counts (host uint64[world]) the rows per rank.  A point of column c >= 1 whose owner
 * differs from owner(c - 1) is also packed into halo_pts / halo_ids (device, room for n rows)
 * for rank owner(c - 1) -- the LID-UNICOMP forward cells lie at most one column ahead (P:174,
 * Alg. 3) -- with halo_counts (host uint64[world]).  ids: device uint32[n] global ids, or NULL
 * (ids = local positions).  1 <= world <= 2^20. */
int sj_part_pack(const double *points, const uint32_t *ids, uint64_t n, int dim, double origin0, double eps,
                 const uint64_t *hist, uint64_t ncol, int world, double *own_pts, uint32_t *own_ids,
                 uint64_t *own_counts, double *halo_pts, uint32_t *halo_ids, uint64_t *halo_counts);

/* ---- host-only helpers (no GPU needed) ------------------------------------ */

/* LID-UNICOMP forward offsets (Alg. 3): the neighbour offsets o in
 * {-1,0,1}^dim whose cell has a higher row-major linear id than the origin, i.e.
 * whose first non-zero component is +1.  Writes F*dim int8 values (F = (3^dim-1)/2)
 * if out != NULL and cap >= F*dim.  Returns F, or SJ_EINVAL. */
int sj_forward_offsets(int dim, int8_t *out, uint64_t cap);

/* WorkQueue chunks of slice (rank, world) out of n_chunks (sj_stats.n_chunks):
 * writes them ascending into out (if out != NULL and cap is large enough) and
 * returns their number, or a negative sj_status. */
int64_t sj_slice_chunks(uint64_t n_chunks, int rank, int world, uint32_t *out, uint64_t cap);

/* Virtual WorkQueue chunks of staged batch `batch` out of `n_batches` over a slice of
 * n_chunks chunks: queue = 1 (WorkQueue) -> the contiguous range
 * [n_chunks*batch/n_batches, n_chunks*(batch+1)/n_batches) (reading c14); queue = 0
 * (SortByWL only) -> the strided D'_l: batch, batch + n_batches, ... (Fig. 1).  Writes them
 * ascending into out (if out != NULL and cap is large enough) and returns their number, or
 * SJ_EINVAL.  sj_self_join cuts its estimated batches with exactly this rule. */
int64_t sj_batch_chunks(uint64_t n_chunks, uint64_t n_batches, uint64_t batch, int queue, uint32_t *out,
                        uint64_t cap);

/* ---- diagnostics (GPU microbenchmarks for the roofline denominators) ------ */

/* FP64 pipe throughput of the current device: DADD/DMUL dependent chains on all
 * SMs; *instr_per_s receives FP64 warp-lane instructions per second.  */
int sj_measure_fp64(double *instr_per_s, double *ms);

/* Same-address global atomicAdd rate (one lane per warp), ops per second. */
int sj_measure_atomics(double *ops_per_s, double *ms);

#ifdef __cplusplus
}
#endif

#endif /* SJ_H */
