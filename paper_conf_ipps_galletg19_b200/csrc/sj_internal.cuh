// sj_internal.cuh -- internal declarations shared by the libsj.so translation units.
// Product code (CUDA for sm_100a + C++ host runtime).  Never includes or links the
// oracle (oracle/), see DESIGN.md §3.
#pragma once

#include <cuda_runtime.h>
#include <stdint.h>

#include <atomic>
#include <string>

#include "../../include/sj.h"

#define SJ_MAX_DIM 8
#define SJ_MAX_FWD 6560  // 3^8 - 1 rows (UNICOMP in 8-D)

// WorkQueue chunk: at most kChunk D' positions; cells with at least kBigCell points get
// chunks of their own.
constexpr unsigned kChunk = 32;
// Empty WorkQueue chunks written after the last one: a device-sized join (the host does not know
// the chunk count yet) may dequeue past it by < grab * world chunks (the runtime checks the bound)
constexpr unsigned kChunkPad = 4096;
#ifndef SJ_BIGCELL
#define SJ_BIGCELL 8
#endif
constexpr unsigned kBigCell = SJ_BIGCELL;

namespace sj {

// --------------------------------------------------------------------------- errors
void set_error(const char *fmt, ...);
struct Status {
    int code = SJ_OK;
};

#define SJ_CUDA_TRY(expr)                                                                       \
    do {                                                                                        \
        cudaError_t _e = (expr);                                                                \
        if (_e != cudaSuccess) {                                                                \
            ::sj::set_error("%s:%d %s: %s", __FILE__, __LINE__, #expr, cudaGetErrorString(_e)); \
            return (_e == cudaErrorMemoryAllocation) ? SJ_ENOMEM : SJ_ECUDA;                    \
        }                                                                                       \
    } while (0)

#define SJ_TRY(expr)                 \
    do {                             \
        int _rc = (expr);            \
        if (_rc < 0) return _rc;     \
    } while (0)

// Process-wide count of kernels libsj.so launched (sj_kernel_launches()).
extern std::atomic<unsigned long long> g_launches;
inline void note_launch() { g_launches.fetch_add(1, std::memory_order_relaxed); }

// Host-side phase timer printed to stderr when SJ_DEBUG=1 (diagnostics only).
void debug_mark(const char *label);

// The caller's stream of the calling thread (sj_set_stream; the legacy default stream by default).
cudaStream_t caller_stream();

// --------------------------------------------------------------------------- memory
// Stream-ordered allocations from the device's default memory pool.  The pool's
// release threshold is raised once, so repeated create/destroy cycles reuse memory
// instead of returning it to the driver (DESIGN.md §4 "memory").
int dev_alloc(void **p, size_t bytes, cudaStream_t s);
void dev_free(void *p, cudaStream_t s);
template <class T>
inline int dev_alloc_t(T **p, size_t count, cudaStream_t s) {
    return dev_alloc(reinterpret_cast<void **>(p), count * sizeof(T) + 16, s);
}

// Build workspace (one stream-ordered block per sj_create): a bump region for the build's
// temporaries and a region zeroed ONCE up front for the small counters and the look-back
// status words of every scan, so the build issues one allocation and one memset instead of
// one of each per temporary and per scan (the host's API calls, not the GPU, paced the
// short build kernels).  take*() return nullptr when the region is exhausted; callers then
// fall back to dev_alloc (+ memset).
struct Workspace {
    char *base = nullptr;
    size_t cap = 0, off = 0;
    char *zbase = nullptr;
    size_t zcap = 0, zoff = 0;
    static size_t round(size_t b) { return (b + 255) & ~(size_t)255; }
    void *take(size_t bytes) {
        bytes = round(bytes);
        if (!base || off + bytes > cap) return nullptr;
        void *p = base + off;
        off += bytes;
        return p;
    }
    void *take_zero(size_t bytes) {
        bytes = round(bytes);
        if (!zbase || zoff + bytes > zcap) return nullptr;
        void *p = zbase + zoff;
        zoff += bytes;
        return p;
    }
};

// Process-wide free list of 4 KiB pinned host blocks ("mailboxes" for small D2H reads);
// cudaMallocHost costs far more than a whole small join, so blocks are recycled.
constexpr size_t kMailBytes = 4096;
void *pinned_acquire();
void pinned_release(void *p);

// Zero-copy host waits: a kernel writes its result into pinned host memory, then `epoch` into
// *flag (after a system-scope fence); the host spins on the flag, polling the stream for errors
// (and for a stream that drained without the flag: an error).  next_epoch() never returns 0.
unsigned next_epoch();
int wait_flag(volatile unsigned *flag, unsigned epoch, cudaStream_t s);

// --------------------------------------------------------------------------- primitives
// Exclusive scan of u32 (out may alias in).  total (device, optional) receives the sum.
int scan_exclusive_u32(const uint32_t *in, uint32_t *out, uint64_t n, uint32_t *d_total, cudaStream_t s,
                       Workspace *ws = nullptr);

// Exclusive scans with 64-bit sums (pair counts, CSR row offsets; totals < 2^62).  out may
// alias in; d_total (device, optional) receives the sum, e.g. out + n for an (n+1)-entry
// offset array.
int scan_exclusive_u64(const uint64_t *in, uint64_t *out, uint64_t n, uint64_t *d_total, cudaStream_t s);
int scan_exclusive_u32_to_u64(const uint32_t *in, uint64_t *out, uint64_t n, uint64_t *d_total, cudaStream_t s);

// Stable LSD radix sort of (key, value) pairs on the low `bits` bits of the keys.
// Hand-written: per 8-bit pass a tile histogram, a digit-major scan and a stable
// scatter through shared memory (DESIGN.md §4 a4).  Buffers are ping-ponged; the
// result pointer pair is returned through *keys_out / *vals_out (one of the inputs
// or the alternates).
// hist0 (optional): the first pass's tile histogram (digit-major [256][tiles of 2048 keys]),
// already counted by the kernel that produced the keys; it also serves as the histogram buffer.
// vals_identity: the values are the identity 0..n-1, generated by the first pass (`vals` is then
// uninitialised scratch of n entries).
constexpr int kRadixTileKeys = 2048;
int radix_sort_u32(uint32_t *keys, uint32_t *vals, uint32_t *keys_alt, uint32_t *vals_alt, uint64_t n, int bits,
                   uint32_t **keys_out, uint32_t **vals_out, cudaStream_t s, Workspace *ws = nullptr,
                   uint32_t *hist0 = nullptr, bool vals_identity = false);
int radix_sort_u64(uint64_t *keys, uint32_t *vals, uint64_t *keys_alt, uint32_t *vals_alt, uint64_t n, int bits,
                   uint64_t **keys_out, uint32_t **vals_out, cudaStream_t s, Workspace *ws = nullptr,
                   uint32_t *hist0 = nullptr, bool vals_identity = false);

// --------------------------------------------------------------------------- index
// The index I in its B200 layout, DESIGN.md §4.  Points are stored in the
// SortByWL queue order D' so the WorkQueue hands out contiguous storage positions.
struct Index {
    uint64_t n = 0;
    int dim = 0;
    int pad = 0;              // doubles per stored point (dim rounded up to even; 1 for dim 1)
    double eps = 0, e2 = 0, w = 0;
    double mins[SJ_MAX_DIM] = {0};
    uint64_t nc[SJ_MAX_DIM] = {0};
    uint64_t stride[SJ_MAX_DIM] = {0};
    int key_bits = 0;
    int pattern = SJ_PATTERN_LID_UNICOMP;  // cell access pattern (sj_create_ex)
    int order = SJ_ORDER_WORKLOAD;         // D' order (sj_create_ex)
    uint64_t n_cells = 0;     // M
    uint64_t n_runs = 0;      // E, forward runs over all cells
    uint64_t dist_calcs = 0;  // D_alg
    uint32_t max_w = 0;
    int lookup_hash = 0;      // a6's lid -> cell lookup: 0 dense table, 1 open-addressing hash

    double *pts = nullptr;      // [n * pad]  points in lid (spatial) order, padded AoS
    uint32_t *orig = nullptr;   // [n]        lid position -> input id
    uint2 *qmap = nullptr;      // [n]        D' (queue) position -> {lid position, queue-order cell}
    uint4 *cellq = nullptr;     // [M]        queue-order cell: {lid begin, m, first run, sum of run lengths}
    uint2 *runs = nullptr;      // [E]        forward run: {lid begin, length}
    uint64_t *cell_lid = nullptr; // [M]      queue-order cell -> linear id (export / tests)
    uint32_t *chunks = nullptr; // [C+1]      WorkQueue chunk c = D' positions [chunks[c], chunks[c+1])
    uint64_t n_chunks = 0;      // C
    uint64_t n_query = 0;       // queries: D' positions [0, n_query) (n unless partitioned)
    uint32_t *d_meta = nullptr; // [4]        device {n_chunks, E}, written by the build
    uint64_t runs_cap = 0;      // entries allocated for runs (>= E + 2)
    uint64_t runs_len = 0;      // entries the cells' run indices span: M * rows in the slot
                                // layout (cell r's runs at r * rows), 0 = compact (E)
    // the build's arrays carved from ONE stream-ordered allocation (bounds from n: M <= n), so a
    // build and a destroy cost one allocation call each; runs are outside it when runs_own
    void *block = nullptr;
    bool runs_own = true;
};
inline uint64_t runs_entries(const Index &ix) { return ix.runs_len ? ix.runs_len : ix.n_runs; }

struct BuildTimes {
    float ms = 0;
};

// Spatial partition of a join (sj_create_part): the grid origin is given (the
// global per-dimension minimum, so every partition's cells align), only the first n_query
// points are queries (the rest is the halo: candidates only), and the output carries the
// caller's global ids.
struct BuildPart {
    double origin[SJ_MAX_DIM];
    const uint32_t *d_ids = nullptr;  // [n] device, or null (ids = input positions)
    uint64_t n_query = 0;
};

// Side stream of the build (the gather of the points into cell order and D' run there,
// overlapping the main stream's forward runs, cell sort and queue); ea: main -> side, eg: the
// gather done, eq: D' done, ej: side -> main at exit.  nullptr: everything on the main stream.
struct BuildSide {
    cudaStream_t s2;
    cudaEvent_t ea, eg, eq, ej;
};

// Builds the index from device-resident raw points (n x dim AoS).  Returns sj_status.
int build_index(Index &ix, const double *d_raw, uint64_t n, int dim, double eps, cudaStream_t s,
                cudaEvent_t ev0, cudaEvent_t ev1, float *ms, const BuildPart *part = nullptr,
                uint64_t *tail_mail = nullptr, const BuildSide *side = nullptr,
                unsigned long long *zero_ctr = nullptr, int zero_words = 0);
// zero_ctr: zero_words device words the build's last kernel zeroes (the join's counters).
// tail_mail (pinned host, 2 words): the build ends without a host round trip; {n_chunks, E}
// arrive there once the stream passes ev1, and ix.n_chunks / ix.n_runs / *ms stay unset
// until the caller reads them (sj_runtime.cu: ix_ready).  nullptr: synchronous, all set.
void free_index(Index &ix, cudaStream_t s);
// LID-UNICOMP forward offsets (host): F = (3^dim - 1)/2 offsets, int8 each dim.
int forward_offsets_public(int dim, int8_t *out, uint64_t cap);

// --------------------------------------------------------------------------- join
struct JoinArgs {
    const double *pts;
    const uint32_t *orig;
    const uint2 *qmap;
    const uint4 *cellq;
    const uint2 *runs;
    const uint32_t *chunks;       // WorkQueue chunks of D'
    uint32_t n_chunks;
    uint64_t n_runs;              // entries of runs (bounds of the staged copies)
    double e2;
    unsigned long long *head;     // WorkQueue counter (chunks taken), zeroed before the launch
    unsigned long long v_begin;   // batch = virtual chunks v_begin, v_begin + v_stride, ... < v_end
    unsigned long long v_end;     //   of this slice (v_stride 1: a contiguous range)
    uint32_t v_stride;
    uint32_t v_count;             // the batch's chunks (set by launch_join)
    uint32_t static_q;            // 1: static warp -> chunk assignment (SortByWL only), 0: WorkQueue
    uint32_t grab;                // chunks per dequeue
    uint32_t gcg;                 // 1: GCG pattern (full neighbourhood, one pair per hit)
    uint32_t rank, world;         // queue slice: virtual chunk v -> chunk v*world + rank
    uint32_t *out;                // interleaved pairs, or nullptr (count-only)
    unsigned long long *emit_ctr; // pairs emitted (may exceed out_cap -> overflow)
    unsigned long long out_cap;   // capacity of out in pairs
    unsigned long long *calcs;    // instrumented distance calculations, or nullptr
    // kPairs, mirrored patterns: the output space is taken in BLOCKS of blk pairs, one atomic
    // on emit_ctr per block and warp, instead of one per warp flush -- a single counter taking
    // every flush congests its L2 slice and halves the join (measured).  Each warp's last block
    // stays partly empty: its gap {start, length} goes to gaps[global warp index] and
    // compact_output() closes the gaps afterwards.  Positions from
    // out_cap & ~1 on go to scratch (scratch_cap pairs).  blk = 0: one atomic per flush.
    unsigned long long blk;
    unsigned long long *gaps;
    uint32_t *scratch;
    unsigned long long scratch_cap;
    // kPairs: the batch estimator fused into the join (a9): pairs of the virtual chunks
    // [v_begin, sample_v1) are added to *sample_ctr (sample_v1 = 0: off)
    unsigned long long *sample_ctr;
    unsigned long long sample_v1;
    // device-sized launch (the build's chunk count not yet on the host): the slice's virtual
    // chunk count V is computed from *d_nchunks in the kernel (v_begin 0, stride 1, v_end V),
    // and with sample_ppm the fused estimator's sample is the first ceil(V * ppm / 1e6) chunks
    const uint32_t *d_nchunks;
    uint32_t sample_ppm;
    // exact two-pass sizing
    unsigned long long *vcount;       // kChunkCount: pairs of virtual chunk v (written per chunk)
    const unsigned long long *voff;   // kExact: pair offset of virtual chunk v (exclusive scan of vcount);
    unsigned long long out_base;      //   out holds pairs [out_base, ..)
    // device CSR (GCG pattern: every query owns its row)
    uint32_t *qdeg;                   // kDegree: degree by input id
    const unsigned long long *row_off; // kRows: row start by input id
    uint32_t *nbrs;                   // kRows: neighbour ids
};

// Join kernel modes: count pairs; emit the pair list; fill CSR rows; count CSR degrees;
// count pairs per WorkQueue chunk (exact sizing pass 1); emit at chunk offsets (pass 2).
// kPairsB: kPairs with the blocked output (JoinArgs::blk) -- a kernel of its own, so the default
// one carries none of its code.
enum JoinMode : int { kCount = 0, kPairs = 1, kRows = 2, kDegree = 3, kChunkCount = 4, kExact = 5, kPairsB = 6 };

// Launch the join kernel for dim/k/mode (kRows / kDegree need the GCG pattern).
int launch_join(const JoinArgs &a, int dim, int k, int mode, int blocks, cudaStream_t s);
// After a blocked kPairs launch (JoinArgs::blk): move the pairs past the total into the warps'
// gaps so the output is [0, total) again; total -> *d_total.  ws: device workspace of
// compact_ws_bytes(blocks) bytes.  Two launches on s, no host round trip.
size_t compact_ws_bytes(int blocks);
constexpr int kCompactMaxGaps = 8192;  // warps (gaps) compact_output handles
int compact_output(const JoinArgs &a, int blocks, unsigned long long *d_total, void *ws, cudaStream_t s);
// Max resident CTAs per SM of the join kernel configuration.
int join_occupancy(int dim, int k, int mode, bool gcg, int *blocks_per_sm);
constexpr int kJoinThreads = 256;

// --------------------------------------------------------------------------- misc kernels
int launch_fill_u64(unsigned long long *p, const unsigned long long *vals_host_pinned, int count, cudaStream_t s);

}  // namespace sj
