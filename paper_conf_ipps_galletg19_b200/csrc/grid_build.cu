// grid_build.cu -- the eps-grid index I built on the GPU, plus the
// per-cell workload and SortByWL.  Steps a2..a8 of
// DESIGN.md §1:
//   a2 bounding box (exact min/max per dimension)
//   a3 cell linearisation  c_d = floor(fl(fl(x_d - min_d) / w)),  w = eps(1+2^-20)
//      (readings c5, c6); lid = sum_d c_d * stride_d, row-major, dim 0 most significant (c7)
//   a4 hand-written radix sort of (lid, point id) on the significant bits
//   a5 run-length compaction -> non-empty cells B + point lookup
//   a6 LID-UNICOMP forward neighbours (Alg. 3) resolved once per cell into
//      contiguous runs of the lid-ordered point storage
//   a7 workload W(A) = ceil((m_A-1)/2) + sum_{B in fwd(A)} m_B and D_alg
//   a8 SortByWL: cells in non-increasing W (stable, ties by lid, c10) -> D' (index array)
#include <algorithm>
#include <cmath>
#include <cstring>
#include <vector>

#include "scan.cuh"
#include "sj_internal.cuh"

namespace sj {


namespace {

constexpr int kThreads = 256;

inline unsigned grid_for(uint64_t n, int threads = kThreads) {
    uint64_t b = (n + threads - 1) / threads;
    if (b == 0) b = 1;
    return (unsigned)b;
}

__device__ __forceinline__ unsigned long long ordered_key(double x) {
    unsigned long long b = (unsigned long long)__double_as_longlong(x);
    return (b >> 63) ? ~b : (b | 0x8000000000000000ull);
}
__host__ __device__ inline double from_ordered_key(unsigned long long k) {
    unsigned long long b = (k >> 63) ? (k & 0x7FFFFFFFFFFFFFFFull) : ~k;
    double d;
    memcpy(&d, &b, sizeof d);
    return d;
}

// Zero-initialised (it lives in the build workspace's pre-zeroed region): the minimum is kept
// as the maximum of the complemented ordered key, so 0 is the neutral element of both.
struct BBox {
    unsigned long long mn_c[SJ_MAX_DIM];  // ~ordered_key(min)
    unsigned long long mx[SJ_MAX_DIM];
    unsigned int nonfinite;
    unsigned int done;  // blocks finished (the last one derives the grid geometry)
};

// The grid geometry (a3, readings c5-c7), derived on the device by the bounding box's last
// block: the cell-id kernel reads it from device memory and the host reads the copy written
// into its pinned mailbox (zero-copy, behind `flag`), so the first kernels after the bounding
// box are queued without a host round trip in between.
struct GeomDev {
    double mins[SJ_MAX_DIM];
    unsigned long long nc[SJ_MAX_DIM];
    unsigned long long stride[SJ_MAX_DIM];
    double w;
    double errq;
    int dim, key_bits;
    int err;     // 0 ok, 1 non-finite coordinate, 2 below the given origin, 3 quotient >= 2^30, 4 cells >= 2^64
    int errdim;
    unsigned flag;  // host copy: the build's epoch once the fields are written
    unsigned pad;
};
struct GeomArgs {
    double w;
    double origin[SJ_MAX_DIM];
    int has_origin;
    GeomDev *dev;        // device copy (read by cell_id_kernel)
    GeomDev *host;       // pinned host copy, or nullptr
    unsigned epoch;
};

// Called by the first warp of the bounding box's last block: lane d handles dimension d.
__device__ void derive_geometry(const BBox *bb, int dim, const GeomArgs &ga) {
    const int lane = threadIdx.x & 31;
    const volatile BBox *vb = bb;
    int err = vb->nonfinite ? 1 : 0, errdim = 0;
    double mn = 0, q = 0;
    unsigned long long nc = 1;
    int my_err = 0;
    if (lane < dim && !err) {
        mn = from_ordered_key(~vb->mn_c[lane]);
        const double mx = from_ordered_key(vb->mx[lane]);
        if (ga.has_origin) {  // partition of a larger grid: its origin (all partitions' cells align)
            if (!(ga.origin[lane] <= mn) || !isfinite(ga.origin[lane])) my_err = 2;
            mn = ga.origin[lane];
        }
        // nc_d = max c_d + 1; c_d is monotone in x_d so max c_d = c_d(max x_d)
        q = __ddiv_rn(__dsub_rn(mx, mn), ga.w);
        if (!my_err && !(q < 0x1p30)) my_err = 3;
        if (!my_err) nc = (unsigned long long)floor(q) + 1ull;
    }
    const unsigned emask = __ballot_sync(0xffffffffu, my_err != 0);
    if (!err && emask) {
        errdim = __ffs(emask) - 1;
        err = __shfl_sync(0xffffffffu, my_err, errdim);
    }
    const double errq = __shfl_sync(0xffffffffu, q, errdim);
    GeomDev *g = ga.dev;
    if (lane < SJ_MAX_DIM) {  // every entry written (the host copy reads all of them)
        g->mins[lane] = lane < dim ? mn : 0.0;
        g->nc[lane] = lane < dim ? nc : 1ull;
        g->stride[lane] = 0;
    }
    __syncwarp();
    unsigned long long ncd[SJ_MAX_DIM];  // every lane: the counts of all dimensions
#pragma unroll
    for (int d = 0; d < SJ_MAX_DIM; ++d) ncd[d] = __shfl_sync(0xffffffffu, nc, d);
    if (lane == 0) {
        unsigned long long total = 1;
        for (int d = 0; d < dim && !err; ++d) {
            if (total > ~0ull / ncd[d] || total * ncd[d] == ~0ull) err = 4;
            else total *= ncd[d];
        }
        unsigned long long st = 1;
        for (int d = dim - 1; d >= 0; --d) {
            g->stride[d] = st;
            st *= ncd[d];
        }
        const unsigned long long mx_id = total - 1ull;
        g->key_bits = err ? 0 : (mx_id ? 64 - __clzll((long long)mx_id) : 0);
        g->dim = dim;
        g->w = ga.w;
        g->err = err;
        g->errdim = errdim;
        g->errq = errq;
    }
}

// The host copy of the geometry (first block of the cell-id kernel, so the host reads it while
// the cell ids are computed): fields, a system-scope fence, then the flag.
__device__ void publish_geometry(const GeomDev *g, const GeomArgs &ga) {
    volatile GeomDev *h = ga.host;
    for (int d = 0; d < SJ_MAX_DIM; ++d) {
        h->mins[d] = g->mins[d];
        h->nc[d] = g->nc[d];
        h->stride[d] = g->stride[d];
    }
    h->w = g->w;
    h->errq = g->errq;
    h->dim = g->dim;
    h->key_bits = g->key_bits;
    h->err = g->err;
    h->errdim = g->errdim;
    __threadfence_system();
    h->flag = ga.epoch;
}

__global__ void __launch_bounds__(kThreads) bbox_kernel(const double *raw, uint64_t n, int dim, BBox *bb,
                                                        GeomArgs ga) {
    const uint64_t total = n * (uint64_t)dim;  // doubles
    const uint64_t T = (uint64_t)gridDim.x * blockDim.x;
    const uint64_t t = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
    const int d0 = (int)((2 * t) % dim), d1 = (int)((2 * t + 1) % dim);
    unsigned long long mn0 = ~0ull, mx0 = 0, mn1 = ~0ull, mx1 = 0;
    unsigned bad = 0;
    const double2 *r2 = reinterpret_cast<const double2 *>(raw);
    const uint64_t pairs = total / 2;
    auto take = [&](const double2 v) {
        bad |= !isfinite(v.x) | !isfinite(v.y);
        const unsigned long long k0 = ordered_key(v.x), k1 = ordered_key(v.y);
        mn0 = min(mn0, k0);
        mx0 = max(mx0, k0);
        mn1 = min(mn1, k1);
        mx1 = max(mx1, k1);
    };
    // four independent 16-B loads in flight per thread (a stride of T keeps the dimensions)
    uint64_t e = t;
    for (; e + 3 * T < pairs; e += 4 * T) {
        const double2 v0 = __ldg(r2 + e), v1 = __ldg(r2 + e + T), v2 = __ldg(r2 + e + 2 * T), v3 = __ldg(r2 + e + 3 * T);
        take(v0);
        take(v1);
        take(v2);
        take(v3);
    }
    for (; e < pairs; e += T) take(__ldg(r2 + e));
    if ((total & 1) && t == 0) {  // odd element count: the last double (dimension dim-1)
        const double x = raw[total - 1];
        bad |= !isfinite(x);
        const unsigned long long k = ordered_key(x);
        atomicMax(&bb->mn_c[dim - 1], ~k);
        atomicMax(&bb->mx[dim - 1], k);
    }
    // block reduction per dimension in shared memory, then ONE atomic per dimension and block
    __shared__ unsigned long long s_mn[SJ_MAX_DIM], s_mx[SJ_MAX_DIM];
    __shared__ unsigned s_bad;
    if (threadIdx.x < SJ_MAX_DIM) {
        s_mn[threadIdx.x] = ~0ull;
        s_mx[threadIdx.x] = 0;
    }
    if (threadIdx.x == 0) s_bad = 0;
    __syncthreads();
    if (t < pairs) {
        atomicMin(&s_mn[d0], mn0);
        atomicMax(&s_mx[d0], mx0);
        atomicMin(&s_mn[d1], mn1);
        atomicMax(&s_mx[d1], mx1);
    }
    if (__any_sync(0xffffffffu, bad) && (threadIdx.x & 31) == 0) s_bad = 1;
    __syncthreads();
    if (threadIdx.x < (unsigned)dim) {
        atomicMax(&bb->mn_c[threadIdx.x], ~s_mn[threadIdx.x]);
        atomicMax(&bb->mx[threadIdx.x], s_mx[threadIdx.x]);
    }
    if (threadIdx.x == 0 && s_bad) atomicOr(&bb->nonfinite, 1u);
    // the last block to finish derives the grid geometry from the final box (its first warp)
    __syncthreads();
    __shared__ unsigned s_last;
    if (threadIdx.x == 0) {
        __threadfence();
        s_last = atomicAdd(&bb->done, 1u) == gridDim.x - 1u ? 1u : 0u;
        if (s_last) __threadfence();
    }
    __syncthreads();
    if (s_last && threadIdx.x < 32) derive_geometry(bb, dim, ga);
}


// a3: cell linearisation.  IEEE RN intrinsics so the result does not depend on
// contraction flags (reading c1): c_d = floor( (x_d - min_d) / w ).
// The geometry comes from device memory (bbox_kernel's last block); keys are 32-bit when the
// grid has at most 2^32 cells, else 64-bit (the host picks the buffer once it reads key_bits).
// One block per radix tile (kRadixTileKeys points): it also counts the tile's low 8-bit digits,
// the first pass of the point sort (a4) -- its histogram kernel is not launched.  The sort's
// values (input ids) are the identity, generated by its first scatter: not written here.
// threads per block: 1-D..3-D 512 (4 points per thread, loaded before any division), 4-D+ 1024
// (2 points: their coordinates fill the registers, and the divisions need the parallelism)
template <int DIM>
struct CellIdThreads {
    static constexpr int value = DIM <= 3 ? 512 : 1024;
};
template <int DIM>
__global__ void __launch_bounds__(CellIdThreads<DIM>::value) cell_id_kernel(const double *raw, uint64_t n,
                                                           const GeomDev *__restrict__ gp, uint32_t *keys32,
                                                           unsigned long long *keys64, GeomArgs ga,
                                                           uint32_t *hist0, uint32_t ntiles) {
    constexpr int kCellIdThreads = CellIdThreads<DIM>::value;
    constexpr int PPT = kRadixTileKeys / kCellIdThreads;
    __shared__ uint32_t h[256];
    if (threadIdx.x < 256) h[threadIdx.x] = 0;
    if (blockIdx.x == 0 && threadIdx.x == 0 && ga.host) publish_geometry(gp, ga);
    __syncthreads();
    const double w = gp->w;
    const bool ok = !gp->err, narrow = gp->key_bits <= 32;
    double mins[DIM];
    unsigned long long stride[DIM];
#pragma unroll
    for (int d = 0; d < DIM; ++d) {
        mins[d] = gp->mins[d];
        stride[d] = gp->stride[d];
    }
    const uint64_t base = (uint64_t)blockIdx.x * kRadixTileKeys;
    double x[PPT][DIM];
#pragma unroll
    for (int it = 0; it < PPT; ++it) {
        const uint64_t i = base + (uint64_t)it * kCellIdThreads + threadIdx.x;
#pragma unroll
        for (int d = 0; d < DIM; ++d) x[it][d] = (i < n && ok) ? __ldg(raw + i * DIM + d) : 0.0;
    }
#pragma unroll
    for (int it = 0; it < PPT; ++it) {
        const uint64_t i = base + (uint64_t)it * kCellIdThreads + threadIdx.x;
        if (i >= n || !ok) continue;
        unsigned long long lid = 0;
#pragma unroll
        for (int d = 0; d < DIM; ++d) {
            const double q = __ddiv_rn(__dsub_rn(x[it][d], mins[d]), w);
            lid += __double2ull_rd(q) * stride[d];
        }
        if (narrow)
            keys32[i] = (uint32_t)lid;
        else
            keys64[i] = lid;
        atomicAdd(&h[(uint32_t)lid & 0xFFu], 1u);
    }
    __syncthreads();
    if (threadIdx.x < 256) hist0[(uint64_t)threadIdx.x * ntiles + blockIdx.x] = h[threadIdx.x];
}

// a5: run-length compaction of the sorted ids, fused into one single-pass scan:
// flag(p) = (p == 0 || key[p] != key[p-1]); a flagged p starts cell ex = excl(p).
template <class K>
struct RleLoad {
    const K *ks;
    __device__ unsigned operator()(uint64_t p) const { return (p == 0 || ks[p] != ks[p - 1]) ? 1u : 0u; }
};
template <class K>
struct RleStore {
    const K *ks;
    uint32_t *cellof;
    unsigned long long *cell_lid;
    uint32_t *cell_start;
    uint32_t *dense;  // a6's dense lid -> cell table (pre-filled with ~0), or null (hashed lookup)
    __device__ void operator()(uint64_t p, unsigned ex, unsigned flag) const {
        if (flag) {
            cell_lid[ex] = (unsigned long long)ks[p];
            cell_start[ex] = (uint32_t)p;
            if (dense) dense[ks[p]] = ex;
        }
        cellof[p] = flag ? ex : ex - 1;  // point (sorted position) -> cell rank
    }
};
struct RleDone {
    uint64_t n;
    uint32_t *cell_start;
    uint64_t *d_M;
    __device__ void operator()(unsigned total) const {
        cell_start[total] = (uint32_t)n;
        *d_M = total;
    }
};

// ---------------------------------------------------------------- lid -> cell rank lookup
struct Lookup {
    const uint32_t *dense;           // dense table over all prod(nc) cells, or null
    const unsigned long long *hkeys; // open-addressing hash (linear probing)
    const uint32_t *hvals;
    unsigned long long hmask;
};

__device__ __forceinline__ unsigned long long hash_lid(unsigned long long x) {
    x ^= x >> 33;
    x *= 0xff51afd7ed558ccdull;
    x ^= x >> 33;
    x *= 0xc4ceb9fe1a85ec53ull;
    x ^= x >> 33;
    return x;
}

__device__ __forceinline__ uint32_t lookup_cell(const Lookup &L, unsigned long long lid) {
    if (L.dense) return L.dense[lid];
    unsigned long long h = hash_lid(lid) & L.hmask;
    for (;;) {
        unsigned long long k = L.hkeys[h];
        if (k == lid) return L.hvals[h];
        if (k == ~0ull) return 0xFFFFFFFFu;
        h = (h + 1) & L.hmask;
    }
}

__global__ void __launch_bounds__(kThreads) hash_insert_kernel(const unsigned long long *cell_lid, const uint64_t *d_M,
                                                               unsigned long long *hkeys, uint32_t *hvals,
                                                               unsigned long long hmask) {
    uint64_t r = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (r >= *d_M) return;
    unsigned long long lid = cell_lid[r];
    unsigned long long h = hash_lid(lid) & hmask;
    for (;;) {
        unsigned long long prev = atomicCAS(&hkeys[h], ~0ull, lid);
        if (prev == ~0ull || prev == lid) {
            hvals[h] = (uint32_t)r;
            return;
        }
        h = (h + 1) & hmask;
    }
}

struct FwdGeom {
    unsigned long long nc[SJ_MAX_DIM];
    unsigned long long stride[SJ_MAX_DIM];
    int dim;
    int rows;   // rows of the cell pattern (see pattern_rows())
    int small;  // prod(nc) < 2^32: 32-bit lid arithmetic
    int full;   // GCG: the rows cover the whole 3^n neighbourhood incl. the home cell
    // rows of the cell pattern, resolved against this grid (RowEnt), in this build's workspace:
    // read through L1 (lanes of a 32-lane cell read different rows)
    const struct RowEnt *rows_ent;
    // partitioned index (sj_create_part): a cell is a query cell iff its first member (lowest
    // input id, the sort is stable) is < nq; halo cells get no runs and no workload
    const uint32_t *idx;  // sorted position -> input id, or null (every cell is a query cell)
    uint32_t nq;
    unsigned int *mixed;  // set if a cell holds both query and halo points
};

struct BuildTotals {
    unsigned long long M;
    unsigned long long E;
    unsigned long long dist_calcs;
    unsigned int max_w;
    unsigned int done;  // blocks of the counting pass finished (the last one publishes)
};

// Zero-copy publication of the counting pass (the host's second wait): {M, E, D_alg, max W,
// mixed cells} into pinned memory, then the epoch into word 5.
struct TotalsPub {
    unsigned long long *host;  // pinned host words [6], or nullptr (copy + synchronisation)
    unsigned epoch;
};

// a6 + a7.  LID-UNICOMP (Alg. 3) visits the neighbour cells with a higher linear
// id.  With row-major ids those form "rows" along the last dimension: for every offset
// o' of the first n-1 dimensions whose first non-zero component is +1, the three cells
// o' x {-1, 0, +1}; plus, in the home row (o' = 0), the single cell +1.  The non-empty
// cells of one row have consecutive ranks in the lid-sorted cell array, so their points
// are ONE contiguous run of the lid-ordered point storage.  Each cell's forward
// neighbourhood is therefore a short list of runs {begin, length}.
//   W(A) = ceil((m_A - 1)/2)            (balanced circulant home-cell half scan, reading c8)
//        + sum_{B in fwd(A)} m_B
//   D_alg = sum_A C(m_A, 2) + m_A * sum_{B in fwd(A)} m_B
// Cell coordinates from a row-major linear id (c_0 most significant): n-1 divisions,
// 32-bit when the whole grid has < 2^32 cells.
// (DIM: the grid's dimensionality, a template parameter so each dimensionality's kernels carry
// only their own loops)
template <int DIM>
__device__ __forceinline__ void decode_lid(unsigned long long lid, const FwdGeom &g, long long (&c)[SJ_MAX_DIM]) {
    if (g.small) {
        unsigned rem = (unsigned)lid;
#pragma unroll
        for (int d = 0; d < SJ_MAX_DIM; ++d) {
            if (d < DIM - 1) {
                const unsigned st = (unsigned)g.stride[d];
                const unsigned q = rem / st;
                c[d] = q;
                rem -= q * st;
            } else if (d == DIM - 1) {
                c[d] = rem;
            }
        }
    } else {
        unsigned long long rem = lid;
#pragma unroll
        for (int d = 0; d < SJ_MAX_DIM; ++d) {
            if (d < DIM - 1) {
                const unsigned long long q = rem / g.stride[d];
                c[d] = (long long)q;
                rem -= q * g.stride[d];
            } else if (d == DIM - 1) {
                c[d] = (long long)rem;
            }
        }
    }
}

// One row of the cell pattern resolved against the grid (host, row_entries()): the linear-id
// delta of its first cell (offsets o' of the first n-1 dimensions and lo in the last), the
// dimensions it steps down (neg) / up (pos) in, and its meta byte (see pattern_rows()).
struct RowEnt {
    long long delta;  // sum_{d<last} o_d * stride_d + lo
    unsigned nm;      // bits 0-7: o_d == -1, bits 8-15: o_d == +1 (d < last)
    unsigned meta;    // lo+1 | (hi+1) << 2 | (pdim+1) << 4
};

// Per-cell data the rows are tested against: coordinates at the grid's edges and parities.
struct CellPos {
    unsigned long long lid;
    long long clast;  // coordinate in the last dimension
    unsigned lo_mask, hi_mask, odd_mask;  // c_d == 0 / c_d == nc_d - 1 (d < last); c_d odd (all d)
};

template <int DIM>
__device__ __forceinline__ CellPos cell_pos(unsigned long long lid, const FwdGeom &g) {
    long long c[SJ_MAX_DIM];
    decode_lid<DIM>(lid, g, c);
    CellPos p;
    p.lid = lid;
    p.lo_mask = p.hi_mask = p.odd_mask = 0;
    p.clast = 0;
#pragma unroll
    for (int d = 0; d < SJ_MAX_DIM; ++d) {
        if (d < DIM - 1) {
            p.lo_mask |= (c[d] == 0 ? 1u : 0u) << d;
            p.hi_mask |= (c[d] == (long long)g.nc[d] - 1 ? 1u : 0u) << d;
        }
        if (d < DIM) p.odd_mask |= (unsigned)(c[d] & 1) << d;
        if (d == DIM - 1) p.clast = c[d];
    }
    return p;
}

// The non-empty cells among the row's <= 3 cells (consecutive along the last dimension) have
// consecutive ranks, so their points are one run [b, b+len) of the lid-ordered storage.  The
// <= 3 lookups are issued together.
template <int DIM>
__device__ __forceinline__ bool eval_row(int j, const CellPos &cp, const FwdGeom &g, const Lookup &L,
                                         const uint32_t *cell_start, uint32_t &b, uint32_t &len) {
    const RowEnt e = g.rows_ent[j];
    const int pdim = (int)(e.meta >> 4) - 1;
    if (pdim >= 0 && !((cp.odd_mask >> pdim) & 1u)) return false;  // UNICOMP rule (Alg. 2)
    if ((e.nm & cp.lo_mask) | ((e.nm >> 8) & cp.hi_mask)) return false;  // leaves the grid
    const int lo = (int)(e.meta & 3u) - 1, hi = (int)((e.meta >> 2) & 3u) - 1;
    const long long x0 = cp.clast + lo;
    const int nx = hi - lo + 1;
    const long long ncl = (long long)g.nc[DIM - 1];
    const unsigned long long base = cp.lid + (unsigned long long)e.delta;
    uint32_t nb[3];
#pragma unroll
    for (int u = 0; u < 3; ++u) {
        const long long x = x0 + u;
        const bool ok = u < nx && x >= 0 && x < ncl;
        nb[u] = ok ? lookup_cell(L, base + (unsigned long long)u) : 0xFFFFFFFFu;
    }
    uint32_t r_lo = 0xFFFFFFFFu, r_hi = 0xFFFFFFFFu;
#pragma unroll
    for (int u = 2; u >= 0; --u)
        if (nb[u] != 0xFFFFFFFFu) r_lo = nb[u];
#pragma unroll
    for (int u = 0; u < 3; ++u)
        if (nb[u] != 0xFFFFFFFFu) r_hi = nb[u];
    if (r_lo == 0xFFFFFFFFu) return false;
    b = cell_start[r_lo];
    len = cell_start[r_hi + 1] - b;
    return true;
}

// a6 + a7 over the forward rows; LPC lanes per cell (1, or 32 when there are many rows:
// 6-D has 122) so the independent lookups of a cell run in parallel.
template <int DIM, bool FILL, int LPC>
__global__ void __launch_bounds__(kThreads) runs_kernel(const unsigned long long *cell_lid, const uint32_t *cell_start,
                                                        const uint64_t *d_M, FwdGeom g, Lookup L, uint32_t *rcnt,
                                                        uint32_t *wload, const uint32_t *rbegin, uint2 *runs,
                                                        BuildTotals *tot, TotalsPub pub, uint32_t *wkey,
                                                        uint32_t *wval) {
    // grid-stride over the cells (M is only known on the device): a bounded grid, so the block
    // reduction below runs once per resident block, not once per n-sized block
    const uint64_t M = *d_M;
    const uint64_t gt = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
    const uint64_t cstride = (uint64_t)gridDim.x * blockDim.x / LPC;
    const unsigned sub = (unsigned)(gt % LPC);
    const unsigned lane = threadIdx.x & 31;
    unsigned long long calcs = 0, nruns = 0;
    uint32_t w = 0;
    if (!FILL && gt == 0) rcnt[M] = 0;  // the scan runs over M + 1 entries
    for (uint64_t r = gt / LPC; r < M; r += cstride) {  // uniform across the LPC lanes of a cell
        const CellPos cp = cell_pos<DIM>(cell_lid[r], g);
        const uint32_t m = cell_start[r + 1] - cell_start[r];
        // FILL: the compacted layout (rbegin = scan of the counts); counting with `runs` set: the
        // slot layout, cell r's runs at r * rows (no second pass, no scan)
        uint32_t out = FILL ? rbegin[r] : (uint32_t)(r * (uint64_t)g.rows);
        bool qcell = true;
        if (g.idx) {
            qcell = g.idx[cell_start[r]] < g.nq;
            if (!FILL && sub == 0 && qcell != (g.idx[cell_start[r + 1] - 1] < g.nq)) atomicOr(g.mixed, 1u);
        }
        uint32_t cnt = 0;
        unsigned long long summ = 0;
        for (int jb = 0; jb < g.rows; jb += LPC) {
            const int j = jb + (int)sub;
            uint32_t b = 0, len = 0;
            const bool found = qcell && j < g.rows && eval_row<DIM>(j, cp, g, L, cell_start, b, len);
            if (FILL || runs) {
                if (LPC == 1) {
                    if (found) runs[out++] = make_uint2(b, len);
                } else {
                    const unsigned fm = __ballot_sync(0xffffffffu, found);
                    if (found) runs[out + __popc(fm & ((1u << lane) - 1u))] = make_uint2(b, len);
                    out += __popc(fm);
                }
            }
            if (!FILL && found) {
                ++cnt;
                summ += len;
            }
        }
        // slot layout: the cell's unused slots among its first five are cleared, so the join's
        // fixed-size staging of a cell's first runs (flat / generic paths, 1-D..3-D) never reads
        // uninitialised memory
        if (!FILL && runs && LPC == 1)
            for (uint32_t e = out, end = (uint32_t)(r * (uint64_t)g.rows) + (uint32_t)min(g.rows, 5); e < end; ++e)
                runs[e] = make_uint2(0, 0);
        if (!FILL) {
            if (LPC == 32) {
#pragma unroll
                for (int o = 16; o > 0; o >>= 1) {
                    cnt += __shfl_xor_sync(0xffffffffu, cnt, o);
                    summ += __shfl_xor_sync(0xffffffffu, summ, o);
                }
            }
            if (sub == 0) {
                rcnt[r] = cnt;
                nruns += cnt;
                uint32_t wr;
                if (!qcell) {  // halo cell (partitioned index): candidates only
                    wr = 0;
                } else if (g.full) {  // GCG: every candidate of the 3^n neighbourhood but the query itself
                    wr = (uint32_t)(summ - 1);
                    calcs += (unsigned long long)m * (summ - 1);
                } else {       // half patterns: ceil((m-1)/2) = floor(m/2) home + the forward runs
                    wr = (uint32_t)(m / 2 + summ);
                    calcs += (unsigned long long)m * (m - 1) / 2 + (unsigned long long)m * summ;
                }
                wload[r] = wr;
                // a8's SortByWL keys (the counting pass writes them: no key kernel): sorted on their
                // low bits_for(max W) bits, ~W ascending is W non-increasing, ties in lid order (the
                // value r); a partitioned index sorts on bits_for(max W + 1) bits, its query cells
                // keyed ~(W + 1) and its halo cells ~0, after every query cell
                wkey[r] = g.idx ? (qcell ? ~(wr + 1u) : ~0u) : ~wr;
                wval[r] = (uint32_t)r;
                w = max(w, wr);
            }
        }
    }
    if (!FILL) {  // block reduction, then ONE pair of global atomics per block
        __shared__ unsigned long long s_calcs[kThreads / 32], s_runs[kThreads / 32];
        __shared__ uint32_t s_w[kThreads / 32];
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) {
            calcs += __shfl_xor_sync(0xffffffffu, calcs, o);
            nruns += __shfl_xor_sync(0xffffffffu, nruns, o);
            w = max(w, __shfl_xor_sync(0xffffffffu, w, o));
        }
        if (lane == 0) {
            s_calcs[threadIdx.x >> 5] = calcs;
            s_runs[threadIdx.x >> 5] = nruns;
            s_w[threadIdx.x >> 5] = w;
        }
        __syncthreads();
        if (threadIdx.x == 0) {
            for (int i = 1; i < kThreads / 32; ++i) {
                calcs += s_calcs[i];
                nruns += s_runs[i];
                w = max(w, s_w[i]);
            }
            if (calcs) atomicAdd(&tot->dist_calcs, calcs);
            if (nruns) atomicAdd(&tot->E, nruns);
            if (w) atomicMax(&tot->max_w, w);
            if (pub.host) {  // the last block publishes the totals
                __threadfence();
                if (atomicAdd(&tot->done, 1u) == gridDim.x - 1u) {
                    __threadfence();
                    const volatile BuildTotals *vt = tot;
                    volatile unsigned long long *hp = pub.host;
                    hp[0] = M;
                    hp[1] = vt->E;
                    hp[2] = vt->dist_calcs;
                    hp[3] = vt->max_w;
                    hp[4] = g.mixed ? *(const volatile unsigned *)g.mixed : 0u;
                    __threadfence_system();
                    *reinterpret_cast<volatile unsigned *>(pub.host + 5) = pub.epoch;
                }
            }
        }
    }
}

// Empty chunks after the last one (kChunkPad): chunks[C + 1 + t] = the end of the queries.
// Also (block 0) the build's tail for the host -- the chunk count into the pinned mailbox
// (zero-copy, no copy on the stream between the build and the join) -- and the join's counters
// zeroed (the first join after sj_create launches without a memset of its own).
__global__ void __launch_bounds__(kThreads) chunk_pad_kernel(uint32_t *chunks, const uint32_t *d_nc, uint32_t end,
                                                             unsigned long long *tail_host,
                                                             unsigned long long *zero_ctr, int zero_words) {
    const uint32_t nc = *d_nc;
    chunks[nc + 1u + blockIdx.x * kThreads + threadIdx.x] = end;
    if (blockIdx.x == 0) {
        if ((int)threadIdx.x < zero_words) zero_ctr[threadIdx.x] = 0ull;
        if (threadIdx.x == 0 && tail_host) {
            *reinterpret_cast<volatile unsigned long long *>(tail_host) = nc;
            __threadfence_system();
        }
    }
}

// a8's queue cells, one fused scan (no count kernel, no separate finalize): load(i) = m of the
// i-th cell of the queue order, store(i, qb) = its record at queue position i, qb = its first D'
// position (the exclusive prefix of the counts).
struct QueueLoad {
    const uint32_t *qorder, *cell_start;
    __device__ unsigned operator()(uint64_t i) const {
        const uint32_t r = qorder[i];
        return cell_start[r + 1] - cell_start[r];
    }
};
struct QueueStore {
    const uint32_t *qorder, *cell_start, *rbegin;
    uint32_t slot_rows;
    const uint32_t *wload;
    const unsigned long long *cell_lid;
    int full;
    uint4 *cellq;
    uint32_t *r2q, *qbr, *qb;
    uint64_t *lid_q;
    const uint32_t *idx;
    uint32_t nq;
    __device__ void operator()(uint64_t i, unsigned ex, unsigned m) const {
        const uint32_t r = qorder[i];
        const uint32_t rb = rbegin ? rbegin[r] : r * slot_rows;  // first forward run
        qb[i] = ex;
        r2q[r] = (uint32_t)i;
        qbr[r] = ex;
        lid_q[i] = cell_lid[r];
        if (idx && idx[cell_start[r]] >= nq) {  // halo cell: never queued (m = 0 in its record)
            cellq[i] = make_uint4(cell_start[r], 0u, rb, 0u);
            return;
        }
        // {begin in the lid-ordered storage, m, first run, S = sum of the runs' lengths}
        // (half patterns: W = floor(m/2) + S; GCG: W = S - 1, the query itself excluded)
        cellq[i] = make_uint4(cell_start[r], m, rb, full ? wload[r] + 1 : wload[r] - m / 2);
    }
};

// Points gathered into lid (spatial) order, padded AoS, plus D' = the queue as an index
// array: qmap[D' position] = {lid-storage position, queue-order cell}.  With
// input_order the queue is the input order itself (the ablation's unsorted D).
// Two kernels, so the gather (the larger, depending only on the point sort) runs on a side
// stream while the main stream resolves runs, sorts cells and builds the queue.
__global__ void __launch_bounds__(kThreads) gather_kernel(const double *raw, uint64_t n, int dim, int pad,
                                                          const uint32_t *idx_sorted, double *pts, uint32_t *orig,
                                                          const uint32_t *ids) {
    uint64_t p = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (p >= n) return;
    const uint32_t src = idx_sorted[p];
    if (pad == 2 && dim == 2) {
        reinterpret_cast<double2 *>(pts)[p] = reinterpret_cast<const double2 *>(raw)[src];
    } else {
        for (int d = 0; d < pad; ++d) pts[p * pad + d] = d < dim ? raw[(uint64_t)src * dim + d] : 0.0;
    }
    orig[p] = ids ? ids[src] : src;  // partitioned index: the caller's global ids
}
__global__ void __launch_bounds__(kThreads) qmap_kernel(uint64_t n, const uint32_t *idx_sorted, const uint32_t *cellof,
                                                        const uint32_t *cell_start, const uint32_t *qbr,
                                                        const uint32_t *r2q, uint2 *qmap, int input_order) {
    uint64_t p = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (p >= n) return;
    const uint32_t r = cellof[p];
    const uint64_t dest = input_order ? (uint64_t)idx_sorted[p] : (uint64_t)qbr[r] + (p - cell_start[r]);
    qmap[dest] = make_uint2((uint32_t)p, r2q[r]);
}

// WorkQueue chunks: D' is cut into chunks of at most kChunk positions so that
// a chunk of a "big" cell (m >= big_min) never contains another cell, and consecutive small
// cells are packed together.  A boundary sits at
//   big cell:   every kChunk positions from the cell's first D' position;
//   small cell: every kChunk-aligned position, and where a big cell ended.
// Flags, their scan and the boundary scatter are one fused single-pass scan.
struct ChunkLoad {
    const uint2 *qmap;
    const uint4 *cellq;
    const uint32_t *qb;
    uint32_t big_min;
    __device__ unsigned operator()(uint64_t p) const {
        const uint32_t iq = qmap[p].y;
        const uint32_t m = cellq[iq].y, beg = qb[iq];
        bool f;
        if (m >= big_min)
            f = ((p - beg) % kChunk) == 0;
        else
            f = (p % kChunk) == 0 || (p == beg && p > 0 && cellq[qmap[p - 1].y].y >= big_min);
        return f ? 1u : 0u;
    }
};
// The same boundaries counted and written per queue CELL (cells are contiguous in D' in the
// SortByWL and cell orders): a scan over the M cells instead of a gather per D' position.
// Cell i = [beg, beg + m): a big cell has a boundary every kChunk positions from beg; a small
// one at its kChunk-aligned positions, plus beg itself when the previous cell was big.
struct CellChunkLoad {
    const uint4 *cellq;
    const uint32_t *qb;
    uint32_t big_min;
    __device__ unsigned operator()(uint64_t i) const {
        const uint32_t beg = qb[i], m = cellq[i].y;
        if (m == 0) return 0;  // halo cell of a partitioned index: not queued
        if (m >= big_min) return (m + kChunk - 1) / kChunk;
        unsigned c = (beg + m + kChunk - 1) / kChunk - (beg + kChunk - 1) / kChunk;
        if (beg % kChunk != 0 && i > 0 && cellq[i - 1].y >= big_min) ++c;
        return c;
    }
};
struct CellChunkStore {
    const uint4 *cellq;
    const uint32_t *qb;
    uint32_t big_min;
    uint32_t *chunks;
    __device__ void operator()(uint64_t i, unsigned ex, unsigned cnt) const {
        if (!cnt) return;
        const uint32_t beg = qb[i], m = cellq[i].y;
        if (m >= big_min) {
            for (unsigned j = 0; j < cnt; ++j) chunks[ex + j] = beg + j * kChunk;
            return;
        }
        unsigned o = ex;
        if (beg % kChunk != 0 && i > 0 && cellq[i - 1].y >= big_min) chunks[o++] = beg;
        for (uint32_t p = (beg + kChunk - 1) / kChunk * kChunk; p < beg + m; p += kChunk) chunks[o++] = p;
    }
};

struct ChunkStore {
    uint32_t *chunks;
    __device__ void operator()(uint64_t p, unsigned ex, unsigned flag) const {
        if (flag) chunks[ex] = (uint32_t)p;
    }
};
struct ChunkDone {
    uint64_t n;
    uint32_t *chunks;
    uint32_t *d_nc;
    __device__ void operator()(unsigned total) const {
        chunks[total] = (uint32_t)n;
        *d_nc = total;
    }
};

int bits_for(unsigned long long maxval) {
    int b = 0;
    while (b < 64 && (maxval >> b) != 0) ++b;
    return b;
}

}  // namespace

// ------------------------------------------------------------------------------ host

// Forward offsets of LID-UNICOMP: o in {-1,0,1}^dim whose row-major linear id
// delta is positive <=> first non-zero component is +1 (reading c7).
static int forward_offsets(int dim, std::vector<int8_t> &offs) {
    offs.clear();
    int total = 1;
    for (int d = 0; d < dim; ++d) total *= 3;
    for (int t = 0; t < total; ++t) {
        int8_t o[SJ_MAX_DIM];
        int v = t;
        for (int d = dim - 1; d >= 0; --d) {
            o[d] = (int8_t)(v % 3 - 1);
            v /= 3;
        }
        int first = 0;
        for (int d = 0; d < dim; ++d)
            if (o[d] != 0) {
                first = o[d];
                break;
            }
        if (first == 1)
            for (int d = 0; d < dim; ++d) offs.push_back(o[d]);
    }
    return (int)(offs.size() / (dim ? dim : 1));
}

int forward_offsets_public(int dim, int8_t *out, uint64_t cap) {
    if (dim < 1 || dim > SJ_MAX_DIM) return SJ_EINVAL;
    std::vector<int8_t> offs;
    int F = forward_offsets(dim, offs);
    if (out) {
        if (cap < offs.size()) return SJ_EINVAL;
        memcpy(out, offs.data(), offs.size());
    }
    return F;
}

void free_index(Index &ix, cudaStream_t s) {
    if (ix.block) {  // one allocation holds every array but (possibly) the runs
        dev_free(ix.block, s);
        if (ix.runs_own) dev_free(ix.runs, s);
    } else {
        dev_free(ix.d_meta, s);
        dev_free(ix.pts, s);
        dev_free(ix.orig, s);
        dev_free(ix.qmap, s);
        dev_free(ix.cellq, s);
        dev_free(ix.runs, s);
        dev_free(ix.cell_lid, s);
        dev_free(ix.chunks, s);
    }
    ix.block = nullptr;
    ix.runs_own = true;
    ix.d_meta = nullptr;
    ix.chunks = nullptr;
    ix.pts = nullptr;
    ix.orig = nullptr;
    ix.qmap = nullptr;
    ix.cellq = nullptr;
    ix.runs = nullptr;
    ix.cell_lid = nullptr;
}

// Rows of a cell pattern (see eval_row for the encoding):
//  * LID-UNICOMP (Alg. 3): the home row's +1 cell, then every o' in {-1,0,1}^(dim-1)
//    whose first non-zero component is +1, with last-dimension offsets -1..+1 -- exactly the
//    neighbours with a higher row-major linear id (reading c7);
//  * GCG (GPUCALCGLOBAL, Alg. 1): every o' with offsets -1..+1 -- the whole 3^n
//    neighbourhood including the home cell;
//  * UNICOMP ([18] as given in Alg. 2): a cell whose coordinate in dimension j is
//    odd compares to the neighbours that differ in dimension j, are free in the dimensions
//    before j and equal in the dimensions after it; one single-cell row per such offset.
static int pattern_rows(int dim, int pattern, std::vector<uint64_t> &rows) {
    rows.clear();
    auto pack = [dim](const int8_t *o, int lo, int hi, int pdim) {
        uint64_t p = 0;
        for (int d = 0; d < dim - 1; ++d) p |= (uint64_t)(uint8_t)o[d] << (8 * d);
        const unsigned meta = (unsigned)(lo + 1) | ((unsigned)(hi + 1) << 2) | ((unsigned)(pdim + 1) << 4);
        return p | ((uint64_t)meta << 56);
    };
    int total = 1;
    for (int d = 0; d < dim - 1; ++d) total *= 3;
    auto prefix = [dim](int t, int8_t *o) {
        for (int d = dim - 2; d >= 0; --d) {
            o[d] = (int8_t)(t % 3 - 1);
            t /= 3;
        }
    };
    if (pattern == SJ_PATTERN_UNICOMP) {
        int all = total * 3;
        for (int t = 0; t < all; ++t) {
            int8_t o[SJ_MAX_DIM] = {0};
            int v = t;
            for (int d = dim - 1; d >= 0; --d) {
                o[d] = (int8_t)(v % 3 - 1);
                v /= 3;
            }
            int j = -1;
            for (int d = dim - 1; d >= 0; --d)
                if (o[d] != 0) {
                    j = d;
                    break;
                }
            if (j < 0) continue;  // the home cell: circulant half scan in the kernel
            rows.push_back(pack(o, o[dim - 1], o[dim - 1], j));
        }
        return (int)rows.size();
    }
    if (pattern == SJ_PATTERN_GCG) {
        for (int t = 0; t < total; ++t) {
            int8_t o[SJ_MAX_DIM] = {0};
            prefix(t, o);
            rows.push_back(pack(o, -1, 1, -1));
        }
        return (int)rows.size();
    }
    int8_t zero[SJ_MAX_DIM] = {0};
    rows.push_back(pack(zero, 1, 1, -1));
    for (int t = 0; t < total; ++t) {
        int8_t o[SJ_MAX_DIM] = {0};
        prefix(t, o);
        int first = 0;
        for (int d = 0; d < dim - 1; ++d)
            if (o[d] != 0) {
                first = o[d];
                break;
            }
        if (first == 1) rows.push_back(pack(o, -1, 1, -1));
    }
    return (int)rows.size();
}

namespace {
// The build's temporaries: one stream-ordered block (Workspace: bump region + pre-zeroed
// region), freed on the stream at scope exit; requests that do not fit fall back to the pool.
struct Temps {
    cudaStream_t s;
    Workspace ws;
    void *block = nullptr;
    std::vector<void *> ptrs;  // fallback allocations
    explicit Temps(cudaStream_t st) : s(st) {}
    ~Temps() {
        for (void *p : ptrs) dev_free(p, s);
        dev_free(block, s);
    }
    int reserve(size_t bytes, size_t zbytes) {
        bytes = Workspace::round(bytes);
        zbytes = Workspace::round(zbytes);
        SJ_TRY(dev_alloc(&block, bytes + zbytes, s));
        ws.base = static_cast<char *>(block);
        ws.cap = bytes;
        ws.zbase = ws.base + bytes;
        ws.zcap = zbytes;
        SJ_CUDA_TRY(cudaMemsetAsync(ws.zbase, 0, zbytes, s));
        return SJ_OK;
    }
    template <class T>
    int alloc(T **p, size_t count) {
        if (void *q = ws.take(count * sizeof(T) + 16)) {
            *p = static_cast<T *>(q);
            return SJ_OK;
        }
        int rc = dev_alloc_t(p, count, s);
        if (rc == SJ_OK) ptrs.push_back(*p);
        return rc;
    }
    template <class T>
    int alloc_zero(T **p, size_t count) {  // zero-filled
        if (void *q = ws.take_zero(count * sizeof(T))) {
            *p = static_cast<T *>(q);
            return SJ_OK;
        }
        SJ_TRY(alloc(p, count));
        SJ_CUDA_TRY(cudaMemsetAsync(*p, 0, count * sizeof(T), s));
        return SJ_OK;
    }
};
}  // namespace

template <class K>
static int sort_points(Temps &tmp, K *ka, uint32_t *va, uint64_t n, int bits, cudaStream_t s, K **keys_sorted,
                       uint32_t **idx_sorted, uint32_t *hist0) {
    K *kb;
    uint32_t *vb;
    SJ_TRY(tmp.alloc(&kb, n));
    SJ_TRY(tmp.alloc(&vb, n));
    if constexpr (sizeof(K) == 4)
        SJ_TRY(radix_sort_u32(ka, va, kb, vb, n, bits, keys_sorted, idx_sorted, s, &tmp.ws, hist0, true));
    else
        SJ_TRY(radix_sort_u64(ka, va, kb, vb, n, bits, keys_sorted, idx_sorted, s, &tmp.ws, hist0, true));
    return SJ_OK;
}

template <class K>
static int rle(const K *ks, uint64_t n, uint32_t *cellof, unsigned long long *cell_lid, uint32_t *cell_start,
               uint64_t *d_M, cudaStream_t s, Workspace *ws, uint32_t *dense) {  // d_M: zero-filled
    return scan_fused(n, RleLoad<K>{ks}, RleStore<K>{ks, cellof, cell_lid, cell_start, dense}, s,
                      RleDone{n, cell_start, d_M}, ws);
}

int build_index(Index &ix, const double *d_raw, uint64_t n, int dim, double eps, cudaStream_t s, cudaEvent_t ev0,
                cudaEvent_t ev1, float *ms, const BuildPart *part, uint64_t *tail_mail, const BuildSide *side,
                unsigned long long *zero_ctr, int zero_words) {
    Temps tmp(s);
    // on every exit, the main stream waits for the side stream before the temporaries are freed
    // (stream-ordered, on s) -- also on the error returns
    struct SideJoin {
        const BuildSide *side;
        cudaStream_t s;
        ~SideJoin() {
            if (side && cudaEventRecord(side->ej, side->s2) == cudaSuccess) cudaStreamWaitEvent(s, side->ej, 0);
        }
    } side_join{side, s};
    ix.n = n;
    const uint64_t nq = part ? part->n_query : n;  // queries: input points [0, nq)
    ix.n_query = nq;
    ix.dim = dim;
    ix.pad = dim == 1 ? 1 : ((dim + 1) & ~1);
    ix.eps = eps;
    ix.e2 = eps * eps;                 // e2 = fl(eps*eps)
    ix.w = eps * (1.0 + 0x1p-20);      // reading c5
    if (ev0) SJ_CUDA_TRY(cudaEventRecord(ev0, s));

    // pinned mailbox (from the process-wide pool) for the two host round trips
    static_assert(sizeof(BBox) <= 256, "bbox");
    void *mail = pinned_acquire();
    if (!mail) return SJ_ENOMEM;
    struct MailFree {
        void *p;
        ~MailFree() { pinned_release(p); }
    } mail_free{mail};

    // One workspace for every temporary (upper bounds from n; M <= n): sort keys/values
    // (8-byte keys at most), the per-point and per-cell arrays, the radix histograms; the
    // zeroed region holds the counters and every scan's look-back status words.
    {
        const uint64_t tiles = (n + 2047) / 2048 + 1;
        const size_t bytes = (size_t)n * 100 + (size_t)2 * 256 * 4 * tiles + 64 * 512;
        const size_t zbytes = (size_t)8 * (12 * tiles + 64) + 48 * 512;
        SJ_TRY(tmp.reserve(bytes, zbytes));
    }

    // ---- a2: bounding box + non-finite check; its last block derives the grid geometry (a3)
    BBox *d_bb;
    GeomDev *d_geo;
    SJ_TRY(tmp.alloc_zero(&d_bb, 1));
    SJ_TRY(tmp.alloc(&d_geo, 1));
    GeomArgs ga{};
    ga.w = ix.w;
    if (part) {
        ga.has_origin = 1;
        for (int d = 0; d < dim; ++d) ga.origin[d] = part->origin[d];
    }
    ga.dev = d_geo;
    // zero-copy: the last block writes the geometry into the pinned mailbox (the device alias of
    // the same pages), and the host waits on its flag instead of a copy + stream synchronisation
    volatile GeomDev *h_geo = static_cast<volatile GeomDev *>(mail);
    // (unified addressing: the device alias of pinned host memory is the host pointer itself --
    // checked once per process, then used directly)
    static const int uva = [&] {
        void *d_alias = nullptr;
        const bool ok = cudaHostGetDevicePointer(&d_alias, mail, 0) == cudaSuccess && d_alias == mail;
        if (!ok) cudaGetLastError();
        return ok ? 1 : 0;
    }();
    const bool zero_copy = uva != 0;
    ga.host = zero_copy ? static_cast<GeomDev *>(mail) : nullptr;
    ga.epoch = next_epoch();
    h_geo->flag = 0;
    {
        // 2 * threads must be a multiple of dim (see bbox_kernel): blocks a multiple of dim
        const uint64_t pairs = n * (uint64_t)dim / 2;
        unsigned blocks = (unsigned)std::min<uint64_t>((pairs + kThreads * 8 - 1) / (kThreads * 8), 148ull * 8);
        blocks = std::max(1u, blocks);
        blocks = ((blocks + dim - 1) / dim) * dim;
        bbox_kernel<<<blocks, kThreads, 0, s>>>(d_raw, n, dim, d_bb, ga);
        note_launch();
    }
    SJ_CUDA_TRY(cudaGetLastError());
    if (!zero_copy) SJ_CUDA_TRY(cudaMemcpyAsync(mail, d_geo, sizeof(GeomDev), cudaMemcpyDeviceToHost, s));
    // a3: cell ids, queued at once (they read the device copy of the geometry); 32- or 64-bit keys
    uint32_t *keys32, *vals0;
    unsigned long long *keys64;
    SJ_TRY(tmp.alloc(&keys32, n));
    SJ_TRY(tmp.alloc(&keys64, n));
    SJ_TRY(tmp.alloc(&vals0, n));
    const uint32_t ntiles = (uint32_t)((n + kRadixTileKeys - 1) / kRadixTileKeys);
    uint32_t *hist0;  // the point sort's first-pass tile histogram, counted by the cell-id kernel
    SJ_TRY(tmp.alloc(&hist0, (uint64_t)256 * ntiles));
    switch (dim) {
#define SJ_CELL_ID(D)                                                                                          \
    case D:                                                                                                    \
        cell_id_kernel<D><<<ntiles, CellIdThreads<D>::value, 0, s>>>(d_raw, n, d_geo, keys32, keys64, ga, hist0, \
                                                                     ntiles);                              \
        break;
        SJ_CELL_ID(1) SJ_CELL_ID(2) SJ_CELL_ID(3) SJ_CELL_ID(4) SJ_CELL_ID(5) SJ_CELL_ID(6) SJ_CELL_ID(7) SJ_CELL_ID(8)
#undef SJ_CELL_ID
    }
    note_launch();
    SJ_CUDA_TRY(cudaGetLastError());
    if (zero_copy) {
        SJ_TRY(wait_flag(&h_geo->flag, ga.epoch, s));
    } else {
        SJ_CUDA_TRY(cudaStreamSynchronize(s));
    }
    debug_mark("build: geometry");
    GeomDev g;
    memcpy(&g, const_cast<const GeomDev *>(h_geo), sizeof g);
    if (g.err == 1) {
        set_error("sj_create: non-finite coordinate");
        return SJ_EINVAL;
    }
    if (g.err == 2) {
        set_error("sj_create_part: a coordinate in dimension %d lies below the grid origin", g.errdim);
        return SJ_EINVAL;
    }
    if (g.err == 3) {
        set_error("sj_create: grid too large in dimension %d (%.3g cells >= 2^30)", g.errdim, g.errq);
        return SJ_EGRID;
    }
    if (g.err) {
        set_error("sj_create: grid too large (prod nc_d >= 2^64)");
        return SJ_EGRID;
    }
    unsigned long long ncells_total = 1;
    for (int d = 0; d < dim; ++d) {
        ix.mins[d] = g.mins[d];
        ix.nc[d] = g.nc[d];
        ix.stride[d] = g.stride[d];
        ncells_total *= g.nc[d];
    }
    ix.key_bits = g.key_bits;

    // ---- a3 + a4 + a5: cell ids, point -> cell sort, compaction of the non-empty cells
    uint32_t *idx_sorted = nullptr;
    uint32_t *cellof;
    unsigned long long *cell_lid;
    uint32_t *cell_start;
    uint64_t *d_M;
    SJ_TRY(tmp.alloc(&cellof, n));
    SJ_TRY(tmp.alloc(&cell_lid, n));
    SJ_TRY(tmp.alloc(&cell_start, n + 1));
    SJ_TRY(tmp.alloc_zero(&d_M, 1));
    // lid -> rank lookup: a dense table when prod(nc) is small, else a hash table
    Lookup L{};
    const bool dense = ncells_total <= (1ull << 27) && ncells_total <= 64ull * n + 4096;
    ix.lookup_hash = dense ? 0 : 1;
    // the dense table is cleared on the side stream while the points sort, and filled by the
    // compaction's store (a5) -- no kernel of its own
    uint32_t *tab = nullptr;
    if (dense) {
        SJ_TRY(tmp.alloc(&tab, ncells_total));
        cudaStream_t st = side ? side->s2 : s;
        if (side) {
            SJ_CUDA_TRY(cudaEventRecord(side->ea, s));
            SJ_CUDA_TRY(cudaStreamWaitEvent(st, side->ea, 0));
        }
        SJ_CUDA_TRY(cudaMemsetAsync(tab, 0xFF, ncells_total * sizeof(uint32_t), st));
        if (side) {
            SJ_CUDA_TRY(cudaEventRecord(side->eq, st));
        }
        L.dense = tab;
    }
    if (ix.key_bits <= 32) {
        uint32_t *ks;
        SJ_TRY(sort_points<uint32_t>(tmp, keys32, vals0, n, ix.key_bits, s, &ks, &idx_sorted, hist0));
        if (dense && side) SJ_CUDA_TRY(cudaStreamWaitEvent(s, side->eq, 0));
        SJ_TRY(rle<uint32_t>(ks, n, cellof, cell_lid, cell_start, d_M, s, &tmp.ws, tab));
    } else {
        uint64_t *ks;
        SJ_TRY(sort_points<uint64_t>(tmp, reinterpret_cast<uint64_t *>(keys64), vals0, n, ix.key_bits, s, &ks,
                                     &idx_sorted, hist0));
        if (dense && side) SJ_CUDA_TRY(cudaStreamWaitEvent(s, side->eq, 0));
        SJ_TRY(rle<uint64_t>(ks, n, cellof, cell_lid, cell_start, d_M, s, &tmp.ws, tab));
    }
    // the gather of the points into cell order needs only the point sort: side stream
    // the index arrays: one allocation, each array at its bound (M <= n cells); the slot-layout
    // runs (n * rows entries, up to 4 GB) join it when they fit the slot bound
    std::vector<uint64_t> rows;
    const int R = pattern_rows(dim, ix.pattern, rows);
    const bool slots = (uint64_t)n * R * sizeof(uint2) <= (4ull << 30);
    {
        auto al = [](size_t b) { return (b + 255) & ~(size_t)255; };
        const size_t b_pts = al(n * ix.pad * sizeof(double)), b_orig = al(n * sizeof(uint32_t)),
                     b_qmap = al(n * sizeof(uint2)), b_cellq = al(n * sizeof(uint4)),
                     b_lid = al(n * sizeof(uint64_t)), b_chunks = al((n + 1 + kChunkPad) * sizeof(uint32_t)),
                     b_meta = al(4 * sizeof(uint32_t)),
                     b_runs = slots ? al(((uint64_t)n * R + 2) * sizeof(uint2)) : 0;
        char *blk = nullptr;
        SJ_TRY(dev_alloc(reinterpret_cast<void **>(&blk),
                         b_pts + b_orig + b_qmap + b_cellq + b_lid + b_chunks + b_meta + b_runs, s));
        ix.block = blk;
        ix.pts = reinterpret_cast<double *>(blk);
        blk += b_pts;
        ix.orig = reinterpret_cast<uint32_t *>(blk);
        blk += b_orig;
        ix.qmap = reinterpret_cast<uint2 *>(blk);
        blk += b_qmap;
        ix.cellq = reinterpret_cast<uint4 *>(blk);
        blk += b_cellq;
        ix.cell_lid = reinterpret_cast<uint64_t *>(blk);
        blk += b_lid;
        ix.chunks = reinterpret_cast<uint32_t *>(blk);
        blk += b_chunks;
        ix.d_meta = reinterpret_cast<uint32_t *>(blk);
        blk += b_meta;
        if (slots) {
            ix.runs = reinterpret_cast<uint2 *>(blk);
            ix.runs_cap = (uint64_t)n * R + 2;
            ix.runs_own = false;
        }
    }
    cudaStream_t sg = side ? side->s2 : s;
    if (side) {
        SJ_CUDA_TRY(cudaEventRecord(side->ea, s));
        SJ_CUDA_TRY(cudaStreamWaitEvent(sg, side->ea, 0));
    }
    gather_kernel<<<grid_for(n), kThreads, 0, sg>>>(d_raw, n, dim, ix.pad, idx_sorted, ix.pts, ix.orig,
                                                     part ? part->d_ids : nullptr);
    note_launch();
    if (side) SJ_CUDA_TRY(cudaEventRecord(side->eg, sg));
    if (!dense) {
        unsigned long long cap = 1024;
        while (cap < 2 * n) cap <<= 1;
        unsigned long long *hk;
        uint32_t *hv;
        SJ_TRY(tmp.alloc(&hk, cap));
        SJ_TRY(tmp.alloc(&hv, cap));
        SJ_CUDA_TRY(cudaMemsetAsync(hk, 0xFF, cap * sizeof(unsigned long long), s));
        hash_insert_kernel<<<grid_for(n), kThreads, 0, s>>>(cell_lid, d_M, hk, hv, cap - 1);
        note_launch();
        L.hkeys = hk;
        L.hvals = hv;
        L.hmask = cap - 1;
    }
    SJ_CUDA_TRY(cudaGetLastError());

    // ---- a6 + a7: forward runs, workload, D_alg (rows R: above)
    // the rows resolved against this grid: linear-id delta, edge masks, meta (eval_row)
    std::vector<RowEnt> ents(R);
    for (int j = 0; j < R; ++j) {
        const uint64_t off = rows[j];
        const unsigned meta = (unsigned)(off >> 56);
        long long delta = (long long)(meta & 3u) - 1;  // lo
        unsigned nm = 0;
        for (int d = 0; d < dim - 1; ++d) {
            const int o = (int)(signed char)((off >> (8 * d)) & 0xFF);
            delta += (long long)o * (long long)ix.stride[d];
            if (o < 0) nm |= 1u << d;
            if (o > 0) nm |= 1u << (8 + d);
        }
        ents[j] = RowEnt{delta, nm, meta};
    }
    RowEnt *d_rows;
    SJ_TRY(tmp.alloc(&d_rows, R));
    const size_t rbytes = R * sizeof(RowEnt);
    if (rbytes <= 3072) {  // through the pinned mailbox: a truly asynchronous copy
        memcpy((char *)mail + 1024, ents.data(), rbytes);
        SJ_CUDA_TRY(cudaMemcpyAsync(d_rows, (char *)mail + 1024, rbytes, cudaMemcpyHostToDevice, s));
    } else {  // pageable: staged by the driver before the call returns
        SJ_CUDA_TRY(cudaMemcpyAsync(d_rows, ents.data(), rbytes, cudaMemcpyHostToDevice, s));
    }
    FwdGeom fg{};
    fg.dim = dim;
    fg.rows = R;
    fg.small = ncells_total <= 0xFFFFFFFFull ? 1 : 0;
    fg.full = ix.pattern == SJ_PATTERN_GCG ? 1 : 0;
    fg.rows_ent = d_rows;
    unsigned int *d_mixed = nullptr;
    if (part) {
        SJ_TRY(tmp.alloc_zero(&d_mixed, 1));
        fg.idx = idx_sorted;
        fg.nq = (uint32_t)nq;
        fg.mixed = d_mixed;
    }
    for (int d = 0; d < dim; ++d) {
        fg.nc[d] = ix.nc[d];
        fg.stride[d] = ix.stride[d];
    }
    uint32_t *rcnt, *wload;
    BuildTotals *d_tot;
    SJ_TRY(tmp.alloc(&rcnt, n + 1));
    SJ_TRY(tmp.alloc(&wload, n));
    SJ_TRY(tmp.alloc_zero(&d_tot, 1));
    const bool wide = R >= 16;  // one warp per cell for many rows
    // Slot layout: cell r's runs at r * R, written by the counting pass itself -- no scan, no
    // second pass, no third host round trip; the array is sized by n >= M before M is known
    // (up to 4 GB of the 180 GB: every configuration, 6-D at 2M points included: 1.95 GB).
    // (slots: the runs are part of the index block, allocated above)
    // grid-stride kernels (M is on the device): at most 8 resident blocks per SM
    int nsm = 148;
    {
        int dev = 0;
        if (cudaGetDevice(&dev) == cudaSuccess) cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev);
    }
    auto runs_grid = [&](uint64_t cells, int lpc) {
        return std::min<unsigned>(grid_for(cells * (uint64_t)lpc), (unsigned)nsm * 8u);
    };
    volatile unsigned long long *h_pub = reinterpret_cast<volatile unsigned long long *>((char *)mail + 768);
    TotalsPub pub{};
    if (zero_copy) {
        pub.host = reinterpret_cast<unsigned long long *>((char *)mail + 768);
        pub.epoch = next_epoch();
        h_pub[5] = 0;
    }
    // a8's SortByWL keys and values, written by the counting pass (M <= n cells)
    uint32_t *wk, *wv;
    SJ_TRY(tmp.alloc(&wk, n));
    SJ_TRY(tmp.alloc(&wv, n));
    // (per dimensionality: the counting pass's per-cell loops are the build's ALU work)
#define SJ_RUNS_COUNT(D, LPC)                                                                                  \
    runs_kernel<D, false, LPC><<<runs_grid(n, LPC), kThreads, 0, s>>>(cell_lid, cell_start, d_M, fg, L, rcnt,     \
                                                                      wload, nullptr, slots ? ix.runs : nullptr, \
                                                                      d_tot, pub, wk, wv)
#define SJ_RUNS_COUNT_D(D)         \
    case D:                        \
        if (wide)                  \
            SJ_RUNS_COUNT(D, 32);  \
        else                       \
            SJ_RUNS_COUNT(D, 1);   \
        break;
    switch (dim) { SJ_RUNS_COUNT_D(1) SJ_RUNS_COUNT_D(2) SJ_RUNS_COUNT_D(3) SJ_RUNS_COUNT_D(4) SJ_RUNS_COUNT_D(5)
                   SJ_RUNS_COUNT_D(6) SJ_RUNS_COUNT_D(7) SJ_RUNS_COUNT_D(8) }
#undef SJ_RUNS_COUNT_D
#undef SJ_RUNS_COUNT
    note_launch();
    SJ_CUDA_TRY(cudaGetLastError());
    uint32_t *rbegin = nullptr;
    if (!slots) SJ_TRY(tmp.alloc(&rbegin, n + 1));
    // host wait 2: M, plus the workload totals (max W sizes the SortByWL keys, D_alg)
    uint64_t M;
    BuildTotals bt{};
    unsigned int mixed = 0;
    if (zero_copy) {  // published by the counting pass's last block
        SJ_TRY(wait_flag(reinterpret_cast<volatile unsigned *>(h_pub + 5), pub.epoch, s));
        M = h_pub[0];
        bt.E = h_pub[1];
        bt.dist_calcs = h_pub[2];
        bt.max_w = (unsigned)h_pub[3];
        mixed = (unsigned)h_pub[4];
    } else {
        SJ_CUDA_TRY(cudaMemcpyAsync(mail, d_M, sizeof(uint64_t), cudaMemcpyDeviceToHost, s));
        SJ_CUDA_TRY(cudaMemcpyAsync((char *)mail + 64, d_tot, sizeof(BuildTotals), cudaMemcpyDeviceToHost, s));
        if (d_mixed)
            SJ_CUDA_TRY(cudaMemcpyAsync((char *)mail + 128, d_mixed, sizeof(unsigned int), cudaMemcpyDeviceToHost, s));
        SJ_CUDA_TRY(cudaStreamSynchronize(s));
        memcpy(&M, mail, sizeof M);
        memcpy(&bt, (char *)mail + 64, sizeof bt);
        if (d_mixed) memcpy(&mixed, (char *)mail + 128, sizeof mixed);
    }
    debug_mark("build: sort+rle+runcount wait");
    ix.n_cells = M;
    if (d_mixed) {
        if (mixed) {
            set_error("sj_create_part: a grid cell holds both query and halo points (partition the data by "
                      "whole cell columns)");
            return SJ_EINVAL;
        }
    }
    ix.dist_calcs = bt.dist_calcs;
    ix.max_w = bt.max_w;
    // persistent device words {n_chunks, E}: the join reads the chunk count from here (a
    // device-sized launch needs no host round trip after the build)
    // (d_meta: part of the index block)
    uint32_t *d_E32 = ix.d_meta + 1;
    if (!slots) SJ_TRY(scan_exclusive_u32(rcnt, rbegin, M + 1, d_E32, s, &tmp.ws));
    // The runs array is allocated at its bound M * rows when that is small (every 1-D..4-D
    // index), so the run total E is read with the final round trip instead of a third one.
    const uint64_t runs_bound = M * (uint64_t)R + 2;
    const bool bounded = slots || runs_bound * sizeof(uint2) <= (256ull << 20);
    uint64_t E = 0;
    if (slots) {
        E = bt.E;
        ix.n_runs = E;
        ix.runs_len = M * (uint64_t)R;
    } else if (!bounded) {
        SJ_CUDA_TRY(cudaMemcpyAsync((char *)mail + 256, d_E32, sizeof(uint32_t), cudaMemcpyDeviceToHost, s));
        SJ_CUDA_TRY(cudaStreamSynchronize(s));
        debug_mark("build: scan sync");
        uint32_t E32;
        memcpy(&E32, (char *)mail + 256, sizeof E32);
        E = E32;
        ix.n_runs = E;
    }
    if (!slots) {
        ix.runs_cap = bounded ? runs_bound : E + 2;
        SJ_TRY(dev_alloc_t(&ix.runs, ix.runs_cap, s));
    }
    if (slots) {
        // (the counting pass wrote them)
    } else {
#define SJ_RUNS_FILL(D, LPC)                                                                                   \
    runs_kernel<D, true, LPC><<<runs_grid(M, LPC), kThreads, 0, s>>>(cell_lid, cell_start, d_M, fg, L, nullptr,  \
                                                                     nullptr, rbegin, ix.runs, nullptr,        \
                                                                     TotalsPub{}, nullptr, nullptr)
#define SJ_RUNS_FILL_D(D)         \
    case D:                       \
        if (wide)                 \
            SJ_RUNS_FILL(D, 32);  \
        else                      \
            SJ_RUNS_FILL(D, 1);   \
        break;
        switch (dim) { SJ_RUNS_FILL_D(1) SJ_RUNS_FILL_D(2) SJ_RUNS_FILL_D(3) SJ_RUNS_FILL_D(4) SJ_RUNS_FILL_D(5)
                       SJ_RUNS_FILL_D(6) SJ_RUNS_FILL_D(7) SJ_RUNS_FILL_D(8) }
#undef SJ_RUNS_FILL_D
#undef SJ_RUNS_FILL
        note_launch();
    }
    SJ_CUDA_TRY(cudaGetLastError());

    // ---- a8: SortByWL over cells -> D' (queue of points in non-increasing W)
    uint32_t *wk2, *wv2, *qorder_keys, *qorder;
    SJ_TRY(tmp.alloc(&wk2, M));
    SJ_TRY(tmp.alloc(&wv2, M));
    if (ix.order == SJ_ORDER_WORKLOAD) {
        SJ_TRY(radix_sort_u32(wk, wv, wk2, wv2, M, bits_for(part ? ix.max_w + 1ull : ix.max_w), &qorder_keys, &qorder,
                              s, &tmp.ws));
    } else {  // ablation orders: cells stay in lid order (no SortByWL)
        qorder_keys = wk;
        qorder = wv;
    }
    uint32_t *qb;
    SJ_TRY(tmp.alloc(&qb, M));

    // ---- final arrays
    // (cellq, cell_lid, qmap: part of the index block)
    uint32_t *r2q, *qbr;
    SJ_TRY(tmp.alloc(&r2q, M));
    SJ_TRY(tmp.alloc(&qbr, M));
    SJ_TRY(scan_fused(M, QueueLoad{qorder, cell_start},
                      QueueStore{qorder, cell_start, rbegin, (uint32_t)R, wload, cell_lid, fg.full, ix.cellq, r2q, qbr,
                                 qb, ix.cell_lid, part ? idx_sorted : nullptr, (uint32_t)nq},
                      s, NoDone(), &tmp.ws));
    // D' (qmap): after the cells' queue positions; on the side stream too (the chunk scan below
    // needs it only in input order), the main stream waits for it before the build ends
    if (side) {
        SJ_CUDA_TRY(cudaEventRecord(side->ea, s));
        SJ_CUDA_TRY(cudaStreamWaitEvent(sg, side->ea, 0));
    }
    qmap_kernel<<<grid_for(n), kThreads, 0, sg>>>(n, idx_sorted, cellof, cell_start, qbr, r2q, ix.qmap,
                                                  ix.order == SJ_ORDER_INPUT ? 1 : 0);
    note_launch();
    if (side) {
        SJ_CUDA_TRY(cudaEventRecord(side->eq, sg));
        if (ix.order == SJ_ORDER_INPUT) SJ_CUDA_TRY(cudaStreamWaitEvent(s, side->eq, 0));
    }
    SJ_CUDA_TRY(cudaGetLastError());

    // ---- WorkQueue chunks over D'
    uint32_t *d_nc = ix.d_meta;
    // (chunks: part of the index block)
    // in input order a cell's points are scattered: no chunk may claim a cell
    const uint32_t big_min = ix.order == SJ_ORDER_INPUT ? 0xFFFFFFFFu : kBigCell;
    if (ix.order == SJ_ORDER_INPUT)
        SJ_TRY(scan_fused(n, ChunkLoad{ix.qmap, ix.cellq, qb, big_min}, ChunkStore{ix.chunks}, s,
                          ChunkDone{n, ix.chunks, d_nc}, &tmp.ws));
    else
        SJ_TRY(scan_fused(M, CellChunkLoad{ix.cellq, qb, big_min}, CellChunkStore{ix.cellq, qb, big_min, ix.chunks}, s,
                          ChunkDone{nq, ix.chunks, d_nc}, &tmp.ws));
    if (tail_mail) tail_mail[0] = tail_mail[1] = 0;
    chunk_pad_kernel<<<kChunkPad / kThreads, kThreads, 0, s>>>(
        ix.chunks, d_nc, ix.order == SJ_ORDER_INPUT ? (uint32_t)n : (uint32_t)nq,
        (tail_mail && zero_copy) ? reinterpret_cast<unsigned long long *>(tail_mail) : nullptr, zero_ctr,
        zero_ctr ? zero_words : 0);
    note_launch();
    if (side) {
        SJ_CUDA_TRY(cudaStreamWaitEvent(s, side->eq, 0));  // points, ids and D' complete
        // the caller's points are read by the gather last: done before sj_create returns
        SJ_CUDA_TRY(cudaEventSynchronize(side->eg));
    }
    if (tail_mail) {
        // no final round trip: {n_chunks, E} land in the caller's pinned mailbox (n_chunks written
        // by the pad kernel when the mailbox is device-mapped), read once the stream has passed
        // ev1 (the join reads n_chunks on the device meanwhile)
        if (!zero_copy) SJ_CUDA_TRY(cudaMemcpyAsync(tail_mail, d_nc, sizeof(uint32_t), cudaMemcpyDeviceToHost, s));
        if (bounded && !slots)  // E from the scan of the counts
            SJ_CUDA_TRY(cudaMemcpyAsync(tail_mail + 1, d_E32, sizeof(uint32_t), cudaMemcpyDeviceToHost, s));
        else
            tail_mail[1] = E;
        if (ev1) SJ_CUDA_TRY(cudaEventRecord(ev1, s));
        return SJ_OK;
    }
    SJ_CUDA_TRY(cudaMemcpyAsync((char *)mail + 512, d_nc, sizeof(uint32_t), cudaMemcpyDeviceToHost, s));
    if (bounded && !slots)
        SJ_CUDA_TRY(cudaMemcpyAsync((char *)mail + 256, d_E32, sizeof(uint32_t), cudaMemcpyDeviceToHost, s));
    if (ev1) SJ_CUDA_TRY(cudaEventRecord(ev1, s));
    debug_mark("build: tail issued");
    SJ_CUDA_TRY(cudaStreamSynchronize(s));
    debug_mark("build: final sync");
    if (ms && ev0 && ev1) SJ_CUDA_TRY(cudaEventElapsedTime(ms, ev0, ev1));
    uint32_t nchunks;
    memcpy(&nchunks, (char *)mail + 512, sizeof nchunks);
    ix.n_chunks = nchunks;
    if (bounded && !slots) {
        uint32_t E32;
        memcpy(&E32, (char *)mail + 256, sizeof E32);
        ix.n_runs = E32;
    }
    return SJ_OK;
}

}  // namespace sj
