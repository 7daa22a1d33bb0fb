// partition.cu -- the slab partition of a multi-GPU join:
// the arithmetic of cutting the global eps-grid into slabs of whole dimension-0 cell columns,
// on the device, behind the C ABI (sj_part_*), so the Python side only issues the collectives
// (all-reduce of the bounds and of the column histogram, all-to-all of the packed rows).
//
//   column  c(x) = floor(fl(fl(x_0 - origin_0) / w)), w = fl(eps (1 + 2^-20))   (readings c5, c6:
//           the same RN intrinsics as the build's cell ids, so the cut never splits a cell)
//   owner   of column c: min(world - 1, floor(start_c * world / total)), start_c = points in the
//           columns before c (global histogram): slabs of whole columns balanced by points
//   halo    a point of column c >= 1 whose owner differs from owner(c - 1) is also sent to
//           owner(c - 1): LID-UNICOMP's forward cells are at most one column ahead (Alg. 3)
//
// Rows are packed per destination rank in ascending rank order, input order inside a rank
// (a stable radix sort of the destination keys), ready for all_to_all_single.
#include <algorithm>
#include <cmath>
#include <cstring>
#include <vector>

#include "sj_internal.cuh"

namespace sj {

namespace {

constexpr int kT = 256;

inline unsigned blocks_for(uint64_t n) { return (unsigned)std::max<uint64_t>(1, std::min<uint64_t>((n + kT - 1) / kT, 148ull * 16)); }

// ordered 64-bit keys of doubles: min/max with integer atomics (exact)
__device__ __forceinline__ unsigned long long okey(double x) {
    const unsigned long long b = (unsigned long long)__double_as_longlong(x);
    return (b >> 63) ? ~b : (b | 0x8000000000000000ull);
}
// per-dimension min / max of n points (grid-stride); out[0..dim) = max of ~okey (min), out[dim..2dim) = max okey
__global__ void __launch_bounds__(kT) part_bounds_kernel(const double *p, uint64_t n, int dim,
                                                         unsigned long long *out, unsigned *bad) {
    unsigned long long lo[SJ_MAX_DIM], hi[SJ_MAX_DIM];
#pragma unroll
    for (int d = 0; d < SJ_MAX_DIM; ++d) lo[d] = hi[d] = 0;
    bool nonfinite = false;
    for (uint64_t i = (uint64_t)blockIdx.x * kT + threadIdx.x; i < n; i += (uint64_t)gridDim.x * kT) {
#pragma unroll
        for (int d = 0; d < SJ_MAX_DIM; ++d)
            if (d < dim) {
                const double x = p[i * dim + d];
                nonfinite |= !isfinite(x);
                const unsigned long long k = okey(x);
                lo[d] = max(lo[d], ~k);
                hi[d] = max(hi[d], k);
            }
    }
#pragma unroll
    for (int d = 0; d < SJ_MAX_DIM; ++d)
        if (d < dim) {
#pragma unroll
            for (int o = 16; o > 0; o >>= 1) {
                lo[d] = max(lo[d], __shfl_xor_sync(0xffffffffu, lo[d], o));
                hi[d] = max(hi[d], __shfl_xor_sync(0xffffffffu, hi[d], o));
            }
            if ((threadIdx.x & 31) == 0) {
                if (lo[d]) atomicMax(out + d, lo[d]);
                if (hi[d]) atomicMax(out + dim + d, hi[d]);
            }
        }
    if (__any_sync(0xffffffffu, nonfinite) && (threadIdx.x & 31) == 0) atomicOr(bad, 1u);
}

__device__ __forceinline__ unsigned long long column_of(double x0, double o0, double w) {
    return __double2ull_rd(__ddiv_rn(__dsub_rn(x0, o0), w));  // x0 >= o0: floor of a non-negative
}

__global__ void __launch_bounds__(kT) part_hist_kernel(const double *p, uint64_t n, int dim, double o0, double w,
                                                       uint64_t ncol, unsigned long long *hist, unsigned *bad) {
    for (uint64_t i = (uint64_t)blockIdx.x * kT + threadIdx.x; i < n; i += (uint64_t)gridDim.x * kT) {
        const double x = p[i * dim];
        if (!(x >= o0)) {  // below the origin (or NaN)
            atomicOr(bad, 2u);
            continue;
        }
        const unsigned long long c = column_of(x, o0, w);
        if (c >= ncol) {
            atomicOr(bad, 4u);
            continue;
        }
        atomicAdd(hist + c, 1ull);
    }
}

// owner of every column from the exclusive scan of the global histogram
__global__ void __launch_bounds__(kT) part_owner_kernel(const unsigned long long *start, uint64_t ncol,
                                                        const unsigned long long *total, unsigned world,
                                                        uint32_t *owner) {
    const uint64_t c = (uint64_t)blockIdx.x * kT + threadIdx.x;
    if (c >= ncol) return;
    const unsigned long long t = *total;
    const unsigned long long r = t ? (start[c] * (unsigned long long)world) / t : 0ull;
    owner[c] = (uint32_t)min(r, (unsigned long long)(world - 1u));
}

// per point: destination of its own row, and of its halo copy (world = none)
__global__ void __launch_bounds__(kT) part_route_kernel(const double *p, uint64_t n, int dim, double o0, double w,
                                                        uint64_t ncol, const uint32_t *owner, unsigned world,
                                                        uint32_t *okey_, uint32_t *hkey, uint32_t *idx0,
                                                        uint32_t *idx1, unsigned long long *counts, unsigned *bad) {
    __shared__ unsigned long long sc[2 * 65];
    const bool small = world <= 64;
    for (int k = threadIdx.x; k < 2 * 65; k += kT) sc[k] = 0;
    __syncthreads();
    for (uint64_t i = (uint64_t)blockIdx.x * kT + threadIdx.x; i < n; i += (uint64_t)gridDim.x * kT) {
        const double x = p[i * dim];
        unsigned long long c = (x >= o0) ? column_of(x, o0, w) : ncol;
        if (c >= ncol) {
            atomicOr(bad, 4u);
            c = 0;
        }
        const uint32_t own = owner[c];
        const uint32_t prev = c ? owner[c - 1] : own;
        const uint32_t h = prev != own ? prev : world;
        okey_[i] = own;
        hkey[i] = h;
        idx0[i] = idx1[i] = (uint32_t)i;
        if (small) {
            atomicAdd(sc + own, 1ull);
            if (h < world) atomicAdd(sc + 65 + h, 1ull);
        } else {
            atomicAdd(counts + own, 1ull);
            if (h < world) atomicAdd(counts + world + h, 1ull);
        }
    }
    __syncthreads();
    if (small)
        for (unsigned k = threadIdx.x; k < world; k += kT) {
            if (sc[k]) atomicAdd(counts + k, sc[k]);
            if (sc[65 + k]) atomicAdd(counts + world + k, sc[65 + k]);
        }
}

// rows in sorted order -> the send buffers
__global__ void __launch_bounds__(kT) part_pack_kernel(const double *p, const uint32_t *ids, uint64_t rows, int dim,
                                                       const uint32_t *order, double *out_p, uint32_t *out_ids) {
    for (uint64_t k = (uint64_t)blockIdx.x * kT + threadIdx.x; k < rows; k += (uint64_t)gridDim.x * kT) {
        const uint64_t i = order[k];
        for (int d = 0; d < dim; ++d) out_p[k * dim + d] = p[i * dim + d];
        out_ids[k] = ids ? ids[i] : (uint32_t)i;
    }
}

int bits_of(unsigned long long v) {
    int b = 0;
    while (b < 64 && (v >> b)) ++b;
    return std::max(b, 1);
}

struct Tmp {  // stream-ordered temporaries freed at scope exit
    cudaStream_t s;
    std::vector<void *> ptrs;
    template <class T>
    int get(T **p, size_t count) {
        SJ_TRY(dev_alloc_t(p, count, s));
        ptrs.push_back(*p);
        return SJ_OK;
    }
    ~Tmp() {
        for (void *q : ptrs) dev_free(q, s);
    }
};

int check_points(const double *p, uint64_t n, int dim) {
    if ((n && !p) || dim < 1 || dim > SJ_MAX_DIM || n >= (1ull << 32)) {
        set_error("sj_part: invalid argument (points=%p n=%llu dim=%d)", (const void *)p, (unsigned long long)n, dim);
        return SJ_EINVAL;
    }
    return SJ_OK;
}

}  // namespace

int part_bounds(const double *p, uint64_t n, int dim, double *mn, double *mx) {
    SJ_TRY(check_points(p, n, dim));
    if (!mn || !mx) return SJ_EINVAL;
    for (int d = 0; d < dim; ++d) {
        mn[d] = INFINITY;
        mx[d] = -INFINITY;
    }
    if (n == 0) return SJ_OK;
    cudaStream_t s = caller_stream();
    Tmp t{s, {}};
    unsigned long long *acc;
    SJ_TRY(t.get(&acc, 2 * SJ_MAX_DIM + 1));
    SJ_CUDA_TRY(cudaMemsetAsync(acc, 0, (2 * SJ_MAX_DIM + 1) * sizeof(unsigned long long), s));
    unsigned *bad = reinterpret_cast<unsigned *>(acc + 2 * SJ_MAX_DIM);
    part_bounds_kernel<<<blocks_for(n), kT, 0, s>>>(p, n, dim, acc, bad);
    note_launch();
    SJ_CUDA_TRY(cudaGetLastError());
    unsigned long long h[2 * SJ_MAX_DIM + 1];
    SJ_CUDA_TRY(cudaMemcpyAsync(h, acc, sizeof h, cudaMemcpyDeviceToHost, s));
    SJ_CUDA_TRY(cudaStreamSynchronize(s));
    if (h[2 * SJ_MAX_DIM] & 0xFFFFFFFFull) {
        set_error("sj_part_bounds: non-finite coordinate");
        return SJ_EINVAL;
    }
    for (int d = 0; d < dim; ++d) {
        const unsigned long long lo = ~h[d], hi = h[dim + d];
        // decode on the host (same bit manipulation as okey_inv)
        auto inv = [](unsigned long long k) {
            const unsigned long long b = (k >> 63) ? (k & 0x7FFFFFFFFFFFFFFFull) : ~k;
            double x;
            memcpy(&x, &b, sizeof x);
            return x;
        };
        mn[d] = inv(lo);
        mx[d] = inv(hi);
    }
    return SJ_OK;
}

int64_t part_columns(double o0, double max0, double eps) {
    if (!(eps > 0.0) || !std::isfinite(eps) || !std::isfinite(o0) || !std::isfinite(max0) || max0 < o0) {
        set_error("sj_part_columns: invalid argument");
        return SJ_EINVAL;
    }
    const double w = eps * (1.0 + 0x1p-20);  // reading c5, as the build computes it
    const double q = (max0 - o0) / w;        // binary64 RN (the host is compiled without contraction)
    if (!(q < 0x1p30)) {
        set_error("sj_part_columns: grid too large in dimension 0 (%.3g cells >= 2^30)", q);
        return SJ_EGRID;
    }
    return (int64_t)std::floor(q) + 1;
}

int part_histogram(const double *p, uint64_t n, int dim, double o0, double eps, uint64_t ncol, uint64_t *hist) {
    SJ_TRY(check_points(p, n, dim));
    if (!hist || ncol == 0 || !(eps > 0.0)) return SJ_EINVAL;
    cudaStream_t s = caller_stream();
    Tmp t{s, {}};
    unsigned *bad;
    SJ_TRY(t.get(&bad, 1));
    SJ_CUDA_TRY(cudaMemsetAsync(bad, 0, sizeof(unsigned), s));
    SJ_CUDA_TRY(cudaMemsetAsync(hist, 0, ncol * sizeof(uint64_t), s));
    const double w = eps * (1.0 + 0x1p-20);
    if (n)
        part_hist_kernel<<<blocks_for(n), kT, 0, s>>>(p, n, dim, o0, w, ncol,
                                                      reinterpret_cast<unsigned long long *>(hist), bad);
    note_launch();
    SJ_CUDA_TRY(cudaGetLastError());
    unsigned hb = 0;
    SJ_CUDA_TRY(cudaMemcpyAsync(&hb, bad, sizeof hb, cudaMemcpyDeviceToHost, s));
    SJ_CUDA_TRY(cudaStreamSynchronize(s));
    if (hb) {
        set_error("sj_part_histogram: a point lies %s", (hb & 2u) ? "below the origin" : "beyond the last column");
        return SJ_EINVAL;
    }
    return SJ_OK;
}

int part_pack(const double *p, const uint32_t *ids, uint64_t n, int dim, double o0, double eps, const uint64_t *hist,
              uint64_t ncol, int world, double *own_p, uint32_t *own_ids, uint64_t *own_counts, double *halo_p,
              uint32_t *halo_ids, uint64_t *halo_counts) {
    SJ_TRY(check_points(p, n, dim));
    if (!hist || ncol == 0 || world < 1 || world > (1 << 20) || !own_counts || !halo_counts || !(eps > 0.0) ||
        (n && (!own_p || !own_ids || !halo_p || !halo_ids))) {
        set_error("sj_part_pack: invalid argument");
        return SJ_EINVAL;
    }
    cudaStream_t s = caller_stream();
    Tmp t{s, {}};
    unsigned long long *start, *counts;
    uint32_t *owner, *ok, *hk, *i0, *i1, *k2, *v2;
    unsigned *bad;
    SJ_TRY(t.get(&start, ncol + 1));
    SJ_TRY(t.get(&owner, ncol));
    SJ_TRY(t.get(&counts, 2 * (size_t)world + 1));
    const uint64_t nn = std::max<uint64_t>(n, 1);
    SJ_TRY(t.get(&ok, nn));
    SJ_TRY(t.get(&hk, nn));
    SJ_TRY(t.get(&i0, nn));
    SJ_TRY(t.get(&i1, nn));
    SJ_TRY(t.get(&k2, nn));
    SJ_TRY(t.get(&v2, nn));
    SJ_CUDA_TRY(cudaMemsetAsync(counts, 0, (2 * (size_t)world + 1) * sizeof(unsigned long long), s));
    bad = reinterpret_cast<unsigned *>(counts + 2 * world);
    SJ_TRY(scan_exclusive_u64(reinterpret_cast<const uint64_t *>(hist), reinterpret_cast<uint64_t *>(start), ncol,
                              reinterpret_cast<uint64_t *>(start + ncol), s));
    part_owner_kernel<<<(unsigned)((ncol + kT - 1) / kT), kT, 0, s>>>(start, ncol, start + ncol, (unsigned)world, owner);
    note_launch();
    const double w = eps * (1.0 + 0x1p-20);
    std::vector<unsigned long long> hc(2 * (size_t)world + 1, 0);
    if (n) {
        part_route_kernel<<<blocks_for(n), kT, 0, s>>>(p, n, dim, o0, w, ncol, owner, (unsigned)world, ok, hk, i0, i1,
                                                       counts, bad);
        note_launch();
        SJ_CUDA_TRY(cudaGetLastError());
        const int bits = bits_of((unsigned long long)world);  // keys 0 .. world (world = no halo)
        uint32_t *ko, *vo;
        SJ_TRY(radix_sort_u32(ok, i0, k2, v2, n, bits, &ko, &vo, s));
        part_pack_kernel<<<blocks_for(n), kT, 0, s>>>(p, ids, n, dim, vo, own_p, own_ids);
        note_launch();
        SJ_TRY(radix_sort_u32(hk, i1, k2, v2, n, bits, &ko, &vo, s));
        SJ_CUDA_TRY(cudaMemcpyAsync(hc.data(), counts, hc.size() * sizeof(unsigned long long), cudaMemcpyDeviceToHost, s));
        SJ_CUDA_TRY(cudaStreamSynchronize(s));
        uint64_t nh = 0;
        for (int r = 0; r < world; ++r) nh += hc[world + r];
        if (nh)
            part_pack_kernel<<<blocks_for(nh), kT, 0, s>>>(p, ids, nh, dim, vo, halo_p, halo_ids);
        note_launch();
        SJ_CUDA_TRY(cudaGetLastError());
    }
    SJ_CUDA_TRY(cudaStreamSynchronize(s));
    if (hc[2 * world] & 0xFFFFFFFFull) {
        set_error("sj_part_pack: a point lies outside the histogram's columns");
        return SJ_EINVAL;
    }
    for (int r = 0; r < world; ++r) {
        own_counts[r] = hc[r];
        halo_counts[r] = hc[world + r];
    }
    return SJ_OK;
}

}  // namespace sj

extern "C" {

int sj_part_bounds(const double *points, uint64_t n, int dim, double *mn, double *mx) {
    sj::set_error("");
    return sj::part_bounds(points, n, dim, mn, mx);
}

int64_t sj_part_columns(double origin0, double max0, double eps) {
    sj::set_error("");
    return sj::part_columns(origin0, max0, eps);
}

int sj_part_histogram(const double *points, uint64_t n, int dim, double origin0, double eps, uint64_t ncol,
                      uint64_t *hist) {
    sj::set_error("");
    return sj::part_histogram(points, n, dim, origin0, eps, ncol, hist);
}

int sj_part_pack(const double *points, const uint32_t *ids, uint64_t n, int dim, double origin0, double eps,
                 const uint64_t *hist, uint64_t ncol, int world, double *own_pts, uint32_t *own_ids,
                 uint64_t *own_counts, double *halo_pts, uint32_t *halo_ids, uint64_t *halo_counts) {
    sj::set_error("");
    return sj::part_pack(points, ids, n, dim, origin0, eps, hist, ncol, world, own_pts, own_ids, own_counts, halo_pts,
                         halo_ids, halo_counts);
}

}  // extern "C"
