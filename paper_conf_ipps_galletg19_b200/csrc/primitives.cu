// primitives.cu -- hand-written scan and LSD radix sort for sm_100a.
//
// The radix sort orders point->cell ids for the eps-grid index ("GPU Grid
// Index", north_star "a hand-written radix sort of point-to-cell IDs") and orders
// cells by workload for SortByWL.  Per 8-bit pass:
//   1. tile histogram (2048 keys per CTA, shared-memory counters), digit-major,
//   2. single-pass exclusive scan (decoupled look-back) of the [256 x tiles] histogram,
//   3. stable scatter: per-warp ranks from ballots over the digit bits, a block-wide prefix over
//      warps and digits, a shared-memory reorder of the tile so the global writes of one
//      digit run are contiguous (coalesced).
#include <cstdio>

#include <algorithm>

#include "scan.cuh"
#include "sj_internal.cuh"

namespace sj {

namespace {


template <class T>
__device__ __forceinline__ T warp_inclusive_scan(T x) {
    const int lane = threadIdx.x & 31;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        T y = __shfl_up_sync(0xffffffffu, x, o);
        if (lane >= o) x += y;
    }
    return x;
}

// Block-wide exclusive scan; every thread of the block must call it.
template <class T>
__device__ __forceinline__ T block_exclusive_scan(T v, T *total) {
    __shared__ T warp_sums[32];
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    const int nw = (blockDim.x + 31) >> 5;
    T x = warp_inclusive_scan(v);
    __syncthreads();
    if (lane == 31) warp_sums[wid] = x;
    __syncthreads();
    if (wid == 0) {
        T w = lane < nw ? warp_sums[lane] : T(0);
        w = warp_inclusive_scan(w);
        warp_sums[lane] = w;
    }
    __syncthreads();
    T pre = wid > 0 ? warp_sums[wid - 1] : T(0);
    if (total) *total = warp_sums[nw - 1];
    return pre + x - v;
}

// ------------------------------------------------------------------ radix sort

constexpr int kRadixThreads = 256;
constexpr int kRadixWarps = kRadixThreads / 32;
constexpr int kRadixItems = 8;  // per lane
constexpr int kRadixTile = kRadixThreads * kRadixItems;
static_assert(kRadixTile == kRadixTileKeys, "the cell-id kernel counts the first pass per tile of this size");
constexpr int kRadixBins = 256;

// Per-tile digit counts, digit-major: hist[d * ntiles + tile].
// (warp-private counters: the 256 bins of one shared histogram serialise a warp's atomics on
// the frequent digits of clustered keys; the keys are loaded first, then counted)
template <class K>
__global__ void __launch_bounds__(kRadixThreads) radix_hist_kernel(const K *keys, uint64_t n, int shift,
                                                                   uint32_t *hist, uint32_t ntiles) {
    __shared__ uint32_t h[kRadixWarps][kRadixBins];
#pragma unroll
    for (int w = 0; w < kRadixWarps; ++w) h[w][threadIdx.x] = 0;
    __syncthreads();
    const int warp = threadIdx.x >> 5;
    const uint64_t base = (uint64_t)blockIdx.x * kRadixTile;
    uint32_t d[kRadixItems];
#pragma unroll
    for (int it = 0; it < kRadixItems; ++it) {
        const uint64_t i = base + (uint64_t)it * kRadixThreads + threadIdx.x;
        d[it] = i < n ? (uint32_t)(keys[i] >> shift) & 0xFFu : kRadixBins;
    }
#pragma unroll
    for (int it = 0; it < kRadixItems; ++it)
        if (d[it] < kRadixBins) atomicAdd(&h[warp][d[it]], 1u);
    __syncthreads();
    uint32_t t = 0;
#pragma unroll
    for (int w = 0; w < kRadixWarps; ++w) t += h[w][threadIdx.x];
    hist[(uint64_t)threadIdx.x * ntiles + blockIdx.x] = t;
}

// Stable scatter of one tile: per-warp ranks from 8 ballots over the digit bits, a block-wide prefix
// over warps and digits, global starts from the scanned digit-major histogram, and a
// shared-memory reorder so each digit's run is written contiguously.
#ifndef SJ_SCATTER_MINB
#define SJ_SCATTER_MINB 4
#endif
template <class K>
__global__ void __launch_bounds__(kRadixThreads, SJ_SCATTER_MINB) radix_scatter_kernel(const K *keys_in, const uint32_t *vals_in,
                                                                      K *keys_out, uint32_t *vals_out, uint64_t n,
                                                                      int shift, const uint32_t *hist_scanned,
                                                                      uint32_t ntiles) {
    __shared__ uint32_t cnt[kRadixWarps][kRadixBins];
    __shared__ uint32_t dstart[kRadixBins];
    __shared__ uint32_t gstart[kRadixBins];
    __shared__ K skeys[kRadixTile];
    __shared__ uint32_t svals[kRadixTile];

    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const uint32_t lt = (1u << lane) - 1u;
#pragma unroll
    for (int w = 0; w < kRadixWarps; ++w) cnt[w][threadIdx.x] = 0;
    const uint64_t base = (uint64_t)blockIdx.x * kRadixTile;
    const uint64_t wbase = base + (uint64_t)warp * (32 * kRadixItems);

    K key[kRadixItems];
    uint32_t val[kRadixItems];
    uint32_t dig[kRadixItems];
    uint32_t rank[kRadixItems];
#pragma unroll
    for (int it = 0; it < kRadixItems; ++it) {
        uint64_t i = wbase + (uint64_t)it * 32 + lane;
        if (i < n) {
            key[it] = keys_in[i];
            val[it] = vals_in ? vals_in[i] : (uint32_t)i;  // null: the identity (first pass of the point sort)
            dig[it] = (uint32_t)(key[it] >> shift) & 0xFFu;
        } else {
            key[it] = 0;
            val[it] = 0;
            dig[it] = kRadixBins;  // sentinel: not counted
        }
    }
    __syncthreads();
    // (only the last tile has empty slots: their sentinel digit matches no key's below)
    const bool full_tile = base + (uint64_t)kRadixTile <= n;
#pragma unroll
    for (int it = 0; it < kRadixItems; ++it) {
        const uint32_t d = dig[it];
        // the lanes of this item with the same digit, from 8 ballots over the digit's bits
        // (__match_any_sync runs on the ADU pipe at ~70 cycles a warp: it bound this kernel)
        uint32_t peers = full_tile ? 0xffffffffu : __ballot_sync(0xffffffffu, d < kRadixBins);
#pragma unroll
        for (int b = 0; b < 8; ++b) {
            const uint32_t bit = (d >> b) & 1u;
            const uint32_t bb = __ballot_sync(0xffffffffu, bit);
            peers &= bit ? bb : ~bb;
        }
        uint32_t before = 0;
        if (d < kRadixBins) before = cnt[warp][d];
        rank[it] = before + __popc(peers & lt);
        __syncwarp();
        if (d < kRadixBins && (peers & lt) == 0) cnt[warp][d] = before + __popc(peers);
        __syncwarp();
    }
    __syncthreads();
    {
        const uint32_t d = threadIdx.x;
        uint32_t tc = 0;
#pragma unroll
        for (int w = 0; w < kRadixWarps; ++w) {
            const uint32_t t = cnt[w][d];
            cnt[w][d] = tc;
            tc += t;
        }
        dstart[d] = block_exclusive_scan<uint32_t>(tc, nullptr);
        gstart[d] = hist_scanned[(uint64_t)d * ntiles + blockIdx.x];
    }
    __syncthreads();
#pragma unroll
    for (int it = 0; it < kRadixItems; ++it) {
        const uint32_t d = dig[it];
        if (d < kRadixBins) {
            const uint32_t lpos = dstart[d] + cnt[warp][d] + rank[it];
            skeys[lpos] = key[it];
            svals[lpos] = val[it];
        }
    }
    __syncthreads();
    const uint64_t rem = n - base;
    const uint32_t tcount = rem < (uint64_t)kRadixTile ? (uint32_t)rem : (uint32_t)kRadixTile;
    for (uint32_t i = threadIdx.x; i < tcount; i += kRadixThreads) {
        const K k = skeys[i];
        const uint32_t d = (uint32_t)(k >> shift) & 0xFFu;
        const uint64_t dest = (uint64_t)gstart[d] + (i - dstart[d]);
        keys_out[dest] = k;
        vals_out[dest] = svals[i];
    }
}

__global__ void __launch_bounds__(kRadixThreads) iota_kernel(uint32_t *v, uint64_t n) {
    const uint64_t i = (uint64_t)blockIdx.x * kRadixThreads + threadIdx.x;
    if (i < n) v[i] = (uint32_t)i;
}

// vals_identity: `vals` holds no values yet -- they are the identity 0..n-1, generated by the
// first pass's scatter (the point sort: no kernel writes the input ids), and `vals` is scratch.
template <class K>
int radix_sort(K *keys, uint32_t *vals, K *keys_alt, uint32_t *vals_alt, uint64_t n, int bits, K **keys_out,
               uint32_t **vals_out, cudaStream_t s, Workspace *ws, uint32_t *hist0, bool vals_identity) {
    *keys_out = keys;
    *vals_out = vals;
    if (n <= 1 || bits <= 0) {
        if (vals_identity && n) {
            iota_kernel<<<(unsigned)((n + kRadixThreads - 1) / kRadixThreads), kRadixThreads, 0, s>>>(vals, n);
            note_launch();
            SJ_CUDA_TRY(cudaGetLastError());
        }
        return SJ_OK;
    }
    if (n >= (1ull << 32)) {
        set_error("radix_sort: n >= 2^32");
        return SJ_EINVAL;
    }
    const uint32_t ntiles = (uint32_t)((n + kRadixTile - 1) / kRadixTile);
    const uint64_t hbytes = (uint64_t)kRadixBins * ntiles * sizeof(uint32_t);
    // hist0: the first pass's tile histogram, already counted by the producer of the keys
    uint32_t *hist = hist0 ? hist0 : ws ? static_cast<uint32_t *>(ws->take(hbytes)) : nullptr;
    const bool own = hist == nullptr;
    if (own) SJ_TRY(dev_alloc(reinterpret_cast<void **>(&hist), hbytes + 16, s));
    K *ka = keys, *kb = keys_alt;
    uint32_t *va = vals, *vb = vals_alt;
    for (int shift = 0; shift < bits; shift += 8) {
        if (!(hist0 && shift == 0)) {
            radix_hist_kernel<K><<<ntiles, kRadixThreads, 0, s>>>(ka, n, shift, hist, ntiles);
            note_launch();
        }
        SJ_TRY(scan_exclusive_u32(hist, hist, (uint64_t)kRadixBins * ntiles, nullptr, s, ws));
        radix_scatter_kernel<K><<<ntiles, kRadixThreads, 0, s>>>(ka, (vals_identity && shift == 0) ? nullptr : va, kb,
                                                                 vb, n, shift, hist, ntiles);
        note_launch();
        SJ_CUDA_TRY(cudaGetLastError());
        K *tk = ka; ka = kb; kb = tk;
        uint32_t *tv = va; va = vb; vb = tv;
    }
    if (own) dev_free(hist, s);
    *keys_out = ka;
    *vals_out = va;
    return SJ_OK;
}

struct LoadArr {
    const uint32_t *in;
    __device__ unsigned operator()(uint64_t i) const { return in[i]; }
};
struct StoreArr {
    uint32_t *out;
    __device__ void operator()(uint64_t i, unsigned ex, unsigned) const { out[i] = ex; }
};
struct DoneTotal {
    uint32_t *total;
    __device__ void operator()(unsigned t) const {
        if (total) *total = t;
    }
};

}  // namespace

int scan_exclusive_u32(const uint32_t *in, uint32_t *out, uint64_t n, uint32_t *d_total, cudaStream_t s,
                       Workspace *ws) {
    if (n == 0) {
        if (d_total) SJ_CUDA_TRY(cudaMemsetAsync(d_total, 0, sizeof(uint32_t), s));
        return SJ_OK;
    }
    return scan_fused(n, LoadArr{in}, StoreArr{out}, s, DoneTotal{d_total}, ws);
}
namespace {
template <class In>
struct LoadArr64 {
    const In *in;
    __device__ unsigned long long operator()(uint64_t i) const { return (unsigned long long)in[i]; }
};
struct StoreArr64 {
    uint64_t *out;
    __device__ void operator()(uint64_t i, unsigned long long ex, unsigned long long) const { out[i] = ex; }
};
struct DoneTotal64 {
    uint64_t *total;
    __device__ void operator()(unsigned long long t) const {
        if (total) *total = t;
    }
};
}  // namespace

int scan_exclusive_u64(const uint64_t *in, uint64_t *out, uint64_t n, uint64_t *d_total, cudaStream_t s) {
    if (n == 0) {
        if (d_total) SJ_CUDA_TRY(cudaMemsetAsync(d_total, 0, sizeof(uint64_t), s));
        return SJ_OK;
    }
    return scan_fused<unsigned long long>(n, LoadArr64<uint64_t>{in}, StoreArr64{out}, s, DoneTotal64{d_total});
}

int scan_exclusive_u32_to_u64(const uint32_t *in, uint64_t *out, uint64_t n, uint64_t *d_total, cudaStream_t s) {
    if (n == 0) {
        if (d_total) SJ_CUDA_TRY(cudaMemsetAsync(d_total, 0, sizeof(uint64_t), s));
        return SJ_OK;
    }
    return scan_fused<unsigned long long>(n, LoadArr64<uint32_t>{in}, StoreArr64{out}, s, DoneTotal64{d_total});
}

int radix_sort_u32(uint32_t *keys, uint32_t *vals, uint32_t *keys_alt, uint32_t *vals_alt, uint64_t n, int bits,
                   uint32_t **keys_out, uint32_t **vals_out, cudaStream_t s, Workspace *ws, uint32_t *hist0,
                   bool vals_identity) {
    return radix_sort<uint32_t>(keys, vals, keys_alt, vals_alt, n, bits, keys_out, vals_out, s, ws, hist0,
                                vals_identity);
}
int radix_sort_u64(uint64_t *keys, uint32_t *vals, uint64_t *keys_alt, uint32_t *vals_alt, uint64_t n, int bits,
                   uint64_t **keys_out, uint32_t **vals_out, cudaStream_t s, Workspace *ws, uint32_t *hist0,
                   bool vals_identity) {
    return radix_sort<uint64_t>(keys, vals, keys_alt, vals_alt, n, bits, keys_out, vals_out, s, ws, hist0,
                                vals_identity);
}

}  // namespace sj
