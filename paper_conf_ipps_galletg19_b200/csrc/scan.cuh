// scan.cuh -- single-pass exclusive scan (decoupled look-back) with fused load / store
// functors, so a flag computation, its scan and the scatter that consumes it are ONE
// kernel (run-length compaction of the sorted cell ids, WorkQueue chunk boundaries, ...).
#pragma once

#include "sj_internal.cuh"

namespace sj {
namespace scan_detail {

constexpr int kThreads = 256;
constexpr int kItems = 8;
constexpr int kTile = kThreads * kItems;
// tile status word: [63:62] flag (0 = not ready, 1 = tile aggregate, 2 = inclusive prefix),
// [61:0] value (u32 scans, and u64 scans of totals below 2^62)
constexpr unsigned long long kFlagA = 1ull << 62;
constexpr unsigned long long kFlagP = 2ull << 62;
constexpr unsigned long long kValMask = (1ull << 62) - 1ull;

template <class T>
__device__ __forceinline__ T warp_incl(T x) {
    const int lane = threadIdx.x & 31;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        T y = __shfl_up_sync(0xffffffffu, x, o);
        if (lane >= o) x += y;
    }
    return x;
}

template <class T>
__device__ __forceinline__ T block_excl(T v, T *total, T *ws) {
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    constexpr int nw = kThreads / 32;
    T x = warp_incl(v);
    __syncthreads();
    if (lane == 31) ws[wid] = x;
    __syncthreads();
    if (wid == 0) {
        T w = lane < nw ? ws[lane] : T(0);
        w = warp_incl(w);
        if (lane < nw) ws[lane] = w;
    }
    __syncthreads();
    *total = ws[nw - 1];
    return (wid > 0 ? ws[wid - 1] : T(0)) + x - v;
}

__device__ __forceinline__ void publish(unsigned long long *status, unsigned tile, unsigned long long word) {
    atomicExch(status + tile, word);
}

// Returns the exclusive prefix of `tile` (sum of all earlier tiles).  Called by the whole
// first warp; the look-back inspects 32 predecessors per step (decoupled look-back with a
// warp-wide window), so the dependency chain is ~32x shorter than a one-tile walk.
template <class T>
__device__ __forceinline__ T look_back_warp(unsigned long long *status, unsigned tile, T agg) {
    const int lane = threadIdx.x & 31;
    if (tile == 0) {
        if (lane == 0) publish(status, 0, kFlagP | (unsigned long long)agg);
        return T(0);
    }
    if (lane == 0) publish(status, tile, kFlagA | (unsigned long long)agg);
    T prefix = 0;
    int j = (int)tile - 1;  // newest predecessor of the window
    for (;;) {
        const int idx = j - lane;
        unsigned long long st = kFlagP;  // before tile 0: an inclusive prefix of 0
        if (idx >= 0) {
            do {
                st = *((volatile unsigned long long *)(status + idx));
            } while ((st & (3ull << 62)) == 0);  // predecessor started earlier: no deadlock
        }
        const unsigned pmask = __ballot_sync(0xffffffffu, (st & (3ull << 62)) == kFlagP);
        const int first_p = pmask ? __ffs(pmask) - 1 : 32;  // nearest inclusive prefix
        T v = lane <= first_p ? (T)(st & kValMask) : T(0);
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
        prefix += v;
        if (pmask) break;
        j -= 32;
    }
    if (lane == 0) publish(status, tile, kFlagP | ((unsigned long long)(prefix + agg) & kValMask));
    return prefix;
}

// load(i) -> unsigned value of item i (< n); store(i, excl, value) consumes the exclusive
// prefix; done(total) runs once, in the last tile, after every earlier prefix is known.
template <class T, class Load, class Store, class Done>
__global__ void __launch_bounds__(kThreads) scan_kernel(uint64_t n, Load load, Store store, Done done,
                                                        unsigned long long *status, unsigned *tile_ctr) {
    __shared__ unsigned s_tile;
    __shared__ T s_prefix;
    __shared__ T ws[32];
    __shared__ T vals[kTile];
    if (threadIdx.x == 0) s_tile = atomicAdd(tile_ctr, 1u);  // dynamic tile order
    __syncthreads();
    const unsigned tile = s_tile;
    const uint64_t base = (uint64_t)tile * kTile;
#pragma unroll
    for (int it = 0; it < kItems; ++it) {
        const uint64_t i = base + (uint64_t)it * kThreads + threadIdx.x;
        vals[it * kThreads + threadIdx.x] = i < n ? (T)load(i) : T(0);
    }
    __syncthreads();
    T v[kItems], s = 0;
#pragma unroll
    for (int j = 0; j < kItems; ++j) {
        v[j] = vals[threadIdx.x * kItems + j];
        s += v[j];
    }
    T agg;
    T ex = block_excl<T>(s, &agg, ws);
    if (threadIdx.x < 32) {
        const T pre = look_back_warp<T>(status, tile, agg);
        if (threadIdx.x == 0) s_prefix = pre;
    }
    __syncthreads();
    ex += s_prefix;
    // per-item exclusive prefixes back to shared memory (blocked), then the stores run in the
    // same striped (coalesced) order as the loads
    __shared__ T exs[kTile];
#pragma unroll
    for (int j = 0; j < kItems; ++j) {
        exs[threadIdx.x * kItems + j] = ex;
        ex += v[j];
    }
    if (base + kTile >= n && threadIdx.x == kThreads - 1) done(ex);  // ex = grand total here
    __syncthreads();
#pragma unroll
    for (int it = 0; it < kItems; ++it) {
        const int k = it * kThreads + threadIdx.x;
        const uint64_t i = base + (uint64_t)k;
        if (i < n) store(i, exs[k], vals[k]);
    }
}

}  // namespace scan_detail

struct NoDone {
    template <class T>
    __device__ void operator()(T) const {}
};

// Exclusive scan of load(0..n-1) in one launch (value type T: unsigned, or unsigned long
// long for totals below 2^62).  Temporaries from the stream-ordered pool.
// With a workspace the tile status words come from its pre-zeroed region (no memset, no
// allocation); without one, or when that region is exhausted, from the pool.
template <class T = unsigned, class Load, class Store, class Done = NoDone>
int scan_fused(uint64_t n, Load load, Store store, cudaStream_t s, Done done = Done(), Workspace *ws = nullptr) {
    using namespace scan_detail;
    if (n == 0) return SJ_OK;
    const uint64_t nt = (n + kTile - 1) / kTile;
    const size_t bytes = nt * sizeof(unsigned long long) + 64;
    unsigned long long *status = ws ? static_cast<unsigned long long *>(ws->take_zero(bytes)) : nullptr;
    const bool own = status == nullptr;
    if (own) {
        SJ_TRY(dev_alloc(reinterpret_cast<void **>(&status), bytes, s));
        SJ_CUDA_TRY(cudaMemsetAsync(status, 0, bytes, s));
    }
    unsigned *ctr = reinterpret_cast<unsigned *>(status + nt);
    scan_kernel<T><<<(unsigned)nt, kThreads, 0, s>>>(n, load, store, done, status, ctr);
    note_launch();
    SJ_CUDA_TRY(cudaGetLastError());
    if (own) dev_free(status, s);
    return SJ_OK;
}

}  // namespace sj
