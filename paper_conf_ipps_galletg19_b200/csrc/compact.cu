// compact.cu -- closes the gaps a blocked in-place join leaves in its output (JoinArgs::blk).
//
// A blocked join hands out the output in blocks of blk pairs, one atomic per block and warp;
// every block is filled completely except each warp's last one, whose unused rest is a gap.  So
// after the join the pairs are [0, A) minus at most one gap per warp (A = the allocation
// counter), positions from cap_e = out_cap & ~1 on in the scratch buffer.  With G = the gaps' total, the join produced T = A - G pairs.  This moves
// the pairs lying at or past T into the gaps below T (both add up to the same count), so the
// output is [0, T) again: the k-th pair past T (in position order, gaps skipped) goes to the
// k-th hole below T.  Holes and sources are disjoint, so one parallel copy does it.
#include <algorithm>

#include "sj_internal.cuh"

namespace sj {

namespace {

constexpr int kMaxGaps = kCompactMaxWarps;  // >= the blocked join's warps (the runtime checks)
static_assert(kMaxGaps == 8192, "the sort keys carry a 13-bit gap index");
constexpr int kPrepThreads = 1024;

struct CompactWs {
    unsigned long long moved;  // pairs to move (= hole pairs below T)
    unsigned long long nh, ns;
    unsigned long long h_start[kMaxGaps], h_pre[kMaxGaps + 1];
    unsigned long long s_start[kMaxGaps + 1], s_pre[kMaxGaps + 2];
};

// Exclusive scan of v[0, n) in shared memory (one block of kPrepThreads; n <= kMaxGaps + 2):
// thread t scans its contiguous run of entries; returns the total.
__device__ unsigned long long block_scan(unsigned long long *v, int n, unsigned long long *part) {
    const int t = threadIdx.x;
    const int per = (n + kPrepThreads - 1) / kPrepThreads;
    const int lo = min(n, t * per), hi = min(n, lo + per);
    unsigned long long sum = 0;
    for (int i = lo; i < hi; ++i) sum += v[i];
    part[t] = sum;
    __syncthreads();
    for (int o = 1; o < kPrepThreads; o <<= 1) {  // Hillis-Steele inclusive scan of the runs' sums
        const unsigned long long x = t >= o ? part[t - o] : 0ull;
        __syncthreads();
        part[t] += x;
        __syncthreads();
    }
    unsigned long long run = part[t] - sum;
    for (int i = lo; i < hi; ++i) {
        const unsigned long long x = v[i];
        v[i] = run;
        run += x;
    }
    const unsigned long long total = part[kPrepThreads - 1];
    __syncthreads();
    return total;
}

// One block: sort the gaps by start, T, the holes below T and the source segments past it, with
// their prefix sums.  Dynamic shared memory: three arrays of kMaxGaps + 2 words (192 KB).
__global__ void __launch_bounds__(kPrepThreads) compact_prep_kernel(const unsigned long long *gaps, int ngap,
                                                                   const unsigned long long *d_alloc,
                                                                   unsigned long long cap_e, CompactWs *w,
                                                                   unsigned long long *d_total) {
    extern __shared__ unsigned long long smem[];
    unsigned long long *key = smem, *ln = smem + (kMaxGaps + 2), *tmp = smem + 2 * (kMaxGaps + 2);
    __shared__ unsigned long long part[kPrepThreads];
    __shared__ int s_m;
    const int t = threadIdx.x;
    int np = 2;  // the sort's size: a power of two >= ngap
    while (np < ngap) np <<= 1;
    // keys (start / 2) << 13 | gap index: starts are even and distinct (the gaps are disjoint),
    // gap index < kMaxGaps = 2^13; empty gaps sort last
    for (int i = t; i < np; i += kPrepThreads) {
        const bool ok = i < ngap && gaps[2 * i + 1] > 0;
        key[i] = ok ? ((gaps[2 * i] >> 1) << 13) | (unsigned long long)i : ~0ull;
    }
    if (t == 0) s_m = 0;
    __syncthreads();
    for (int k = 2; k <= np; k <<= 1)  // bitonic sort
        for (int j = k >> 1; j > 0; j >>= 1) {
            for (int i = t; i < np; i += kPrepThreads) {
                const int p = i ^ j;
                if (p > i) {
                    const bool up = (i & k) == 0;
                    const unsigned long long x = key[i], y = key[p];
                    if ((x > y) == up) {
                        key[i] = y;
                        key[p] = x;
                    }
                }
            }
            __syncthreads();
        }
    // the sorted gaps: key[i] becomes the start, ln[i] the length
    int mine = 0;
    for (int i = t; i < np; i += kPrepThreads) {
        const unsigned long long kk = key[i];
        const bool ok = kk != ~0ull;
        const int g = (int)(kk & 8191ull);
        key[i] = ok ? gaps[2 * g] : ~0ull;
        ln[i] = ok ? gaps[2 * g + 1] : 0ull;
        tmp[i] = ln[i];
        mine += ok ? 1 : 0;
    }
    atomicAdd(&s_m, mine);
    __syncthreads();
    const int m = s_m;
    unsigned long long *st = key;
    const unsigned long long G = block_scan(tmp, np, part);
    const unsigned long long A = *d_alloc;
    const unsigned long long T = A - G;
    // holes: the gaps' parts below T
    for (int i = t; i < m; i += kPrepThreads) {
        w->h_start[i] = st[i];
        tmp[i] = st[i] < T ? min(st[i] + ln[i], T) - st[i] : 0ull;
    }
    __syncthreads();
    const unsigned long long H = block_scan(tmp, m, part);
    for (int i = t; i < m; i += kPrepThreads) w->h_pre[i] = tmp[i];
    __syncthreads();
    // sources: [T, A) outside the gaps -- the segments between consecutive gaps, clipped to >= T
    for (int i = t; i <= m; i += kPrepThreads) {
        const unsigned long long lo0 = i == 0 ? 0ull : st[i - 1] + ln[i - 1];
        const unsigned long long hi = i == m ? A : st[i];
        const unsigned long long lo = max(lo0, T);
        w->s_start[i] = lo;
        tmp[i] = hi > lo ? hi - lo : 0ull;
    }
    __syncthreads();
    const unsigned long long S = block_scan(tmp, m + 1, part);
    for (int i = t; i <= m; i += kPrepThreads) w->s_pre[i] = tmp[i];
    if (t == 0) {
        w->h_pre[m] = H;
        w->s_pre[m + 1] = S;
        w->nh = (unsigned long long)m;
        w->ns = (unsigned long long)m + 1;
        // (H == S by construction; T > cap_e: the output overflowed, the caller re-runs staged)
        w->moved = (T <= cap_e && H == S) ? H : 0ull;
        *d_total = T;
    }
}

// the last index i of pre[0, n) with pre[i] <= x (pre ascending, pre[0] = 0)
__device__ __forceinline__ unsigned long long seg_of(const unsigned long long *pre, unsigned long long n,
                                                     unsigned long long x) {
    unsigned long long lo = 0, hi = n;  // invariant: pre[lo] <= x, answer in [lo, hi)
    while (hi - lo > 1) {
        const unsigned long long mid = (lo + hi) / 2;
        if (pre[mid] <= x) lo = mid; else hi = mid;
    }
    return lo;
}

__global__ void __launch_bounds__(256) compact_copy_kernel(uint4 *out, const uint4 *scratch, unsigned long long cap_e,
                                                           const CompactWs *w) {
    // each thread moves a contiguous run of records (2 pairs each: every gap and segment is
    // even), locating its first hole and source once and walking the segments from there
    const unsigned long long recs = w->moved / 2;
    const unsigned long long nth = (unsigned long long)gridDim.x * blockDim.x;
    const unsigned long long per = (recs + nth - 1) / nth;
    const unsigned long long r0 = ((unsigned long long)blockIdx.x * blockDim.x + threadIdx.x) * per;
    const unsigned long long r1 = min(recs, r0 + per);
    if (r0 >= r1) return;
    const unsigned long long nh = w->nh, ns = w->ns;
    unsigned long long hj = seg_of(w->h_pre, nh, 2 * r0), sj_ = seg_of(w->s_pre, ns, 2 * r0);
    for (unsigned long long r = r0; r < r1; ++r) {
        const unsigned long long p = 2 * r;
        while (w->h_pre[hj + 1] <= p) ++hj;  // next non-empty hole / source
        while (w->s_pre[sj_ + 1] <= p) ++sj_;
        const unsigned long long dst = w->h_start[hj] + (p - w->h_pre[hj]);
        const unsigned long long src = w->s_start[sj_] + (p - w->s_pre[sj_]);
        const uint4 v = src < cap_e ? out[src >> 1] : scratch[(src - cap_e) >> 1];
        out[dst >> 1] = v;
    }
}

}  // namespace

size_t compact_ws_bytes(int blocks) {
    (void)blocks;
    return sizeof(CompactWs);
}

int compact_output(const JoinArgs &a, int blocks, unsigned long long *d_total, void *ws, cudaStream_t s) {
    const int nwarps = blocks * (kJoinThreads / 32);
    if (nwarps > kMaxGaps) {
        set_error("compact_output: %d warps > %d", nwarps, kMaxGaps);
        return SJ_EINVAL;
    }
    CompactWs *w = static_cast<CompactWs *>(ws);
    const unsigned long long cap_e = a.out_cap & ~1ull;
    static bool attr = false;
    if (!attr) {
        SJ_CUDA_TRY(cudaFuncSetAttribute(compact_prep_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                         3 * (kMaxGaps + 2) * (int)sizeof(unsigned long long)));
        attr = true;
    }
    compact_prep_kernel<<<1, kPrepThreads, 3 * (kMaxGaps + 2) * sizeof(unsigned long long), s>>>(
        a.gaps, nwarps, a.emit_ctr, cap_e, w, d_total);
    note_launch();
    compact_copy_kernel<<<148 * 4, 256, 0, s>>>(reinterpret_cast<uint4 *>(a.out),
                                               reinterpret_cast<const uint4 *>(a.scratch), cap_e, w);
    note_launch();
    SJ_CUDA_TRY(cudaGetLastError());
    return SJ_OK;
}

}  // namespace sj
