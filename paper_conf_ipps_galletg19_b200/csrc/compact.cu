// compact.cu -- closes the gaps a blocked in-place join leaves in its output (JoinArgs::blk).
//
// A blocked join hands out the output in blocks of blk pairs, one atomic per block and warp;
// every block is filled completely except each warp's last one, whose unused rest is a gap.  So
// after the join the pairs are [0, A) minus at most one gap per warp (A = the allocation
// counter), positions from cap_e = out_cap & ~1 on in the scratch buffer.  With G = the gaps'
// total, the join produced T = A - G pairs.  This moves the pairs lying at or past T into the
// gaps below T (both add up to the same count), so the output is [0, T) again: the k-th pair past
// T (in position order, gaps skipped) goes to the k-th hole below T (holes in warp order).  Holes
// and sources are disjoint, so one parallel copy does it.
#include <algorithm>

#include "sj_internal.cuh"

namespace sj {

namespace {

constexpr int kMaxGaps = kCompactMaxGaps;  // >= the blocked join's warps (the runtime checks)
constexpr int kPrepThreads = 1024;

struct CompactWs {
    unsigned long long moved;  // pairs to move (= hole pairs below T)
    unsigned long long nh, ns;
    unsigned long long h_start[kMaxGaps], h_pre[kMaxGaps + 1];
    unsigned long long s_start[kMaxGaps + 1], s_pre[kMaxGaps + 2];
};

// Exclusive scan of v[0, n) in shared memory (one block of kPrepThreads; n <= kMaxGaps + 2):
// thread t scans its contiguous run of entries, the runs' sums by warp shuffles; returns the total.
__device__ unsigned long long block_scan(unsigned long long *v, int n, unsigned long long *part) {
    const int t = threadIdx.x, lane = t & 31, wid = t >> 5;
    const int per = (n + kPrepThreads - 1) / kPrepThreads;
    const int lo = min(n, t * per), hi = min(n, lo + per);
    unsigned long long sum = 0;
    for (int i = lo; i < hi; ++i) sum += v[i];
    unsigned long long x = sum;  // inclusive scan of the runs' sums within the warp
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const unsigned long long y = __shfl_up_sync(0xffffffffu, x, o);
        if (lane >= o) x += y;
    }
    if (lane == 31) part[wid] = x;
    __syncthreads();
    if (wid == 0) {  // the warps' totals (kPrepThreads / 32 = 32 of them)
        unsigned long long z = part[lane];
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const unsigned long long y = __shfl_up_sync(0xffffffffu, z, o);
            if (lane >= o) z += y;
        }
        part[lane] = z;
    }
    __syncthreads();
    unsigned long long run = (wid ? part[wid - 1] : 0ull) + x - sum;
    for (int i = lo; i < hi; ++i) {
        const unsigned long long y = v[i];
        v[i] = run;
        run += y;
    }
    const unsigned long long total = part[kPrepThreads / 32 - 1];
    __syncthreads();
    return total;
}

// One block, no sort.  The allocation counter hands out blocks of blk pairs in order, so [0, A) is
// blocks 0 .. A/blk - 1, every one full except each warp's LAST block, which holds the gap at its
// end (gaps[2w] = its start, gaps[2w+1] = its length).  With T = A - sum of the gaps:
//   holes   = the gaps' parts below T, listed in warp order;
//   sources = the filled parts of the blocks b >= T / blk, clipped to >= T, in block order: a
//             block is full unless it is some warp's last block (then filled up to its gap);
//             there are at most (A - T) / blk + 1 <= warps + 1 such blocks.
// The k-th source pair goes to the k-th hole pair (any pairing of equal totals closes the gaps).
// Dynamic shared memory: two arrays of kMaxGaps + 2 words.
__global__ void __launch_bounds__(kPrepThreads) compact_prep_kernel(const unsigned long long *gaps, int ngap,
                                                                   const unsigned long long *d_alloc,
                                                                   unsigned long long blk, unsigned long long cap_e,
                                                                   CompactWs *w, unsigned long long *d_total) {
    extern __shared__ unsigned long long smem[];
    unsigned long long *hv = smem, *sv = smem + (kMaxGaps + 2);
    __shared__ unsigned long long part[kPrepThreads / 32];
    const int t = threadIdx.x;
    // G = the gaps' total (the lengths through hv, scanned in place)
    for (int i = t; i < ngap; i += kPrepThreads) hv[i] = gaps[2 * i + 1];
    __syncthreads();
    const unsigned long long G = block_scan(hv, ngap, part);
    const unsigned long long A = *d_alloc;
    const unsigned long long T = A - G;
    const unsigned long long b0 = T / blk, b1 = (A + blk - 1) / blk;  // source blocks [b0, b1)
    // <= ngap + 1: A - T = G < ngap * blk (a warp opens a block only to write into it); the clamp
    // only guards the shared arrays -- a violation would leave H != S, and nothing is moved
    const int nb = (int)min(b1 - b0, (unsigned long long)kMaxGaps + 1ull);
    // holes below T, in warp order; the source blocks' fill (blk unless a warp's last block)
    for (int i = t; i < ngap; i += kPrepThreads) {
        const unsigned long long st = gaps[2 * i], ln = gaps[2 * i + 1];
        w->h_start[i] = st;
        hv[i] = (ln > 0 && st < T) ? min(st + ln, T) - st : 0ull;
    }
    for (int i = t; i < nb; i += kPrepThreads) sv[i] = blk;
    __syncthreads();
    for (int i = t; i < ngap; i += kPrepThreads) {
        const unsigned long long st = gaps[2 * i], ln = gaps[2 * i + 1];
        const unsigned long long b = st / blk;  // the gap's block (a gap never spans two)
        if (ln > 0 && b >= b0 && b < b1) sv[b - b0] = st - b * blk;
    }
    __syncthreads();
    for (int i = t; i < nb; i += kPrepThreads) {
        const unsigned long long bs = (b0 + (unsigned long long)i) * blk, lo = max(bs, T), hi = bs + sv[i];
        w->s_start[i] = lo;
        sv[i] = hi > lo ? hi - lo : 0ull;
    }
    __syncthreads();
    const unsigned long long H = block_scan(hv, ngap, part);
    const unsigned long long S = block_scan(sv, nb, part);
    for (int i = t; i < ngap; i += kPrepThreads) w->h_pre[i] = hv[i];
    for (int i = t; i < nb; i += kPrepThreads) w->s_pre[i] = sv[i];
    if (t == 0) {
        w->h_pre[ngap] = H;
        w->s_pre[nb] = S;
        w->nh = (unsigned long long)ngap;
        w->ns = (unsigned long long)nb;
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
    // each warp moves a contiguous run of records (2 pairs each: every gap and segment is even),
    // its lanes 32 consecutive records per step (coalesced 16-B loads and stores); a lane locates
    // its first hole and source once and walks the segments from there
    const unsigned long long recs = w->moved / 2;
    const unsigned long long nw = (unsigned long long)gridDim.x * blockDim.x / 32;
    const unsigned long long per = ((recs + nw - 1) / nw + 31) / 32 * 32;
    const unsigned long long gw = ((unsigned long long)blockIdx.x * blockDim.x + threadIdx.x) / 32;
    const unsigned long long r0 = gw * per + (threadIdx.x & 31);
    const unsigned long long r1 = min(recs, gw * per + per);
    if (r0 >= r1) return;
    const unsigned long long nh = w->nh, ns = w->ns;
    unsigned long long hj = seg_of(w->h_pre, nh, 2 * r0), sj_ = seg_of(w->s_pre, ns, 2 * r0);
    for (unsigned long long r = r0; r < r1; r += 32) {
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
                                         2 * (kMaxGaps + 2) * (int)sizeof(unsigned long long)));
        attr = true;
    }
    compact_prep_kernel<<<1, kPrepThreads, 2 * (kMaxGaps + 2) * sizeof(unsigned long long), s>>>(
        a.gaps, nwarps, a.emit_ctr, a.blk, cap_e, w, d_total);
    note_launch();
    compact_copy_kernel<<<148 * 4, 256, 0, s>>>(reinterpret_cast<uint4 *>(a.out),
                                               reinterpret_cast<const uint4 *>(a.scratch), cap_e, w);
    note_launch();
    SJ_CUDA_TRY(cudaGetLastError());
    return SJ_OK;
}

}  // namespace sj
