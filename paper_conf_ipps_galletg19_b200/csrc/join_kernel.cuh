// join_kernel.cu -- the hot loop (DESIGN.md §1 a10): WorkQueue + k threads per query
// point + LID-UNICOMP + mirrored, warp-aggregated emission.  sm_100a, FP64 CUDA cores.
//
// Paper mapping:
//   * GPUCALCGLOBAL structure, P:75 (Alg. 1 prose): get the query point, its
//     neighbouring cells, for every candidate compute the distance, if <= eps add
//     the pair.
//   * WorkQueue, P:194-198 (§III-D): a global counter persistent for the batch is
//     the queue head; an atomic increment hands D' (sorted by workload)
//     out in order.  With k > 1 only a leader increments the counter and shuffles
//     the result to its group; here the leader is lane 0 of the warp, and a
//     dequeue hands out a chunk of <= 32 consecutive D' positions.
//   * k threads per query point, P:161-170 (§III-A, Fig. 4): the k lanes of a
//     group split the query's candidates -- lane t takes candidates t, t+k, t+2k...
//     of the concatenated candidate list, so the split stays balanced across cell
//     boundaries (reading c11).
//   * LID-UNICOMP, P:172-185 (§III-B, Alg. 3): only neighbour cells with a higher
//     linear id are scanned (pre-resolved per cell into the forward list), every
//     distance calculation emits both (q, c) and (c, q); in the home cell the
//     query at position r compares to r+1 .. r+floor((m-1)/2) (mod m), plus r+m/2
//     when m is even and r < m/2 (balanced circulant half scan, reading c8), so
//     every in-cell pair is evaluated exactly once.
//   * Distance: s = sum_d fl(t_d*t_d) with t_d = fl(q_d - c_d), RN intrinsics,
//     dimension order, no FMA; hit iff s <= fl(eps^2) (readings c1, c2).
//   * Emission: hits of a warp step are ranked with __ballot_sync/__popc into a
//     per-warp shared-memory buffer; a full buffer is flushed with ONE atomicAdd on
//     the batch's output counter and coalesced 16-byte streaming stores.
//   * Cell tiles in shared memory: a chunk whose queries all lie in one cell of >= 8
//     points shares that cell's forward runs; the warp stages them 32 candidates at a
//     time in shared memory and every query of the chunk is evaluated against each
//     tile (loads per distance calculation / (chunk size / k)).
#pragma once
#include "sj_internal.cuh"

namespace sj {

// Shared by the per-dimension translation units (join_dim.cu, SJ_JOIN_DIM = 1..8) and the
// launcher (join_kernel.cu).
typedef void (*join_fn)(const JoinArgs);
struct KernelInfo {
    join_fn f = nullptr;
    size_t smem = 0;
    int occ = 0;  // resident CTAs per SM
};
// The kernel of (mode, pattern, k) for one dimensionality (defined in join_dim.cu per D).
template <int D>
KernelInfo join_pick(int mode, bool gcg, int k);

namespace {

constexpr unsigned kFull = 0xffffffffu;
constexpr int kWarps = kJoinThreads / 32;
// 1-D / 2-D: hits buffered per warp ({orig q, orig c}, 8 B each): 624 fills a warp's 7 KB share of
// four CTAs per SM (measured against 512: fewer flushes, C5 0.914 -> 0.906 ms, C5 eps 0.2 2.90 ->
// 2.85 ms; 600 was slower than both)
#ifndef SJ_BUF2
#define SJ_BUF2 624
#endif
constexpr int kBufHits = SJ_BUF2;
#ifndef SJ_BUF_HI
#define SJ_BUF_HI 96
#endif
// 4..8-D: few hits per calculation; the small buffer keeps a warp's shared memory under
// 7 KB, so four 256-thread CTAs fit an SM (occupancy of the FP64-bound kernels)
constexpr int kBufHitsHi = SJ_BUF_HI;
// A cell segment of >= 2 queries is tiled when its forward list has at least this many
// candidates (6-D: ~1300 per cell of ~4 points), so staging pays for itself.
constexpr unsigned kTileMinCand = 128;

template <int DIM>
struct PointPad {
    static constexpr int value = DIM == 1 ? 1 : ((DIM + 1) & ~1);
};

// Compile-time traits of the kernel modes (JoinMode): exact sizing and the per-chunk counts
// are modes of their own so the default kernels carry none of their code.
template <int MODE>
struct Mode {
    static constexpr bool pairs = MODE == kPairs || MODE == kExact || MODE == kPairsB;  // emits the pair list
    static constexpr bool inplace = MODE == kPairs || MODE == kPairsB;  // overflow stop, fused estimator
    static constexpr bool blocked = MODE == kPairsB;                    // blocked output (JoinArgs::blk)
    static constexpr bool exact = MODE == kExact;                     // ... at chunk offsets
};

#ifndef SJ_BUF3
#define SJ_BUF3 512
#endif
template <int DIM>
struct BufCap {
    static constexpr int value = DIM <= 2 ? kBufHits : DIM == 3 ? SJ_BUF3 : kBufHitsHi;
};

// Per-warp shared memory: emission buffer, the chunk's queries, one candidate tile.
#ifndef SJ_GSTAGE
#define SJ_GSTAGE 1  // generic path: stage the chunk's query data and first runs in shared memory
#endif
// Generic path staging: the LID-UNICOMP forward runs of one cell (3-D: 5, the rows of
// pattern_rows()); other patterns' further runs are read from global memory.  Measured (join
// ms, B200): 3-D C3 K64 0.721 -> 0.697, K256 1.814 -> 1.679; 2-D C5 1.027 -> 1.035, C5 eps 0.2
// 2.97 -> 3.10 (the staging's wait costs more than the run loads it hides), so 3-D only.
template <int DIM>
struct GStage {
    static constexpr int runs = !SJ_GSTAGE ? 0 : DIM == 3 ? 5 : 0;
};
#ifndef SJ_FLAT_W
#define SJ_FLAT_W 128  // flat path for chunks whose longest candidate list is <= this (0: off;
                       // measured 32 / 64 / 128 / 256: C3 K64 0.679 / 0.676 / 0.669 / 0.670 ms)
#endif
// flat path: independent (query, candidate) pairs per lane and step -- their candidate loads are
// in flight together (measured: 2-D 4 (C2 K16 join 0.216 -> 0.201 ms), 3-D 2)
#ifndef SJ_FLAT_U
#define SJ_FLAT_U 0
#endif
template <int DIM>
struct FlatU {
    static constexpr int value = SJ_FLAT_U ? SJ_FLAT_U : DIM <= 2 ? 4 : 2;
};
// Flat path (flat_chunk): 1-D..3-D, half patterns, the pair / count modes.  runs = the
// LID-UNICOMP forward runs per cell (pattern_rows()), staged per query.
template <int DIM, int MODE, bool GCG>
struct Flat {
    static constexpr int runs = DIM == 1 ? 1 : DIM == 2 ? 2 : DIM == 3 ? 5 : 0;
    static constexpr bool on = SJ_FLAT_W > 0 && runs > 0 && !GCG && MODE != kRows && MODE != kDegree;
};
template <int DIM>
struct StagedRuns {  // entries of WarpSmem::gruns per query
    static constexpr int a = GStage<DIM>::runs, b = Flat<DIM, kPairs, false>::runs;
    static constexpr int value = (a > b ? a : b) > 0 ? (a > b ? a : b) : 1;
};
// Per-warp control words (shared memory, lane 0 writes).
struct WarpCtl {
    // kExact: next output slot of the current chunk; kPairs: nonzero once a flush of this warp
    // found the output full (the warp stops dequeuing: the caller re-runs the join staged)
    unsigned long long wcur;
    // kPairs with the fused estimator (a9): hits this warp has flushed so far, and its
    // hits in the sample chunks, taken when it first dequeues a chunk past the sample (a warp
    // meets its chunks in increasing order), so no state is live across a chunk
    unsigned long long wtot, samp;
    unsigned sclosed;
    unsigned long long sv1;  // end of the fused estimator's sample (virtual chunks [0, sv1))
    unsigned vcount;         // the batch's virtual chunks (in shared memory: no register in the loops)
    unsigned long long ocur, oend;  // the warp's output block (blocked kPairs launches): [ocur, oend) free
};

template <int DIM, int MODE>
struct WarpSmem {
    // (2-D / 3-D: the staging fits inside the tiles; 4-D+ stage one run per query, and their
    // shared memory is what limits the occupancy: 6-D must stay under 7 KB per warp)
    static_assert(DIM < 2 || DIM > 3 ||
                      2 * 32 * PointPad<DIM>::value * 8 + 2 * 32 * 4 >=
                          32 * 8 * StagedRuns<DIM>::value + 32 * 4 + 32 * 16,
                  "the staging union must not grow the warp's shared memory");
    static constexpr int PAD = PointPad<DIM>::value;
    // the tiled path's candidate tiles and the generic / flat paths' per-query staging are
    // never live together (a chunk's tiled segments finish before its generic queries start)
    union {
        struct {
            alignas(16) double tile[2][32 * PAD];  // staged candidates (lid order), double-buffered
            unsigned tile_orig[2][32];             // input ids of the staged candidates
        };
        struct {
            uint2 gruns[32 * StagedRuns<DIM>::value];  // generic (3-D) / flat: the queries' first runs
            unsigned char neq[32];                     // flat: lanes of the non-empty lists, in order
            uint4 fq[32];                              // flat: per query {home begin, m, rr, S}
        };
    };
    alignas(16) double qry[32 * PAD];   // the chunk's query points
    unsigned qorig[32];                 // input ids of the chunk's queries
    unsigned qrr[32];                   // the queries' positions in their (common) cell
    unsigned char glist[32];            // generic path: lanes of the chunk's remaining queries
    // 4-D..6-D: the segment cell's forward runs (<= 122) staged once, so the per-tile run walk
    // reads shared memory instead of chasing L2 latency run by run
    uint2 runs_s[(DIM >= 4 && DIM <= 6) ? 128 : 1];
    // hits buffered before a flush: fewer in high dimensions (few hits per calculation,
    // and the smaller footprint buys occupancy)
    alignas(16) uint2 buf[Mode<MODE>::pairs ? BufCap<DIM>::value : 2];
    WarpCtl ctl;
    unsigned snext;  // SortByWL only (static assignment): this warp's next chunk index
    // kRows: the segment's per-query row cursors; kDegree: their running neighbour counts
    unsigned long long qcur[(MODE == kRows || MODE == kDegree) ? 32 : 1];
};
static_assert(sizeof(WarpSmem<6, kPairs>) <= 7168, "6-D: four 256-thread CTAs per SM");
static_assert(sizeof(WarpSmem<2, kPairsB>) <= 7168 && sizeof(WarpSmem<2, kPairs>) <= 7168,
              "2-D: four 256-thread CTAs per SM");

template <int DIM>
__device__ __forceinline__ void load_point(const double *__restrict__ p, double (&x)[DIM]) {
    if constexpr (DIM == 1) {
        x[0] = __ldg(p);
    } else {
#pragma unroll
        for (int d = 0; d < DIM; d += 2) {
            const double2 v = __ldg(reinterpret_cast<const double2 *>(p + d));
            x[d] = v.x;
            if (d + 1 < DIM) x[d + 1] = v.y;
        }
    }
}

template <int DIM>
__device__ __forceinline__ void load_smem_point(const double *p, double (&x)[DIM]) {
    if constexpr (DIM == 1) {
        x[0] = p[0];
    } else {
#pragma unroll
        for (int d = 0; d < DIM; d += 2) {
            const double2 v = *reinterpret_cast<const double2 *>(p + d);
            x[d] = v.x;
            if (d + 1 < DIM) x[d + 1] = v.y;
        }
    }
}

template <int DIM>
__device__ __forceinline__ void copy_point_to_smem(const double *__restrict__ src, double *dst) {
    constexpr int PAD = PointPad<DIM>::value;
    if constexpr (PAD == 1) {
        dst[0] = __ldg(src);
    } else {
#pragma unroll
        for (int d = 0; d < PAD; d += 2)
            *reinterpret_cast<double2 *>(dst + d) = __ldg(reinterpret_cast<const double2 *>(src + d));
    }
}

// Asynchronous global->shared copies (cp.async, LDGSTS): tile staging without registers.
__device__ __forceinline__ void cp_async_16(void *smem, const void *gmem) {
    const unsigned sa = (unsigned)__cvta_generic_to_shared(smem);
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16;\n" ::"r"(sa), "l"(gmem));
}
__device__ __forceinline__ void cp_async_8(void *smem, const void *gmem) {
    const unsigned sa = (unsigned)__cvta_generic_to_shared(smem);
    asm volatile("cp.async.ca.shared.global [%0], [%1], 8;\n" ::"r"(sa), "l"(gmem));
}
__device__ __forceinline__ void cp_async_4(void *smem, const void *gmem) {
    const unsigned sa = (unsigned)__cvta_generic_to_shared(smem);
    asm volatile("cp.async.ca.shared.global [%0], [%1], 4;\n" ::"r"(sa), "l"(gmem));
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;\n" ::); }
template <int N>
__device__ __forceinline__ void cp_async_wait() {
    asm volatile("cp.async.wait_group %0;\n" ::"n"(N) : "memory");
}
template <int DIM>
__device__ __forceinline__ void cp_async_point(double *dst, const double *src) {
    constexpr int PAD = PointPad<DIM>::value;
    if constexpr (PAD == 1) {
        cp_async_8(dst, src);
    } else {
#pragma unroll
        for (int d = 0; d < PAD; d += 2) cp_async_16(dst + d, src + d);
    }
}

// s = fl(...fl(fl(t0*t0) + fl(t1*t1)) + ...), t_d = fl(q_d - c_d)  (readings c1/c2)
template <int DIM>
__device__ __forceinline__ double sqdist(const double (&q)[DIM], const double (&c)[DIM]) {
    double t = __dsub_rn(q[0], c[0]);
    double s = __dmul_rn(t, t);
#pragma unroll
    for (int d = 1; d < DIM; ++d) {
        t = __dsub_rn(q[d], c[d]);
        s = __dadd_rn(s, __dmul_rn(t, t));
    }
    return s;
}

// Flush a warp's staged hits and return how many stay buffered (0, or the rest of a flush that
// filled its output block).  The lanes write coalesced streaming stores: both mirrored pairs of a
// hit as one 16-B store {q, c, c, q} (half patterns), or the single pair {q, c} (GCG, which
// meets every pair twice).  The output slots:
//   * default: ONE atomicAdd on the output counter per flush;
//   * blocked output (JoinArgs::blk, half patterns, kPairs): from the warp's current block; a
//     block is taken with ONE atomicAdd of blk per block and warp.  A flush that does not fit in
//     its block's rest fills the rest and keeps the other hits buffered (moved to the buffer's
//     front) for the next flush, which starts a new block -- so every block but each warp's last
//     is full and the one write loop stays a single contiguous segment;
//   * exact sizing (kExact): the chunk's own cursor, so the output order is deterministic; the
//     counter still totals the pairs.
// Positions from cap_e = out_cap & ~1 on go to the scratch buffer of a blocked launch
// (compact_output moves them back), past it they are dropped and the warp stops (overflow).
template <bool GCG, bool EXACT, bool BLOCKED>
__device__ __forceinline__ int flush(uint2 *buf, int nbuf, const JoinArgs &a, int lane, WarpCtl *wc) {
    __syncwarp();
    constexpr unsigned long long kPer = GCG ? 1ull : 2ull;  // pairs per buffered hit
    unsigned long long base = 0;
    unsigned take = (unsigned)nbuf;  // hits written by this flush
    if (lane == 0) {
        if (BLOCKED && !GCG && !EXACT) {
            // the warp's own output block (no lock): a new one (ONE atomicAdd of blk) when full
            unsigned long long c = wc->ocur, e = wc->oend;
            if (c == e) {
                c = atomicAdd(a.emit_ctr, a.blk);
                e = c + a.blk;
                wc->oend = e;
            }
            take = min((unsigned)nbuf, (unsigned)((e - c) >> 1));
            wc->ocur = c + 2ull * take;
            base = c;
        } else {
            base = atomicAdd(a.emit_ctr, kPer * (unsigned long long)nbuf);
        }
        wc->wtot += (unsigned long long)take;
        if (EXACT) {
            base = wc->wcur;
            wc->wcur = base + kPer * (unsigned long long)nbuf;
        } else if (base + kPer * (unsigned long long)take > (a.out_cap & ~1ull) + a.scratch_cap) {
            wc->wcur = 1;  // overflow: stop dequeuing
        }
    }
    base = __shfl_sync(kFull, base, 0);
    take = __shfl_sync(kFull, take, 0);
    uint2 *out2 = reinterpret_cast<uint2 *>(a.out);
    if constexpr (GCG) {
        const bool fits = base + (unsigned long long)nbuf <= a.out_cap;
        for (int k = lane; k < nbuf; k += 32)
            if (fits || base + (unsigned long long)k < a.out_cap) __stcs(out2 + base + k, buf[k]);
    } else {
        uint4 *out4 = reinterpret_cast<uint4 *>(a.out) + (base >> 1);  // base is even
        if (base + 2ull * (unsigned long long)take <= a.out_cap) {
#pragma unroll 4
            for (int k = lane; k < (int)take; k += 32) {
                const uint2 v = buf[k];  // {orig q, orig c}
                __stcs(out4 + k, make_uint4(v.x, v.y, v.y, v.x));  // (q,c) and (c,q)
            }
        } else {  // past the buffer: the scratch of a blocked launch, else dropped (overflow)
            const unsigned long long cap_e = a.out_cap & ~1ull;
            for (int k = lane; k < (int)take; k += 32) {
                const unsigned long long pos = base + 2ull * (unsigned long long)k;
                const uint2 v = buf[k];
                if (pos < cap_e)
                    __stcs(out4 + k, make_uint4(v.x, v.y, v.y, v.x));
                else if (pos - cap_e < a.scratch_cap)
                    __stcs(reinterpret_cast<uint4 *>(a.scratch) + ((pos - cap_e) >> 1), make_uint4(v.x, v.y, v.y, v.x));
            }
        }
        if (take < (unsigned)nbuf) {  // the rest to the buffer's front (forward copy: safe)
            const unsigned rest = (unsigned)nbuf - take;
            for (unsigned k0 = 0; k0 < rest; k0 += 32) {
                const unsigned k = k0 + (unsigned)lane;
                const uint2 v = k < rest ? buf[take + k] : make_uint2(0, 0);
                __syncwarp();
                if (k < rest) buf[k] = v;
                __syncwarp();
            }
            return (int)rest;
        }
    }
    __syncwarp();
    return 0;
}

// Warp-aggregated emission of one evaluation step (all 32 lanes call it): the hits are
// ranked with __ballot_sync/__popc into the warp's shared buffer.  Before each round the
// caller makes room for the round's maximum number of hits (flush_if) instead of checking
// after every step.  kRows: the hits of a k-lane group (gbits) go straight to the group's
// query row at its cursor `cur`, in candidate order.
template <int DIM, int MODE, bool GCG>
__device__ __forceinline__ void emit(bool hit, unsigned oq, unsigned oc, uint2 *buf, int &nbuf,
                                     unsigned long long &nhits, unsigned lt, unsigned gbits,
                                     unsigned long long &cur, const JoinArgs &a, int lane) {
    constexpr bool RARE = DIM >= 4;
    if constexpr (Mode<MODE>::pairs) {
        const unsigned hm = __ballot_sync(kFull, hit);
        if (RARE && hm == 0u) return;  // high dimensions: most steps have no hit in the warp
        if (hit) buf[nbuf + __popc(hm & lt)] = make_uint2(oq, oc);
        nbuf += __popc(hm);
    } else if constexpr (MODE == kRows) {
        const unsigned all = __ballot_sync(kFull, hit);
        if (RARE && all == 0u) return;
        const unsigned hm = all & gbits;
        if (hit) a.nbrs[cur + __popc(hm & lt)] = oc;
        cur += __popc(hm);
        nhits += hit ? 1ull : 0ull;
    } else {
        nhits += hit ? (GCG ? 1ull : 2ull) : 0ull;
    }
}

// Make room before a round: `room` = the most hits the round can add to the warp.
template <int DIM, int MODE, bool GCG>
__device__ __forceinline__ void flush_if(uint2 *buf, int &nbuf, int room, const JoinArgs &a, int lane,
                                         WarpCtl *wc) {
    constexpr int CAP = BufCap<DIM>::value;
    if constexpr (Mode<MODE>::pairs) {
        while (nbuf > CAP - room) nbuf = flush<GCG, Mode<MODE>::exact, Mode<MODE>::blocked>(buf, nbuf, a, lane, wc);
    }
}

// Would a round adding up to `room` hits overflow the warp's buffer?  The tiled rounds return to
// their caller to flush (flush_now): the hot loop's registers are dead there, and the flush's
// own (the output reservation) do not add to them.
template <int DIM, int MODE>
__device__ __forceinline__ bool needs_flush(const uint2 *buf, int nbuf, int room, int lane) {
    constexpr int CAP = BufCap<DIM>::value;
    if constexpr (Mode<MODE>::pairs) {
        return nbuf > CAP - room;
    } else {
        return false;
    }
}
template <int DIM, int MODE, bool GCG>
__device__ __forceinline__ void flush_now(uint2 *buf, int &nbuf, const JoinArgs &a, int lane, WarpCtl *wc) {
    if constexpr (Mode<MODE>::pairs) {
        nbuf = flush<GCG, Mode<MODE>::exact, Mode<MODE>::blocked>(buf, nbuf, a, lane, wc);
    }
}

// Flush whatever is buffered (end of an exact-sizing chunk, end of the kernel).
template <int DIM, int MODE, bool GCG>
__device__ __forceinline__ void flush_all(uint2 *buf, int &nbuf, const JoinArgs &a, int lane,
                                          WarpCtl *wc) {
    if constexpr (Mode<MODE>::pairs) {
        while (nbuf > 0) nbuf = flush<GCG, Mode<MODE>::exact, Mode<MODE>::blocked>(buf, nbuf, a, lane, wc);
    }
}

// Sum over the k lanes of a group (groups are aligned runs of K lanes).
template <int K>
__device__ __forceinline__ unsigned group_sum(unsigned v) {
#pragma unroll
    for (int o = K / 2; o > 0; o >>= 1) v += __shfl_xor_sync(kFull, v, o);
    return v;
}

// Home cell of one query (reading c8): position rr compares to rr+1, rr+2, ... (mod m), the
// first home_count(m, rr) of them --
//   * cells of <= 32 points (one WorkQueue chunk, one tile): the balanced circulant half scan,
//     rr+1 .. rr+floor((m-1)/2) (mod m), plus rr+m/2 when m is even and rr < m/2;
//   * larger cells (several chunks of 32 queries): the upper triangle rr+1 .. m-1, so a chunk
//     at positions [32c, 32c+32) evaluates only the home tiles from its own on, unmasked but for
//     the diagonal one (the circulant windows would mask half of every staged home tile).
// Either way every in-cell pair is evaluated exactly once and the cell's mean per-point load is
// ceil((m-1)/2) (a7's W, reading c9).
constexpr unsigned kTriMin = 33;
__device__ __forceinline__ unsigned home_count(unsigned m, unsigned rr) {
    if (m >= kTriMin) return m - 1u - rr;
    return (m - 1u) / 2u + (((m & 1u) == 0u && rr < m / 2u) ? 1u : 0u);
}

// Generic path: rounds of 32/k queries (possibly from different cells); the k lanes of a
// group walk their query's list -- forward runs first (identical for queries of one cell,
// so their loads coincide), then the home half scan -- taking candidates t, t+k, ...
template <int DIM, int K, int MODE, bool GCG>
__device__ __forceinline__ void generic_chunk(const JoinArgs &a, unsigned gmask, uint2 qm_lane, uint4 ci_lane,
                                              WarpSmem<DIM, MODE> &ws, int &nbuf, unsigned long long &nhits,
                                              unsigned &ncalcs, int lane, unsigned lt) {
    constexpr int PAD = PointPad<DIM>::value;
    constexpr int QPW = 32 / K;
    const int grp = lane / K;
    const unsigned t = (unsigned)(lane % K);
    const unsigned gbits = K == 32 ? kFull : (((1u << K) - 1u) << (lane & ~(K - 1)));
    uint2 *buf = ws.buf;
    unsigned char *glist = ws.glist;
    const unsigned nq = __popc(gmask);  // the chunk's queries handled here: lanes in gmask
    // compacted list of those lanes (a contiguous prefix in the common all-generic case)
    const bool prefix = gmask == (nq >= 32u ? 0xffffffffu : ((1u << nq) - 1u));
    if (!prefix) {
        __syncwarp();
        if ((gmask >> lane) & 1u) glist[__popc(gmask & lt)] = (unsigned char)lane;
        __syncwarp();
    }
    // Every generic query's point, input id and first forward runs are copied into shared
    // memory at once (cp.async, all lanes in parallel): a round then starts from shared memory
    // and its only global loads are the candidates -- one dependent global access per round
    // instead of two (the sparse tail of D' is latency-bound, not issue-bound).
    constexpr int GRS = GStage<DIM>::runs;
    if constexpr (GRS > 0) {
        __syncwarp();
        if ((gmask >> lane) & 1u) {
            cp_async_point<DIM>(ws.qry + lane * PAD, a.pts + (size_t)qm_lane.x * PAD);
            cp_async_4(ws.qorig + lane, a.orig + qm_lane.x);
#pragma unroll
            for (int j = 0; j < GRS; ++j)
                if (ci_lane.z + (unsigned)j < a.n_runs)
                    cp_async_8(ws.gruns + lane * StagedRuns<DIM>::value + j, a.runs + ci_lane.z + j);
        }
        cp_async_commit();
        cp_async_wait<0>();
        __syncwarp();
    }
    for (unsigned r0 = 0; r0 < nq; r0 += QPW) {
        const unsigned qi = r0 + grp;
        const bool valid = qi < nq;
        const int src = prefix ? (int)(qi & 31u) : (int)glist[qi & 31u];  // lane of the qi-th query
        const unsigned qlid = __shfl_sync(kFull, qm_lane.x, src);
        // the cell record was fetched per lane at chunk start: shuffle, do not reload
        uint4 ci;
        ci.x = __shfl_sync(kFull, ci_lane.x, src);
        ci.y = __shfl_sync(kFull, ci_lane.y, src);
        ci.z = __shfl_sync(kFull, ci_lane.z, src);
        ci.w = __shfl_sync(kFull, ci_lane.w, src);
        double qp[DIM];
        unsigned oq = 0;
        uint2 nxt = make_uint2(0, 0);
        if (!valid) ci = make_uint4(0, 0, 0, 0);
        unsigned long long cur = 0;  // kRows: the query's row cursor
        // staged runs of this query: grs[e] for e < elim (GRS > 0)
        const uint2 *grs = ws.gruns + src * StagedRuns<DIM>::value - ci.z;
        const unsigned elim = ci.z + (unsigned)GRS;
        if (valid) {
            if constexpr (GRS > 0) {
                load_smem_point<DIM>(ws.qry + src * PAD, qp);
                oq = ws.qorig[src];
                if (ci.w) nxt = grs[ci.z];
            } else {
                load_point<DIM>(a.pts + (size_t)qlid * PAD, qp);
                oq = __ldg(a.orig + qlid);
                if (ci.w) nxt = __ldg(a.runs + ci.z);  // prefetched next run
            }
            if constexpr (MODE == kRows) cur = __ldg(a.row_off + oq);
        } else {
#pragma unroll
            for (int d = 0; d < DIM; ++d) qp[d] = 0.0;
        }
        const unsigned hb = ci.x, m = ci.y;
        unsigned e = ci.z;
        unsigned rem = ci.w;  // forward candidates not yet entered
        const unsigned rr = qlid - hb;
        // GCG: the home cell is part of the runs (the full neighbourhood) -- no half scan
        const unsigned home_len = (valid && !GCG) ? home_count(m, rr) : 0u;
        const unsigned total = valid ? rem + home_len : 0u;
        unsigned seg_base = 0, seg_len = 0;
        bool home = false;
        unsigned i = t;  // lane t takes candidates t, t+k, ... of the list (Fig. 4)
        const unsigned my_iters = (total + (unsigned)K - 1u - t) / (unsigned)K;
        const unsigned iters = __reduce_max_sync(kFull, my_iters);  // warp-uniform trip count
        ncalcs += my_iters;
        if (GCG && valid && t == 0 && total) ncalcs -= 1;  // the query itself is skipped
        unsigned gi = t;
        const unsigned long long nh0 = nhits;
        for (unsigned it = 0; it < iters; ++it, gi += K) {
            bool hit = false;
            unsigned cidx = 0, oc = 0;
            if (gi < total) {
                while (i >= seg_len) {  // step to the run holding candidate gi
                    i -= seg_len;
                    if (rem) {
                        seg_base = nxt.x;
                        seg_len = nxt.y;
                        rem -= nxt.y;
                        if (rem) {
                            ++e;
                            nxt = (GRS > 0 && e < elim) ? grs[e] : __ldg(a.runs + e);
                        }
                    } else {
                        seg_base = hb;
                        seg_len = home_len;
                        home = true;
                    }
                }
                if (home) {
                    unsigned j = rr + 1u + i;
                    if (j >= m) j -= m;
                    cidx = hb + j;
                } else {
                    cidx = seg_base + i;
                }
                double cp[DIM];
                load_point<DIM>(a.pts + (size_t)cidx * PAD, cp);
                if (Mode<MODE>::pairs || MODE == kRows) oc = __ldg(a.orig + cidx);  // issued with the point, not after the test
                hit = sqdist<DIM>(qp, cp) <= a.e2;
                if (GCG) hit = hit && cidx != qlid;  // GCG scans its own cell: skip (q, q)
                i += K;
            }
            flush_if<DIM, MODE, GCG>(buf, nbuf, 32, a, lane, &ws.ctl);
            emit<DIM, MODE, GCG>(hit, oq, oc, buf, nbuf, nhits, lt, gbits, cur, a, lane);
        }
        if constexpr (MODE == kDegree) {  // the query's degree: its group's hits
            const unsigned deg = group_sum<K>((unsigned)(nhits - nh0));
            if (valid && t == 0) a.qdeg[oq] = deg;
        }
    }
}

// Flat path for short candidate lists (the sparse tail of D', whose chunks hold queries of
// small cells with similar W): the (query, candidate) pairs of all the chunk's generic queries
// are numbered f = 0 .. T-1 (query by query, each query's list as in generic_chunk: forward runs,
// then the home half scan) and lane l evaluates pairs l, l+32, ... -- FlatU per step, independent,
// so their candidate loads are in flight together.  The k-lane rounds of generic_chunk instead
// walk 32/k queries per round with a dependent global load chain each round, which is what the
// sparse tail's time is made of (it is latency-bound, not issue-bound).  The queries' points,
// ids and forward runs are staged in shared memory first; the query of pair f is the r-th
// non-empty list, r counted with a ballot and an OR-reduction of the lists' start bits.
// Returns false (nothing evaluated) when a list is longer than SJ_FLAT_W or a cell has more runs
// than are staged (UNICOMP).
template <int DIM, int MODE, bool GCG>
__device__ __forceinline__ bool flat_chunk(const JoinArgs &a, unsigned gmask, uint2 qm_lane, uint4 ci_lane,
                                           WarpSmem<DIM, MODE> &ws, int &nbuf, unsigned long long &nhits,
                                           unsigned &ncalcs, int lane, unsigned lt) {
    constexpr int PAD = PointPad<DIM>::value;
    constexpr int FRS = Flat<DIM, MODE, GCG>::runs;
    constexpr int SR = StagedRuns<DIM>::value;
    const bool mine = (gmask >> lane) & 1u;
    const unsigned rr_l = qm_lane.x - ci_lane.x;
    const unsigned W = mine ? ci_lane.w + home_count(ci_lane.y, rr_l) : 0u;
    if (__reduce_max_sync(kFull, W) > (unsigned)SJ_FLAT_W) return false;
    __syncwarp();
    if (mine) {
        cp_async_point<DIM>(ws.qry + lane * PAD, a.pts + (size_t)qm_lane.x * PAD);
        cp_async_4(ws.qorig + lane, a.orig + qm_lane.x);
#pragma unroll
        for (int j = 0; j < FRS; ++j)
            if (ci_lane.z + (unsigned)j < a.n_runs) cp_async_8(ws.gruns + lane * SR + j, a.runs + ci_lane.z + j);
    }
    unsigned incl = W;  // inclusive warp scan of the list lengths
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const unsigned v = __shfl_up_sync(kFull, incl, o);
        if (lane >= o) incl += v;
    }
    const unsigned T = __shfl_sync(kFull, incl, 31);
    const unsigned start = incl - W;  // the lane's first pair number
    const unsigned nem = __ballot_sync(kFull, W > 0u);
    if (W > 0u) ws.neq[__popc(nem & lt)] = (unsigned char)lane;
    ws.fq[lane] = make_uint4(ci_lane.x, ci_lane.y, rr_l, ci_lane.w);
    cp_async_commit();
    cp_async_wait<0>();
    __syncwarp();
    // the staged runs must cover the forward list (LID-UNICOMP: always; UNICOMP may have more)
    bool covered = true;
    if (mine) {
        unsigned acc = 0;
#pragma unroll
        for (int j = 0; j < FRS; ++j)
            if (acc < ci_lane.w) acc += ws.gruns[lane * SR + j].y;
        covered = acc == ci_lane.w;
    }
    if (!__all_sync(kFull, covered)) return false;
    ncalcs += W;
    unsigned long long cur = 0;
    constexpr int FU = FlatU<DIM>::value;
    for (unsigned f0 = 0; f0 < T; f0 += 32 * FU) {
        double qq[FU][DIM], cp[FU][DIM];
        unsigned oq[FU], oc[FU];
        bool ok[FU];
#pragma unroll
        for (int u = 0; u < FU; ++u) {
            const unsigned fb = f0 + (unsigned)(u * 32), f = fb + (unsigned)lane;
            ok[u] = f < T;
            // the query of pair f: the r-th non-empty list, r = the non-empty lists starting at
            // or before f (the starts of non-empty lists are distinct) -- those before the
            // window, plus the window's start bits up to f
            const unsigned rel = start - fb;
            const unsigned before = __ballot_sync(kFull, W > 0u && start < fb);
            const unsigned win = __reduce_or_sync(kFull, (W > 0u && rel < 32u) ? 1u << rel : 0u);
            const int r = __popc(before) + __popc(win & ((2u << lane) - 1u));  // >= 1: the first list starts at 0
            const unsigned q = ws.neq[r - 1];
            unsigned j = f - __shfl_sync(kFull, start, q);
            const uint4 d = ws.fq[q];  // {home begin, m, rr, S}
            unsigned idx;
            if (j < d.w) {  // forward runs, in order
                idx = 0;
                bool found = false;
#pragma unroll
                for (int r = 0; r < FRS; ++r) {
                    const uint2 run = ws.gruns[q * SR + r];
                    if (!found && j < run.y) {
                        idx = run.x + j;
                        found = true;
                    }
                    if (!found) j -= run.y;
                }
            } else {  // home cell: circulant half scan, offset j - S past rr (reading c8)
                unsigned p = d.z + 1u + (j - d.w);
                if (p >= d.y) p -= d.y;
                idx = d.x + p;
            }
            if (!ok[u]) idx = d.x;  // a valid address; masked below
            load_point<DIM>(a.pts + (size_t)idx * PAD, cp[u]);
            oc[u] = Mode<MODE>::pairs ? __ldg(a.orig + idx) : 0u;
            load_smem_point<DIM>(ws.qry + q * PAD, qq[u]);
            oq[u] = ws.qorig[q];
        }
        bool hit[FU];
#pragma unroll
        for (int u = 0; u < FU; ++u) hit[u] = ok[u] && sqdist<DIM>(qq[u], cp[u]) <= a.e2;
        flush_if<DIM, MODE, GCG>(ws.buf, nbuf, 32 * FU, a, lane, &ws.ctl);
#pragma unroll
        for (int u = 0; u < FU; ++u) emit<DIM, MODE, GCG>(hit[u], oq[u], oc[u], ws.buf, nbuf, nhits, lt, kFull, cur, a, lane);
    }
    return true;
}

// Evaluate one staged tile against every query of the chunk.  HOME != 0: the tile holds
// home-cell positions tb.. and a (query, slot) pair is inside the query's half scan (reading c8)
// iff (p - rr - 1) mod m < home_count(m, rr) -- HOME = 1, the circulant windows of cells of
// <= 32 points -- or iff p > rr -- HOME = 2, the upper triangle of larger cells.
// FULL (1-D..3-D register path): the tile holds 32 candidates and every round 32/k queries, so
// no slot or query validity is tested (the dense cells' common case).
template <int DIM, int K, int MODE, bool GCG, int HOME, bool FULL = false>
__device__ __forceinline__ unsigned tile_rounds(const JoinArgs &a, unsigned nq, unsigned nt, unsigned tb, unsigned m,
                                                WarpSmem<DIM, MODE> &ws, int b, int &nbuf, unsigned long long &nhits,
                                                int lane, unsigned lt, unsigned r_start) {
    const double *tile = ws.tile[b];
    const unsigned *tile_orig = ws.tile_orig[b];
    constexpr int PAD = PointPad<DIM>::value;
    constexpr int QPW = 32 / K;
    constexpr int SPL = 32 / K;  // tile slots per lane
    const int grp = lane / K;
    const unsigned t = (unsigned)(lane % K);
    const unsigned gbits = K == 32 ? kFull : (((1u << K) - 1u) << (lane & ~(K - 1)));
    // kRows / kDegree: the round's query cursor (count) lives in ws.qcur between rounds
    auto round_end = [&](unsigned qi, bool qv, unsigned long long cur, unsigned long long nh0) {
        if constexpr (MODE == kRows) {
            __syncwarp();  // every lane of the group read the cursor before it is advanced (racecheck)
            if (t == 0 && qv) ws.qcur[qi] = cur;
        } else if constexpr (MODE == kDegree) {
            const unsigned d = group_sum<K>((unsigned)(nhits - nh0));
            if (t == 0 && qv) ws.qcur[qi] += d;
        }
    };
    if constexpr (SPL <= 4 && DIM <= 3) {  // tile slots in registers (register budget)
        double cp[SPL][DIM];
        unsigned co[SPL];
        bool cv[SPL];
#pragma unroll
        for (int s = 0; s < SPL; ++s) {
            const unsigned j = t + (unsigned)(K * s);
            cv[s] = FULL || j < nt;
            load_smem_point<DIM>(tile + (j & 31) * PAD, cp[s]);
            co[s] = tile_orig[j & 31];
        }
        for (unsigned r0 = r_start; r0 < nq; r0 += QPW) {
            if (needs_flush<DIM, MODE>(ws.buf, nbuf, 32 * SPL, lane)) return r0;  // the caller flushes
            const unsigned qi = (r0 + grp) & 31;
            const bool qv = FULL || r0 + grp < nq;
            double qq[DIM];
            load_smem_point<DIM>(ws.qry + qi * PAD, qq);
            const unsigned oq = ws.qorig[qi];
            unsigned rr = 0, hl = 0;
            if (HOME) rr = ws.qrr[qi];
            if (HOME == 1) hl = home_count(m, rr);
            unsigned long long cur = MODE == kRows ? ws.qcur[qi] : 0ull;
            const unsigned long long nh0 = nhits;
            // all SPL distances first (independent FP64 chains -> ILP), then the emissions;
            // evaluated unconditionally and masked after (invalid slots may hold stale or
            // uninitialised bits; FP64 arithmetic on them cannot trap)
            bool close[SPL];
#pragma unroll
            for (int s = 0; s < SPL; ++s) close[s] = sqdist<DIM>(qq, cp[s]) <= a.e2;
#pragma unroll
            for (int s = 0; s < SPL; ++s) {
                bool ok = qv & cv[s];
                if (GCG) ok = ok & (co[s] != oq);  // GCG: skip (q, q)
                if (HOME == 1) {
                    int d = (int)(tb + t + (unsigned)(K * s)) - (int)rr - 1;
                    if (d < 0) d += (int)m;
                    ok = ok & ((unsigned)d < hl);
                } else if (HOME == 2) {
                    ok = ok & (tb + t + (unsigned)(K * s) > rr);
                }
                emit<DIM, MODE, GCG>(close[s] & ok, oq, co[s], ws.buf, nbuf, nhits, lt, gbits, cur, a, lane);
            }
            round_end(qi, qv, cur, nh0);
        }
    } else if constexpr (DIM >= 4) {
        // Higher dimensions: a lane keeps ONE tile slot (its candidate, 2*DIM registers) for the
        // whole tile and the warp walks the segment's queries two at a time; the query reads are
        // shared-memory broadcasts, so each staged coordinate is read once per lane per tile
        // instead of once per round (the k-lane split of the rounds above is a register-budget
        // device of the low-dimensional path; all 32 lanes serve one query here).
        const bool cv = (unsigned)lane < nt;
        double cp[DIM];
        load_smem_point<DIM>(tile + lane * PAD, cp);
        const unsigned co = tile_orig[lane];
        int dh = (int)(tb + (unsigned)lane) - 1;  // HOME: slot position - 1, minus rr below
        for (unsigned q0 = r_start; q0 < nq; q0 += 2) {
            if (needs_flush<DIM, MODE>(ws.buf, nbuf, 64, lane)) return q0;  // the caller flushes
            const unsigned q1 = q0 + 1;
            const bool v1 = q1 < nq;
            double qa[DIM], qb[DIM];
            load_smem_point<DIM>(ws.qry + q0 * PAD, qa);
            load_smem_point<DIM>(ws.qry + (q1 & 31) * PAD, qb);
            const bool ca = sqdist<DIM>(qa, cp) <= a.e2;  // two independent FP64 chains
            const bool cb = sqdist<DIM>(qb, cp) <= a.e2;
            const unsigned oqa = ws.qorig[q0], oqb = ws.qorig[q1 & 31];
            bool oka = cv, okb = cv & v1;
            if (GCG) {  // skip (q, q)
                oka = oka & (co != oqa);
                okb = okb & (co != oqb);
            }
            if (HOME == 1) {
                const unsigned rra = ws.qrr[q0], rrb = ws.qrr[q1 & 31];
                int da = dh - (int)rra, db = dh - (int)rrb;
                if (da < 0) da += (int)m;
                if (db < 0) db += (int)m;
                oka = oka & ((unsigned)da < home_count(m, rra));
                okb = okb & ((unsigned)db < home_count(m, rrb));
            } else if (HOME == 2) {
                oka = oka & (dh >= (int)ws.qrr[q0]);
                okb = okb & (dh >= (int)ws.qrr[q1 & 31]);
            }
            const bool ha = ca & oka, hb = cb & okb;
            unsigned long long cura = 0, curb = 0;
            if constexpr (MODE == kRows) {
                cura = ws.qcur[q0];
                curb = ws.qcur[q1 & 31];
            }
            emit<DIM, MODE, GCG>(ha, oqa, co, ws.buf, nbuf, nhits, lt, kFull, cura, a, lane);
            emit<DIM, MODE, GCG>(hb, oqb, co, ws.buf, nbuf, nhits, lt, kFull, curb, a, lane);
            if constexpr (MODE == kRows) {
                __syncwarp();
                if (lane == 0) {
                    ws.qcur[q0] = cura;
                    if (v1) ws.qcur[q1] = curb;
                }
                __syncwarp();
            } else if constexpr (MODE == kDegree) {
                const unsigned na = __popc(__ballot_sync(kFull, ha)), nb = __popc(__ballot_sync(kFull, hb));
                if (lane == 0) {
                    ws.qcur[q0] += na;
                    if (v1) ws.qcur[q1] += nb;
                }
                __syncwarp();
            }
        }
    } else {  // tile slots read from shared memory each step (low dimensions, k < 8)
        for (unsigned r0 = r_start; r0 < nq; r0 += QPW) {
            const unsigned qi = (r0 + grp) & 31;
            const bool qv = r0 + grp < nq;
            double qq[DIM];
            load_smem_point<DIM>(ws.qry + qi * PAD, qq);
            const unsigned oq = ws.qorig[qi];
            unsigned rr = 0, hl = 0;
            if (HOME) rr = ws.qrr[qi];
            if (HOME == 1) hl = home_count(m, rr);
            unsigned long long cur = MODE == kRows ? ws.qcur[qi] : 0ull;
            const unsigned long long nh0 = nhits;
#pragma unroll 2
            for (int s = 0; s < SPL; s += 2) {  // two slots per step: two independent FP64 chains
                flush_if<DIM, MODE, GCG>(ws.buf, nbuf, 64, a, lane, &ws.ctl);
                const unsigned j0 = t + (unsigned)(K * s), j1 = j0 + (unsigned)K;
                double c0[DIM], c1[DIM];
                load_smem_point<DIM>(tile + (j0 & 31) * PAD, c0);
                load_smem_point<DIM>(tile + (j1 & 31) * PAD, c1);
                // evaluated unconditionally and masked after (see above)
                const bool close0 = sqdist<DIM>(qq, c0) <= a.e2;
                const bool close1 = sqdist<DIM>(qq, c1) <= a.e2;
                bool ok0 = qv & (j0 < nt), ok1 = qv & (s + 1 < SPL) & (j1 < nt);
                if (GCG) {  // skip (q, q)
                    ok0 = ok0 & (tile_orig[j0 & 31] != oq);
                    ok1 = ok1 & (tile_orig[j1 & 31] != oq);
                }
                if (HOME == 1) {
                    int d0 = (int)(tb + j0) - (int)rr - 1, d1 = (int)(tb + j1) - (int)rr - 1;
                    if (d0 < 0) d0 += (int)m;
                    if (d1 < 0) d1 += (int)m;
                    ok0 = ok0 & ((unsigned)d0 < hl);
                    ok1 = ok1 & ((unsigned)d1 < hl);
                } else if (HOME == 2) {
                    ok0 = ok0 & (tb + j0 > rr);
                    ok1 = ok1 & (tb + j1 > rr);
                }
                const bool hit0 = close0 & ok0, hit1 = close1 & ok1;
                emit<DIM, MODE, GCG>(hit0, oq, hit0 ? tile_orig[j0 & 31] : 0u, ws.buf, nbuf, nhits, lt, gbits,
                                            cur, a, lane);
                emit<DIM, MODE, GCG>(hit1, oq, hit1 ? tile_orig[j1 & 31] : 0u, ws.buf, nbuf, nhits, lt, gbits,
                                            cur, a, lane);
            }
            round_end(qi, qv, cur, nh0);
        }
    }
    return nq;
}

#ifndef SJ_HOMEWIN
#define SJ_HOMEWIN 1
#endif
// Home cell of at most 32 points (one staged tile, tb = 0): instead of evaluating every
// (query, slot) pair of the tile and masking half of them out (tile_rounds<HOME>), lane t of
// a group evaluates only the query's circulant window (reading c8): window offsets i = t,
// t+k, ... < home_count(m, rr) <= 16, slot (rr + 1 + i) mod m read from shared memory.
template <int DIM, int K, int MODE, bool GCG>
__device__ __forceinline__ unsigned home_window_rounds(const JoinArgs &a, unsigned nq, unsigned m,
                                                       WarpSmem<DIM, MODE> &ws, int b, int &nbuf,
                                                       unsigned long long &nhits, int lane, unsigned lt,
                                                       unsigned r_start) {
    constexpr int PAD = PointPad<DIM>::value;
    constexpr int QPW = 32 / K;
    constexpr int WS = (16 + K - 1) / K;  // window slots per lane
    const double *tile = ws.tile[b];
    const unsigned *tile_orig = ws.tile_orig[b];
    const int grp = lane / K;
    const unsigned t = (unsigned)(lane % K);
    const unsigned gbits = K == 32 ? kFull : (((1u << K) - 1u) << (lane & ~(K - 1)));
    for (unsigned r0 = r_start; r0 < nq; r0 += QPW) {
        if (needs_flush<DIM, MODE>(ws.buf, nbuf, 32 * WS, lane)) return r0;  // the caller flushes
        const unsigned qi = (r0 + grp) & 31;
        const bool qv = r0 + grp < nq;
        double qq[DIM];
        load_smem_point<DIM>(ws.qry + qi * PAD, qq);
        const unsigned oq = ws.qorig[qi];
        const unsigned rr = ws.qrr[qi];
        const unsigned hl = home_count(m, rr);
        unsigned long long cur = 0;
        double cp[WS][DIM];
        unsigned co[WS];
        bool ok[WS], close[WS];
#pragma unroll
        for (int s = 0; s < WS; ++s) {
            const unsigned i = t + (unsigned)(K * s);
            ok[s] = qv && i < hl;
            unsigned p = rr + 1u + i;
            if (p >= m) p -= m;
            p &= 31u;
            load_smem_point<DIM>(tile + p * PAD, cp[s]);
            co[s] = tile_orig[p];
        }
#pragma unroll
        for (int s = 0; s < WS; ++s) close[s] = sqdist<DIM>(qq, cp[s]) <= a.e2;
#pragma unroll
        for (int s = 0; s < WS; ++s)
            emit<DIM, MODE, GCG>(close[s] & ok[s], oq, co[s], ws.buf, nbuf, nhits, lt, gbits, cur, a, lane);
    }
    return nq;
}

// Tiled path: all nq queries of the chunk lie in one cell (hb, m, runs rb.., S forward
// candidates).  The forward runs, then the home cell, are staged 32 candidates at a time in
// shared memory (points + input ids); lane t of a group holds tile slots t, t+k, ... and
// evaluates them against one query per round of 32/k queries, so each staged candidate
// serves the whole chunk.
template <int DIM, int K, int MODE, bool GCG>
__device__ __forceinline__ void tiled_chunk(const JoinArgs &a, unsigned s0, unsigned nq, uint2 qm_lane, uint4 ci,
                                            WarpSmem<DIM, MODE> &ws, int &nbuf, unsigned long long &nhits,
                                            unsigned &ncalcs, int lane, unsigned lt) {
    constexpr int PAD = PointPad<DIM>::value;
    const unsigned hb = ci.x, m = ci.y, S = ci.w;
    __syncwarp();
    const unsigned slot = (unsigned)lane - s0;  // the segment's queries are lanes s0 .. s0+nq-1
    if (slot < nq) {
        copy_point_to_smem<DIM>(a.pts + (size_t)qm_lane.x * PAD, ws.qry + slot * PAD);
        const unsigned oq = __ldg(a.orig + qm_lane.x);
        ws.qorig[slot] = oq;
        if constexpr (MODE == kRows) ws.qcur[slot] = __ldg(a.row_off + oq);
        if constexpr (MODE == kDegree) ws.qcur[slot] = 0;
        const unsigned rr = qm_lane.x - hb;
        ws.qrr[slot] = rr;
        // this query's distance calculations
        ncalcs += GCG ? S - 1u : S + home_count(m, rr);
    }
    // ---- forward runs (LID-UNICOMP): tiles staged with cp.async, double-buffered, so the
    // next tile's global loads overlap this tile's distance calculations
    const uint2 *runs = a.runs + ci.z;
    bool runs_smem = false;
    if constexpr (DIM >= 4 && DIM <= 6) {  // copy the cell's runs until their lengths add up to S
        unsigned acc = 0;
        for (unsigned k0 = 0; acc < S && k0 < 128u; k0 += 32) {
            const unsigned k = k0 + (unsigned)lane;
            const uint2 f = (ci.z + k < a.n_runs) ? __ldg(a.runs + ci.z + k) : make_uint2(0, 0);
            ws.runs_s[k] = f;
            acc += __reduce_add_sync(kFull, f.y);
        }
        __syncwarp();
        runs_smem = acc >= S;  // GCG / UNICOMP lists can exceed 128 runs: keep reading L2 then
        if (runs_smem) runs = ws.runs_s;
    }
    unsigned e = 0, seg_base = 0, seg_len = 0, i = (unsigned)lane;
    auto stage_fwd = [&](int b, unsigned tb) {
        if (tb + (unsigned)lane < S) {
            while (i >= seg_len) {
                i -= seg_len;
                const uint2 f = runs_smem ? runs[e++] : __ldg(runs + (e++));
                seg_base = f.x;
                seg_len = f.y;
            }
            const unsigned cidx = seg_base + i;
            cp_async_point<DIM>(ws.tile[b] + lane * PAD, a.pts + (size_t)cidx * PAD);
            cp_async_4(ws.tile_orig[b] + lane, a.orig + cidx);
            i += 32;
        }
        cp_async_commit();
    };
    if (S) stage_fwd(0, 0);
    int it = 0;
    for (unsigned tb = 0; tb < S; tb += 32, ++it) {
        const bool more = tb + 32 < S;
        if (more) stage_fwd((it + 1) & 1, tb + 32);
        if (more)
            cp_async_wait<1>();
        else
            cp_async_wait<0>();
        __syncwarp();
        const unsigned nt = min(32u, S - tb);
        const bool full = DIM <= 3 && nt == 32u && nq % (32u / K) == 0u;
        for (unsigned r = 0; r < nq;) {  // (the rounds return to flush the buffer)
            if (full)
                r = tile_rounds<DIM, K, MODE, GCG, 0, true>(a, nq, nt, tb, m, ws, it & 1, nbuf, nhits, lane, lt, r);
            else
                r = tile_rounds<DIM, K, MODE, GCG, 0>(a, nq, nt, tb, m, ws, it & 1, nbuf, nhits, lane, lt, r);
            if (r < nq) flush_now<DIM, MODE, GCG>(ws.buf, nbuf, a, lane, &ws.ctl);
        }
        __syncwarp();
    }
    // ---- home cell: the half scan (reading c8) as a mask over staged home tiles; in the upper
    // triangle of a large cell the tiles before the segment's first query hold no candidate
    auto stage_home = [&](int b, unsigned tb) {
        if (tb + (unsigned)lane < m) {
            const unsigned cidx = hb + tb + (unsigned)lane;
            cp_async_point<DIM>(ws.tile[b] + lane * PAD, a.pts + (size_t)cidx * PAD);
            cp_async_4(ws.tile_orig[b] + lane, a.orig + cidx);
        }
        cp_async_commit();
    };
    if constexpr (GCG) {  // GCG: the home cell was one of the runs
        if constexpr (MODE == kDegree) {
            if (slot < nq) a.qdeg[ws.qorig[slot]] = (unsigned)ws.qcur[slot];
            __syncwarp();
        }
        return;
    }
    unsigned tb0 = 0;
    if (m >= kTriMin) {
        // (re-read from shared memory: nothing of the segment's set-up stays live across the
        // forward tiles, which would cost the 1-D..3-D kernels their 64-register budget)
        const unsigned rmin = __reduce_min_sync(kFull, (unsigned)lane < nq ? ws.qrr[lane] : 0xFFFFFFFFu);
        tb0 = ((rmin + 1u) / 32u) * 32u;
    }
    stage_home(0, tb0);
    if constexpr (SJ_HOMEWIN && !GCG && DIM <= 3 && K >= 4 && MODE != kRows && MODE != kDegree) {
        if (m <= 32u) {  // one tile: evaluate the circulant windows only
            cp_async_wait<0>();
            __syncwarp();
            for (unsigned r = 0; r < nq;) {  // (the rounds return to flush the buffer)
                r = home_window_rounds<DIM, K, MODE, GCG>(a, nq, m, ws, 0, nbuf, nhits, lane, lt, r);
                if (r < nq) flush_now<DIM, MODE, GCG>(ws.buf, nbuf, a, lane, &ws.ctl);
            }
            __syncwarp();
            return;
        }
    }
    it = 0;
    for (unsigned tb = tb0; tb < m; tb += 32, ++it) {
        const bool more = tb + 32 < m;
        if (more) stage_home((it + 1) & 1, tb + 32);
        if (more)
            cp_async_wait<1>();
        else
            cp_async_wait<0>();
        __syncwarp();
        // (with the circulant windows of small cells evaluated above, only the triangle remains
        // for the 1-D..3-D pair kernels; the others take either)
        constexpr bool kOnlyTri = SJ_HOMEWIN && DIM <= 3 && K >= 4 && MODE != kRows && MODE != kDegree;
        // 3-D: full triangle tiles without validity tests too (C3 K64 -1 %; in 2-D the extra
        // instantiation spilled and cost 1.7 % on C5, measured)
        const bool hfull = DIM == 3 && m - tb >= 32u && nq % (32u / K) == 0u;
        for (unsigned r = 0; r < nq;) {  // (the rounds return to flush the buffer)
            if ((kOnlyTri || m >= kTriMin) && hfull)
                r = tile_rounds<DIM, K, MODE, GCG, 2, DIM == 3>(a, nq, 32u, tb, m, ws, it & 1, nbuf, nhits, lane, lt, r);
            else if (kOnlyTri || m >= kTriMin)
                r = tile_rounds<DIM, K, MODE, GCG, 2>(a, nq, min(32u, m - tb), tb, m, ws, it & 1, nbuf, nhits, lane, lt, r);
            else
                r = tile_rounds<DIM, K, MODE, GCG, 1>(a, nq, min(32u, m - tb), tb, m, ws, it & 1, nbuf, nhits, lane, lt, r);
            if (r < nq) flush_now<DIM, MODE, GCG>(ws.buf, nbuf, a, lane, &ws.ctl);
        }
        __syncwarp();
    }
}

// 3-D kernels are held to three resident CTAs per SM (their shared-memory limit), i.e. up to 85
// registers: ptxas' own choice otherwise drifts between 64 with spills and 80 with small changes.
#ifndef SJ_MINB3
#define SJ_MINB3 3
#endif
template <int DIM>
struct MinBlocks {
    static constexpr int value = DIM == 3 ? SJ_MINB3 : 0;
};

template <int DIM, int K, int MODE, bool GCG>
__global__ void __launch_bounds__(kJoinThreads, MinBlocks<DIM>::value) join_kernel(const JoinArgs a) {
    static_assert(32 % K == 0, "k must divide 32");
    constexpr int QPW = 32 / K;
    extern __shared__ __align__(16) unsigned char smem_raw[];
    const int lane = threadIdx.x & 31;
    const int warp = threadIdx.x >> 5;
    const unsigned lt = (1u << lane) - 1u;
    WarpSmem<DIM, MODE> &ws = reinterpret_cast<WarpSmem<DIM, MODE> *>(smem_raw)[warp];
    int nbuf = 0;  // hits in the warp's buffer (pair modes)
    unsigned long long nhits = 0;
    unsigned ncalcs = 0;  // this lane's distance calculations (instrumented runs; 32 bits per lane)
    // The batch: virtual chunks v_begin, v_begin + v_stride, ... < v_end (contiguous, or the
    // strided D'_l of the SortByWL-only batches); i indexes them.  A device-sized
    // launch reads the build's chunk count here: V = the slice's chunks (rank, world).
    if (lane == 0) {
        unsigned vc = a.v_count;
        unsigned long long sv1 = a.sample_v1;
        if (a.d_nchunks) {
            const unsigned nch = *a.d_nchunks;  // 32-bit arithmetic: no division subroutine
            const unsigned long long V = nch > a.rank ? (nch - a.rank + a.world - 1u) / a.world : 0u;
            vc = (unsigned)V;
            if (a.sample_ppm) {  // the estimator's sample: the first ceil(V * ppm / 1e6) chunks
                sv1 = (V * a.sample_ppm + 999999ull) / 1000000ull;
                if (sv1 < 1) sv1 = 1;
                sv1 = (sv1 + a.grab - 1) / a.grab * a.grab;  // whole dequeues (as the host rounds)
                if (sv1 > V) sv1 = V;
            }
        }
        ws.ctl.vcount = vc;
        ws.ctl.sv1 = sv1;
        ws.ctl.wcur = ws.ctl.wtot = ws.ctl.samp = 0;
        ws.ctl.sclosed = 0;
        ws.ctl.ocur = ws.ctl.oend = 0;
    }

    // a kernel parameter, not a register: the dequeue compares against the constant bank (a
    // register here costs the 1-D..3-D kernels 16 registers and a quarter of their occupancy)
    const unsigned vcount = a.v_count;
    if (lane == 0) ws.snext = (blockIdx.x * (unsigned)kWarps + (unsigned)warp) * a.grab;  // static assignment
    for (;;) {
        // WorkQueue dequeue: one atomic per warp, result shuffled.  SortByWL only
        // (static_q): warp w takes w, w + #warps, ... in D' order, no atomics (the
        // cursor lives in shared memory, not in a register of the hot loops).
        // kPairs: a warp whose flush found the output full stops (the caller re-runs staged).
        unsigned ib = 0;
        if (lane == 0) {
            if (Mode<MODE>::inplace && ws.ctl.wcur) {
                ib = vcount;
            } else if (a.static_q) {
                ib = ws.snext;
                ws.snext = ib + gridDim.x * (unsigned)kWarps * a.grab;
            } else {
                ib = (unsigned)atomicAdd(a.head, (unsigned long long)a.grab);
            }
            // device-sized launch (a.v_count = ~0u): the bound the prologue read (grab 1)
            if (ib >= ws.ctl.vcount) ib = 0xFFFFFFFFu;
            // fused estimator (a9; v_begin 0, stride 1; the sample is whole dequeues): on the
            // first dequeue past the sample, this warp's hits so far all came from sample chunks
            if (Mode<MODE>::inplace && !ws.ctl.sclosed && ib >= ws.ctl.sv1) {
                ws.ctl.samp = ws.ctl.wtot + (unsigned long long)nbuf;
                ws.ctl.sclosed = 1;
            }
        }
        ib = __shfl_sync(kFull, ib, 0);
        if (ib >= vcount) break;
        const unsigned iend = min(ib + a.grab, vcount);
        for (unsigned i = ib; i < iend; ++i) {
            const unsigned long long v = a.v_begin + (unsigned long long)i * a.v_stride;
            const unsigned long long c = v * a.world + a.rank;  // queue slice (multi-GPU)
            // (a device-sized launch bounds this by 0xFFFFFFFF: its last dequeue may pass the
            // build's chunk count by < grab * world chunks, which the build pads with empty ones)
            if (c >= a.n_chunks) break;
            if constexpr (MODE == kExact) {  // exact sizing: the chunk's pairs start at voff[v]
                if (lane == 0) ws.ctl.wcur = __ldg(a.voff + v) - a.out_base;
                __syncwarp();
            }
            const unsigned long long nh0 = nhits;
            const unsigned qs = __ldg(a.chunks + c), qe = __ldg(a.chunks + c + 1);
            const unsigned nq = qe - qs;  // 1..32 D' positions
            const bool lv = (unsigned)lane < nq;
            const uint2 qm = lv ? __ldg(a.qmap + qs + lane) : make_uint2(0, 0xFFFFFFFFu);
            // The chunk's queries form segments of one cell each (D' keeps cells contiguous).
            // A segment whose cell has a long candidate list is evaluated tile by tile from
            // shared memory (each staged candidate serves every query of the segment); the
            // remaining queries go through the generic per-query path together.
            const unsigned prev = __shfl_up_sync(kFull, qm.y, 1);
            const bool head = lv && (lane == 0 || qm.y != prev);
            const unsigned heads = __ballot_sync(kFull, head);
            // every lane fetches its own cell record in parallel; heads decide for their segment
            const uint4 ci = lv ? __ldg(a.cellq + qm.y) : make_uint4(0, 0, 0, 0);
            const unsigned later = heads & ~(0xffffffffu >> (31 - lane));  // heads after this lane
            const unsigned seg_end = later ? (unsigned)(__ffs(later) - 1) : nq;
            const unsigned nseg = seg_end - (unsigned)lane;  // meaningful on head lanes
            const bool tiled = head && ((nseg >= 2u * QPW && ci.y >= kBigCell) ||
                                        (DIM >= 4 && nseg >= 2u && ci.w >= kTileMinCand));
            unsigned theads = __ballot_sync(kFull, tiled);
            const int my_head = 31 - __clz(heads & (0xffffffffu >> (31 - lane)));
            const unsigned gmask = __ballot_sync(kFull, lv && !((theads >> (my_head & 31)) & 1u));
            while (theads) {
                const int s0 = __ffs(theads) - 1;
                theads &= theads - 1;
                uint4 cs;
                cs.x = __shfl_sync(kFull, ci.x, s0);
                cs.y = __shfl_sync(kFull, ci.y, s0);
                cs.z = __shfl_sync(kFull, ci.z, s0);
                cs.w = __shfl_sync(kFull, ci.w, s0);
                const unsigned n0 = __shfl_sync(kFull, nseg, s0);
                tiled_chunk<DIM, K, MODE, GCG>(a, (unsigned)s0, n0, qm, cs, ws, nbuf, nhits, ncalcs, lane, lt);
            }
            if (gmask) {
                bool done = false;
                if constexpr (Flat<DIM, MODE, GCG>::on)
                    done = flat_chunk<DIM, MODE, GCG>(a, gmask, qm, ci, ws, nbuf, nhits, ncalcs, lane, lt);
                if (!done) generic_chunk<DIM, K, MODE, GCG>(a, gmask, qm, ci, ws, nbuf, nhits, ncalcs, lane, lt);
            }
            if constexpr (MODE == kExact) {  // exact sizing: a chunk's pairs never share a flush
                flush_all<DIM, MODE, GCG>(ws.buf, nbuf, a, lane, &ws.ctl);
            } else if constexpr (MODE == kChunkCount) {  // exact sizing, pass 1: pairs per chunk
                unsigned long long d = nhits - nh0;
#pragma unroll
                for (int o = 16; o > 0; o >>= 1) d += __shfl_xor_sync(kFull, d, o);
                if (lane == 0) a.vcount[v] = d;
            }
            (void)nh0;
        }
    }
    if constexpr (Mode<MODE>::pairs) {
        flush_all<DIM, MODE, GCG>(ws.buf, nbuf, a, lane, &ws.ctl);
        if (Mode<MODE>::inplace && a.sample_ctr && lane == 0) {
            const unsigned long long sh = ws.ctl.sclosed ? ws.ctl.samp : ws.ctl.wtot;
            if (sh) atomicAdd(a.sample_ctr, (GCG ? 1ull : 2ull) * sh);
        }
    } else {
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) nhits += __shfl_xor_sync(kFull, nhits, o);
        if (lane == 0 && nhits) atomicAdd(a.emit_ctr, nhits);
    }
    if (a.calcs) {
#pragma unroll
        unsigned long long c = ncalcs;
        for (int o = 16; o > 0; o >>= 1) c += __shfl_xor_sync(kFull, c, o);
        if (lane == 0 && c) atomicAdd(a.calcs, c);
    }
    if (Mode<MODE>::blocked && lane == 0) {  // the warp's last block: its unused rest is a gap
        const unsigned gw = blockIdx.x * (unsigned)kWarps + (unsigned)warp;
        a.gaps[2 * gw] = ws.ctl.ocur;
        a.gaps[2 * gw + 1] = ws.ctl.oend - ws.ctl.ocur;
    }
}

}  // namespace

}  // namespace sj
