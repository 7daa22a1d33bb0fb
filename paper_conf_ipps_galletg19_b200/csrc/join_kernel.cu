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
//     the result to its group; here the leader is lane 0 of the warp and
//     the warp takes SJ_OPT_GRAB consecutive positions per atomic.
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
#include "sj_internal.cuh"

namespace sj {

namespace {

constexpr unsigned kFull = 0xffffffffu;
constexpr int kWarps = kJoinThreads / 32;
constexpr int kBufHits = 256;  // hits (= 2 pairs = 16 B) buffered per warp

template <int DIM>
struct PointPad {
    static constexpr int value = DIM == 1 ? 1 : ((DIM + 1) & ~1);
};

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

__device__ __forceinline__ void flush(uint4 *buf, int nbuf, const JoinArgs &a, int lane) {
    __syncwarp();
    unsigned long long base = 0;
    if (lane == 0) base = atomicAdd(a.emit_ctr, 2ull * (unsigned long long)nbuf);
    base = __shfl_sync(kFull, base, 0);
    uint4 *out4 = reinterpret_cast<uint4 *>(a.out);
    uint2 *out2 = reinterpret_cast<uint2 *>(a.out);
    for (int k = lane; k < nbuf; k += 32) {
        const unsigned long long slot = base + 2ull * (unsigned long long)k;  // even
        const uint4 v = buf[k];
        if (slot + 2 <= a.out_cap)
            __stcs(out4 + (slot >> 1), v);
        else if (slot < a.out_cap)
            __stcs(out2 + slot, make_uint2(v.x, v.y));
    }
    __syncwarp();
}

template <int DIM, int K, bool EMIT>
__global__ void __launch_bounds__(kJoinThreads) join_kernel(const JoinArgs a) {
    static_assert(32 % K == 0, "k must divide 32");
    constexpr int PAD = PointPad<DIM>::value;
    constexpr int QPW = 32 / K;  // query points per warp step
    __shared__ uint4 sbuf[EMIT ? kWarps : 1][EMIT ? kBufHits : 1];

    const int lane = threadIdx.x & 31;
    const int warp = threadIdx.x >> 5;
    const int grp = lane / K;
    const unsigned t = (unsigned)(lane % K);
    const unsigned lt = (1u << lane) - 1u;
    uint4 *buf = sbuf[EMIT ? warp : 0];
    int nbuf = 0;
    unsigned long long nhits = 0;
    unsigned long long ncalcs = 0;

    for (;;) {
        // WorkQueue dequeue: one atomic per warp, result shuffled
        unsigned long long vb = 0;
        if (lane == 0) vb = atomicAdd(a.head, (unsigned long long)a.grab);
        vb = __shfl_sync(kFull, vb, 0);
        if (vb >= a.v_end) break;
        // queue slice (multi-GPU): virtual chunk -> physical chunk
        const unsigned long long pchunk = (vb / a.grab) * a.world + a.rank;
        const unsigned long long qbase = pchunk * a.grab;
        const unsigned long long qlim = min(qbase + a.grab, (unsigned long long)a.n);

        for (unsigned r0 = 0; r0 < a.grab; r0 += QPW) {
            const unsigned long long q = qbase + r0 + grp;
            const bool valid = q < qlim;
            if (!__any_sync(kFull, valid)) break;

            double qp[DIM];
            unsigned oq = 0;
            uint4 ci = make_uint4(0, 0, 0, 0);
            if (valid) {
                load_point<DIM>(a.pts + q * PAD, qp);
                oq = __ldg(a.orig + q);
                ci = __ldg(a.cellq + __ldg(a.pcell + q));
            } else {
#pragma unroll
                for (int d = 0; d < DIM; ++d) qp[d] = 0.0;
            }
            const unsigned hb = ci.x, m = ci.y;
            unsigned e = ci.z;
            const unsigned fe = ci.w;
            const unsigned rr = (unsigned)(q - hb);
            // home cell: balanced circulant half scan (reading c8)
            unsigned seg_len = valid ? ((m - 1u) / 2u + (((m & 1u) == 0u && rr < m / 2u) ? 1u : 0u)) : 0u;
            unsigned seg_base = hb;
            bool home = true;
            bool done = !valid;
            unsigned i = t;  // lane t takes candidates t, t+k, ... (Fig. 4)

            for (;;) {
                while (!done && i >= seg_len) {
                    i -= seg_len;
                    if (e >= fe) {
                        done = true;
                    } else {
                        const uint2 f = __ldg(a.fwd + e);  // next forward cell (LID-UNICOMP)
                        ++e;
                        seg_base = f.x;
                        seg_len = f.y;
                        home = false;
                    }
                }
                if (__ballot_sync(kFull, !done) == 0u) break;
                bool hit = false;
                unsigned cidx = 0;
                if (!done) {
                    if (home) {
                        unsigned j = rr + 1u + i;
                        if (j >= m) j -= m;
                        cidx = hb + j;
                    } else {
                        cidx = seg_base + i;
                    }
                    double cp[DIM];
                    load_point<DIM>(a.pts + (size_t)cidx * PAD, cp);
                    hit = sqdist<DIM>(qp, cp) <= a.e2;
                    i += K;
                    ++ncalcs;
                }
                if constexpr (EMIT) {
                    const unsigned hm = __ballot_sync(kFull, hit);
                    if (hm) {
                        if (hit) {
                            const unsigned oc = __ldg(a.orig + cidx);
                            buf[nbuf + __popc(hm & lt)] = make_uint4(oq, oc, oc, oq);  // (q,c) and (c,q)
                        }
                        nbuf += __popc(hm);
                        if (nbuf > kBufHits - 32) {
                            flush(buf, nbuf, a, lane);
                            nbuf = 0;
                        }
                    }
                } else {
                    nhits += hit ? 2ull : 0ull;
                }
            }
        }
    }
    if constexpr (EMIT) {
        if (nbuf > 0) flush(buf, nbuf, a, lane);
    } else {
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) nhits += __shfl_xor_sync(kFull, nhits, o);
        if (lane == 0 && nhits) atomicAdd(a.emit_ctr, nhits);
    }
    if (a.calcs) {
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) ncalcs += __shfl_xor_sync(kFull, ncalcs, o);
        if (lane == 0 && ncalcs) atomicAdd(a.calcs, ncalcs);
    }
}

typedef void (*join_fn)(const JoinArgs);

template <int DIM, bool EMIT>
join_fn pick_k(int k) {
    switch (k) {
        case 1: return join_kernel<DIM, 1, EMIT>;
        case 2: return join_kernel<DIM, 2, EMIT>;
        case 4: return join_kernel<DIM, 4, EMIT>;
        case 8: return join_kernel<DIM, 8, EMIT>;
        case 16: return join_kernel<DIM, 16, EMIT>;
        case 32: return join_kernel<DIM, 32, EMIT>;
    }
    return nullptr;
}

template <bool EMIT>
join_fn pick(int dim, int k) {
    switch (dim) {
        case 1: return pick_k<1, EMIT>(k);
        case 2: return pick_k<2, EMIT>(k);
        case 3: return pick_k<3, EMIT>(k);
        case 4: return pick_k<4, EMIT>(k);
        case 5: return pick_k<5, EMIT>(k);
        case 6: return pick_k<6, EMIT>(k);
        case 7: return pick_k<7, EMIT>(k);
        case 8: return pick_k<8, EMIT>(k);
    }
    return nullptr;
}

}  // namespace

int join_occupancy(int dim, int k, bool emit, int *blocks_per_sm) {
    join_fn f = emit ? pick<true>(dim, k) : pick<false>(dim, k);
    if (!f) {
        set_error("join: unsupported dim=%d k=%d", dim, k);
        return SJ_EINVAL;
    }
    SJ_CUDA_TRY(cudaOccupancyMaxActiveBlocksPerMultiprocessor(blocks_per_sm, f, kJoinThreads, 0));
    return SJ_OK;
}

int launch_join(const JoinArgs &a, int dim, int k, bool emit, int blocks, cudaStream_t s) {
    join_fn f = emit ? pick<true>(dim, k) : pick<false>(dim, k);
    if (!f) {
        set_error("join: unsupported dim=%d k=%d", dim, k);
        return SJ_EINVAL;
    }
    f<<<blocks, kJoinThreads, 0, s>>>(a);
    note_launch();
    SJ_CUDA_TRY(cudaGetLastError());
    return SJ_OK;
}

}  // namespace sj
