// join_dim.cu -- one dimensionality of the join kernel family (compiled once per
// SJ_JOIN_DIM = 1..8, so the eight instantiation sets build in parallel); the templates are in
// join_kernel.cuh, the launcher in join_kernel.cu.
#include "join_kernel.cuh"

#ifndef SJ_JOIN_DIM
#error "compile with -DSJ_JOIN_DIM=<1..8>"
#endif

namespace sj {

namespace {
template <int DIM, int K, int MODE, bool GCG>
KernelInfo info() {
    KernelInfo ki;
    ki.f = join_kernel<DIM, K, MODE, GCG>;
    ki.smem = sizeof(WarpSmem<DIM, MODE>) * kWarps;
    return ki;
}

// The LID-UNICOMP / UNICOMP kernels exist for every k; the GCG kernels (ablation, and the
// row-owner CSR modes) for the k the paper evaluates (1 and 8) and 32.
template <int DIM, int MODE, bool GCG>
KernelInfo pick_k(int k) {
#ifdef SJ_QUICK  // register / SASS experiments: one k only
    return k == 8 ? info<DIM, 8, MODE, GCG>() : KernelInfo();
#else
    switch (k) {
        case 1: return info<DIM, 1, MODE, GCG>();
        case 8: return info<DIM, 8, MODE, GCG>();
        case 32: return info<DIM, 32, MODE, GCG>();
    }
    if constexpr (!GCG) {
        switch (k) {
            case 2: return info<DIM, 2, MODE, false>();
            case 4: return info<DIM, 4, MODE, false>();
            case 16: return info<DIM, 16, MODE, false>();
        }
    }
    return KernelInfo();
#endif
}

}  // namespace

template <>
KernelInfo join_pick<SJ_JOIN_DIM>(int mode, bool gcg, int k) {
    constexpr int D = SJ_JOIN_DIM;
    switch (mode) {
        case kCount: return gcg ? pick_k<D, kCount, true>(k) : pick_k<D, kCount, false>(k);
        case kPairs: return gcg ? pick_k<D, kPairs, true>(k) : pick_k<D, kPairs, false>(k);
        case kPairsB: return gcg ? KernelInfo() : pick_k<D, kPairsB, false>(k);
        case kChunkCount: return gcg ? pick_k<D, kChunkCount, true>(k) : pick_k<D, kChunkCount, false>(k);
        case kExact: return gcg ? pick_k<D, kExact, true>(k) : pick_k<D, kExact, false>(k);
        case kRows: return gcg ? pick_k<D, kRows, true>(k) : KernelInfo();
        case kDegree: return gcg ? pick_k<D, kDegree, true>(k) : KernelInfo();
    }
    return KernelInfo();
}

}  // namespace sj
