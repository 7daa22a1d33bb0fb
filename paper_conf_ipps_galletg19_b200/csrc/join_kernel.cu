// join_kernel.cu -- launcher of the join kernel family (DESIGN.md §1 a10): picks the
// instantiation of (dim, k, mode, pattern) -- compiled per dimensionality in join_dim.cu --
// sets its shared-memory attribute once per device, and launches the persistent grid.
#include <map>
#include <mutex>
#include <utility>

#include "join_kernel.cuh"

namespace sj {

namespace {

std::mutex g_prep_mu;
std::map<std::pair<int, const void *>, int> g_prep;  // (device, kernel) -> occupancy, attribute set

KernelInfo pick_any(int dim, int mode, bool gcg, int k) {
    switch (dim) {
        case 1: return join_pick<1>(mode, gcg, k);
        case 2: return join_pick<2>(mode, gcg, k);
        case 3: return join_pick<3>(mode, gcg, k);
        case 4: return join_pick<4>(mode, gcg, k);
        case 5: return join_pick<5>(mode, gcg, k);
        case 6: return join_pick<6>(mode, gcg, k);
        case 7: return join_pick<7>(mode, gcg, k);
        case 8: return join_pick<8>(mode, gcg, k);
    }
    return KernelInfo();
}

int prepare(int dim, int k, int mode, bool gcg, KernelInfo *out) {
    KernelInfo ki = pick_any(dim, mode, gcg, k);
    if (!ki.f) {
        set_error("join: unsupported dim=%d k=%d mode=%d%s", dim, k, mode,
                  gcg ? " for the GCG pattern (k in {1, 8, 32})" : " (CSR modes need the GCG pattern)");
        return SJ_EINVAL;
    }
    // the shared-memory attribute and the occupancy are per (device, kernel): set / queried once
    // (each costs the host microseconds, on the path from sj_create to the join's launch)
    int dev = 0;
    SJ_CUDA_TRY(cudaGetDevice(&dev));
    {
        std::lock_guard<std::mutex> lk(g_prep_mu);
        auto it = g_prep.find(std::make_pair(dev, (const void *)ki.f));
        if (it != g_prep.end()) {
            ki.occ = it->second;
            *out = ki;
            return SJ_OK;
        }
    }
    SJ_CUDA_TRY(cudaFuncSetAttribute(ki.f, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)ki.smem));
    SJ_CUDA_TRY(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&ki.occ, ki.f, kJoinThreads, ki.smem));
    {
        std::lock_guard<std::mutex> lk(g_prep_mu);
        g_prep[std::make_pair(dev, (const void *)ki.f)] = ki.occ;
    }
    *out = ki;
    return SJ_OK;
}

}  // namespace

int join_occupancy(int dim, int k, int mode, bool gcg, int *blocks_per_sm) {
    KernelInfo ki;
    SJ_TRY(prepare(dim, k, mode, gcg, &ki));
    *blocks_per_sm = ki.occ;
    return SJ_OK;
}

int launch_join(const JoinArgs &a0, int dim, int k, int mode, int blocks, cudaStream_t s) {
    KernelInfo ki;
    SJ_TRY(prepare(dim, k, mode, a0.gcg != 0, &ki));
    JoinArgs a = a0;
    const uint64_t st = a.v_stride ? a.v_stride : 1;
    a.v_stride = (uint32_t)st;
    a.v_count = a.v_end > a.v_begin ? (uint32_t)((a.v_end - a.v_begin + st - 1) / st) : 0u;
    ki.f<<<blocks, kJoinThreads, ki.smem, s>>>(a);
    note_launch();
    SJ_CUDA_TRY(cudaGetLastError());
    return SJ_OK;
}

}  // namespace sj
