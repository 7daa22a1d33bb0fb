// diag.cu -- microbenchmarks for the roofline denominators that MEASURED_PEAKS.json
// does not provide: FP64 pipe throughput and same-address global
// atomic throughput (the WorkQueue head and the emission counter are such atomics).
#include "sj_internal.cuh"

namespace sj {
namespace {

constexpr int kChains = 8;
constexpr int kIters = 2048;

// Each thread runs kChains independent x = x*a + b chains with separate DMUL and
// DADD (no FMA) -> 2 * kChains * kIters FP64 lane-instructions per thread.
__global__ void __launch_bounds__(256) fp64_kernel(double *sink, double a, double b) {
    double x[kChains];
#pragma unroll
    for (int c = 0; c < kChains; ++c) x[c] = (double)(threadIdx.x + c) * 1e-3;
    for (int it = 0; it < kIters; ++it) {
#pragma unroll
        for (int c = 0; c < kChains; ++c) x[c] = __dadd_rn(__dmul_rn(x[c], a), b);
    }
    double s = 0;
#pragma unroll
    for (int c = 0; c < kChains; ++c) s += x[c];
    if (s == 12345.678) sink[0] = s;  // never true; keeps the chains live
}

__global__ void __launch_bounds__(256) atomic_kernel(unsigned long long *ctr, int iters, unsigned long long *sink) {
    unsigned long long acc = 0;
    if ((threadIdx.x & 31) == 0) {
        for (int i = 0; i < iters; ++i) acc += atomicAdd(ctr, 32ull);
    }
    if (acc == 1ull) sink[0] = acc;
}

}  // namespace
}  // namespace sj

using namespace sj;

extern "C" int sj_measure_fp64(double *instr_per_s, double *ms_out) {
    int dev = 0, sms = 0;
    SJ_CUDA_TRY(cudaGetDevice(&dev));
    SJ_CUDA_TRY(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev));
    double *sink;
    SJ_CUDA_TRY(cudaMalloc(&sink, 64));
    cudaEvent_t e0, e1;
    SJ_CUDA_TRY(cudaEventCreate(&e0));
    SJ_CUDA_TRY(cudaEventCreate(&e1));
    const int blocks = sms * 8;
    fp64_kernel<<<blocks, 256>>>(sink, 0.999999, 1e-7);  // warm-up
    SJ_CUDA_TRY(cudaEventRecord(e0));
    const int reps = 5;
    for (int r = 0; r < reps; ++r) fp64_kernel<<<blocks, 256>>>(sink, 0.999999, 1e-7);
    SJ_CUDA_TRY(cudaEventRecord(e1));
    SJ_CUDA_TRY(cudaEventSynchronize(e1));
    float ms = 0;
    SJ_CUDA_TRY(cudaEventElapsedTime(&ms, e0, e1));
    const double instr = (double)reps * blocks * 256.0 * kIters * kChains * 2.0;
    if (instr_per_s) *instr_per_s = instr / (ms * 1e-3);
    if (ms_out) *ms_out = ms / reps;
    cudaEventDestroy(e0);
    cudaEventDestroy(e1);
    cudaFree(sink);
    return SJ_OK;
}

extern "C" int sj_measure_atomics(double *ops_per_s, double *ms_out) {
    int dev = 0, sms = 0;
    SJ_CUDA_TRY(cudaGetDevice(&dev));
    SJ_CUDA_TRY(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev));
    unsigned long long *ctr;
    SJ_CUDA_TRY(cudaMalloc(&ctr, 64));
    SJ_CUDA_TRY(cudaMemset(ctr, 0, 64));
    cudaEvent_t e0, e1;
    SJ_CUDA_TRY(cudaEventCreate(&e0));
    SJ_CUDA_TRY(cudaEventCreate(&e1));
    const int blocks = sms * 4, iters = 256;
    atomic_kernel<<<blocks, 256>>>(ctr, iters, ctr + 4);
    SJ_CUDA_TRY(cudaEventRecord(e0));
    atomic_kernel<<<blocks, 256>>>(ctr, iters, ctr + 4);
    SJ_CUDA_TRY(cudaEventRecord(e1));
    SJ_CUDA_TRY(cudaEventSynchronize(e1));
    float ms = 0;
    SJ_CUDA_TRY(cudaEventElapsedTime(&ms, e0, e1));
    const double ops = (double)blocks * 8.0 * iters;
    if (ops_per_s) *ops_per_s = ops / (ms * 1e-3);
    if (ms_out) *ms_out = ms;
    cudaEventDestroy(e0);
    cudaEventDestroy(e1);
    cudaFree(ctr);
    return SJ_OK;
}
