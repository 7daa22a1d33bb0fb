// sj_runtime.cu -- host runtime behind the C ABI of include/sj.h (L1 + L2 of
// DESIGN.md §2): handle state, stream-ordered memory, the batch estimator and the
// batch loop, overflow retry, SJ_MORE continuation, statistics,
// index export/import for the NCCL broadcast, and the host-only helpers.
#include <algorithm>
#include <chrono>
#include <cstdlib>
#include <cmath>
#include <cstdarg>
#include <cstdio>
#include <cstring>
#include <deque>
#include <mutex>
#include <vector>

#include "sj_internal.cuh"

namespace sj {

std::atomic<unsigned long long> g_launches{0};

// ------------------------------------------------------------------------- errors
static thread_local char g_err[1024] = "";

void set_error(const char *fmt, ...) {
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(g_err, sizeof g_err, fmt, ap);
    va_end(ap);
}

void debug_mark(const char *label) {
    static const bool on = [] {
        const char *e = getenv("SJ_DEBUG");
        return e && e[0] == '1';
    }();
    if (!on) return;
    static thread_local std::chrono::steady_clock::time_point last = std::chrono::steady_clock::now();
    auto now = std::chrono::steady_clock::now();
    fprintf(stderr, "[sj] %-28s %9.3f ms\n", label, std::chrono::duration<double, std::milli>(now - last).count());
    last = now;
}

// ------------------------------------------------------------------------- memory
static std::mutex g_pool_mu;
static bool g_pool_ready[64] = {false};

static void pool_setup(int dev) {
    std::lock_guard<std::mutex> lk(g_pool_mu);
    if (dev < 0 || dev >= 64 || g_pool_ready[dev]) return;
    cudaMemPool_t pool;
    if (cudaDeviceGetDefaultMemPool(&pool, dev) == cudaSuccess) {
        uint64_t thr = UINT64_MAX;
        cudaMemPoolSetAttribute(pool, cudaMemPoolAttrReleaseThreshold, &thr);
    }
    g_pool_ready[dev] = true;
}

int dev_alloc(void **p, size_t bytes, cudaStream_t s) {
    *p = nullptr;
    if (bytes == 0) bytes = 16;
    cudaError_t e = cudaMallocAsync(p, bytes, s);
    if (e != cudaSuccess) {
        cudaGetLastError();
        set_error("device allocation of %zu bytes failed: %s", bytes, cudaGetErrorString(e));
        return e == cudaErrorMemoryAllocation ? SJ_ENOMEM : SJ_ECUDA;
    }
    return SJ_OK;
}

void dev_free(void *p, cudaStream_t s) {
    if (p) cudaFreeAsync(p, s);
}

static std::mutex g_pin_mu;
static std::vector<void *> g_pin_free;

void *pinned_acquire() {
    {
        std::lock_guard<std::mutex> lk(g_pin_mu);
        if (!g_pin_free.empty()) {
            void *p = g_pin_free.back();
            g_pin_free.pop_back();
            return p;
        }
    }
    void *p = nullptr;
    if (cudaMallocHost(&p, kMailBytes) != cudaSuccess) {
        cudaGetLastError();
        set_error("pinned host allocation failed");
        return nullptr;
    }
    return p;
}

void pinned_release(void *p) {
    if (!p) return;
    std::lock_guard<std::mutex> lk(g_pin_mu);
    g_pin_free.push_back(p);
}

// ------------------------------------------------------------------------- zero-copy waits
static std::atomic<unsigned> g_epoch{0};

unsigned next_epoch() {
    unsigned e = g_epoch.fetch_add(1, std::memory_order_relaxed) + 1;
    if (e == 0) e = g_epoch.fetch_add(1, std::memory_order_relaxed) + 1;
    return e;
}

int wait_flag(volatile unsigned *flag, unsigned epoch, cudaStream_t s) {
    for (unsigned long long spin = 0;; ++spin) {
        if (*flag == epoch) {
            std::atomic_thread_fence(std::memory_order_acquire);
            return SJ_OK;
        }
        if ((spin & 255) == 255) {
            const cudaError_t e = cudaStreamQuery(s);
            if (e == cudaSuccess) {  // the stream drained: the flag must be there
                if (*flag == epoch) {
                    std::atomic_thread_fence(std::memory_order_acquire);
                    return SJ_OK;
                }
                set_error("zero-copy wait: the stream completed without the result flag");
                return SJ_ECUDA;
            }
            if (e != cudaErrorNotReady) {
                set_error("zero-copy wait: %s", cudaGetErrorString(e));
                return SJ_ECUDA;
            }
        }
    }
}

// ------------------------------------------------------------------------- caller stream
// The stream the caller produced its inputs on (sj_set_stream; thread-local).  Every entry point
// that reads or writes caller memory first makes the handle's stream wait for it, so device
// inputs written asynchronously by the caller (e.g. torch kernels on its current stream) are
// complete before the library reads them, and caller buffers are not written under pending work.
static thread_local cudaStream_t g_caller_stream = cudaStreamLegacy;
cudaStream_t caller_stream() { return g_caller_stream; }

// ------------------------------------------------------------------------- small kernels
__global__ void set_u64_kernel(unsigned long long *p, unsigned long long v) { *p = v; }

}  // namespace sj

using namespace sj;

// ------------------------------------------------------------------------- handle
namespace {

constexpr int kMaxStreams = 8;
// Device counters of a join: [0] pairs emitted (one atomic per output flush), [kHead] the
// WorkQueue head (one atomic per dequeue), [2] distance calculations, [4] the fused estimator's
// sample pairs, [kHead + 2] a separate estimator's queue head.  The two hot atomics live in
// different 128-byte lines: in one line they serialise on one L2 slice, and the join then falls
// into a congested mode (C5: 0.95 -> 1.8 ms, C5 eps 0.2: 3.1 -> 6.1 ms, measured).
constexpr int kHead = 16;
constexpr int kTotal = 8;  // a blocked in-place join's pair total (compact_output)
constexpr int kCtrWords = 24;
// Blocked in-place output (JoinArgs::blk): pairs per warp block.  One atomic per block and warp
// instead of one per warp flush (~900 pairs); the warps' last blocks leave gaps that
// compact_output closes (on average half a block per warp to move, from a scratch of one block
// per warp past the buffer).  SJ_OUT_BLK (environment, even) overrides it for measurements.
// (Blocks shared by the warps of a CTA -- a packed {block, offset} word in shared memory, one
// shared atomic per flush -- were measured slower: C5 join 0.93 -> 1.06 ms.)
constexpr unsigned long long kOutBlkDefault = 4096;
static unsigned long long out_blk() {
    static const unsigned long long v = [] {
        const char *e = getenv("SJ_OUT_BLK");
        const unsigned long long x = e ? strtoull(e, nullptr, 10) : 0ull;
        return (x >= 1024 && x <= (1ull << 22) && x % 2 == 0) ? x : kOutBlkDefault;
    }();
    return v;
}
// pinned mailbox layout (uint64 words): [0, kCtrWords) counters; [48, 50) the build's tail;
// [64 + 4 s, 64 + 4 s + 3) staged slot s's counters
constexpr int kMailSlots = 64;

struct Job {
    uint64_t v0, v1;  // virtual chunks v0, v0 + stride, ... < v1 of this handle's slice
    uint64_t stride = 1;             // 1: contiguous (WorkQueue); nbBatches: strided D'_l
    uint64_t base = 0;               // exact sizing: pair offset of chunk v0 in the whole join
    uint64_t expect = UINT64_MAX;    // exact sizing: the batch's pairs (UINT64_MAX: estimated)
    int slot = -1;
    bool launched = false, complete = false;
    uint64_t cnt = 0, consumed = 0;
};

struct Slot {
    cudaStream_t stream = nullptr;
    uint32_t *buf = nullptr;
    uint64_t cap = 0;                      // pairs
    unsigned long long *d_ctr = nullptr;   // [0]=emit, [1]=head, [2]=calcs
    cudaEvent_t ev_start = nullptr, ev_stop = nullptr, ev_done = nullptr;
    bool busy = false;
};

}  // namespace

struct sj_handle {
    int device = 0;
    int state = 0;  // 0 ready, 1 continuing (staged path), -1 error
    cudaStream_t s_main = nullptr;
    cudaEvent_t ev_a = nullptr, ev_b = nullptr, ev_c = nullptr, ev_d = nullptr, ev_e = nullptr;
    cudaEvent_t ev_ba = nullptr, ev_bb = nullptr;  // build start / end
    cudaEvent_t ev_in = nullptr;  // the caller's stream, recorded at entry (order_after_caller)
    sj::BuildSide side{};                         // the build's side stream and its events
    int pending = 0;  // 1: the build's tail {n_chunks, E} and its timing not read yet (ix_ready)
    bool ctr_zeroed = false;  // the build's last kernel zeroed d_ctr (no join has used it since)
    sj::Index ix;
    bool owns_index = true;
    int num_sms = 148;

    // options
    int k = 8;
    uint64_t batch_pairs = 100000000ull;
    int streams = 3;
    uint32_t sample_ppm = 10000;
    uint32_t grab = 4;  // WorkQueue chunks per dequeue (fewer same-address atomics, measured)
    int count_calcs = 0;
    int blocks_per_sm = 0;
    int fast_path = 1;
    int exact = 0;
    int queue = 1;  // 1: WorkQueue; 0: SortByWL only (static assignment, strided batches)
    int rank = 0, world = 1;

    uint64_t *d_voff = nullptr;  // exact sizing: per-chunk pairs -> offsets, [V+1]
    uint64_t voff_cap = 0;
    char *outws = nullptr;       // blocked in-place output: gaps, compaction workspace, scratch
    size_t outws_bytes = 0;
    int out_blocks = 2;          // SJ_OPT_OUT_BLOCKS

    unsigned long long *d_ctr = nullptr;  // [0]=emit [1]=head [2]=calcs [3..] spare
    uint64_t *mail = nullptr;             // pinned host mailbox [64]
    Slot slots[kMaxStreams];
    std::deque<Job> jobs;

    sj_stats st{};
};

namespace {

int fail(sj_handle *h, int rc) {
    if (h && rc < 0) h->state = -1;
    return rc;
}

int ensure_device(const sj_handle *h) {
    SJ_CUDA_TRY(cudaSetDevice(h->device));
    return SJ_OK;
}

bool is_device_ptr(const void *p, int dev) {
    cudaPointerAttributes at;
    if (cudaPointerGetAttributes(&at, p) != cudaSuccess) {
        cudaGetLastError();
        return false;
    }
    if (at.type == cudaMemoryTypeDevice) return at.device == dev;
    if (at.type == cudaMemoryTypeManaged) return true;
    return false;
}

// Per-handle CUDA objects (main stream, 5 timing events, device counters, pinned mailbox)
// are recycled process-wide per device: creating and destroying them costs ~0.1 ms per
// handle, a visible fraction of a millisecond-scale join.
struct Core {
    int device;
    int num_sms;
    cudaStream_t s;
    cudaEvent_t ev[8];
    sj::BuildSide side;
    unsigned long long *d_ctr;
    uint64_t *mail;
    char *outws;  // the blocked output's workspace (gaps, compaction, scratch), kept with the core
    size_t outws_bytes;
};
std::mutex g_core_mu;
std::vector<Core> g_core_cache;

int handle_init_common(sj_handle *h) {
    SJ_CUDA_TRY(cudaGetDevice(&h->device));
    {
        std::lock_guard<std::mutex> lk(g_core_mu);
        for (size_t k = 0; k < g_core_cache.size(); ++k)
            if (g_core_cache[k].device == h->device) {
                const Core c = g_core_cache[k];
                g_core_cache.erase(g_core_cache.begin() + (long)k);
                h->num_sms = c.num_sms;
                h->s_main = c.s;
                h->ev_a = c.ev[0];
                h->ev_b = c.ev[1];
                h->ev_c = c.ev[2];
                h->ev_d = c.ev[3];
                h->ev_e = c.ev[4];
                h->ev_ba = c.ev[5];
                h->ev_bb = c.ev[6];
                h->ev_in = c.ev[7];
                h->side = c.side;
                h->d_ctr = c.d_ctr;
                h->mail = c.mail;
                h->outws = c.outws;
                h->outws_bytes = c.outws_bytes;
                return SJ_OK;
            }
    }
    pool_setup(h->device);
    SJ_CUDA_TRY(cudaDeviceGetAttribute(&h->num_sms, cudaDevAttrMultiProcessorCount, h->device));
    // priorities: the build's side stream (the gather of the points, D') yields the SMs to the
    // main stream's critical path, block by block
    int prio_least = 0, prio_greatest = 0;
    SJ_CUDA_TRY(cudaDeviceGetStreamPriorityRange(&prio_least, &prio_greatest));
    SJ_CUDA_TRY(cudaStreamCreateWithPriority(&h->s_main, cudaStreamNonBlocking, prio_greatest));
    SJ_CUDA_TRY(cudaEventCreate(&h->ev_a));
    SJ_CUDA_TRY(cudaEventCreate(&h->ev_b));
    SJ_CUDA_TRY(cudaEventCreate(&h->ev_c));
    SJ_CUDA_TRY(cudaEventCreate(&h->ev_d));
    SJ_CUDA_TRY(cudaEventCreate(&h->ev_e));
    SJ_CUDA_TRY(cudaEventCreate(&h->ev_ba));
    SJ_CUDA_TRY(cudaEventCreate(&h->ev_bb));
    SJ_CUDA_TRY(cudaEventCreateWithFlags(&h->ev_in, cudaEventDisableTiming));
    SJ_CUDA_TRY(cudaStreamCreateWithPriority(&h->side.s2, cudaStreamNonBlocking, prio_least));
    SJ_CUDA_TRY(cudaEventCreateWithFlags(&h->side.ea, cudaEventDisableTiming));
    SJ_CUDA_TRY(cudaEventCreateWithFlags(&h->side.eg, cudaEventDisableTiming));
    SJ_CUDA_TRY(cudaEventCreateWithFlags(&h->side.eq, cudaEventDisableTiming));
    SJ_CUDA_TRY(cudaEventCreateWithFlags(&h->side.ej, cudaEventDisableTiming));
    h->mail = static_cast<uint64_t *>(pinned_acquire());
    if (!h->mail) return SJ_ENOMEM;
    SJ_TRY(dev_alloc_t(&h->d_ctr, kCtrWords, h->s_main));
    return SJ_OK;
}

// Returns the handle's core to the cache (stream drained first); false if it must be freed.
bool core_release(sj_handle *h) {
    if (!h->s_main || !h->ev_a || !h->ev_b || !h->ev_c || !h->ev_d || !h->ev_e || !h->ev_ba || !h->ev_bb || !h->ev_in || !h->d_ctr ||
        !h->mail || !h->side.s2 || !h->side.ea || !h->side.eg || !h->side.eq || !h->side.ej)
        return false;
    if (cudaStreamSynchronize(h->side.s2) != cudaSuccess) {
        cudaGetLastError();
        return false;
    }
    if (cudaStreamSynchronize(h->s_main) != cudaSuccess) {
        cudaGetLastError();
        return false;
    }
    std::lock_guard<std::mutex> lk(g_core_mu);
    if (g_core_cache.size() >= 64) return false;
    g_core_cache.push_back(Core{h->device, h->num_sms, h->s_main, {h->ev_a, h->ev_b, h->ev_c, h->ev_d, h->ev_e, h->ev_ba, h->ev_bb, h->ev_in}, h->side, h->d_ctr,
                                h->mail, h->outws, h->outws_bytes});
    h->outws = nullptr;
    h->outws_bytes = 0;
    return true;
}

// Staged-path slots (stream + events + b_s result buffer) are recycled process-wide per
// device: creating/destroying streams and multi-GB buffers per join costs tens of ms.
std::mutex g_slot_mu;
std::vector<std::pair<int, Slot>> g_slot_cache;  // (device, idle slot)

int slot_init(sj_handle *h, int i) {
    Slot &s = h->slots[i];
    if (s.stream) return SJ_OK;
    {
        std::lock_guard<std::mutex> lk(g_slot_mu);
        for (size_t k = 0; k < g_slot_cache.size(); ++k)
            if (g_slot_cache[k].first == h->device) {
                s = g_slot_cache[k].second;
                g_slot_cache.erase(g_slot_cache.begin() + (long)k);
                s.busy = false;
                return SJ_OK;
            }
    }
    SJ_CUDA_TRY(cudaStreamCreateWithFlags(&s.stream, cudaStreamNonBlocking));
    SJ_CUDA_TRY(cudaEventCreate(&s.ev_start));
    SJ_CUDA_TRY(cudaEventCreate(&s.ev_stop));
    SJ_CUDA_TRY(cudaEventCreateWithFlags(&s.ev_done, cudaEventDisableTiming));
    SJ_TRY(dev_alloc_t(&s.d_ctr, kCtrWords, s.stream));
    return SJ_OK;
}

int slot_buffer(sj_handle *h, Slot &s, uint64_t pairs) {
    if (s.cap >= pairs && s.buf) return SJ_OK;
    dev_free(s.buf, s.stream);
    s.buf = nullptr;
    s.cap = 0;
    SJ_TRY(dev_alloc(reinterpret_cast<void **>(&s.buf), pairs * 2 * sizeof(uint32_t), s.stream));
    s.cap = pairs;
    return SJ_OK;
}

void slots_release(sj_handle *h) {
    for (int i = 0; i < kMaxStreams; ++i) {
        Slot &s = h->slots[i];
        if (!s.stream) continue;
        cudaStreamSynchronize(s.stream);
        {
            std::lock_guard<std::mutex> lk(g_slot_mu);
            if (g_slot_cache.size() < 2 * kMaxStreams) {
                g_slot_cache.emplace_back(h->device, s);
                s = Slot();
                continue;
            }
        }
        dev_free(s.buf, s.stream);
        dev_free(s.d_ctr, s.stream);
        cudaStreamSynchronize(s.stream);
        cudaStreamDestroy(s.stream);
        cudaEventDestroy(s.ev_start);
        cudaEventDestroy(s.ev_stop);
        cudaEventDestroy(s.ev_done);
        s = Slot();
    }
}

// number of WorkQueue chunks of this handle's slice (chunk c belongs to rank c mod world)
// Batch l of nb over the nch virtual chunks of a slice: WorkQueue batches are
// contiguous ranges of D' (reading c14); SortByWL-only batches are the strided D'_l =
// {v : v mod nb = l} of Fig. 1.  Returned as {v0, v1, stride}: chunks v0, v0 + stride, ... < v1.
Job batch_job(uint64_t nch, uint64_t nb, uint64_t l, bool queue) {
    Job j;
    if (queue) {
        j.v0 = nch * l / nb;
        j.v1 = nch * (l + 1) / nb;
    } else {
        j.v0 = l;
        j.v1 = nch;
        j.stride = nb;
    }
    return j;
}

uint64_t slice_chunks(const sj_handle *h) {
    const uint64_t nchunks = h->ix.n_chunks;
    if (nchunks <= (uint64_t)h->rank) return 0;
    return (nchunks - (uint64_t)h->rank + (uint64_t)h->world - 1) / (uint64_t)h->world;
}

JoinArgs base_args(const sj_handle *h) {
    JoinArgs a{};
    a.pts = h->ix.pts;
    a.orig = h->ix.orig;
    a.qmap = h->ix.qmap;
    a.cellq = h->ix.cellq;
    a.runs = h->ix.runs;
    a.chunks = h->ix.chunks;
    a.n_chunks = (uint32_t)h->ix.n_chunks;
    a.n_runs = h->ix.runs_cap ? h->ix.runs_cap : h->ix.n_runs;  // bound of the run reads: the allocation
    a.e2 = h->ix.e2;
    a.grab = h->grab;
    a.v_stride = 1;
    a.static_q = h->queue ? 0u : 1u;
    a.gcg = h->ix.pattern == SJ_PATTERN_GCG ? 1 : 0;
    a.rank = (uint32_t)h->rank;
    a.world = (uint32_t)h->world;
    return a;
}

void fill_static_stats(sj_handle *h) {
    sj_stats &st = h->st;
    st.n = h->ix.n;
    st.dim = (uint32_t)h->ix.dim;
    st.key_bits = (uint32_t)h->ix.key_bits;
    st.n_cells = h->ix.n_cells;
    st.fwd_runs = h->ix.n_runs;
    st.dist_calcs = h->ix.dist_calcs;
    st.max_cell_load = h->ix.max_w;
    st.k = (uint32_t)h->k;
    for (int d = 0; d < SJ_MAX_DIM; ++d) st.nc[d] = d < h->ix.dim ? (uint32_t)h->ix.nc[d] : 0;
    st.n_chunks = h->ix.n_chunks;
    st.tiled_min = kBigCell;
    st.pattern = (uint32_t)h->ix.pattern;
    st.order = (uint32_t)h->ix.order;
    st.lookup_hash = (uint32_t)h->ix.lookup_hash;
}

// The build's tail (sj_create returns without a final round trip): {n_chunks, E} from the
// handle's mailbox once the stream passed the build's end event, the build time, the static
// statistics.  Every host path that needs them calls this first; the in-place fast path does
// so only after its join (the kernel reads n_chunks on the device).
int ix_ready(sj_handle *h) {
    if (!h->pending) return SJ_OK;
    SJ_CUDA_TRY(cudaEventSynchronize(h->ev_bb));
    h->ix.n_chunks = h->mail[48];
    h->ix.n_runs = h->mail[49];
    float ms = 0;
    SJ_CUDA_TRY(cudaEventElapsedTime(&ms, h->ev_ba, h->ev_bb));
    h->pending = 0;
    fill_static_stats(h);
    h->st.ms_build = ms;
    return SJ_OK;
}

// The handle's main stream waits for the work queued so far on the caller's stream.
int order_after_caller(sj_handle *h) {
    SJ_CUDA_TRY(cudaEventRecord(h->ev_in, g_caller_stream));
    SJ_CUDA_TRY(cudaStreamWaitEvent(h->s_main, h->ev_in, 0));
    return SJ_OK;
}

int join_blocks(const sj_handle *h, int mode, int *blocks) {
    int occ = 0;
    SJ_TRY(join_occupancy(h->ix.dim, h->k, mode, h->ix.pattern == SJ_PATTERN_GCG, &occ));
    if (h->blocks_per_sm > 0 && h->blocks_per_sm < occ) occ = h->blocks_per_sm;
    if (occ < 1) occ = 1;
    *blocks = occ * h->num_sms;
    return SJ_OK;
}

// Count-only join over virtual range [v0, v1) on the main stream.  Synchronous.  With
// vcount, every chunk's pairs are recorded and scanned in place into chunk offsets
// (exact sizing, pass 1): vcount[V] receives the total.
int count_range(sj_handle *h, uint64_t v0, uint64_t v1, uint64_t *pairs, float *ms, uint64_t *vcount = nullptr,
                uint64_t stride = 1) {
    cudaStream_t s = h->s_main;
    SJ_CUDA_TRY(cudaMemsetAsync(h->d_ctr, 0, kCtrWords * sizeof(unsigned long long), s));
    JoinArgs a = base_args(h);
    a.head = h->d_ctr + kHead;  // zeroed above
    a.v_begin = v0;
    a.v_end = v1;
    a.v_stride = (uint32_t)stride;
    a.out = nullptr;
    a.emit_ctr = h->d_ctr;
    a.out_cap = 0;
    a.calcs = h->count_calcs ? h->d_ctr + 2 : nullptr;
    a.vcount = reinterpret_cast<unsigned long long *>(vcount);
    const int mode = vcount ? kChunkCount : kCount;
    int blocks;
    SJ_TRY(join_blocks(h, mode, &blocks));
    SJ_CUDA_TRY(cudaEventRecord(h->ev_c, s));
    if (v1 > v0) SJ_TRY(launch_join(a, h->ix.dim, h->k, mode, blocks, s));
    if (vcount) SJ_TRY(scan_exclusive_u64(vcount + v0, vcount + v0, v1 - v0, vcount + v1, s));
    SJ_CUDA_TRY(cudaEventRecord(h->ev_d, s));
    SJ_CUDA_TRY(cudaMemcpyAsync(h->mail, h->d_ctr, kCtrWords * sizeof(uint64_t), cudaMemcpyDeviceToHost, s));
    SJ_CUDA_TRY(cudaStreamSynchronize(s));
    *pairs = h->mail[0];
    if (h->count_calcs) h->st.calcs_measured = h->mail[2];
    if (ms) SJ_CUDA_TRY(cudaEventElapsedTime(ms, h->ev_c, h->ev_d));
    return SJ_OK;
}

// ------------------------------------------------------------------ staged batches
int launch_job(sj_handle *h, Job &j, int slot_idx) {
    Slot &s = h->slots[slot_idx];
    SJ_TRY(slot_buffer(h, s, j.expect != UINT64_MAX ? std::max<uint64_t>(h->batch_pairs, j.expect) : h->batch_pairs));
    SJ_CUDA_TRY(cudaMemsetAsync(s.d_ctr, 0, kCtrWords * sizeof(unsigned long long), s.stream));
    JoinArgs a = base_args(h);
    a.head = s.d_ctr + kHead;  // zeroed above
    a.v_begin = j.v0;
    a.v_end = j.v1;
    a.v_stride = (uint32_t)j.stride;
    a.out = s.buf;
    a.emit_ctr = s.d_ctr;
    a.out_cap = s.cap;
    a.calcs = h->count_calcs ? s.d_ctr + 2 : nullptr;
    const bool exact = j.expect != UINT64_MAX;
    if (exact) {  // exact sizing: every chunk writes at its own offset
        a.voff = reinterpret_cast<const unsigned long long *>(h->d_voff);
        a.out_base = j.base;
    }
    int blocks;
    SJ_TRY(join_blocks(h, exact ? kExact : kPairs, &blocks));
    SJ_CUDA_TRY(cudaEventRecord(s.ev_start, s.stream));
    SJ_TRY(launch_join(a, h->ix.dim, h->k, exact ? kExact : kPairs, blocks, s.stream));
    SJ_CUDA_TRY(cudaEventRecord(s.ev_stop, s.stream));
    SJ_CUDA_TRY(cudaMemcpyAsync(h->mail + kMailSlots + 4 * slot_idx, s.d_ctr, 3 * sizeof(uint64_t), cudaMemcpyDeviceToHost,
                                s.stream));
    SJ_CUDA_TRY(cudaEventRecord(s.ev_done, s.stream));
    j.slot = slot_idx;
    j.launched = true;
    s.busy = true;
    h->st.join_launches++;
    return SJ_OK;
}

int fill_pipeline(sj_handle *h) {
    for (Job &j : h->jobs) {
        if (j.launched) continue;
        int free_slot = -1;
        for (int i = 0; i < h->streams; ++i)
            if (!h->slots[i].busy) {
                free_slot = i;
                break;
            }
        if (free_slot < 0) break;
        SJ_TRY(launch_job(h, j, free_slot));
    }
    return SJ_OK;
}

// Drives the staged batch pipeline until the caller's buffer is full or the join ends.
int continue_staged(sj_handle *h, uint32_t *out, uint64_t cap, uint64_t *count) {
    uint64_t written = 0;
    // the copies into the caller's buffer run on the slot streams: order them after the caller
    // (sj_self_join made s_main wait for the caller's stream)
    SJ_CUDA_TRY(cudaEventRecord(h->ev_in, h->s_main));
    for (int i = 0; i < h->streams; ++i)
        if (h->slots[i].stream) SJ_CUDA_TRY(cudaStreamWaitEvent(h->slots[i].stream, h->ev_in, 0));
    for (;;) {
        SJ_TRY(fill_pipeline(h));
        if (h->jobs.empty()) break;
        Job &j = h->jobs.front();
        Slot &s = h->slots[j.slot];
        if (!j.complete) {
            SJ_CUDA_TRY(cudaEventSynchronize(s.ev_done));
            const uint64_t *m = h->mail + kMailSlots + 4 * j.slot;
            j.cnt = m[0];
            if (h->count_calcs) h->st.calcs_measured += m[2];
            float ms = 0;
            SJ_CUDA_TRY(cudaEventElapsedTime(&ms, s.ev_start, s.ev_stop));
            h->st.ms_join_sum += ms;
            if (getenv("SJ_DEBUG_BATCH"))
                fprintf(stderr, "[sj] batch chunks [%llu, %llu) pairs %llu  %.3f ms  %.1f GB/s\n",
                        (unsigned long long)j.v0, (unsigned long long)j.v1, (unsigned long long)j.cnt, ms,
                        j.cnt * 8.0 / (ms * 1e6));
            if (j.expect != UINT64_MAX && j.cnt != j.expect) {
                set_error("sj_self_join: exact sizing mismatch in chunks [%llu, %llu): counted %llu, emitted %llu",
                          (unsigned long long)j.v0, (unsigned long long)j.v1, (unsigned long long)j.expect,
                          (unsigned long long)j.cnt);
                return SJ_ECUDA;
            }
            if (j.cnt > s.cap) {
                // overflow (estimate too low): split the range, or grow the buffer if it is one chunk
                h->st.retries++;
                if (h->count_calcs) h->st.calcs_measured -= m[2];
                const Job old = j;
                const uint64_t chunks = (old.v1 - old.v0 + old.stride - 1) / old.stride;
                h->jobs.pop_front();
                s.busy = false;
                if (chunks <= 1) {
                    SJ_TRY(slot_buffer(h, s, old.cnt));
                    Job again;
                    again.v0 = old.v0;
                    again.v1 = old.v1;
                    again.stride = old.stride;
                    h->jobs.push_front(again);
                    SJ_TRY(launch_job(h, h->jobs.front(), old.slot));
                } else {
                    const uint64_t parts = std::min<uint64_t>(chunks, old.cnt / s.cap + 2);
                    for (uint64_t p = parts; p-- > 0;) {
                        Job nj;
                        if (old.stride == 1) {  // WorkQueue batches stay contiguous ranges of D' (c14)
                            nj.v0 = old.v0 + chunks * p / parts;
                            nj.v1 = old.v0 + chunks * (p + 1) / parts;
                        } else {  // strided batches split into interleaved sub-batches
                            nj.v0 = old.v0 + p * old.stride;
                            nj.v1 = old.v1;
                            nj.stride = old.stride * parts;
                        }
                        if (nj.v1 > nj.v0) h->jobs.push_front(nj);
                    }
                    h->st.batches += (uint32_t)(parts - 1);
                }
                continue;
            }
            j.complete = true;
        }
        const uint64_t take = std::min<uint64_t>(j.cnt - j.consumed, cap - written);
        if (take) {
            SJ_CUDA_TRY(cudaMemcpyAsync(out + 2 * written, s.buf + 2 * j.consumed, take * 2 * sizeof(uint32_t),
                                        cudaMemcpyDefault, s.stream));
            written += take;
            j.consumed += take;
            h->st.pairs += take;
        }
        if (j.consumed == j.cnt) {
            s.busy = false;  // the next job on this slot is ordered after the copy (same stream)
            h->jobs.pop_front();
            continue;
        }
        if (written == cap) break;  // leftover pairs in j -> SJ_MORE
    }
    for (int i = 0; i < h->streams; ++i)
        if (h->slots[i].stream) SJ_CUDA_TRY(cudaStreamSynchronize(h->slots[i].stream));
    *count = written;
    if (h->jobs.empty()) {
        h->state = 0;
        SJ_CUDA_TRY(cudaEventRecord(h->ev_b, h->s_main));
        SJ_CUDA_TRY(cudaEventSynchronize(h->ev_b));
        float tot = 0;
        SJ_CUDA_TRY(cudaEventElapsedTime(&tot, h->ev_a, h->ev_b));
        h->st.ms_total = tot;
        h->st.ms_join = h->st.ms_join_sum;
        return SJ_OK;
    }
    h->state = 1;
    return SJ_MORE;
}

// One persistent launch over the slice's chunks [v0, v1) writing the caller's device buffer in
// place (no staging, no D2D copy).  *emitted = the pairs the kernel produced (> cap: overflow,
// only the first cap were written).  exact: chunk offsets from h->d_voff.
int run_in_place(sj_handle *h, uint32_t *out, uint64_t cap, uint64_t v0, uint64_t v1, bool exact,
                 uint64_t *emitted) {
    cudaStream_t s = h->s_main;
    SJ_CUDA_TRY(cudaMemsetAsync(h->d_ctr, 0, kCtrWords * sizeof(unsigned long long), s));
    JoinArgs a = base_args(h);
    a.head = h->d_ctr + kHead;  // zeroed above
    a.v_begin = v0;
    a.v_end = v1;
    a.out = out;
    a.emit_ctr = h->d_ctr;
    a.out_cap = cap;
    a.calcs = h->count_calcs ? h->d_ctr + 2 : nullptr;
    if (exact) {
        a.voff = reinterpret_cast<const unsigned long long *>(h->d_voff);
        a.out_base = 0;
    }
    const int mode = exact ? kExact : kPairs;
    int blocks;
    SJ_TRY(join_blocks(h, mode, &blocks));
    SJ_CUDA_TRY(cudaEventRecord(h->ev_c, s));
    if (v1 > v0) SJ_TRY(launch_join(a, h->ix.dim, h->k, mode, blocks, s));
    SJ_CUDA_TRY(cudaEventRecord(h->ev_d, s));
    SJ_CUDA_TRY(cudaMemcpyAsync(h->mail, h->d_ctr, kCtrWords * sizeof(uint64_t), cudaMemcpyDeviceToHost, s));
    SJ_CUDA_TRY(cudaStreamSynchronize(s));
    float ms = 0;
    SJ_CUDA_TRY(cudaEventElapsedTime(&ms, h->ev_c, h->ev_d));
    h->st.join_launches = 1;
    h->st.batches = 1;
    h->st.ms_join = h->st.ms_join_sum = ms;
    *emitted = h->mail[0];
    return SJ_OK;
}

// Fast path (caller's HBM buffer, in place): the estimator (a9) and the join of the
// whole queue [0, V) into the caller's buffer.  In place there are no batches to size, so the
// join never waits for the estimate; it is reported, and sizes the staged fallback if the
// buffer overflows.  WorkQueue: the estimator is FUSED into the join -- the sample is the first
// sch chunks of D', which are exactly the first chunks the queue hands out, so the join
// adds the pairs of chunks [0, sv1) to a counter of their own: the same number a separate
// count-only launch over [0, sv1) returns, without evaluating the heaviest 1 % twice (a
// separate launch of it cannot fill the GPU: 84 us on C5).  Every dequeued chunk is finished,
// so the sample is complete whenever the queue head passed sv1 -- always, unless the output
// overflowed early; then the separate estimator runs.  SortByWL only (strided sample, static
// assignment): the separate count-only launch first, back to back on the main stream.
// (Running it concurrently on a side stream was measured: it wins ~0.04 ms on C5 but loses
// 3 ms on C5 eps=0.2, where estimator and join fight over the same heaviest head of D'.)
// *spairs = the sample's pairs, *total = all pairs emitted (> cap: overflow, only the first
// cap were written).
// Blocked output for an in-place kPairs launch of `blocks` CTAs (JoinArgs::blk, mode kPairsB):
// the gaps array, the compaction workspace and the scratch, from one per-handle allocation.  Half
// patterns only (GCG emits single pairs).  SJ_OPT_OUT_BLOCKS: 1 on, 0 off, 2 (default) on when
// the caller's buffer holds at least kBlockedMinCap pairs (a large result: the output counter's
// congestion doubles the join, measured on C5 eps 0.2 every time and on C5 on some boxes -- 0.88
// vs 1.3-1.4 ms, with blocks 0.93 on every box; below it the compaction's fixed cost (a prep
// launch, ~15 us, and a copy of half a block per warp) outweighs the risk: C2 K64 0.28 vs 0.34).
constexpr uint64_t kBlockedMinCap = 300000000ull;
int blocked_out(sj_handle *h, JoinArgs &a, int blocks, uint64_t cap, bool *on) {
    *on = h->out_blocks == 1 || (h->out_blocks == 2 && cap >= kBlockedMinCap);
    *on = *on && h->ix.pattern != SJ_PATTERN_GCG && blocks * (kJoinThreads / 32) <= kCompactMaxGaps;
    if (!*on) return SJ_OK;
    const size_t gbytes = ((size_t)blocks * kJoinThreads / 32 * 16 + 255) & ~(size_t)255;  // a gap per warp
    const size_t wbytes = (compact_ws_bytes(blocks) + 255) & ~(size_t)255;
    const size_t sbytes = (size_t)blocks * kJoinThreads / 32 * out_blk() * 8;
    const size_t need = gbytes + wbytes + sbytes;
    if (h->outws_bytes < need) {
        dev_free(h->outws, h->s_main);
        h->outws = nullptr;
        h->outws_bytes = 0;
        SJ_TRY(dev_alloc(reinterpret_cast<void **>(&h->outws), need, h->s_main));
        h->outws_bytes = need;
    }
    a.blk = out_blk();
    a.gaps = reinterpret_cast<unsigned long long *>(h->outws);
    a.scratch = reinterpret_cast<uint32_t *>(h->outws + gbytes + wbytes);
    a.scratch_cap = (unsigned long long)blocks * kJoinThreads / 32 * out_blk();
    return SJ_OK;
}

void *blocked_ws(sj_handle *h, int blocks) {
    return h->outws + (((size_t)blocks * kJoinThreads / 32 * 16 + 255) & ~(size_t)255);
}

int run_in_place_est(sj_handle *h, uint32_t *out, uint64_t cap, uint64_t sch, uint64_t sv1, uint64_t sstride,
                     uint64_t V, uint64_t *spairs, uint64_t *total) {
    cudaStream_t s = h->s_main;
    const bool fused = sstride == 1 && h->queue && sch && !getenv("SJ_SEPARATE_EST");
    SJ_CUDA_TRY(cudaMemsetAsync(h->d_ctr, 0, kCtrWords * sizeof(unsigned long long), s));
    SJ_CUDA_TRY(cudaEventRecord(h->ev_c, s));
    if (!fused) {
        JoinArgs e = base_args(h);
        e.head = h->d_ctr + kHead + 2;
        e.emit_ctr = h->d_ctr + 4;
        e.v_begin = 0;
        e.v_end = sv1;  // the sample: chunks 0, sstride, ... < sv1 (sch of them)
        e.v_stride = (uint32_t)sstride;
        int blocks_e;
        SJ_TRY(join_blocks(h, kCount, &blocks_e));
        if (sch) SJ_TRY(launch_join(e, h->ix.dim, h->k, kCount, blocks_e, s));
    }
    SJ_CUDA_TRY(cudaEventRecord(h->ev_e, s));
    JoinArgs a = base_args(h);
    a.out = out;
    a.emit_ctr = h->d_ctr;
    a.out_cap = cap;
    a.calcs = h->count_calcs ? h->d_ctr + 2 : nullptr;
    a.head = h->d_ctr + kHead;
    a.v_begin = 0;
    a.v_end = V;
    if (fused) {
        a.sample_ctr = h->d_ctr + 4;
        a.sample_v1 = sv1;
    }
    int blocks;
    SJ_TRY(join_blocks(h, kPairs, &blocks));
    bool blocked = false;
    SJ_TRY(blocked_out(h, a, blocks, cap, &blocked));
    if (V) SJ_TRY(launch_join(a, h->ix.dim, h->k, blocked ? kPairsB : kPairs, blocks, s));
    if (V && blocked) SJ_TRY(compact_output(a, blocks, h->d_ctr + kTotal, blocked_ws(h, blocks), s));
    SJ_CUDA_TRY(cudaEventRecord(h->ev_d, s));
    SJ_CUDA_TRY(cudaMemcpyAsync(h->mail, h->d_ctr, kCtrWords * sizeof(uint64_t), cudaMemcpyDeviceToHost, s));
    SJ_CUDA_TRY(cudaStreamSynchronize(s));
    if (blocked) h->mail[0] = h->mail[kTotal];  // pairs emitted (the counter itself counts blocks)
    float ms_est = 0, ms = 0;
    SJ_CUDA_TRY(cudaEventElapsedTime(&ms_est, h->ev_c, h->ev_e));
    SJ_CUDA_TRY(cudaEventElapsedTime(&ms, h->ev_e, h->ev_d));
    h->st.join_launches = V ? 1u : 0u;
    h->st.batches = 1;
    h->st.ms_estimate = fused ? 0.0 : ms_est;  // fused: inside the join launch
    h->st.ms_join = h->st.ms_join_sum = ms;   // the join launch
    h->st.est_fused = fused ? 1u : 0u;
    *spairs = h->mail[4];
    *total = h->mail[0];
    if (fused && h->mail[kHead] < sv1) {  // overflowed before the sample was handed out: count it apart
        const uint64_t emitted = *total;
        const uint64_t calcs = h->mail[2];
        float ms_c = 0;
        SJ_TRY(count_range(h, 0, sv1, spairs, &ms_c));
        h->st.ms_estimate = ms_c;
        h->st.est_fused = 0;
        h->mail[0] = emitted;
        h->mail[2] = calcs;
    }
    return SJ_OK;
}

// The fast path right after sj_create, before the build's tail reached the host: ONE
// device-sized launch (the kernel reads the chunk count the build left in ix.d_meta and sizes
// the fused estimator's sample from it), so the GPU goes from the last build kernel straight
// into the join.  *spairs = the sample's pairs, *total = all pairs emitted.
int run_in_place_lazy(sj_handle *h, uint32_t *out, uint64_t cap, uint64_t *spairs, uint64_t *total, bool zeroed) {
    cudaStream_t s = h->s_main;
    if (!zeroed) SJ_CUDA_TRY(cudaMemsetAsync(h->d_ctr, 0, kCtrWords * sizeof(unsigned long long), s));
    SJ_CUDA_TRY(cudaEventRecord(h->ev_e, s));
    JoinArgs a = base_args(h);
    a.n_chunks = 0xFFFFFFFFu;      // bounded by the device-side V instead
    a.n_runs = h->ix.runs_cap;     // the allocation (>= E): bounds of the staged run copies
    a.d_nchunks = h->ix.d_meta;
    a.sample_ppm = h->sample_ppm;
    a.sample_ctr = h->d_ctr + 4;
    a.out = out;
    a.emit_ctr = h->d_ctr;
    a.out_cap = cap;
    a.calcs = h->count_calcs ? h->d_ctr + 2 : nullptr;
    a.head = h->d_ctr + kHead;
    a.v_begin = 0;
    a.v_end = 0xFFFFFFFFull;  // v_count = ~0u: the kernel bounds the queue by the device-side V
    int blocks;
    SJ_TRY(join_blocks(h, kPairs, &blocks));
    bool blocked = false;
    SJ_TRY(blocked_out(h, a, blocks, cap, &blocked));
    SJ_TRY(launch_join(a, h->ix.dim, h->k, blocked ? kPairsB : kPairs, blocks, s));
    if (blocked) SJ_TRY(compact_output(a, blocks, h->d_ctr + kTotal, blocked_ws(h, blocks), s));
    SJ_CUDA_TRY(cudaEventRecord(h->ev_d, s));
    SJ_CUDA_TRY(cudaMemcpyAsync(h->mail, h->d_ctr, kCtrWords * sizeof(uint64_t), cudaMemcpyDeviceToHost, s));
    SJ_CUDA_TRY(cudaStreamSynchronize(s));
    if (blocked) h->mail[0] = h->mail[kTotal];  // pairs emitted (the counter itself counts blocks)
    SJ_TRY(ix_ready(h));
    float ms = 0;
    SJ_CUDA_TRY(cudaEventElapsedTime(&ms, h->ev_e, h->ev_d));
    h->st.join_launches = 1;
    h->st.batches = 1;
    h->st.ms_estimate = 0.0;
    h->st.ms_join = h->st.ms_join_sum = ms;
    h->st.est_fused = 1;
    *spairs = h->mail[4];
    *total = h->mail[0];
    return SJ_OK;
}

int finish_in_place(sj_handle *h, uint64_t total, uint64_t *count) {
    if (h->count_calcs) h->st.calcs_measured = h->mail[2];
    h->st.pairs = total;
    h->st.fast_path = 1;
    *count = total;
    SJ_CUDA_TRY(cudaEventRecord(h->ev_b, h->s_main));
    SJ_CUDA_TRY(cudaEventSynchronize(h->ev_b));
    float tot = 0;
    SJ_CUDA_TRY(cudaEventElapsedTime(&tot, h->ev_a, h->ev_b));
    h->st.ms_total = tot;
    h->state = 0;
    return SJ_OK;
}

// Staged path: the queued jobs run round-robin over `streams` streams, each into its
// own b_s buffer, and are copied out in batch order.
int start_staged(sj_handle *h, uint32_t *out, uint64_t cap, uint64_t *count) {
    for (int i = 0; i < h->streams; ++i) SJ_TRY(slot_init(h, i));
    SJ_CUDA_TRY(cudaEventRecord(h->ev_c, h->s_main));
    for (int i = 0; i < h->streams; ++i) SJ_CUDA_TRY(cudaStreamWaitEvent(h->slots[i].stream, h->ev_c, 0));
    h->st.batches = (uint32_t)h->jobs.size();
    h->state = 1;
    return continue_staged(h, out, cap, count);
}

// Exact two-pass sizing (SJ_OPT_EXACT): pass 1 counts every
// chunk's pairs and scans them into chunk offsets; batches are cut at exact sizes <= b_s
// (a single chunk larger than b_s gets a batch -- and buffer -- of its own); pass 2 writes
// each chunk at its offset.  No estimator, no overflow retry, deterministic output order.
int start_exact(sj_handle *h, uint32_t *out, uint64_t cap, uint64_t *count, bool dev_out) {
    const uint64_t V = slice_chunks(h);
    if (h->voff_cap < V + 1) {
        dev_free(h->d_voff, h->s_main);
        h->d_voff = nullptr;
        h->voff_cap = 0;
        SJ_TRY(dev_alloc_t(&h->d_voff, V + 1, h->s_main));
        h->voff_cap = V + 1;
    }
    uint64_t total = 0;
    float ms = 0;
    SJ_TRY(count_range(h, 0, V, &total, &ms, h->d_voff));
    h->st.ms_estimate = ms;
    h->st.est_pairs = total;
    h->st.calcs_measured = 0;
    if (dev_out && h->fast_path && total <= cap) {
        uint64_t emitted = 0;
        SJ_TRY(run_in_place(h, out, cap, 0, V, true, &emitted));
        if (emitted != total) {
            set_error("sj_self_join: exact sizing mismatch: counted %llu pairs, emitted %llu",
                      (unsigned long long)total, (unsigned long long)emitted);
            return SJ_ECUDA;
        }
        return finish_in_place(h, total, count);
    }
    std::vector<uint64_t> off(V + 1);
    SJ_CUDA_TRY(cudaMemcpyAsync(off.data(), h->d_voff, (V + 1) * sizeof(uint64_t), cudaMemcpyDeviceToHost,
                                h->s_main));
    SJ_CUDA_TRY(cudaStreamSynchronize(h->s_main));
    if (off[V] != total) {
        set_error("sj_self_join: exact sizing: scan total %llu != counter %llu", (unsigned long long)off[V],
                  (unsigned long long)total);
        return SJ_ECUDA;
    }
    for (uint64_t v = 0; v < V;) {  // greedy: the longest run of chunks with <= b_s pairs
        uint64_t e = (uint64_t)(std::upper_bound(off.begin() + (long)v + 1, off.end(), off[v] + h->batch_pairs) -
                                off.begin()) - 1;
        if (e <= v) e = v + 1;
        Job j;
        j.v0 = v;
        j.v1 = e;
        j.base = off[v];
        j.expect = off[e] - off[v];
        h->jobs.push_back(j);
        v = e;
    }
    return start_staged(h, out, cap, count);
}

int start_join(sj_handle *h, uint32_t *out, uint64_t cap, uint64_t *count) {
    SJ_TRY(ensure_device(h));
    // a new join: reset per-join statistics
    h->st.pairs = 0;
    h->st.calcs_measured = 0;
    h->st.batches = 0;
    h->st.retries = 0;
    h->st.join_launches = 0;
    h->st.ms_join = h->st.ms_join_sum = h->st.ms_estimate = h->st.ms_transfer = h->st.ms_total = 0;
    h->st.fast_path = 0;
    h->st.est_fused = 0;
    h->st.k = (uint32_t)h->k;
    h->jobs.clear();
    for (int i = 0; i < kMaxStreams; ++i) h->slots[i].busy = false;

    SJ_CUDA_TRY(cudaEventRecord(h->ev_a, h->s_main));
    const bool dev_out = out && is_device_ptr(out, h->device);
    // right after sj_create, the in-place WorkQueue join needs nothing from the build on the
    // host (run_in_place_lazy); every other path reads the build's tail first
    const bool lazy = h->pending && dev_out && h->fast_path && !h->exact && h->queue &&
                      (uint64_t)h->grab * (uint64_t)h->world <= kChunkPad &&
                      !getenv("SJ_DEBUG_VRANGE") && !getenv("SJ_SEPARATE_EST") &&
                      !(reinterpret_cast<uintptr_t>(out) & 15u);
    uint64_t lazy_spairs = 0, lazy_total = 0;
    const bool zeroed = h->ctr_zeroed;  // (only the first join after the build finds them zeroed)
    h->ctr_zeroed = false;
    if (lazy) {
        SJ_TRY(run_in_place_lazy(h, out, cap, &lazy_spairs, &lazy_total, zeroed));
        debug_mark("join: lazy fast path");
    } else {
        SJ_TRY(ix_ready(h));
    }
    const uint64_t nch = slice_chunks(h);
    const uint64_t V = nch;

    if (out == nullptr) {  // count-only (whole slice, one launch)
        uint64_t pairs = 0;
        float ms = 0;
        SJ_TRY(count_range(h, 0, V, &pairs, &ms));
        h->st.ms_join = h->st.ms_join_sum = ms;
        h->st.join_launches = 1;
        h->st.batches = 1;
        h->st.pairs = pairs;
        *count = pairs;
        SJ_CUDA_TRY(cudaEventRecord(h->ev_b, h->s_main));
        SJ_CUDA_TRY(cudaEventSynchronize(h->ev_b));
        float tot = 0;
        SJ_CUDA_TRY(cudaEventElapsedTime(&tot, h->ev_a, h->ev_b));
        h->st.ms_total = tot;
        h->state = 0;
        return SJ_OK;
    }

    if (dev_out && (reinterpret_cast<uintptr_t>(out) & 15u)) {
        set_error("sj_self_join: device out_pairs must be 16-byte aligned");
        return SJ_EINVAL;
    }
    if (h->exact) return start_exact(h, out, cap, count, dev_out);

    // a9: batch estimator -- join over the first sample_ppm of D' (WorkQueue), or over a
    // strided sample of the whole dataset (SortByWL only: "samples a percentage of the
    // dataset"; P:200 contrasts the two)
    uint64_t sch = (nch * (uint64_t)h->sample_ppm + 999999ull) / 1000000ull;
    if (sch < 1) sch = 1;
    // whole dequeues (a WorkQueue dequeue takes `grab` consecutive chunks): the fused estimator's
    // sample then ends where a dequeue ends (the join kernel rounds the same way)
    if (h->queue) sch = (sch + h->grab - 1) / h->grab * h->grab;
    if (sch > nch) sch = nch;
    uint64_t sstride = 1, sv1 = sch;
    if (!h->queue && nch) {
        sstride = (nch + sch - 1) / sch;
        sv1 = nch;
        sch = (nch + sstride - 1) / sstride;  // chunks 0, sstride, 2 sstride, ...
    }
    uint64_t spairs = 0;
    float ms_est = 0;
    debug_mark("join: enter");
    if (dev_out && h->fast_path && !getenv("SJ_DEBUG_VRANGE")) {
        // Fast path: the caller's HBM buffer is the result buffer; the estimator and the join
        // run back to back without a host round trip.  Overflow is detected from the counter
        // (the join stops early) and falls back to the staged path below, whose batches are
        // sized by the estimate.
        uint64_t total = 0;
        if (lazy) {  // already ran; the sample is complete unless the output overflowed early
            spairs = lazy_spairs;
            total = lazy_total;
            if (h->mail[kHead] < sv1) {
                const uint64_t calcs = h->mail[2];
                float ms_c = 0;
                SJ_TRY(count_range(h, 0, sv1, &spairs, &ms_c));
                h->st.ms_estimate = ms_c;
                h->st.est_fused = 0;
                h->mail[0] = total;
                h->mail[2] = calcs;
            }
        } else {
            SJ_TRY(run_in_place_est(h, out, cap, sch, sv1, sstride, V, &spairs, &total));
        }
        debug_mark("join: fast path");
        h->st.est_pairs = nch ? (uint64_t)((double)spairs * (double)nch / (double)sch) : 0;
        if (total <= cap) return finish_in_place(h, total, count);
        ms_est = (float)h->st.ms_estimate;
        h->st.retries++;  // did not fit: fall through to the staged path
        h->st.ms_join = h->st.ms_join_sum = 0;
        h->st.join_launches = 0;
    } else if (nch) {
        SJ_TRY(count_range(h, 0, sv1, &spairs, &ms_est, nullptr, sstride));
    }
    debug_mark("join: estimator");
    h->st.ms_estimate = ms_est;
    h->st.calcs_measured = 0;
    const double est = nch ? (double)spairs * (double)nch / (double)sch : 0.0;
    h->st.est_pairs = (uint64_t)est;
    uint64_t nb = (uint64_t)std::ceil(est / (double)h->batch_pairs);
    if (nb < 1) nb = 1;
    if (nb > nch && nch) nb = nch;

    // The sample's own pairs are part of the result, so spairs is a strict lower bound of the
    // total; the extrapolated estimate is NOT (the first 1% of D' is the heaviest part)
    // and is only used to size the staged batches.
    if (dev_out && h->fast_path && spairs <= cap && getenv("SJ_DEBUG_VRANGE")) {
        // diagnostics: the in-place join of a sub-range only
        unsigned long long dv0 = 0, dv1 = V;
        if (const char *r = getenv("SJ_DEBUG_VRANGE")) {  // diagnostics: join a sub-range only
            sscanf(r, "%llu,%llu", &dv0, &dv1);
            dv1 = std::min<unsigned long long>(dv1, V);
        }
        uint64_t total = 0;
        SJ_TRY(run_in_place(h, out, cap, dv0, dv1, false, &total));
        debug_mark("join: fast path");
        if (total <= cap) return finish_in_place(h, total, count);
        h->st.retries++;  // did not fit: fall through to the staged path
        h->st.ms_join = h->st.ms_join_sum = 0;
        h->st.join_launches = 0;
    }

    // Staged path: nb batches = contiguous ranges of D' (WorkQueue, reading c14), or the
    // strided D'_l = {chunk v : v mod nb = l} of SortByWL only (Fig. 1).
    for (uint64_t b = 0; b < nb; ++b) {
        const Job j = batch_job(nch, nb, b, h->queue != 0);
        if (j.v1 > j.v0) h->jobs.push_back(j);
    }
    return start_staged(h, out, cap, count);
}

// Device CSR (sj_neighbor_csr): degrees (GCG row owners, no atomics) -> exclusive scan ->
// row fill.  Temporaries come from the stream-ordered pool.
int neighbor_csr(sj_handle *h, uint64_t *row_off, uint32_t *nbrs, uint64_t cap, uint64_t *total) {
    SJ_TRY(ix_ready(h));
    if (h->ix.pattern != SJ_PATTERN_GCG) {
        set_error("sj_neighbor_csr: needs a handle created with SJ_PATTERN_GCG (every query owns its row)");
        return SJ_EINVAL;
    }
    if (h->world != 1) {
        set_error("sj_neighbor_csr: needs the whole queue (sj_set_slice world 1)");
        return SJ_EINVAL;
    }
    if (h->state == 1) {
        set_error("sj_neighbor_csr: a staged sj_self_join is pending (SJ_MORE); finish it first");
        return SJ_EINVAL;
    }
    SJ_TRY(ensure_device(h));
    cudaStream_t s = h->s_main;
    const uint64_t n = h->ix.n, V = slice_chunks(h);
    h->st.pairs = 0;
    h->st.calcs_measured = 0;
    h->st.batches = 1;
    h->st.retries = 0;
    h->st.join_launches = 0;
    h->st.ms_join = h->st.ms_join_sum = h->st.ms_estimate = h->st.ms_transfer = h->st.ms_total = 0;
    h->st.fast_path = 0;
    SJ_CUDA_TRY(cudaEventRecord(h->ev_a, s));
    const bool off_dev = row_off && is_device_ptr(row_off, h->device) && !(reinterpret_cast<uintptr_t>(row_off) & 7u);
    uint64_t *d_off = off_dev ? row_off : nullptr;
    uint32_t *d_deg = nullptr, *d_nbrs = nullptr;
    int blocks;
    SJ_TRY(join_blocks(h, kDegree, &blocks));
    auto cleanup = [&]() {
        dev_free(d_deg, s);
        if (!off_dev) dev_free(d_off, s);
        if (d_nbrs != nbrs) dev_free(d_nbrs, s);
    };
    int rc = dev_alloc_t(&d_deg, n, s);
    if (rc == SJ_OK && !off_dev) rc = dev_alloc_t(&d_off, n + 1, s);
    if (rc < 0) {
        cleanup();
        return rc;
    }
    // pass 1: degrees
    JoinArgs a = base_args(h);
    a.head = h->d_ctr + kHead;
    a.emit_ctr = h->d_ctr;
    a.calcs = h->count_calcs ? h->d_ctr + 2 : nullptr;
    a.v_begin = 0;
    a.v_end = V;
    a.qdeg = d_deg;
    rc = [&]() -> int {
        SJ_CUDA_TRY(cudaMemsetAsync(h->d_ctr, 0, kCtrWords * sizeof(unsigned long long), s));
        SJ_CUDA_TRY(cudaEventRecord(h->ev_c, s));
        if (V) SJ_TRY(launch_join(a, h->ix.dim, h->k, kDegree, blocks, s));
        SJ_TRY(scan_exclusive_u32_to_u64(d_deg, d_off, n, d_off + n, s));
        SJ_CUDA_TRY(cudaEventRecord(h->ev_d, s));
        SJ_CUDA_TRY(cudaMemcpyAsync(h->mail, d_off + n, sizeof(uint64_t), cudaMemcpyDeviceToHost, s));
        SJ_CUDA_TRY(cudaMemcpyAsync(h->mail + 1, h->d_ctr, sizeof(uint64_t), cudaMemcpyDeviceToHost, s));
        if (row_off && !off_dev)
            SJ_CUDA_TRY(cudaMemcpyAsync(row_off, d_off, (n + 1) * sizeof(uint64_t), cudaMemcpyDefault, s));
        SJ_CUDA_TRY(cudaStreamSynchronize(s));
        float ms = 0;
        SJ_CUDA_TRY(cudaEventElapsedTime(&ms, h->ev_c, h->ev_d));
        h->st.ms_estimate = ms;
        h->st.join_launches = 1;
        *total = h->mail[0];
        h->st.est_pairs = h->mail[0];
        if (h->mail[0] != h->mail[1]) {
            set_error("sj_neighbor_csr: degree sum %llu != counter %llu", (unsigned long long)h->mail[0],
                      (unsigned long long)h->mail[1]);
            return SJ_ECUDA;
        }
        return SJ_OK;
    }();
    if (rc < 0 || !nbrs) {
        cleanup();
        return rc;
    }
    const uint64_t tot = *total;
    if (cap < tot) {
        cleanup();
        set_error("sj_neighbor_csr: cap %llu < %llu neighbour entries", (unsigned long long)cap,
                  (unsigned long long)tot);
        return SJ_EINVAL;
    }
    // pass 2: row fill
    const bool nb_dev = is_device_ptr(nbrs, h->device) && !(reinterpret_cast<uintptr_t>(nbrs) & 3u);
    d_nbrs = nb_dev ? nbrs : nullptr;
    if (!nb_dev) {
        rc = dev_alloc_t(&d_nbrs, tot, s);
        if (rc < 0) {
            cleanup();
            return rc;
        }
    }
    rc = [&]() -> int {
        JoinArgs b = base_args(h);
        b.head = h->d_ctr + kHead;
        b.emit_ctr = h->d_ctr;
        b.calcs = h->count_calcs ? h->d_ctr + 2 : nullptr;
        b.v_begin = 0;
        b.v_end = V;
        b.row_off = reinterpret_cast<const unsigned long long *>(d_off);
        b.nbrs = d_nbrs;
        int fb;
        SJ_TRY(join_blocks(h, kRows, &fb));
        SJ_CUDA_TRY(cudaMemsetAsync(h->d_ctr, 0, kCtrWords * sizeof(unsigned long long), s));
        SJ_CUDA_TRY(cudaEventRecord(h->ev_c, s));
        if (V) SJ_TRY(launch_join(b, h->ix.dim, h->k, kRows, fb, s));
        SJ_CUDA_TRY(cudaEventRecord(h->ev_d, s));
        SJ_CUDA_TRY(cudaMemcpyAsync(h->mail, h->d_ctr, kCtrWords * sizeof(uint64_t), cudaMemcpyDeviceToHost, s));
        if (!nb_dev && tot)
            SJ_CUDA_TRY(cudaMemcpyAsync(nbrs, d_nbrs, tot * sizeof(uint32_t), cudaMemcpyDefault, s));
        SJ_CUDA_TRY(cudaStreamSynchronize(s));
        float ms = 0;
        SJ_CUDA_TRY(cudaEventElapsedTime(&ms, h->ev_c, h->ev_d));
        h->st.ms_join = h->st.ms_join_sum = ms;
        h->st.join_launches = 2;
        if (h->count_calcs) h->st.calcs_measured = h->mail[2];
        if (h->mail[0] != tot) {
            set_error("sj_neighbor_csr: filled %llu entries, counted %llu", (unsigned long long)h->mail[0],
                      (unsigned long long)tot);
            return SJ_ECUDA;
        }
        h->st.pairs = tot;
        SJ_CUDA_TRY(cudaEventRecord(h->ev_b, s));
        SJ_CUDA_TRY(cudaEventSynchronize(h->ev_b));
        float all = 0;
        SJ_CUDA_TRY(cudaEventElapsedTime(&all, h->ev_a, h->ev_b));
        h->st.ms_total = all;
        return SJ_OK;
    }();
    cleanup();
    return rc;
}

}  // namespace

// =========================================================================== C ABI
extern "C" {

int sj_abi_version(void) { return SJ_ABI_VERSION; }

uint64_t sj_kernel_launches(void) { return g_launches.load(); }

void sj_set_stream(void *stream) {
    g_caller_stream = stream ? static_cast<cudaStream_t>(stream) : cudaStreamLegacy;
}

const char *sj_last_error(void) { return g_err; }

static int create_common(sj_handle **out_h) {
    sj_handle *h = new (std::nothrow) sj_handle();
    if (!h) {
        set_error("out of host memory");
        return SJ_ENOMEM;
    }
    int rc = handle_init_common(h);
    if (rc < 0) {
        sj_destroy(h);
        return rc;
    }
    *out_h = h;
    return SJ_OK;
}


sj_handle *sj_create(const double *points, uint64_t n, int dim, double eps) {
    return sj_create_ex(points, n, dim, eps, SJ_PATTERN_LID_UNICOMP, SJ_ORDER_WORKLOAD);
}

static sj_handle *create_impl(const double *points, uint64_t n, int dim, double eps, int pattern, int order,
                              const uint32_t *ids, uint64_t n_query, const double *origin);

sj_handle *sj_create_ex(const double *points, uint64_t n, int dim, double eps, int pattern, int order) {
    return create_impl(points, n, dim, eps, pattern, order, nullptr, n, nullptr);
}

sj_handle *sj_create_part(const double *points, const uint32_t *ids, uint64_t n, uint64_t n_query, int dim,
                          double eps, const double *origin) {
    set_error("");
    if (!origin || n_query > n) {
        set_error("sj_create_part: invalid argument (origin=%p n=%llu n_query=%llu)", (const void *)origin,
                  (unsigned long long)n, (unsigned long long)n_query);
        return nullptr;
    }
    return create_impl(points, n, dim, eps, SJ_PATTERN_LID_UNICOMP, SJ_ORDER_WORKLOAD, ids, n_query, origin);
}

static sj_handle *create_impl(const double *points, uint64_t n, int dim, double eps, int pattern, int order,
                              const uint32_t *ids, uint64_t n_query, const double *origin) {
    set_error("");
    if (!points || n == 0 || n >= (1ull << 32) || dim < 1 || dim > SJ_MAX_DIM || !(eps > 0.0) || !std::isfinite(eps) ||
        pattern < SJ_PATTERN_LID_UNICOMP || pattern > SJ_PATTERN_UNICOMP || order < SJ_ORDER_WORKLOAD ||
        order > SJ_ORDER_INPUT) {
        set_error("sj_create: invalid argument (points=%p n=%llu dim=%d eps=%g pattern=%d order=%d)",
                  (const void *)points, (unsigned long long)n, dim, eps, pattern, order);
        return nullptr;
    }
    int ndev = 0;
    if (cudaGetDeviceCount(&ndev) != cudaSuccess || ndev == 0) {
        cudaGetLastError();
        set_error("sj_create: no CUDA device available (the CUDA path has no CPU fallback)");
        return nullptr;
    }
    debug_mark("create: enter");
    sj_handle *h = nullptr;
    if (create_common(&h) < 0) return nullptr;
    debug_mark("create: handle init");
    cudaStream_t s = h->s_main;
    const double *d_raw = points;
    double *d_copy = nullptr;
    int rc = order_after_caller(h);  // device points may still be in flight on the caller's stream
    // host input, or a device pointer that is not 16-byte aligned (the build reads double2)
    if (!is_device_ptr(points, h->device) || (reinterpret_cast<uintptr_t>(points) & 15u)) {
        // a1: upload (the library owns its copy; caller keeps `points`)
        rc = dev_alloc_t(&d_copy, n * (uint64_t)dim, s);
        if (rc == SJ_OK) {
            cudaError_t e = cudaMemcpyAsync(d_copy, points, n * (uint64_t)dim * sizeof(double), cudaMemcpyDefault, s);
            if (e != cudaSuccess) {
                set_error("sj_create: upload failed: %s", cudaGetErrorString(e));
                rc = SJ_ECUDA;
            }
        }
        d_raw = d_copy;
    }
    float ms = 0;
    h->ix.pattern = pattern;
    h->ix.order = order;
    // partitioned index (sj_create_part): ids to the device, origin and query count
    BuildPart part;
    uint32_t *d_ids = nullptr;
    if (origin) {
        for (int d = 0; d < dim; ++d) part.origin[d] = origin[d];
        part.n_query = n_query;
        part.d_ids = ids;
        if (rc == SJ_OK && ids && !is_device_ptr(ids, h->device)) {
            rc = dev_alloc_t(&d_ids, n, s);
            if (rc == SJ_OK && cudaMemcpyAsync(d_ids, ids, n * sizeof(uint32_t), cudaMemcpyDefault, s) != cudaSuccess) {
                set_error("sj_create_part: id upload failed: %s", cudaGetErrorString(cudaGetLastError()));
                rc = SJ_ECUDA;
            }
            part.d_ids = d_ids;
        }
    }
    debug_mark("create: upload issued");
    // The build returns without a final host round trip (its tail is read by ix_ready) unless
    // SJ_SYNC_BUILD=1; errors of its last kernels surface at the next synchronisation.
    static const bool sync_build = [] {
        const char *e = getenv("SJ_SYNC_BUILD");
        return e && e[0] == '1';
    }();
    if (rc == SJ_OK)
        rc = build_index(h->ix, d_raw, n, dim, eps, s, h->ev_ba, h->ev_bb, &ms, origin ? &part : nullptr,
                         sync_build ? nullptr : h->mail + 48, h->side.s2 ? &h->side : nullptr, h->d_ctr,
                         kCtrWords);
    h->ctr_zeroed = rc == SJ_OK;  // the build's last kernel zeroed the join's counters
    debug_mark("create: build_index");
    dev_free(d_copy, s);
    dev_free(d_ids, s);
    if (rc == SJ_OK && sync_build && cudaStreamSynchronize(s) != cudaSuccess) {
        set_error("sj_create: %s", cudaGetErrorString(cudaGetLastError()));
        rc = SJ_ECUDA;
    }
    if (rc < 0) {
        std::string keep = g_err;
        sj_destroy(h);
        snprintf(g_err, sizeof g_err, "%s", keep.c_str());
        return nullptr;
    }
    if (dim >= 4) h->grab = 1;  // 4-D+: every chunk is heavy; one per dequeue keeps the end balanced
    if (sync_build) {
        fill_static_stats(h);
        h->st.ms_build = ms;
    } else {
        h->pending = 1;
    }
    return h;
}

int sj_self_join(sj_handle *h, uint32_t *out_pairs, uint64_t cap, uint64_t *count) {
    if (!h || !count) {
        set_error("sj_self_join: NULL handle or count");
        return SJ_EINVAL;
    }
    *count = 0;
    if (h->state < 0) {
        set_error("sj_self_join: handle is in the error state");
        return SJ_ESTATE;
    }
    if ((out_pairs == nullptr) != (cap == 0)) {
        set_error("sj_self_join: out_pairs and cap must both be set, or both NULL/0 for count-only");
        return SJ_EINVAL;
    }
    int rc = ensure_device(h);
    if (rc == SJ_OK) rc = order_after_caller(h);  // the caller's buffer may have pending work
    if (rc < 0) return fail(h, rc);
    if (h->state == 1 && out_pairs) {
        rc = continue_staged(h, out_pairs, cap, count);
    } else {
        rc = start_join(h, out_pairs, cap, count);
    }
    return fail(h, rc);
}

int sj_neighbor_csr(sj_handle *h, uint64_t *row_off, uint32_t *nbrs, uint64_t cap, uint64_t *total) {
    if (!h || !total || ((nbrs == nullptr) != (cap == 0))) {
        set_error("sj_neighbor_csr: NULL handle/total, or nbrs and cap not both set / both NULL-0");
        return SJ_EINVAL;
    }
    *total = 0;
    if (h->state < 0) {
        set_error("sj_neighbor_csr: handle is in the error state");
        return SJ_ESTATE;
    }
    int rc = ensure_device(h);
    if (rc == SJ_OK) rc = order_after_caller(h);
    if (rc == SJ_OK) rc = neighbor_csr(h, row_off, nbrs, cap, total);
    return rc == SJ_EINVAL ? rc : fail(h, rc);
}

void sj_destroy(sj_handle *h) {
    if (!h) return;
    debug_mark("destroy: enter");
    cudaSetDevice(h->device);
    slots_release(h);
    if (h->s_main) dev_free(h->d_voff, h->s_main);
    if (h->s_main && h->owns_index) free_index(h->ix, h->s_main);  // stream-ordered frees
    if (!core_release(h)) {  // (a released core keeps the blocked output's workspace)
        if (h->s_main) {
            dev_free(h->outws, h->s_main);
            cudaStreamSynchronize(h->s_main);
            dev_free(h->d_ctr, h->s_main);
            cudaStreamSynchronize(h->s_main);
            cudaStreamDestroy(h->s_main);
        }
        if (h->ev_a) cudaEventDestroy(h->ev_a);
        if (h->ev_b) cudaEventDestroy(h->ev_b);
        if (h->ev_c) cudaEventDestroy(h->ev_c);
        if (h->ev_d) cudaEventDestroy(h->ev_d);
        if (h->ev_e) cudaEventDestroy(h->ev_e);
        if (h->ev_ba) cudaEventDestroy(h->ev_ba);
        if (h->ev_bb) cudaEventDestroy(h->ev_bb);
        if (h->ev_in) cudaEventDestroy(h->ev_in);
        if (h->side.s2) {
            cudaStreamSynchronize(h->side.s2);
            cudaStreamDestroy(h->side.s2);
        }
        if (h->side.ea) cudaEventDestroy(h->side.ea);
        if (h->side.eg) cudaEventDestroy(h->side.eg);
        if (h->side.eq) cudaEventDestroy(h->side.eq);
        if (h->side.ej) cudaEventDestroy(h->side.ej);
        pinned_release(h->mail);
    }
    delete h;
    debug_mark("destroy: done");
}

int sj_set_option(sj_handle *h, int opt, int64_t v) {
    if (!h) return SJ_EINVAL;
    switch (opt) {
        case SJ_OPT_K:
            if (v != 1 && v != 2 && v != 4 && v != 8 && v != 16 && v != 32) break;
            h->k = (int)v;
            h->st.k = (uint32_t)v;
            return SJ_OK;
        case SJ_OPT_BATCH_PAIRS:
            if (v < 64) break;
            h->batch_pairs = (uint64_t)v;
            return SJ_OK;
        case SJ_OPT_STREAMS:
            if (v < 1 || v > kMaxStreams) break;
            h->streams = (int)v;
            return SJ_OK;
        case SJ_OPT_SAMPLE_PPM:
            if (v < 1 || v > 1000000) break;
            h->sample_ppm = (uint32_t)v;
            return SJ_OK;
        case SJ_OPT_GRAB:
            if (v < 1 || v > 1024) break;
            h->grab = (uint32_t)v;
            return SJ_OK;
        case SJ_OPT_COUNT_CALCS:
            h->count_calcs = v ? 1 : 0;
            return SJ_OK;
        case SJ_OPT_BLOCKS_PER_SM:
            if (v < 0 || v > 32) break;
            h->blocks_per_sm = (int)v;
            return SJ_OK;
        case SJ_OPT_FAST_PATH:
            h->fast_path = v ? 1 : 0;
            return SJ_OK;
        case SJ_OPT_EXACT:
            h->exact = v ? 1 : 0;
            return SJ_OK;
        case SJ_OPT_QUEUE:
            if (v != 0 && v != 1) break;
            h->queue = (int)v;
            return SJ_OK;
        case SJ_OPT_OUT_BLOCKS:
            if (v < 0 || v > 2) break;
            h->out_blocks = (int)v;
            return SJ_OK;

    }
    set_error("sj_set_option: invalid option %d or value %lld", opt, (long long)v);
    return SJ_EINVAL;
}

int sj_set_slice(sj_handle *h, int rank, int world) {
    if (!h || world < 1 || rank < 0 || rank >= world) {
        set_error("sj_set_slice: invalid rank %d / world %d", rank, world);
        return SJ_EINVAL;
    }
    h->rank = rank;
    h->world = world;
    h->state = h->state < 0 ? h->state : 0;
    return SJ_OK;
}

int sj_get_stats(const sj_handle *h, sj_stats *s) {
    if (!h || !s) return SJ_EINVAL;
    SJ_TRY(ix_ready(const_cast<sj_handle *>(h)));
    *s = h->st;
    return SJ_OK;
}

// ---------------------------------------------------------------- index export / import
namespace {
struct BlobHeader {
    uint64_t magic;  // "SJIDX004"
    uint64_t n;
    int32_t dim, pad, key_bits, pattern_order;
    double eps, e2, w;
    double mins[SJ_MAX_DIM];
    uint64_t nc[SJ_MAX_DIM];
    uint64_t stride[SJ_MAX_DIM];
    uint64_t n_cells, n_runs, dist_calcs, n_chunks;
    uint32_t max_w, lookup_hash;
    uint64_t off[7], bytes[7];  // pts, orig, qmap, cellq, runs, cell_lid, chunks
    uint64_t total;
    uint64_t n_query;  // queries of a partitioned index (D' positions [0, n_query))
    uint64_t runs_len; // entries of the runs array (slot layout: M * rows; else = n_runs)
};
constexpr uint64_t kMagic = 0x3430305844494a53ull;  // "SJIDX004"
constexpr uint64_t kHdr = 1024;
static_assert(sizeof(BlobHeader) <= kHdr, "header");

BlobHeader make_header(const Index &ix) {
    BlobHeader b{};
    b.magic = kMagic;
    b.n = ix.n;
    b.dim = ix.dim;
    b.pad = ix.pad;
    b.key_bits = ix.key_bits;
    b.pattern_order = ix.pattern | (ix.order << 8);
    b.eps = ix.eps;
    b.e2 = ix.e2;
    b.w = ix.w;
    for (int d = 0; d < SJ_MAX_DIM; ++d) {
        b.mins[d] = ix.mins[d];
        b.nc[d] = ix.nc[d];
        b.stride[d] = ix.stride[d];
    }
    b.n_cells = ix.n_cells;
    b.n_runs = ix.n_runs;
    b.n_chunks = ix.n_chunks;
    b.dist_calcs = ix.dist_calcs;
    b.max_w = ix.max_w;
    b.lookup_hash = (uint32_t)ix.lookup_hash;
    const uint64_t sz[7] = {ix.n * ix.pad * sizeof(double), ix.n * sizeof(uint32_t), ix.n * sizeof(uint2),
                            ix.n_cells * sizeof(uint4), runs_entries(ix) * sizeof(uint2), ix.n_cells * sizeof(uint64_t),
                            (ix.n_chunks + 1) * sizeof(uint32_t)};
    uint64_t o = kHdr;
    for (int i = 0; i < 7; ++i) {
        b.off[i] = o;
        b.bytes[i] = sz[i];
        o += (sz[i] + 255) & ~255ull;
    }
    b.total = o;
    b.n_query = ix.n_query;
    b.runs_len = ix.runs_len;
    return b;
}
}  // namespace

int sj_export_index(const sj_handle *h, void *dst, uint64_t cap, uint64_t *bytes) {
    if (!h || !bytes) return SJ_EINVAL;
    SJ_TRY(ix_ready(const_cast<sj_handle *>(h)));
    BlobHeader b = make_header(h->ix);
    *bytes = b.total;
    if (!dst) return SJ_OK;
    if (cap < b.total) {
        set_error("sj_export_index: cap %llu < %llu bytes", (unsigned long long)cap, (unsigned long long)b.total);
        return SJ_EINVAL;
    }
    SJ_TRY(ensure_device(h));
    SJ_TRY(order_after_caller(const_cast<sj_handle *>(h)));
    char *d = static_cast<char *>(dst);
    const void *src[7] = {h->ix.pts, h->ix.orig, h->ix.qmap, h->ix.cellq, h->ix.runs, h->ix.cell_lid, h->ix.chunks};
    SJ_CUDA_TRY(cudaMemcpyAsync(d, &b, sizeof b, cudaMemcpyDefault, h->s_main));
    for (int i = 0; i < 7; ++i)
        if (b.bytes[i]) SJ_CUDA_TRY(cudaMemcpyAsync(d + b.off[i], src[i], b.bytes[i], cudaMemcpyDefault, h->s_main));
    SJ_CUDA_TRY(cudaStreamSynchronize(h->s_main));
    return SJ_OK;
}

// Every field of a received blob is checked before anything is copied or read by a kernel: the
// blob crosses process boundaries (NCCL broadcast), so a truncated or corrupt one must give
// SJ_EINVAL, not out-of-bounds copies or device reads.
static bool blob_header_ok(const BlobHeader &b, uint64_t bytes, const char **why) {
    *why = "";
    if (b.magic != kMagic) return *why = "magic (not an SJIDX004 blob of this library version)", false;
    if (b.total > bytes || b.total < kHdr) return *why = "total size exceeds the buffer", false;
    if (b.dim < 1 || b.dim > SJ_MAX_DIM) return *why = "dim", false;
    if (b.n < 1 || b.n >= (1ull << 32)) return *why = "n", false;
    const int pad = b.dim == 1 ? 1 : ((b.dim + 1) & ~1);
    if (b.pad != pad) return *why = "pad", false;
    const int pattern = b.pattern_order & 0xFF, order = (b.pattern_order >> 8) & 0xFF;
    if (pattern > SJ_PATTERN_UNICOMP || order > SJ_ORDER_INPUT || (b.pattern_order >> 16)) return *why = "pattern/order", false;
    if (b.n_cells < 1 || b.n_cells > b.n) return *why = "n_cells", false;
    if (b.n_chunks < 1 || b.n_chunks > b.n || b.n_chunks >= (1ull << 32)) return *why = "n_chunks", false;
    if (b.n_query > b.n) return *why = "n_query", false;
    if (b.runs_len && b.runs_len < b.n_runs) return *why = "runs_len", false;
    if (!(b.e2 > 0.0) || !(b.w > 0.0) || b.key_bits < 0 || b.key_bits > 64) return *why = "eps/w/key_bits", false;
    const uint64_t runs = b.runs_len ? b.runs_len : b.n_runs;
    const uint64_t want[7] = {b.n * (uint64_t)pad * sizeof(double), b.n * sizeof(uint32_t), b.n * sizeof(uint2),
                              b.n_cells * sizeof(uint4), runs * sizeof(uint2), b.n_cells * sizeof(uint64_t),
                              (b.n_chunks + 1) * sizeof(uint32_t)};
    uint64_t end = kHdr;
    for (int i = 0; i < 7; ++i) {
        if (b.bytes[i] != want[i]) return *why = "array size", false;
        if (b.off[i] < end || b.off[i] > b.total || b.bytes[i] > b.total - b.off[i]) return *why = "array extent", false;
        end = b.off[i] + b.bytes[i];
    }
    return true;
}

static sj_handle *from_index_impl(const void *blob, uint64_t bytes, bool view);

sj_handle *sj_create_from_index(const void *blob, uint64_t bytes) { return from_index_impl(blob, bytes, false); }

sj_handle *sj_create_from_index_view(const void *blob, uint64_t bytes) { return from_index_impl(blob, bytes, true); }

static sj_handle *from_index_impl(const void *blob, uint64_t bytes, bool view) {
    set_error("");
    if (!blob || bytes < kHdr) {
        set_error("sj_create_from_index: invalid blob");
        return nullptr;
    }
    int ndev = 0;
    if (cudaGetDeviceCount(&ndev) != cudaSuccess || ndev == 0) {
        cudaGetLastError();
        set_error("sj_create_from_index: no CUDA device available");
        return nullptr;
    }
    sj_handle *h = nullptr;
    if (create_common(&h) < 0) return nullptr;
    if (view && (!is_device_ptr(blob, h->device) || (reinterpret_cast<uintptr_t>(blob) & 255u))) {
        sj_destroy(h);
        set_error("sj_create_from_index_view: the blob must be device memory of the current device, 256-byte aligned");
        return nullptr;
    }
    cudaStream_t s = h->s_main;
    // the blob may have been written on the caller's stream (e.g. the NCCL broadcast's output)
    BlobHeader b;
    int rc = order_after_caller(h);
    if (rc == SJ_OK && (cudaMemcpyAsync(h->mail, blob, sizeof b, cudaMemcpyDefault, s) != cudaSuccess ||
                        cudaStreamSynchronize(s) != cudaSuccess)) {
        set_error("sj_create_from_index: %s", cudaGetErrorString(cudaGetLastError()));
        rc = SJ_ECUDA;
    }
    const char *why = "";
    if (rc == SJ_OK) {
        static_assert(sizeof(BlobHeader) <= kMailBytes, "header through the mailbox");
        memcpy(&b, h->mail, sizeof b);
        if (!blob_header_ok(b, bytes, &why)) {
            set_error("sj_create_from_index: bad header (%s)", why);
            rc = SJ_EINVAL;
        }
    }
    if (rc < 0) {
        std::string keep = g_err;
        sj_destroy(h);
        snprintf(g_err, sizeof g_err, "%s", keep.c_str());
        return nullptr;
    }
    Index &ix = h->ix;
    ix.n = b.n;
    ix.dim = b.dim;
    ix.pad = b.pad;
    ix.key_bits = b.key_bits;
    ix.pattern = b.pattern_order & 0xFF;
    ix.order = (b.pattern_order >> 8) & 0xFF;
    ix.eps = b.eps;
    ix.e2 = b.e2;
    ix.w = b.w;
    for (int d = 0; d < SJ_MAX_DIM; ++d) {
        ix.mins[d] = b.mins[d];
        ix.nc[d] = b.nc[d];
        ix.stride[d] = b.stride[d];
    }
    ix.n_cells = b.n_cells;
    ix.n_runs = b.n_runs;
    ix.runs_len = b.runs_len;
    ix.runs_cap = runs_entries(ix) + 2;
    ix.n_chunks = b.n_chunks;
    ix.n_query = b.n_query ? b.n_query : b.n;
    ix.dist_calcs = b.dist_calcs;
    ix.max_w = b.max_w;
    ix.lookup_hash = (int)b.lookup_hash;
    void **dst[7] = {(void **)&ix.pts,  (void **)&ix.orig,     (void **)&ix.qmap,  (void **)&ix.cellq,
                     (void **)&ix.runs, (void **)&ix.cell_lid, (void **)&ix.chunks};
    if (view) {  // zero copy: the arrays are the blob's (the caller keeps it alive, unchanged)
        for (int i = 0; i < 7; ++i)
            *dst[i] = const_cast<char *>(static_cast<const char *>(blob)) + b.off[i];
        h->owns_index = false;
        if (ix.dim >= 4) h->grab = 1;
        fill_static_stats(h);
        return h;
    }
    for (int i = 0; i < 7 && rc == SJ_OK; ++i) {
        rc = dev_alloc(dst[i], b.bytes[i] + 32, s);
        if (rc == SJ_OK && b.bytes[i] &&
            cudaMemcpyAsync(*dst[i], static_cast<const char *>(blob) + b.off[i], b.bytes[i], cudaMemcpyDefault, s) !=
                cudaSuccess) {
            set_error("sj_create_from_index: copy failed");
            rc = SJ_ECUDA;
        }
    }
    if (rc == SJ_OK && cudaStreamSynchronize(s) != cudaSuccess) rc = SJ_ECUDA;
    if (rc < 0) {
        sj_destroy(h);
        return nullptr;
    }
    if (ix.dim >= 4) h->grab = 1;
    fill_static_stats(h);
    return h;
}

// ---------------------------------------------------------------- host-only helpers
int sj_forward_offsets(int dim, int8_t *out, uint64_t cap) {
    return sj::forward_offsets_public(dim, out, cap);
}

int64_t sj_slice_chunks(uint64_t n_chunks, int rank, int world, uint32_t *out, uint64_t cap) {
    if (world < 1 || rank < 0 || rank >= world || n_chunks >= (1ull << 32)) return SJ_EINVAL;
    int64_t cnt = 0;
    for (uint64_t c = (uint64_t)rank; c < n_chunks; c += (uint64_t)world) {
        if (out) {
            if ((uint64_t)cnt >= cap) return SJ_EINVAL;
            out[cnt] = (uint32_t)c;
        }
        ++cnt;
    }
    return cnt;
}

int64_t sj_batch_chunks(uint64_t n_chunks, uint64_t n_batches, uint64_t batch, int queue, uint32_t *out,
                        uint64_t cap) {
    if (n_batches < 1 || batch >= n_batches || n_chunks >= (1ull << 32) || (queue != 0 && queue != 1))
        return SJ_EINVAL;
    const Job j = batch_job(n_chunks, n_batches, batch, queue != 0);
    int64_t cnt = 0;
    for (uint64_t v = j.v0; v < j.v1; v += j.stride) {
        if (out) {
            if ((uint64_t)cnt >= cap) return SJ_EINVAL;
            out[cnt] = (uint32_t)v;
        }
        ++cnt;
    }
    return cnt;
}

}  // extern "C"
