// dfs_runtime.cu — host runtime + C ABI (include/dfs.h) of the B200 unordered-DFS library.
//
// Owns graph residency (step a1: copy, validate, narrow row_ptr to uint32), per-traversal
// scratch "slots" (visited bitmap,
// per-warp ColdSeg words, chunk table, chunk pool, control block) and the launch sequence
// reset (a2) -> persistent traversal (a3-a8) -> finalize (a9).  A batch (a10) may run K
// traversals concurrently on K slots / streams, each on a 1/K share of the SMs (SURVEY
// §8(f)-2).  "P:a-b" = /root/reference/PAPER.md lines.
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <new>
#include <thread>
#include <vector>

#include "../../include/dfs.h"
#include "dfs_device.cuh"
#include "dfs_walker.cuh"

using namespace b200dfs;

#ifndef DFS_KRING
#define DFS_KRING 256
#endif

namespace {

constexpr int kRing = DFS_KRING;            // HotRing entries per warp (P:367 uses 128)
constexpr int kMaxSlots = 16;                // concurrent traversals per handle (batches)
thread_local int g_last_error = DFS_OK;

int fail(int code) { g_last_error = code; return code; }

bool is_device_ptr(const void* p) {
    cudaPointerAttributes a;
    if (cudaPointerGetAttributes(&a, p) != cudaSuccess) { cudaGetLastError(); return false; }
    return a.type == cudaMemoryTypeDevice || a.type == cudaMemoryTypeManaged;
}

// the 24 instantiations of the persistent kernel: [bulk][cluster tier][vec128][wmax16][stats]
// (the bulk variants without the cluster tier)
// DFS_WMAX_BIG: warps per CTA of the large instantiations (32: 64 registers per thread)
#ifndef DFS_WMAX_BIG
#define DFS_WMAX_BIG 32
#endif
#define DFS_K(V, W, S, C, B) (const void*)dfs_persistent_kernel<kRing, V, (W == 32 ? DFS_WMAX_BIG : W), S, C, B>
const void* const* kernel_table() {
    static const void* const t[24] = {
        DFS_K(1, 32, false, false, false), DFS_K(1, 32, true, false, false), DFS_K(1, 16, false, false, false), DFS_K(1, 16, true, false, false),
        DFS_K(4, 32, false, false, false), DFS_K(4, 32, true, false, false), DFS_K(4, 16, false, false, false), DFS_K(4, 16, true, false, false),
        DFS_K(1, 32, false, true, false), DFS_K(1, 32, true, true, false), DFS_K(1, 16, false, true, false), DFS_K(1, 16, true, true, false),
        DFS_K(4, 32, false, true, false), DFS_K(4, 32, true, true, false), DFS_K(4, 16, false, true, false), DFS_K(4, 16, true, true, false),
        DFS_K(1, 32, false, false, true), DFS_K(1, 32, true, false, true), DFS_K(1, 16, false, false, true), DFS_K(1, 16, true, false, true),
        DFS_K(4, 32, false, false, true), DFS_K(4, 32, true, false, true), DFS_K(4, 16, false, false, true), DFS_K(4, 16, true, false, true)};
    return t;
}
#undef DFS_K
constexpr int kNumKernels = 24;

// sub-warp walker kernels (dfs_walker.cuh): [G = 16, 8, 4, 2][stats], then the vertex-record
// variants [G = 16, 8][stats]; HotRing H = 16 * G entries per walker, so a 32-warp CTA holds
// 128 KB of rings for every G
#define DFS_WK(G, S, R) (const void*)dfs_walker_kernel<G, 16 * G, S, R>
const void* const* walker_table() {
    static const void* const t[12] = {DFS_WK(16, false, false), DFS_WK(16, true, false), DFS_WK(8, false, false),
                                      DFS_WK(8, true, false), DFS_WK(4, false, false), DFS_WK(4, true, false),
                                      DFS_WK(2, false, false), DFS_WK(2, true, false),
                                      DFS_WK(16, false, true), DFS_WK(16, true, true), DFS_WK(8, false, true),
                                      DFS_WK(8, true, true)};
    return t;
}
#undef DFS_WK
constexpr int kNumWalkerKernels = 12;
int walker_lanes_of(int kf) {
    static const int lanes[12] = {16, 16, 8, 8, 4, 4, 2, 2, 16, 16, 8, 8};
    return lanes[kf];
}
int walker_index(int lanes, bool rec) {
    if (rec && lanes >= 8) return lanes == 16 ? 8 : 10;
    return lanes == 16 ? 0 : lanes == 8 ? 2 : lanes == 4 ? 4 : 6;
}
bool valid_walker_lanes(int lanes) { return lanes == 16 || lanes == 8 || lanes == 4 || lanes == 2; }
constexpr int kWalkerMaxWarps = DFS_WALKER_LB / 32;

size_t smem_bytes(int warps) {
    return ((sizeof(SmemCtl) + 15) & ~size_t(15)) + (size_t)warps * kRing * sizeof(unsigned long long);
}
size_t walker_smem_bytes(int warps, int lanes) {
    return ((sizeof(SmemW) + 15) & ~size_t(15)) + (size_t)warps * (32 / lanes) * (16 * lanes) * sizeof(unsigned long long);
}

// per-traversal scratch set
struct Slot {
    bool ready = false;
    uint32_t* bitmap = nullptr;
    uint32_t bstride = 1;                   // bitmap layout of the last launch (1, or 2 = {visited, leaf})
    int32_t* parent = nullptr;              // lazily allocated for host outputs
    int32_t* parent2 = nullptr;             // second row buffer: concurrent batches into host memory
                                            // copy one row while the next traversal fills the other
    cudaStream_t cstream = nullptr;         // device->host copies of the slot's rows (batches)
    cudaEvent_t evt[2] = {nullptr, nullptr};   // traversal into buffer b done (copy may start)
    cudaEvent_t evc[2] = {nullptr, nullptr};   // copy out of buffer b done (buffer reusable)
    unsigned long long* cold_tb = nullptr;
    uint32_t* tab = nullptr;
    unsigned long long* pool = nullptr;
    uint32_t* consumed = nullptr;
    uint32_t* next = nullptr;
    int* block_cold = nullptr;
    Ctl* ctl = nullptr;
    unsigned long long* count2 = nullptr;   // visited count, TEPS numerator (summed over a batch)
    int* status = nullptr;                  // worst status over the slot's traversals in a batch
    unsigned long long* block_claims = nullptr;   // per-block claim counts (stats), else null
    size_t tab_words = 0;
    int64_t n_warps_cap = 0;                // warps (blocks x warps per block) the scratch is sized for
    uint32_t n_chunks = 0;
    bool tab_dirty = false;
    cudaStream_t stream = nullptr;          // own stream (slots >= 1 of a concurrent batch)
    cudaEvent_t ev0 = nullptr, ev1 = nullptr, evk0 = nullptr, evk1 = nullptr;
    cudaEvent_t evq[2] = {nullptr, nullptr};   // completion of the last two traversals issued (batches)
    int64_t issued = 0;                        // traversals issued on this slot in the current batch
};

}  // namespace

struct dfs_graph {
    int device = 0;
    cudaStream_t stream = nullptr;
    int64_t n = 0, m = 0;
    int64_t max_degree = 0;      // maximum out-degree (kernel selection)
    int sms = 0;
    int max_blocks = 0;          // co-resident 32-warp blocks (allocation bound)
    int max_clusters[4] = {0, 0, 0, 0};   // co-resident clusters of 1/2/4/8 CTAs (lazy)
    size_t persist_req = 0;      // l2_persist_mb requested last (bytes)
    size_t persist_bytes = 0;    // persisting-L2 set-aside granted for it (0 = none)
    size_t max_window_bytes = 0; // cudaDevAttrMaxAccessPolicyWindowSize
    int tab_log2 = 0;
    uint32_t* d_rp = nullptr;
    int32_t* d_col = nullptr;    // col_idx (+8 padding for 128-bit window loads)
    uint32_t* d_leaf = nullptr;  // leaf map: ceil(n/32) words (dfs_leaf_*_kernel)
    uint32_t* d_rec = nullptr;   // vertex records: 8 words per vertex (built on first use)
    Slot slots[kMaxSlots];
    int64_t launches = 0;
    unsigned int* d_timeline = nullptr;   // diagnostics (dfs_debug_timeline)
    unsigned int timeline_len = 0, timeline_dt_ns = 0;
    unsigned long long* d_counts = nullptr;   // per-root (n_visited, m_visited) of a stats call
    int32_t counts_cap = 0;
};

static void free_slot(Slot& s) {
    cudaFree(s.bitmap); cudaFree(s.parent); cudaFree(s.parent2); cudaFree(s.cold_tb); cudaFree(s.tab); cudaFree(s.pool);
    cudaFree(s.consumed); cudaFree(s.next); cudaFree(s.block_cold); cudaFree(s.ctl); cudaFree(s.count2);
    cudaFree(s.status); cudaFree(s.block_claims);
    if (s.stream) cudaStreamDestroy(s.stream);
    if (s.cstream) cudaStreamDestroy(s.cstream);
    for (int b = 0; b < 2; ++b) {
        if (s.evt[b]) cudaEventDestroy(s.evt[b]);
        if (s.evc[b]) cudaEventDestroy(s.evc[b]);
    }
    if (s.ev0) cudaEventDestroy(s.ev0);
    if (s.ev1) cudaEventDestroy(s.ev1);
    if (s.evk0) cudaEventDestroy(s.evk0);
    if (s.evk1) cudaEventDestroy(s.evk1);
    if (s.evq[0]) cudaEventDestroy(s.evq[0]);
    if (s.evq[1]) cudaEventDestroy(s.evq[1]);
    s = Slot();
}

static void free_graph(dfs_graph* g) {
    if (!g) return;
    int cur = 0;
    cudaGetDevice(&cur);
    cudaSetDevice(g->device);
    cudaFree(g->d_rp); cudaFree(g->d_col); cudaFree(g->d_leaf); cudaFree(g->d_rec); cudaFree(g->d_timeline); cudaFree(g->d_counts);
    for (int k = 0; k < kMaxSlots; ++k) free_slot(g->slots[k]);
    cudaSetDevice(cur);
    delete g;
}

// allocate scratch slot k for traversals on up to `n_warps` warps (slot 0: every warp of the
// device; the slots of a concurrent batch: their block share).  A slot that is too small is
// reallocated.
static int ensure_slot(dfs_graph* g, int k, int64_t n_warps) {
    Slot& s = g->slots[k];
    if (s.ready && s.n_warps_cap >= n_warps) return DFS_OK;
    if (s.ready) { cudaStreamSynchronize(s.stream ? s.stream : g->stream); free_slot(s); }
    const int64_t n = g->n;
    s.n_warps_cap = n_warps;
    s.tab_words = (size_t)n_warps << g->tab_log2;
    // pool: sum of live spans <= n, plus <= 4 partially used chunks per warp (reading S9)
    s.n_chunks = (uint32_t)(n / kChunk + 4 * n_warps + 16);
    const size_t nwords = (size_t)((n + 31) / 32);
    bool ok = true;
    auto A = [&](void** p, size_t bytes) { if (ok && cudaMalloc(p, bytes ? bytes : 16) != cudaSuccess) ok = false; };
    A((void**)&s.bitmap, 2 * nwords * sizeof(uint32_t));      // room for the {visited, leaf} layout
    A((void**)&s.cold_tb, (size_t)n_warps * sizeof(unsigned long long));
    A((void**)&s.tab, s.tab_words * sizeof(uint32_t));
    A((void**)&s.pool, (size_t)s.n_chunks * kChunk * sizeof(unsigned long long));
    A((void**)&s.consumed, (size_t)s.n_chunks * sizeof(uint32_t));
    A((void**)&s.next, (size_t)s.n_chunks * sizeof(uint32_t));
    A((void**)&s.block_cold, (size_t)g->max_blocks * sizeof(int));
    A((void**)&s.ctl, sizeof(Ctl));
    A((void**)&s.count2, 2 * sizeof(unsigned long long));
    A((void**)&s.status, sizeof(int));
    if (!ok) { cudaGetLastError(); free_slot(s); return DFS_ENOMEM; }
    if (cudaEventCreate(&s.ev0) != cudaSuccess || cudaEventCreate(&s.ev1) != cudaSuccess ||
        cudaEventCreate(&s.evk0) != cudaSuccess || cudaEventCreate(&s.evk1) != cudaSuccess ||
        cudaEventCreateWithFlags(&s.evq[0], cudaEventDisableTiming) != cudaSuccess ||
        cudaEventCreateWithFlags(&s.evq[1], cudaEventDisableTiming) != cudaSuccess ||
        (k > 0 && cudaStreamCreateWithFlags(&s.stream, cudaStreamNonBlocking) != cudaSuccess)) {
        cudaGetLastError(); free_slot(s); return DFS_ECUDA;
    }
    // all chunk slots empty; complete before any stream (the slot streams are non-blocking, so
    // they do not wait for work on the legacy default stream) can launch on this slot
    if (cudaMemset(s.tab, 0xFF, s.tab_words * sizeof(uint32_t)) != cudaSuccess ||
        cudaDeviceSynchronize() != cudaSuccess) {
        cudaGetLastError(); free_slot(s); return DFS_ECUDA;
    }
    s.ready = true;
    return DFS_OK;
}

extern "C" {

void dfs_options_default(dfs_options* o) {
    if (!o) return;
    std::memset(o, 0, sizeof(*o));
    o->blocks = 0;
    o->warps_per_block = 32;
    o->hot_cutoff = 1;           // paper: 32; B200 sweep: 1
    o->cold_cutoff = 1;          // paper: 64; B200 sweep: 1
    o->deterministic = 0;
    o->intra_steal = 1;
    o->inter_steal = 1;
    o->victim_policy = DFS_VICTIM_TWO_CHOICE;
    o->timeout_ms = 120000;
    o->seed = 0x5EEDu;
    o->collect_stats = 0;
    o->spill = 1;
    o->inter_any = 1;
    o->spill_idle = 32;
    o->backoff_max_ns = 2048;
    o->window = 0;
    o->pub_batch = 1;
    o->speculate = 2 | 4 | 8;    // + popped-entry speculation (A/B: road -4%, others neutral)
                                 // + early child window (A/B: road -2%, path -2.6%, det path -4%)
    o->steal_half = 1;
    o->concurrency = 0;
    o->ring_cap = 0;
    o->backoff_min_ns = 32;
    o->max_pool_chunks = 0;
    o->leaf_skip = 2;            // A/B on B200: rmat22 5.20 -> 4.33 ms (bulk), others neutral
    o->steal_tries = 8;          // A/B on B200: road 16.8 -> 15.4 ms, grid -15%, others neutral
    o->bulk_copy = 1;            // A/B on B200: rmat24 -11%, caterpillar -18%, road -2%, path -1%
    o->donate = 1;               // walker kernel: hand pushed entries to idle sibling walkers
    o->records = 0;              // walker kernel (>= 8 lanes): vertex records — measured slower
}

int dfs_last_error(void) { return g_last_error; }

const char* dfs_strerror(int code) {
    switch (code) {
        case DFS_OK: return "ok";
        case DFS_EINVAL: return "invalid argument or malformed CSR";
        case DFS_ENOMEM: return "out of device memory or stack-chunk pool exhausted";
        case DFS_ECUDA: return "CUDA runtime error";
        case DFS_EDEVICE: return "current device differs from the handle's device";
        case DFS_ETIMEOUT: return "traversal watchdog fired";
        case DFS_EINTERNAL: return "internal consistency check failed";
        default: return "unknown dfs_status";
    }
}

dfs_graph* dfs_graph_create(const int64_t* row_ptr, const int32_t* col_idx, int64_t n, int64_t m) {
    if (!row_ptr || n <= 0 || n > (int64_t)0x7FFFFFFC || m < 0 || m >= ((int64_t)1 << 32) ||
        (m > 0 && !col_idx)) {
        fail(DFS_EINVAL);
        return nullptr;
    }
    dfs_graph* g = new (std::nothrow) dfs_graph();
    if (!g) { fail(DFS_ENOMEM); return nullptr; }
    if (cudaGetDevice(&g->device) != cudaSuccess) { cudaGetLastError(); delete g; fail(DFS_ECUDA); return nullptr; }
    g->n = n; g->m = m;
    cudaDeviceProp prop;
    if (cudaGetDeviceProperties(&prop, g->device) != cudaSuccess) { cudaGetLastError(); delete g; fail(DFS_ECUDA); return nullptr; }
    g->sms = prop.multiProcessorCount;
    const size_t sm32 = smem_bytes(32);
    bool attr_ok = true;
    for (int kf = 0; kf < kNumKernels; ++kf) {
        if (cudaFuncSetAttribute(kernel_table()[kf], cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm32) != cudaSuccess)
            attr_ok = false;
    }
    for (int kf = 0; kf < kNumWalkerKernels; ++kf) {
        const int lanes = walker_lanes_of(kf);
        if (cudaFuncSetAttribute(walker_table()[kf], cudaFuncAttributeMaxDynamicSharedMemorySize,
                                 (int)walker_smem_bytes(32, lanes)) != cudaSuccess)
            attr_ok = false;
    }
    if (!attr_ok) { cudaGetLastError(); delete g; fail(DFS_ECUDA); return nullptr; }
    int per_sm = 0;
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, dfs_persistent_kernel<kRing, 4, DFS_WMAX_BIG, false, false, false>, 32 * DFS_WMAX_BIG, sm32) !=
            cudaSuccess || per_sm < 1) {
        cudaGetLastError(); per_sm = 1;
    }
    g->max_blocks = g->sms * per_sm;
    // chunk table: 2^tab_log2 >= (max live span + 2 chunks + flush batch) / chunk  (reading S9)
    const int64_t need = (n + 2 * (int64_t)kChunk + kRing) / kChunk + 2;
    g->tab_log2 = 2;
    while (((int64_t)1 << g->tab_log2) < need) ++g->tab_log2;

    if (cudaMalloc(&g->d_rp, (size_t)(n + 1) * sizeof(uint32_t)) != cudaSuccess ||
        cudaMalloc(&g->d_leaf, (size_t)((n + 31) / 32) * sizeof(uint32_t)) != cudaSuccess ||
        cudaMalloc(&g->d_col, (size_t)(m + 8) * sizeof(int32_t)) != cudaSuccess) {   // padded for 128-bit loads
        cudaGetLastError(); free_graph(g); fail(DFS_ENOMEM); return nullptr;
    }
    const int rc = ensure_slot(g, 0, (int64_t)g->max_blocks * kMaxWarps);
    if (rc != DFS_OK) { free_graph(g); fail(rc); return nullptr; }

    // ---- copy + validate + narrow (step a1) ----
    // Both arrays are staged on the device (host inputs are copied as they are; device inputs are
    // used in place) and validated by kernels: no O(n) host loop on the create path.
    int* d_bad = nullptr;
    int64_t* d_rp64 = nullptr;                 // staging copy of a host row_ptr
    const bool rp_dev = is_device_ptr(row_ptr);
    bool ok = cudaMalloc(&d_bad, 2 * sizeof(int)) == cudaSuccess &&
              (rp_dev || cudaMalloc(&d_rp64, (size_t)(n + 1) * sizeof(int64_t)) == cudaSuccess);
    if (!ok) {
        cudaGetLastError(); cudaFree(d_bad); cudaFree(d_rp64);
        free_graph(g); fail(DFS_ENOMEM); return nullptr;
    }
    cudaMemset(d_bad, 0, 2 * sizeof(int));
    const int64_t* rp_src = row_ptr;
    if (!rp_dev) {
        cudaMemcpy(d_rp64, row_ptr, (size_t)(n + 1) * sizeof(int64_t), cudaMemcpyHostToDevice);
        rp_src = d_rp64;
    }
    {
        const int blocks = (int)std::min<int64_t>((n + 256) / 256 + 1, 65535);
        dfs_validate_rowptr_kernel<<<blocks, 256>>>(rp_src, g->d_rp, n, m, d_bad);
        g->launches++;
    }
    if (m > 0) {
        cudaMemcpy(g->d_col, col_idx, (size_t)m * sizeof(int32_t), cudaMemcpyDefault);
        const int blocks = (int)std::min<int64_t>((m + 255) / 256, 65535);
        dfs_validate_col_kernel<<<blocks, 256>>>(g->d_col, m, n, d_bad);
        g->launches++;
    }
    int hbad2[2] = {0, 0};
    cudaMemcpy(hbad2, d_bad, 2 * sizeof(int), cudaMemcpyDeviceToHost);
    const int hbad = hbad2[0];
    g->max_degree = hbad2[1];
    cudaFree(d_bad);
    cudaFree(d_rp64);
    if (cudaGetLastError() != cudaSuccess) { free_graph(g); fail(DFS_ECUDA); return nullptr; }
    if (hbad) { free_graph(g); fail(DFS_EINVAL); return nullptr; }
    cudaMemset(g->d_col + m, 0xFF, 8 * sizeof(int32_t));            // padding (never a valid position)
    {
        uint32_t* d_inn = nullptr;                                    // unique in-neighbours (temporary)
        if (cudaMalloc(&d_inn, (size_t)n * sizeof(uint32_t)) != cudaSuccess) {
            cudaGetLastError(); free_graph(g); fail(DFS_ENOMEM); return nullptr;
        }
        cudaMemset(d_inn, 0xFF, (size_t)n * sizeof(uint32_t));      // kInUnset
        dfs_leaf_in_kernel<<<(int)std::min<int64_t>((n + 255) / 256, 65535), 256>>>(g->d_rp, g->d_col, (uint32_t)n, d_inn);
        const int blocks = (int)std::min<int64_t>(((n + 31) / 32 + 255) / 256 + 1, 65535);
        dfs_leaf_init_kernel<<<blocks, 256>>>(g->d_rp, g->d_col, d_inn, (uint32_t)n, g->d_leaf);
        g->launches += 2;
        cudaFree(d_inn);
    }
    if (cudaDeviceSynchronize() != cudaSuccess) { cudaGetLastError(); free_graph(g); fail(DFS_ECUDA); return nullptr; }
    return g;
}

void dfs_graph_destroy(dfs_graph* g) { free_graph(g); }

int dfs_set_stream(dfs_graph* g, void* s) {
    if (!g) return fail(DFS_EINVAL);
    g->stream = (cudaStream_t)s;
    return DFS_OK;
}

int dfs_graph_info(const dfs_graph* g, int64_t* n, int64_t* m, int32_t* device) {
    if (!g) return fail(DFS_EINVAL);
    if (n) *n = g->n;
    if (m) *m = g->m;
    if (device) *device = g->device;
    return DFS_OK;
}

int64_t dfs_launch_count(const dfs_graph* g) { return g ? g->launches : -1; }

int dfs_debug_timeline(dfs_graph* g, uint32_t len, uint32_t dt_ns, uint32_t* out) {
    if (!g || (len > 0 && dt_ns == 0)) return fail(DFS_EINVAL);
    if (len == 0) {                       // disable
        cudaFree(g->d_timeline);
        g->d_timeline = nullptr; g->timeline_len = 0;
        return DFS_OK;
    }
    if (g->d_timeline && g->timeline_len == len && out == nullptr) return DFS_OK;
    if (!g->d_timeline || g->timeline_len != len) {
        cudaFree(g->d_timeline);
        g->d_timeline = nullptr;
        if (cudaMalloc(&g->d_timeline, (size_t)len * sizeof(uint32_t)) != cudaSuccess) {
            cudaGetLastError();
            g->timeline_len = 0;
            return fail(DFS_ENOMEM);
        }
        cudaMemset(g->d_timeline, 0, (size_t)len * sizeof(uint32_t));
        g->timeline_len = len; g->timeline_dt_ns = dt_ns;
        return DFS_OK;
    }
    // copy out the samples of the last run, then clear
    if (cudaMemcpy(out, g->d_timeline, (size_t)len * sizeof(uint32_t), cudaMemcpyDeviceToHost) != cudaSuccess) {
        cudaGetLastError();
        return fail(DFS_ECUDA);
    }
    cudaMemset(g->d_timeline, 0, (size_t)len * sizeof(uint32_t));
    return DFS_OK;
}

}  // extern "C"

// ------------------------------------------------------------------------------------------
// one traversal on slot `sl`, stream-ordered on `s` (no synchronisation)
// ------------------------------------------------------------------------------------------
// stack-script mode of the walker STATS kernel (dfs_debug_stack_script)
struct ScriptArgs {
    const int32_t* d_script = nullptr;
    int n_ops = 0;
    int32_t* d_out = nullptr;
    int out_len = 0;
};

static int launch_one(dfs_graph* g, Slot& sl, cudaStream_t s, int32_t root, int32_t* d_out,
                      const dfs_options& o, int blocks, int warps, bool timed, bool cooperative,
                      const ScriptArgs* script = nullptr) {
    const uint32_t nwords = (uint32_t)((g->n + 31) / 32);
    const int rblocks = (int)std::min<int64_t>((std::max<int64_t>(nwords, sl.tab_dirty ? (int64_t)sl.tab_words : 0) + 255) / 256 + 1,
                                               (int64_t)g->sms * 8);
    const uint32_t bstride = 2u;                              // {visited, leaf} pairs (both windows)
    sl.bstride = bstride;
    const int wl = o.walker_lanes;                            // resolved: 32 = warp kernel
    const int owners = blocks * warps * (wl == 32 ? 1 : 32 / wl);   // stack owners (warps or walkers)
    if (owners > sl.n_warps_cap) return DFS_EINTERNAL;
    dfs_reset_kernel<<<rblocks, 256, 0, s>>>(sl.bitmap, nwords, bstride, o.leaf_skip >= 2 ? g->d_leaf : nullptr,
                                            sl.cold_tb, (uint32_t)owners,
                                            sl.block_cold, (uint32_t)blocks, sl.ctl, d_out, root,
                                            sl.tab, sl.tab_dirty ? sl.tab_words : 0);
    g->launches++;
    sl.tab_dirty = false;

    KParams P = {};
    P.rp = g->d_rp; P.col = g->d_col; P.bitmap = sl.bitmap; P.parent = d_out;
    P.cold_tb = sl.cold_tb; P.chunk_tab = sl.tab; P.pool = sl.pool;
    P.chunk_consumed = sl.consumed; P.chunk_next = sl.next; P.block_cold = sl.block_cold;
    P.ctl = sl.ctl;
    P.n = (uint32_t)g->n; P.m = (uint32_t)g->m; P.root = root; P.tab_log2 = g->tab_log2;
    P.n_chunks = (o.max_pool_chunks > 0 && (uint32_t)o.max_pool_chunks < sl.n_chunks) ? (uint32_t)o.max_pool_chunks
                                                                                      : sl.n_chunks;
    P.hot_cutoff = o.hot_cutoff; P.cold_cutoff = o.cold_cutoff;
    P.intra = o.intra_steal; P.inter = o.inter_steal; P.policy = o.victim_policy;
    P.collect_stats = o.collect_stats;
    P.spill = o.spill;
    P.spill_idle = o.spill_idle > 0 ? o.spill_idle : 32;
    P.inter_any = o.inter_any;
    P.backoff_max_ns = o.backoff_max_ns > 0 ? (unsigned)o.backoff_max_ns : 2048u;
    P.backoff_min_ns = o.backoff_min_ns > 0 ? (unsigned)o.backoff_min_ns : 32u;
    P.pub_batch = o.pub_batch > 0 ? (uint32_t)o.pub_batch : 1u;
    P.speculate = o.speculate;
    P.steal_half = o.steal_half;
    P.leaf_skip = o.leaf_skip ? 1 : 0;
    P.ring_cap = (o.ring_cap > 0 && o.ring_cap < kRing) ? (uint32_t)o.ring_cap : (uint32_t)kRing;
    P.block_claims = sl.block_claims;
    P.cluster_late = o.cluster_late;
    P.steal_tries = o.steal_tries > 0 ? o.steal_tries : 1;
    P.bulk_copy = o.bulk_copy;
    P.period_mask = (uint32_t)(o.spill_period > 0 ? o.spill_period : 32) - 1u;
    P.steal_period_mask = (uint32_t)(o.steal_period > 0 ? o.steal_period : 1) - 1u;
    P.donate = o.donate;
    const bool tl = g->d_timeline && &sl == &g->slots[0];
    P.timeline = tl ? g->d_timeline : nullptr;
    P.timeline_len = tl ? (g->timeline_len / 3u) * 2u : 0;   // kernel: three regions of len/3
    P.timeline_dt_ns = tl ? g->timeline_dt_ns : 1;
    P.timeout_ns = (unsigned long long)o.timeout_ms * 1000000ull;
    P.seed = o.seed;
    if (script) {
        P.script = script->d_script; P.script_len = script->n_ops;
        P.script_out = script->d_out; P.script_out_len = script->out_len;
    }
    void* args[] = {(void*)&P};
    const int cl = o.cluster > 1 ? o.cluster : 1;
    // the cluster build has no bulk variant: cluster >= 1 takes precedence over bulk_copy
    P.rec = g->d_rec;
    const bool rec = wl != 32 && wl >= 8 && o.records && g->d_rec;
    const void* kfn = wl != 32 ? walker_table()[walker_index(wl, rec) + (o.collect_stats ? 1 : 0)]
                               : kernel_table()[(o.cluster >= 1 ? 8 : o.bulk_copy ? 16 : 0) + (o.window == 128 ? 4 : 0) +
                                                (warps <= 16 ? 2 : 0) + (o.collect_stats ? 1 : 0)];
    if (timed) cudaEventRecord(sl.evk0, s);
    cudaError_t e;
    // launch attributes: cooperative (single traversals), cluster dimension (cluster tier,
    // blocks is a multiple of cl and at most cl x the co-resident cluster count,
    // resolve_options), and an L2 access-policy window that keeps row_ptr persisting in L2
    // (l2_persist_mb; the window's hits are persisting, its misses streaming)
    cudaLaunchConfig_t cfg = {};
    cudaLaunchAttribute at[3];
    int na = 0;
    at[na].id = cudaLaunchAttributeCooperative;
    at[na].val.cooperative = cooperative ? 1 : 0;
    ++na;
    if (o.cluster >= 1) {
        at[na].id = cudaLaunchAttributeClusterDimension;
        at[na].val.clusterDim.x = (unsigned)cl; at[na].val.clusterDim.y = 1; at[na].val.clusterDim.z = 1;
        ++na;
    }
    if (o.l2_persist_mb > 0 && g->persist_bytes > 0) {
        const size_t rp_bytes = (size_t)(g->n + 1) * sizeof(uint32_t);
        const size_t win = std::min(rp_bytes, g->max_window_bytes);
        at[na].id = cudaLaunchAttributeAccessPolicyWindow;
        at[na].val.accessPolicyWindow.base_ptr = (void*)g->d_rp;
        at[na].val.accessPolicyWindow.num_bytes = win;
        at[na].val.accessPolicyWindow.hitRatio = std::min(1.0f, (float)g->persist_bytes / (float)win);
        at[na].val.accessPolicyWindow.hitProp = cudaAccessPropertyPersisting;
        at[na].val.accessPolicyWindow.missProp = cudaAccessPropertyStreaming;
        ++na;
    }
    cfg.gridDim = dim3(blocks); cfg.blockDim = dim3(32 * warps);
    cfg.dynamicSmemBytes = wl != 32 ? walker_smem_bytes(warps, wl) : smem_bytes(warps); cfg.stream = s;
    cfg.attrs = at; cfg.numAttrs = na;
    // concurrent batch slots launch non-cooperatively: co-residency is not required for progress —
    // a block that starts late finds the traversal done or steals the remaining work
    e = cudaLaunchKernelExC(&cfg, kfn, args);
    if (e != cudaSuccess) { cudaGetLastError(); return DFS_ECUDA; }
    if (timed) cudaEventRecord(sl.evk1, s);
    g->launches++;
    const int fblocks = (int)std::min<int64_t>((g->n + 255) / 256, (int64_t)g->sms * 16);
    dfs_finalize_kernel<<<fblocks, 256, 0, s>>>(sl.bitmap, bstride, d_out, (uint32_t)g->n, sl.ctl, sl.status);
    g->launches++;
    return DFS_OK;
}

// co-resident clusters of `cl` CTAs of the persistent kernel (cudaOccupancyMaxActiveClusters;
// cached per cluster size)
static int max_clusters(dfs_graph* g, int cl, int warps, int window, bool stats) {
    int idx = 0;
    while ((1 << idx) < cl) ++idx;
    if (g->max_clusters[idx] > 0) return g->max_clusters[idx];
    (void)warps;   // the 32-warp instantiation bounds the smaller blocks' footprint
    const void* kfn = kernel_table()[8 + (window == 128 ? 4 : 0) + (stats ? 1 : 0)];
    cudaLaunchConfig_t cfg = {};
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeClusterDimension;
    at[0].val.clusterDim.x = (unsigned)cl; at[0].val.clusterDim.y = 1; at[0].val.clusterDim.z = 1;
    cfg.gridDim = dim3((unsigned)(g->max_blocks / cl * cl)); cfg.blockDim = dim3(32 * DFS_WMAX_BIG);
    cfg.dynamicSmemBytes = smem_bytes(32); cfg.attrs = at; cfg.numAttrs = 1;
    int n = 0;
    if (cudaOccupancyMaxActiveClusters(&n, kfn, &cfg) != cudaSuccess) { cudaGetLastError(); n = 0; }
    g->max_clusters[idx] = n;
    return n;
}

static int resolve_options(dfs_graph* g, const dfs_options* in, int num_roots, dfs_options& o,
                           int& blocks, int& warps, int& conc) {
    dfs_options_default(&o);
    if (in) o = *in;
    if (o.hot_cutoff == 0) o.hot_cutoff = 1;
    if (o.cold_cutoff == 0) o.cold_cutoff = 1;
    if (o.timeout_ms <= 0) o.timeout_ms = 120000;
    // thresholds >= 1; h_s = max(1, hot_cutoff/2) <= 32 (one lane per entry);
    // c_s = max(1, cold_cutoff/2) <= 64
    if (o.hot_cutoff < 1 || o.hot_cutoff / 2 > 32) return DFS_EINVAL;
    if (o.cold_cutoff < 1 || o.cold_cutoff / 2 > 64) return DFS_EINVAL;
    if (o.victim_policy != 0 && o.victim_policy != 1) return DFS_EINVAL;
    if (o.reserved0 != 0) return DFS_EINVAL;
    if (o.spill_period < 0 || o.spill_period > 1024 || (o.spill_period & (o.spill_period - 1))) return DFS_EINVAL;
    if (o.cluster < 0 || o.cluster > 8 || (o.cluster > 1 && (o.cluster & (o.cluster - 1)))) return DFS_EINVAL;
    if (o.walker_lanes != 0 && o.walker_lanes != 32 && !valid_walker_lanes(o.walker_lanes)) return DFS_EINVAL;
    if (o.steal_period < 0 || o.steal_period > 1024 || (o.steal_period & (o.steal_period - 1))) return DFS_EINVAL;
    const bool window_auto = o.window == 0;
    if (o.window == 0) o.window = (g->n > 0 && g->m >= 8 * g->n) ? 128 : 32;   // wide windows for dense lists
    // kernel (auto, measured on B200 — DESIGN.md §5): sub-warp walkers of 4 lanes where work is
    // plentiful on low-degree graphs — batches (several traversals in flight) and path-like
    // graphs (avg degree < 2.2: long unbranched runs, so every steal carries a long path); the
    // warp kernel otherwise (road single roots: small stolen subtrees, walkers 1.5x slower;
    // long lists / hubs: a 4-lane window needs 8x the steps of the 32-wide one)
    if (o.walker_lanes == 0) {
        const bool low_degree = g->m <= 4 * g->n && g->max_degree <= 16;
        const bool batch = num_roots > 1 && o.concurrency != 1;
        const bool pathlike = 10 * g->m < 22 * g->n;
        o.walker_lanes = (low_degree && (batch || pathlike)) ? 4 : 32;
    }
    if (o.steal_period == 0) o.steal_period = 16;   // walker kernel (A/B on B200: batch -13%, road -27%)
    if (o.deterministic || o.cluster >= 1 || (o.window == 128 && !window_auto)) o.walker_lanes = 32;
    if (o.walker_lanes != 32) o.window = 32;
    if (o.records && o.walker_lanes != 32 && o.walker_lanes >= 8 && !g->d_rec) {
        // vertex records (8 words per vertex), built once per handle on first use
        if (cudaMalloc(&g->d_rec, (size_t)g->n * 32) != cudaSuccess) { cudaGetLastError(); g->d_rec = nullptr; return DFS_ENOMEM; }
        const int blocks_r = (int)std::min<int64_t>((g->n + 255) / 256, (int64_t)g->sms * 16);
        dfs_records_kernel<<<blocks_r, 256>>>(g->d_rp, g->d_col, (uint32_t)g->n, reinterpret_cast<uint4*>(g->d_rec));
        g->launches++;
        if (cudaDeviceSynchronize() != cudaSuccess) { cudaGetLastError(); cudaFree(g->d_rec); g->d_rec = nullptr; return DFS_ECUDA; }
    }
    if (o.window != 32 && o.window != 128) return DFS_EINVAL;
    if (o.concurrency < 0 || o.concurrency > kMaxSlots) return DFS_EINVAL;
    warps = o.warps_per_block <= 0 ? 32 : o.warps_per_block;
    if (warps > 32) return DFS_EINVAL;
    // the walker kernel is compiled for CTAs of up to kWalkerMaxWarps warps (DFS_WALKER_LB threads:
    // 28 warps x 72 registers measured faster than 32 x 64 — fewer register rematerialisations;
    // DESIGN.md §5); auto and larger requests get that
    if (o.walker_lanes != 32 && warps > kWalkerMaxWarps) warps = kWalkerMaxWarps;
    if (o.walker_lanes == 32 && warps > DFS_WMAX_BIG) warps = DFS_WMAX_BIG;
    conc = o.concurrency == 0 ? 8 : o.concurrency;       // auto: 8 in flight (B200 sweep)
    if (o.deterministic) conc = 1;
    if (conc > num_roots) conc = std::max(1, num_roots);
    const int share = std::max(1, g->max_blocks / conc);
    blocks = o.blocks <= 0 ? share : o.blocks;
    if (blocks > g->max_blocks || (conc > 1 && blocks * conc > g->max_blocks)) return DFS_EINVAL;
    if (o.deterministic) { blocks = 1; warps = 1; o.intra_steal = 0; o.inter_steal = 0; o.cluster = 0; }
    if (o.l2_persist_mb < -1) return DFS_EINVAL;
    const bool persist_auto = o.l2_persist_mb == 0;
    if (persist_auto) o.l2_persist_mb = o.window == 128 ? 64 : -1;   // auto (A/B: rmat24 -4.8%)
    if (o.l2_persist_mb > 0) {
        // device-wide persisting-L2 set-aside (capped by the device); done once per handle.
        // Where it cannot be granted (MIG: max 0; MPS: the limit is not settable) an explicit
        // request fails with DFS_ECUDA and the auto setting quietly runs without it.
        const size_t want = (size_t)o.l2_persist_mb << 20;
        if (g->persist_req != want) {
            int maxp = 0, maxw = 0;
            cudaDeviceGetAttribute(&maxp, cudaDevAttrMaxPersistingL2CacheSize, g->device);
            cudaDeviceGetAttribute(&maxw, cudaDevAttrMaxAccessPolicyWindowSize, g->device);
            cudaGetLastError();
            const size_t bytes = std::min(want, (size_t)std::max(maxp, 0));
            if (bytes == 0 || maxw <= 0 || cudaDeviceSetLimit(cudaLimitPersistingL2CacheSize, bytes) != cudaSuccess) {
                cudaGetLastError();
                if (!persist_auto) return DFS_ECUDA;
                o.l2_persist_mb = -1;
            } else {
                g->persist_req = want;
                g->persist_bytes = bytes;                 // granted (hitRatio uses this)
                g->max_window_bytes = (size_t)maxw;
            }
        }
    }
    if (o.cluster > 1) {
        // whole clusters only, no more than can be co-resident
        const int maxc = max_clusters(g, o.cluster, warps, o.window, o.collect_stats != 0);
        if (maxc < 1) return DFS_EINVAL;
        blocks = std::min(blocks, maxc * o.cluster) / o.cluster * o.cluster;
        if (blocks < o.cluster) return DFS_EINVAL;
    }
    return DFS_OK;
}

static int check_device(const dfs_graph* g) {
    int cur = -1;
    if (cudaGetDevice(&cur) != cudaSuccess) { cudaGetLastError(); return DFS_ECUDA; }
    return cur == g->device ? DFS_OK : DFS_EDEVICE;
}

static void fill_stats(dfs_stats* stats, const dfs_options& o, int blocks, int warps, float total_ms, float trav_ms,
                       int64_t nv, int64_t mv, const unsigned long long* counters) {
    int64_t* keep = stats->root_counts;
    std::memset(stats, 0, sizeof(*stats));
    stats->root_counts = keep;
    stats->kernel_ms = total_ms;
    stats->traversal_ms = trav_ms;
    stats->blocks = blocks; stats->warps_per_block = warps;
    stats->n_visited = nv; stats->m_visited = mv;
    stats->claims = (int64_t)counters[kCntClaims];
    stats->failed_claims = (int64_t)counters[kCntFailedClaims];
    stats->flushes = (int64_t)counters[kCntFlushes];
    stats->refills = (int64_t)counters[kCntRefills];
    stats->intra_steals = (int64_t)counters[kCntIntraSteals];
    stats->inter_steals = (int64_t)counters[kCntInterSteals];
    stats->steal_attempts = (int64_t)counters[kCntStealAttempts];
    stats->chunks_allocated = (int64_t)counters[kCntChunks];
    stats->windows = (int64_t)counters[kCntWindows];
    stats->idle_ns = (int64_t)counters[kCntIdleNs];
    stats->inter_scans = (int64_t)counters[kCntInterScans];
    stats->spills = (int64_t)counters[kCntSpills];
    stats->cyc_window = (int64_t)counters[kCntTWin];
    stats->cyc_probe = (int64_t)counters[kCntTProbe];
    stats->cyc_claim = (int64_t)counters[kCntTClaim];
    stats->cyc_tail = (int64_t)counters[kCntTTail];
    stats->cyc_outside = (int64_t)counters[kCntTOut];
    stats->cluster_steals = (int64_t)counters[kCntClusterSteals];
    stats->pops = (int64_t)counters[kCntPops];
    stats->dead_pops = (int64_t)counters[kCntDeadPops];
    stats->donations = (int64_t)counters[kCntDonations];
    stats->walker_lanes = o.walker_lanes;
    stats->window = o.window;
}

// per-root count buffer (2 x u64 per root) for stats calls
static int ensure_counts(dfs_graph* g, int32_t k) {
    if (g->counts_cap >= k) return DFS_OK;
    cudaFree(g->d_counts);
    g->d_counts = nullptr; g->counts_cap = 0;
    if (cudaMalloc(&g->d_counts, (size_t)k * 2 * sizeof(unsigned long long)) != cudaSuccess) {
        cudaGetLastError();
        return DFS_ENOMEM;
    }
    g->counts_cap = k;
    return DFS_OK;
}

// copy the per-root counts out (and total them)
static int finish_counts(dfs_graph* g, int32_t k, dfs_stats* stats, int64_t& nv, int64_t& mv) {
    std::vector<unsigned long long> h((size_t)k * 2);
    if (cudaMemcpy(h.data(), g->d_counts, h.size() * sizeof(unsigned long long), cudaMemcpyDeviceToHost) != cudaSuccess) {
        cudaGetLastError();
        return DFS_ECUDA;
    }
    nv = mv = 0;
    for (int32_t q = 0; q < k; ++q) {
        nv += (int64_t)h[2 * q]; mv += (int64_t)h[2 * q + 1];
        if (stats->root_counts) { stats->root_counts[2 * q] = (int64_t)h[2 * q]; stats->root_counts[2 * q + 1] = (int64_t)h[2 * q + 1]; }
    }
    return DFS_OK;
}

// sequential path: one slot, cooperative launch, per-traversal status check and stats
static int run_sequential(dfs_graph* g, const int32_t* roots, int32_t k, int32_t* out, bool out_dev,
                          const dfs_options& o, int blocks, int warps, dfs_stats* stats) {
    Slot& sl = g->slots[0];
    {
        const int64_t owners = (int64_t)blocks * warps * (o.walker_lanes == 32 ? 1 : 32 / o.walker_lanes);
        const int rc = ensure_slot(g, 0, std::max<int64_t>(owners, (int64_t)g->max_blocks * kMaxWarps));
        if (rc != DFS_OK) return fail(rc);
    }
    if (!out_dev && !sl.parent) {
        if (cudaMalloc(&sl.parent, (size_t)g->n * sizeof(int32_t)) != cudaSuccess) {
            cudaGetLastError();
            return fail(DFS_ENOMEM);
        }
    }
    unsigned long long counters[kNumWCounters] = {0};
    float total_ms = 0.f, trav_ms = 0.f;
    int64_t nv = 0, mv = 0;
    cudaStream_t s = g->stream;
    if (stats) {
        const int rc = ensure_counts(g, k);
        if (rc != DFS_OK) return fail(rc);
        cudaMemsetAsync(g->d_counts, 0, (size_t)k * 2 * sizeof(unsigned long long), s);
    }
    const bool want_blocks = stats && stats->block_claims;
    if (want_blocks) {
        if (!sl.block_claims && cudaMalloc(&sl.block_claims, (size_t)g->max_blocks * sizeof(unsigned long long)) != cudaSuccess) {
            cudaGetLastError();
            return fail(DFS_ENOMEM);
        }
        cudaMemsetAsync(sl.block_claims, 0, (size_t)g->max_blocks * sizeof(unsigned long long), s);
    } else if (sl.block_claims) {
        cudaFree(sl.block_claims);           // launch_one passes it to the kernel when non-null
        sl.block_claims = nullptr;
    }
    for (int32_t q = 0; q < k; ++q) {
        int32_t* d_out = out_dev ? out + (size_t)q * g->n : sl.parent;
        cudaMemsetAsync(sl.status, 0, sizeof(int), s);
        cudaEventRecord(sl.ev0, s);
        int rc = launch_one(g, sl, s, roots[q], d_out, o, blocks, warps, stats != nullptr, true);
        if (rc != DFS_OK) return fail(rc);
        cudaEventRecord(sl.ev1, s);
        if (stats) {
            dfs_count_kernel<<<g->sms * 4, 256, 0, s>>>(sl.bitmap, sl.bstride, g->d_rp, (uint32_t)g->n, g->d_counts + 2 * q);
            g->launches++;
        }
        Ctl h;
        if (cudaMemcpyAsync(&h, sl.ctl, sizeof(Ctl), cudaMemcpyDeviceToHost, s) != cudaSuccess ||
            cudaStreamSynchronize(s) != cudaSuccess) {
            cudaGetLastError();
            return fail(DFS_ECUDA);
        }
        if (h.status != 0) { sl.tab_dirty = true; return fail(h.status); }
        if (!out_dev) {
            if (cudaMemcpyAsync(out + (size_t)q * g->n, sl.parent, (size_t)g->n * sizeof(int32_t),
                                cudaMemcpyDeviceToHost, s) != cudaSuccess) {
                cudaGetLastError();
                return fail(DFS_ECUDA);
            }
        }
        if (stats) {
            float ms = 0.f, kms = 0.f;
            cudaEventElapsedTime(&ms, sl.ev0, sl.ev1);
            cudaEventElapsedTime(&kms, sl.evk0, sl.evk1);
            total_ms += ms;
            trav_ms += kms;
            for (int c = 0; c < kNumWCounters; ++c) counters[c] += h.counters[c];
        }
    }
    if (cudaStreamSynchronize(s) != cudaSuccess) { cudaGetLastError(); return fail(DFS_ECUDA); }
    if (stats) {
        const int rc = finish_counts(g, k, stats, nv, mv);
        if (rc != DFS_OK) return fail(rc);
        int64_t* bc = stats->block_claims;
        fill_stats(stats, o, blocks, warps, total_ms, trav_ms, nv, mv, counters);
        stats->block_claims = bc;
        if (bc) {
            std::vector<unsigned long long> h((size_t)blocks);
            cudaMemcpy(h.data(), sl.block_claims, h.size() * sizeof(unsigned long long), cudaMemcpyDeviceToHost);
            for (int b = 0; b < blocks; ++b) bc[b] = (int64_t)h[(size_t)b];
        }
    }
    return DFS_OK;
}

// concurrent path (§8(f)-2): `conc` slots, each on its own stream and a 1/conc share of the
// SMs, take roots round-robin; no host synchronisation until the whole batch is issued
static int run_concurrent(dfs_graph* g, const int32_t* roots, int32_t k, int32_t* out, bool out_dev,
                          const dfs_options& o, int blocks, int warps, int conc, dfs_stats* stats,
                          int extra = 0) {
    for (int c = 0; c < conc; ++c) {
        Slot& sl = g->slots[c];
        if (sl.block_claims) { cudaFree(sl.block_claims); sl.block_claims = nullptr; }
        if (!out_dev) {
            // host rows: two device row buffers and a copy stream per slot, so the copy of one
            // row overlaps the slot's next traversal (double buffering)
            if (!sl.parent && cudaMalloc(&sl.parent, (size_t)g->n * sizeof(int32_t)) != cudaSuccess) {
                cudaGetLastError();
                return fail(DFS_ENOMEM);
            }
            if (!sl.parent2 && cudaMalloc(&sl.parent2, (size_t)g->n * sizeof(int32_t)) != cudaSuccess) {
                cudaGetLastError();                       // one buffer: copies do not overlap
                sl.parent2 = nullptr;
            }
            for (int b = 0; b < 2; ++b) {
                if ((!sl.evt[b] && cudaEventCreateWithFlags(&sl.evt[b], cudaEventDisableTiming) != cudaSuccess) ||
                    (!sl.evc[b] && cudaEventCreateWithFlags(&sl.evc[b], cudaEventDisableTiming) != cudaSuccess)) {
                    cudaGetLastError(); return fail(DFS_ECUDA);
                }
            }
            if (!sl.cstream && cudaStreamCreateWithFlags(&sl.cstream, cudaStreamNonBlocking) != cudaSuccess) {
                cudaGetLastError(); sl.cstream = nullptr; return fail(DFS_ECUDA);
            }
            // the copy stream starts after the handle's stream like the slot stream (below)
        }
    }
    // fork: every slot stream waits for the handle's stream; slot 0 gets its own stream too
    cudaStream_t base = g->stream;
    if (stats) {
        const int rc = ensure_counts(g, k);
        if (rc != DFS_OK) return fail(rc);
        cudaMemsetAsync(g->d_counts, 0, (size_t)k * 2 * sizeof(unsigned long long), base);
    }
    if (!g->slots[0].stream && cudaStreamCreateWithFlags(&g->slots[0].stream, cudaStreamNonBlocking) != cudaSuccess) {
        cudaGetLastError();
        return fail(DFS_ECUDA);
    }
    Slot& s0 = g->slots[0];
    cudaEventRecord(s0.ev0, base);
    for (int c = 0; c < conc; ++c) {
        Slot& sl = g->slots[c];
        cudaStreamWaitEvent(sl.stream, s0.ev0, 0);
        if (!out_dev) cudaStreamWaitEvent(sl.cstream, s0.ev0, 0);
        cudaMemsetAsync(sl.status, 0, sizeof(int), sl.stream);
        cudaMemsetAsync(sl.count2, 0, 2 * sizeof(unsigned long long), sl.stream);
    }
    // dynamic issue: a root goes to whichever slot has room in its two-deep queue (the traversal
    // issued two earlier on it has completed), so slots that draw short traversals take more
    // roots and the batch does not end waiting for the slot that drew the long ones
    for (int c = 0; c < conc; ++c) g->slots[c].issued = 0;
    int32_t q = 0;
    int rr = 0;                                          // round-robin start of the next sweep
    while (q < k) {
        bool any = false;
        for (int t = 0; t < conc && q < k; ++t) {
            const int c = (rr + t) % conc;
            Slot& sl = g->slots[c];
            if (sl.issued >= 2) {
                const cudaError_t qe = cudaEventQuery(sl.evq[sl.issued & 1]);
                if (qe == cudaErrorNotReady) continue;
                if (qe != cudaSuccess) { cudaGetLastError(); return fail(DFS_ECUDA); }
            }
            const int nbuf = sl.parent2 ? 2 : 1;
            const int buf = (int)(sl.issued % nbuf);
            int32_t* d_out = out_dev ? out + (size_t)q * g->n : (buf ? sl.parent2 : sl.parent);
            // host rows: the buffer's previous row must have left for the host first
            if (!out_dev && sl.issued >= nbuf) cudaStreamWaitEvent(sl.stream, sl.evc[buf], 0);
            // the first `extra` slots take one more block: all SMs in use (148 = 4 x 19 + 4 x 18)
            int rc = launch_one(g, sl, sl.stream, roots[q], d_out, o, blocks + (c < extra ? 1 : 0), warps, false, false);
            if (rc != DFS_OK) return fail(rc);
            if (stats) {
                dfs_count_kernel<<<g->sms * 4, 256, 0, sl.stream>>>(sl.bitmap, sl.bstride, g->d_rp, (uint32_t)g->n, g->d_counts + 2 * q);
                g->launches++;
            }
            if (!out_dev) {
                // the row's copy runs on the slot's copy stream, overlapping its next traversal
                cudaEventRecord(sl.evt[buf], sl.stream);
                cudaStreamWaitEvent(sl.cstream, sl.evt[buf], 0);
                if (cudaMemcpyAsync(out + (size_t)q * g->n, d_out, (size_t)g->n * sizeof(int32_t),
                                    cudaMemcpyDeviceToHost, sl.cstream) != cudaSuccess) {
                    cudaGetLastError();
                    return fail(DFS_ECUDA);
                }
                cudaEventRecord(sl.evc[buf], sl.cstream);
            }
            cudaEventRecord(sl.evq[sl.issued & 1], sl.stream);
            ++sl.issued;
            ++q;
            any = true;
            rr = (c + 1) % conc;
        }
        if (!any) std::this_thread::yield();
    }
    // join (host rows: the copy streams too)
    for (int c = 0; c < conc; ++c) {
        Slot& sl = g->slots[c];
        cudaEventRecord(sl.ev1, sl.stream);
        cudaStreamWaitEvent(base, sl.ev1, 0);
        if (!out_dev && sl.issued > 0) {
            cudaEventRecord(sl.ev1, sl.cstream);
            cudaStreamWaitEvent(base, sl.ev1, 0);
        }
    }
    cudaEventRecord(s0.evk1, base);
    if (cudaStreamSynchronize(base) != cudaSuccess) { cudaGetLastError(); return fail(DFS_ECUDA); }
    int worst = 0;
    int64_t nv = 0, mv = 0;
    for (int c = 0; c < conc; ++c) {
        Slot& sl = g->slots[c];
        int st = 0;
        cudaMemcpy(&st, sl.status, sizeof(int), cudaMemcpyDeviceToHost);
        if (st != 0) { sl.tab_dirty = true; worst = std::min(worst, st); }
    }
    if (cudaGetLastError() != cudaSuccess) return fail(DFS_ECUDA);
    if (worst != 0) return fail(worst);
    if (stats) {
        const int rc = finish_counts(g, k, stats, nv, mv);
        if (rc != DFS_OK) return fail(rc);
        float ms = 0.f;
        cudaEventElapsedTime(&ms, s0.ev0, s0.evk1);
        unsigned long long counters[kNumWCounters] = {0};
        fill_stats(stats, o, blocks, warps, ms, ms, nv, mv, counters);
    }
    return DFS_OK;
}

static bool is_pinned_host(const void* p) {
    cudaPointerAttributes a;
    if (cudaPointerGetAttributes(&a, p) != cudaSuccess) { cudaGetLastError(); return false; }
    return a.type == cudaMemoryTypeHost;
}

static int run_many(dfs_graph* g, const int32_t* roots_host, int32_t k, int32_t* out, bool out_dev,
                    const dfs_options* opt, dfs_stats* stats) {
    dfs_options o;
    int blocks = 0, warps = 0, conc = 1;
    int rc = resolve_options(g, opt, k, o, blocks, warps, conc);
    if (rc != DFS_OK) return fail(rc);
    for (int32_t q = 0; q < k; ++q)
        if (roots_host[q] < 0 || roots_host[q] >= g->n) return fail(DFS_EINVAL);
    // concurrent slots: scratch sized for their block share; when the device cannot hold
    // `conc` slots, fewer traversals run concurrently (each on a larger share)
    const bool auto_blocks = o.blocks <= 0;
    while (conc > 1) {
        int c = 0;
        rc = DFS_OK;
        const int64_t owners = (int64_t)(blocks + (auto_blocks ? 1 : 0)) * warps * (o.walker_lanes == 32 ? 1 : 32 / o.walker_lanes);
        for (; c < conc; ++c) {
            rc = ensure_slot(g, c, c == 0 ? std::max<int64_t>(owners, (int64_t)g->max_blocks * kMaxWarps) : owners);
            if (rc != DFS_OK) break;
        }
        if (rc == DFS_OK) break;
        if (rc != DFS_ENOMEM || c == 0) return fail(rc);
        for (int q = c; q < kMaxSlots; ++q) free_slot(g->slots[q]);
        conc = c;
        if (auto_blocks) blocks = std::max(1, g->max_blocks / conc);
        if (conc == 1) blocks = auto_blocks ? g->max_blocks : blocks;
    }
    if (conc <= 1) return run_sequential(g, roots_host, k, out, out_dev, o, blocks, warps, stats);
    // a device->pageable-host copy is synchronous, which would serialise the concurrent
    // traversals: the output range is page-locked for the call (or the batch runs sequentially
    // on the whole GPU when it cannot be)
    bool registered = false;
    if (!out_dev && !is_pinned_host(out)) {
        if (cudaHostRegister(out, (size_t)k * (size_t)g->n * sizeof(int32_t), cudaHostRegisterDefault) != cudaSuccess) {
            cudaGetLastError();
            if (auto_blocks) blocks = g->max_blocks;
            return run_sequential(g, roots_host, k, out, out_dev, o, blocks, warps, stats);
        }
        registered = true;
    }
    // (not with the cluster tier: its grids are whole clusters)
    const int extra = (auto_blocks && o.cluster < 1) ? std::max(0, g->max_blocks - blocks * conc) : 0;
    rc = run_concurrent(g, roots_host, k, out, out_dev, o, blocks, warps, conc, stats, extra);
    if (registered) { cudaHostUnregister(out); cudaGetLastError(); }
    return rc;
}

extern "C" {

int dfs_run_ex(dfs_graph* g, int32_t root, int32_t* parent_out, const dfs_options* opt, dfs_stats* stats) {
    if (!g || !parent_out) return fail(DFS_EINVAL);
    int rc = check_device(g);
    if (rc != DFS_OK) return fail(rc);
    return run_many(g, &root, 1, parent_out, is_device_ptr(parent_out), opt, stats);
}

int dfs_run(dfs_graph* g, int32_t root, int32_t* parent_out) {
    return dfs_run_ex(g, root, parent_out, nullptr, nullptr);
}

int dfs_run_batch_ex(dfs_graph* g, const int32_t* roots, int32_t num_roots, int32_t* parents_out,
                     const dfs_options* opt, dfs_stats* stats) {
    if (!g || num_roots < 0 || (num_roots > 0 && (!roots || !parents_out))) return fail(DFS_EINVAL);
    int rc = check_device(g);
    if (rc != DFS_OK) return fail(rc);
    if (num_roots == 0) return DFS_OK;                          // nothing to do (arrays may be NULL)
    std::vector<int32_t> hroots((size_t)num_roots);
    if (is_device_ptr(roots)) {
        if (cudaMemcpy(hroots.data(), roots, (size_t)num_roots * sizeof(int32_t), cudaMemcpyDeviceToHost) != cudaSuccess) {
            cudaGetLastError();
            return fail(DFS_ECUDA);
        }
    } else {
        std::memcpy(hroots.data(), roots, (size_t)num_roots * sizeof(int32_t));
    }
    return run_many(g, hroots.data(), num_roots, parents_out, is_device_ptr(parents_out), opt, stats);
}

int dfs_run_batch(dfs_graph* g, const int32_t* roots, int32_t num_roots, int32_t* parents_out) {
    return dfs_run_batch_ex(g, roots, num_roots, parents_out, nullptr, nullptr);
}

}  // extern "C"

extern "C" int dfs_debug_stack_script(dfs_graph* g, int32_t lanes, const int32_t* script, int32_t n_ops,
                                      int32_t* out, int32_t out_len, const dfs_options* opt) {
    if (!g || !script || n_ops < 0 || (out_len > 0 && !out) || !valid_walker_lanes(lanes))
        return fail(DFS_EINVAL);
    int rc = check_device(g);
    if (rc != DFS_OK) return fail(rc);
    dfs_options in;
    dfs_options_default(&in);
    if (opt) in = *opt;
    in.walker_lanes = lanes; in.collect_stats = 1; in.deterministic = 0; in.cluster = 0; in.window = 0;
    dfs_options o;
    int blocks = 0, warps = 0, conc = 1;
    rc = resolve_options(g, &in, 1, o, blocks, warps, conc);
    if (rc != DFS_OK) return fail(rc);
    Slot& sl = g->slots[0];
    rc = ensure_slot(g, 0, std::max<int64_t>((int64_t)g->max_blocks * kMaxWarps, (int64_t)warps * (32 / lanes)));
    if (rc != DFS_OK) return fail(rc);
    if (!sl.parent && cudaMalloc(&sl.parent, (size_t)g->n * sizeof(int32_t)) != cudaSuccess) {
        cudaGetLastError();
        return fail(DFS_ENOMEM);
    }
    int32_t *d_script = nullptr, *d_out = nullptr;
    if (cudaMalloc(&d_script, (size_t)n_ops * 6 * sizeof(int32_t) + 16) != cudaSuccess ||
        cudaMalloc(&d_out, (size_t)out_len * sizeof(int32_t) + 16) != cudaSuccess) {
        cudaGetLastError(); cudaFree(d_script); cudaFree(d_out);
        return fail(DFS_ENOMEM);
    }
    cudaMemcpy(d_script, script, (size_t)n_ops * 6 * sizeof(int32_t), cudaMemcpyHostToDevice);
    cudaMemset(d_out, 0xFF, (size_t)out_len * sizeof(int32_t) + 16);
    ScriptArgs sa;
    sa.d_script = d_script; sa.n_ops = n_ops; sa.d_out = d_out; sa.out_len = out_len;
    cudaStream_t s = g->stream;
    rc = launch_one(g, sl, s, 0, sl.parent, o, 1, warps, false, false, &sa);
    if (rc == DFS_OK) {
        if (cudaStreamSynchronize(s) != cudaSuccess ||
            (out_len > 0 && cudaMemcpy(out, d_out, (size_t)out_len * sizeof(int32_t), cudaMemcpyDeviceToHost) != cudaSuccess)) {
            cudaGetLastError();
            rc = DFS_ECUDA;
        }
    }
    sl.tab_dirty = true;                       // the script maps chunks it never returns
    cudaFree(d_script); cudaFree(d_out);
    return rc == DFS_OK ? DFS_OK : fail(rc);
}
