// dfs_runtime.cu — host runtime + C ABI (include/dfs.h) of the B200 unordered-DFS library.
//
// Owns graph residency (step a1: copy, validate, narrow row_ptr to uint32), the per-handle
// scratch (visited bitmap, per-warp ColdSeg words, chunk table, chunk pool, control block),
// and the per-traversal launch sequence: reset (a2) -> persistent traversal (a3-a8) ->
// finalize (a9).  "P:a-b" = /root/reference/PAPER.md lines.
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <new>
#include <vector>

#include "../../include/dfs.h"
#include "dfs_device.cuh"

using namespace b200dfs;

namespace {

constexpr int kRing = 256;                   // HotRing entries per warp (P:367 uses 128)
thread_local int g_last_error = DFS_OK;

int fail(int code) { g_last_error = code; return code; }

bool is_device_ptr(const void* p) {
    cudaPointerAttributes a;
    if (cudaPointerGetAttributes(&a, p) != cudaSuccess) { cudaGetLastError(); return false; }
    return a.type == cudaMemoryTypeDevice || a.type == cudaMemoryTypeManaged;
}

// the 8 instantiations of the persistent kernel: [vec128][wmax16][stats]
const void* const* kernel_table() {
    static const void* const t[8] = {
        (const void*)dfs_persistent_kernel<kRing, 1, 32, false>, (const void*)dfs_persistent_kernel<kRing, 1, 32, true>,
        (const void*)dfs_persistent_kernel<kRing, 1, 16, false>, (const void*)dfs_persistent_kernel<kRing, 1, 16, true>,
        (const void*)dfs_persistent_kernel<kRing, 4, 32, false>, (const void*)dfs_persistent_kernel<kRing, 4, 32, true>,
        (const void*)dfs_persistent_kernel<kRing, 4, 16, false>, (const void*)dfs_persistent_kernel<kRing, 4, 16, true>};
    return t;
}

size_t smem_bytes(int warps) {
    return ((sizeof(SmemCtl) + 15) & ~size_t(15)) + (size_t)warps * kRing * sizeof(unsigned long long);
}

}  // namespace

struct dfs_graph {
    int device = 0;
    cudaStream_t stream = nullptr;
    int64_t n = 0, m = 0;
    int sms = 0;
    int max_blocks = 0;          // co-resident 32-warp blocks (allocation bound)
    uint32_t* d_rp = nullptr;
    uint2* d_adj = nullptr;      // {col_idx[j], row_ptr[col_idx[j]]} per CSR entry (+8 padding)
    uint32_t* d_bitmap = nullptr;
    int32_t* d_parent = nullptr; // lazily allocated for host outputs
    unsigned long long* d_cold_tb = nullptr;
    uint32_t* d_tab = nullptr;
    unsigned long long* d_pool = nullptr;
    uint32_t* d_consumed = nullptr;
    uint32_t* d_next = nullptr;
    int* d_block_cold = nullptr;
    Ctl* d_ctl = nullptr;
    unsigned long long* d_count2 = nullptr;
    int tab_log2 = 0;
    uint32_t n_chunks = 0;
    size_t tab_words = 0;
    bool tab_dirty = false;
    int64_t launches = 0;
    cudaEvent_t ev0 = nullptr, ev1 = nullptr, evk0 = nullptr, evk1 = nullptr;
    unsigned int* d_timeline = nullptr;   // diagnostics (dfs_debug_timeline)
    unsigned int timeline_len = 0, timeline_dt_ns = 0;
};

static void free_graph(dfs_graph* g) {
    if (!g) return;
    int cur = 0;
    cudaGetDevice(&cur);
    cudaSetDevice(g->device);
    cudaFree(g->d_rp); cudaFree(g->d_adj); cudaFree(g->d_bitmap); cudaFree(g->d_parent);
    cudaFree(g->d_cold_tb); cudaFree(g->d_tab); cudaFree(g->d_pool); cudaFree(g->d_consumed);
    cudaFree(g->d_next); cudaFree(g->d_block_cold); cudaFree(g->d_ctl); cudaFree(g->d_count2);
    cudaFree(g->d_timeline);
    if (g->ev0) cudaEventDestroy(g->ev0);
    if (g->ev1) cudaEventDestroy(g->ev1);
    if (g->evk0) cudaEventDestroy(g->evk0);
    if (g->evk1) cudaEventDestroy(g->evk1);
    cudaSetDevice(cur);
    delete g;
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
    o->speculate = 2;
    o->steal_half = 1;
    o->probe_mode = 0;
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
    for (int kf = 0; kf < 8; ++kf) {
        const void* f = kernel_table()[kf];
        if (f && cudaFuncSetAttribute(f, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm32) != cudaSuccess)
            attr_ok = false;
    }
    if (!attr_ok) { cudaGetLastError(); delete g; fail(DFS_ECUDA); return nullptr; }
    int per_sm = 0;
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, dfs_persistent_kernel<kRing, 4, 32, false>, 1024, sm32) !=
            cudaSuccess || per_sm < 1) {
        cudaGetLastError(); per_sm = 1;
    }
    g->max_blocks = g->sms * per_sm;

    const int64_t n_warps = (int64_t)g->max_blocks * kMaxWarps;
    // chunk table: 2^tab_log2 >= (max live span + 2 chunks + flush batch) / chunk  (reading S9)
    int64_t need = (n + 2 * (int64_t)kChunk + kRing) / kChunk + 2;
    g->tab_log2 = 2;
    while (((int64_t)1 << g->tab_log2) < need) ++g->tab_log2;
    g->tab_words = (size_t)n_warps << g->tab_log2;
    // pool: sum of live spans <= n, plus <= 4 partially used chunks per warp
    g->n_chunks = (uint32_t)(n / kChunk + 4 * n_warps + 16);

    const size_t nwords = (size_t)((n + 31) / 32);
    bool ok = true;
    auto A = [&](void** p, size_t bytes) { if (ok && cudaMalloc(p, bytes ? bytes : 16) != cudaSuccess) ok = false; };
    A((void**)&g->d_rp, (size_t)(n + 1) * sizeof(uint32_t));
    A((void**)&g->d_adj, (size_t)(m + 8) * sizeof(uint2));       // padded for 128-bit window loads
    A((void**)&g->d_bitmap, nwords * sizeof(uint32_t));
    A((void**)&g->d_cold_tb, (size_t)n_warps * sizeof(unsigned long long));
    A((void**)&g->d_tab, g->tab_words * sizeof(uint32_t));
    A((void**)&g->d_pool, (size_t)g->n_chunks * kChunk * sizeof(unsigned long long));
    A((void**)&g->d_consumed, (size_t)g->n_chunks * sizeof(uint32_t));
    A((void**)&g->d_next, (size_t)g->n_chunks * sizeof(uint32_t));
    A((void**)&g->d_block_cold, (size_t)g->max_blocks * sizeof(int));
    A((void**)&g->d_ctl, sizeof(Ctl));
    A((void**)&g->d_count2, 2 * sizeof(unsigned long long));
    if (!ok) { cudaGetLastError(); free_graph(g); fail(DFS_ENOMEM); return nullptr; }
    if (cudaEventCreate(&g->ev0) != cudaSuccess || cudaEventCreate(&g->ev1) != cudaSuccess ||
        cudaEventCreate(&g->evk0) != cudaSuccess || cudaEventCreate(&g->evk1) != cudaSuccess) {
        cudaGetLastError(); free_graph(g); fail(DFS_ECUDA); return nullptr;
    }

    // ---- copy + validate + narrow (step a1) ----
    int* d_bad = nullptr;
    if (cudaMalloc(&d_bad, sizeof(int)) != cudaSuccess) { cudaGetLastError(); free_graph(g); fail(DFS_ENOMEM); return nullptr; }
    cudaMemset(d_bad, 0, sizeof(int));
    bool bad = false;
    if (is_device_ptr(row_ptr)) {
        const int blocks = (int)std::min<int64_t>((n + 256) / 256 + 1, 65535);
        dfs_validate_rowptr_kernel<<<blocks, 256>>>(row_ptr, g->d_rp, n, m, d_bad);
        g->launches++;
    } else {
        std::vector<uint32_t> rp32((size_t)n + 1);
        for (int64_t v = 0; v <= n; ++v) {
            const int64_t a = row_ptr[v];
            if (a < 0 || a > m || (v == 0 && a != 0) || (v == n && a != m) || (v < n && row_ptr[v + 1] < a)) { bad = true; break; }
            rp32[(size_t)v] = (uint32_t)a;
        }
        if (!bad) cudaMemcpy(g->d_rp, rp32.data(), (size_t)(n + 1) * sizeof(uint32_t), cudaMemcpyHostToDevice);
    }
    int32_t* d_col = nullptr;   // staging copy of col_idx (freed after the adjacency is built)
    if (!bad && m > 0) {
        if (cudaMalloc(&d_col, (size_t)m * sizeof(int32_t)) != cudaSuccess) {
            cudaGetLastError(); cudaFree(d_bad); free_graph(g); fail(DFS_ENOMEM); return nullptr;
        }
        cudaMemcpy(d_col, col_idx, (size_t)m * sizeof(int32_t), cudaMemcpyDefault);
        const int blocks = (int)std::min<int64_t>((m + 255) / 256, 65535);
        dfs_validate_col_kernel<<<blocks, 256>>>(d_col, m, n, d_bad);
        g->launches++;
    }
    int hbad = 0;
    cudaMemcpy(&hbad, d_bad, sizeof(int), cudaMemcpyDeviceToHost);
    cudaFree(d_bad);
    if (!bad && !hbad && m > 0) {
        const int blocks = (int)std::min<int64_t>((m + 255) / 256, 65535);
        dfs_build_adj_kernel<<<blocks, 256>>>(d_col, g->d_rp, g->d_adj, m);
        g->launches++;
    }
    cudaFree(d_col);
    if (cudaGetLastError() != cudaSuccess) { free_graph(g); fail(DFS_ECUDA); return nullptr; }
    if (bad || hbad) { free_graph(g); fail(DFS_EINVAL); return nullptr; }
    cudaMemset(g->d_tab, 0xFF, g->tab_words * sizeof(uint32_t));   // all chunk slots empty
    cudaMemset(g->d_adj + m, 0xFF, 8 * sizeof(uint2));              // padding (never a valid position)
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
// one traversal on the handle's stream (no synchronisation)
// ------------------------------------------------------------------------------------------
static int launch_one(dfs_graph* g, int32_t root, int32_t* d_out, const dfs_options& o, int blocks,
                      int warps, bool timed) {
    cudaStream_t s = g->stream;
    const uint32_t nwords = (uint32_t)((g->n + 31) / 32);
    const int rblocks = (int)std::min<int64_t>((std::max<int64_t>(nwords, g->tab_dirty ? (int64_t)g->tab_words : 0) + 255) / 256 + 1,
                                               (int64_t)g->sms * 8);
    dfs_reset_kernel<<<rblocks, 256, 0, s>>>(g->d_bitmap, nwords, g->d_cold_tb, (uint32_t)(blocks * warps),
                                            g->d_block_cold, (uint32_t)blocks, g->d_ctl, d_out, root,
                                            g->d_tab, g->tab_dirty ? g->tab_words : 0);
    g->launches++;
    g->tab_dirty = false;

    KParams P;
    P.rp = g->d_rp; P.adj = g->d_adj; P.bitmap = g->d_bitmap; P.parent = d_out;
    P.cold_tb = g->d_cold_tb; P.chunk_tab = g->d_tab; P.pool = g->d_pool;
    P.chunk_consumed = g->d_consumed; P.chunk_next = g->d_next; P.block_cold = g->d_block_cold;
    P.ctl = g->d_ctl;
    P.n = (uint32_t)g->n; P.m = (uint32_t)g->m; P.root = root; P.tab_log2 = g->tab_log2;
    P.n_chunks = g->n_chunks;
    P.hot_cutoff = o.hot_cutoff; P.cold_cutoff = o.cold_cutoff;
    P.intra = o.intra_steal; P.inter = o.inter_steal; P.policy = o.victim_policy;
    P.collect_stats = o.collect_stats;
    P.spill = o.spill;
    P.spill_idle = o.spill_idle > 0 ? o.spill_idle : 32;
    P.inter_any = o.inter_any;
    P.backoff_max_ns = o.backoff_max_ns > 0 ? (unsigned)o.backoff_max_ns : 2048u;
    P.pub_batch = o.pub_batch > 0 ? (uint32_t)o.pub_batch : 4u;
    P.speculate = o.speculate;
    P.steal_half = o.steal_half;
    P.probe_mode = o.probe_mode;
    P.timeline = g->d_timeline;
    P.timeline_len = g->timeline_len;
    P.timeline_dt_ns = g->timeline_dt_ns;
    P.timeout_ns = (unsigned long long)o.timeout_ms * 1000000ull;
    P.seed = o.seed;
    void* args[] = {(void*)&P};
    if (timed) cudaEventRecord(g->evk0, s);
    const void* kfn = kernel_table()[(o.window == 128 ? 4 : 0) + (warps <= 16 ? 2 : 0) + (o.collect_stats ? 1 : 0)];
    cudaError_t e = cudaLaunchCooperativeKernel(kfn, dim3(blocks),
                                                dim3(32 * warps), args, smem_bytes(warps), s);
    if (e != cudaSuccess) { cudaGetLastError(); return DFS_ECUDA; }
    if (timed) cudaEventRecord(g->evk1, s);
    g->launches++;
    const int fblocks = (int)std::min<int64_t>((g->n + 255) / 256, (int64_t)g->sms * 16);
    dfs_finalize_kernel<<<fblocks, 256, 0, s>>>(g->d_bitmap, d_out, (uint32_t)g->n);
    g->launches++;
    return DFS_OK;
}

static int resolve_options(const dfs_graph* g, const dfs_options* in, dfs_options& o, int& blocks, int& warps) {
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
    if (o.window == 0) o.window = (g->n > 0 && g->m >= 8 * g->n) ? 128 : 32;   // wide windows for dense lists
    if (o.window != 32 && o.window != 128) return DFS_EINVAL;
    warps = o.warps_per_block <= 0 ? 32 : o.warps_per_block;
    if (warps > 32) return DFS_EINVAL;
    blocks = o.blocks <= 0 ? g->max_blocks : o.blocks;
    if (blocks > g->max_blocks) return DFS_EINVAL;
    if (o.deterministic) { blocks = 1; warps = 1; o.intra_steal = 0; o.inter_steal = 0; }
    return DFS_OK;
}

static int check_device(const dfs_graph* g) {
    int cur = -1;
    if (cudaGetDevice(&cur) != cudaSuccess) { cudaGetLastError(); return DFS_ECUDA; }
    return cur == g->device ? DFS_OK : DFS_EDEVICE;
}

static int run_many(dfs_graph* g, const int32_t* roots_host, int32_t k, int32_t* out, bool out_dev,
                    const dfs_options* opt, dfs_stats* stats) {
    dfs_options o;
    int blocks = 0, warps = 0;
    int rc = resolve_options(g, opt, o, blocks, warps);
    if (rc != DFS_OK) return fail(rc);
    for (int32_t q = 0; q < k; ++q)
        if (roots_host[q] < 0 || roots_host[q] >= g->n) return fail(DFS_EINVAL);
    if (!out_dev && !g->d_parent) {
        if (cudaMalloc(&g->d_parent, (size_t)g->n * sizeof(int32_t)) != cudaSuccess) {
            cudaGetLastError();
            return fail(DFS_ENOMEM);
        }
    }
    unsigned long long counters[kNumCounters] = {0};
    float total_ms = 0.f, trav_ms = 0.f;
    int64_t nv = 0, mv = 0;
    for (int32_t q = 0; q < k; ++q) {
        int32_t* d_out = out_dev ? out + (size_t)q * g->n : g->d_parent;
        cudaEventRecord(g->ev0, g->stream);
        rc = launch_one(g, roots_host[q], d_out, o, blocks, warps, stats != nullptr);
        if (rc != DFS_OK) return fail(rc);
        cudaEventRecord(g->ev1, g->stream);
        if (stats) {
            cudaMemsetAsync(g->d_count2, 0, 2 * sizeof(unsigned long long), g->stream);
            dfs_count_kernel<<<g->sms * 4, 256, 0, g->stream>>>(g->d_bitmap, g->d_rp, (uint32_t)g->n, g->d_count2);
            g->launches++;
        }
        Ctl h;
        if (cudaMemcpyAsync(&h, g->d_ctl, sizeof(Ctl), cudaMemcpyDeviceToHost, g->stream) != cudaSuccess ||
            cudaStreamSynchronize(g->stream) != cudaSuccess) {
            cudaGetLastError();
            return fail(DFS_ECUDA);
        }
        if (h.status != 0) { g->tab_dirty = true; return fail(h.status); }
        if (!out_dev) {
            if (cudaMemcpyAsync(out + (size_t)q * g->n, g->d_parent, (size_t)g->n * sizeof(int32_t),
                                cudaMemcpyDeviceToHost, g->stream) != cudaSuccess) {
                cudaGetLastError();
                return fail(DFS_ECUDA);
            }
        }
        if (stats) {
            float ms = 0.f, kms = 0.f;
            cudaEventElapsedTime(&ms, g->ev0, g->ev1);
            cudaEventElapsedTime(&kms, g->evk0, g->evk1);
            total_ms += ms;
            trav_ms += kms;
            for (int c = 0; c < kNumCounters; ++c) counters[c] += h.counters[c];
            {
                unsigned long long c2[2];
                cudaMemcpyAsync(c2, g->d_count2, sizeof(c2), cudaMemcpyDeviceToHost, g->stream);
                cudaStreamSynchronize(g->stream);
                nv += (int64_t)c2[0]; mv += (int64_t)c2[1];
            }
        }
    }
    if (cudaStreamSynchronize(g->stream) != cudaSuccess) { cudaGetLastError(); return fail(DFS_ECUDA); }
    if (stats) {
        std::memset(stats, 0, sizeof(*stats));
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
    }
    return DFS_OK;
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
    if (!g || !roots || !parents_out || num_roots < 0) return fail(DFS_EINVAL);
    int rc = check_device(g);
    if (rc != DFS_OK) return fail(rc);
    if (num_roots == 0) return DFS_OK;
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
