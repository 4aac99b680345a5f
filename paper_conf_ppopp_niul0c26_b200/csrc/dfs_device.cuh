// dfs_device.cuh — sm_100a device code of the unordered-DFS hot path.
//
// The method is DiggerBees (PPoPP '26); "P:a-b" = /root/reference/PAPER.md lines.  The kernel
// re-designs the paper's H100 kernel for B200:
//
//   * persistent grid, one 32-warp CTA per SM (subsystem 1; "1 block per SM")
//   * per-warp two-level stack (subsystem 2; §3.2, Fig 2):
//       HotRing  = circular buffer in shared memory; head/tail are 16-bit counters packed in
//                  one 32-bit word updated only by shared-memory atomics (no SC fences)
//       ColdSeg  = per-warp virtual linear segment in global memory, backed by a chunk table
//                  and a global chunk pool (the paper's fixed n_v/n_w capacity overflows on deep
//                  graphs; reading S9)
//       flush oldest entries from tail -> ColdSeg top; refill from ColdSeg top
//   * warp-level expansion (subsystem 3; §3.3): the 32 lanes load a VEC*32-position
//     window of col_idx (VEC = 4: one 128-bit load per lane), probe the visited bitmap,
//     __ballot_sync + __ffs pick the FIRST unvisited neighbour in CSR order, lane 0 claims it
//     with atomicOr on the bitmap word (Alg 1 l.9-10 made atomic).  The top entry lives in
//     registers; the child's row_ptr pair and first window are loaded speculatively so they
//     overlap the probe and the claim.
//   * intra-block stealing (subsystem 4; §3.4, Alg 3): an idle warp takes h_s =
//     hot_cutoff/2 entries from the TAIL of the peer HotRing with max hot_rest >= hot_cutoff,
//     reserving them with a CAS on the packed head/tail word under the victim's lock (S12)
//   * inter-block stealing (subsystem 5; §3.5, Alg 4): two random active blocks,
//     the heavier by cumulative ColdSeg load (S14); the warp with max cold_rest >= cold_cutoff;
//     c_s = cold_cutoff/2 entries reserved from the ColdSeg BOTTOM by a 64-bit CAS on the packed
//     {top,bottom} word and copied into the thief's HotRing.
//   * demand-driven spill (B200 addition): when many warps are idle, a busy warp
//     moves the oldest half of a deep HotRing to its ColdSeg so other blocks can steal it.
//   * global termination (unspecified in the paper, reading S13): hierarchical busy counters — a
//     shared-memory count per block of warps that hold work plus registered thieves, and a global
//     count of blocks whose local count is non-zero (changed only on the local 0<->1
//     transitions); the global atomic that brings it to 0 raises `done`.
//
// Memory-ordering notes: CTA-scope release (MEMBAR.ALL.CTA) publishes HotRing
// entries; CTA-scope acquire is free.  GPU-scope publication of ColdSeg data uses
// fence.release.gpu (MEMBAR.ALL.GPU, no L1 invalidation); readers of ColdSeg data use L2
// (.cg / .relaxed.gpu) loads whose addresses depend on the reserving atomic.
#pragma once
#include <cstdint>

namespace b200dfs {

constexpr uint32_t kFull = 0xffffffffu;
constexpr uint32_t kEmptySlot = 0xffffffffu;
constexpr int kChunkLog2 = 11;                     // ColdSeg chunk = 2048 entries (16 KB)
constexpr uint32_t kChunk = 1u << kChunkLog2;
constexpr int kMaxWarps = 32;                      // 32-bit warp mask

// error codes written to Ctl::status (mirrors dfs_status)
constexpr int kStatusENOMEM = -2;
constexpr int kStatusETIMEOUT = -5;
constexpr int kStatusEINTERNAL = -6;

struct Ctl {
    unsigned int busy;                 // blocks whose local busy count is non-zero (S13)
    unsigned int done;                 // set once busy reaches 0 (or on error)
    int status;                        // 0 or a negative dfs_status
    unsigned int pool_bump;            // bump allocator over the chunk pool
    unsigned long long free_head;      // tagged free-stack head: (tag << 32) | chunk id
    unsigned long long counters[24];   // stats (collect_stats)
    unsigned long long claims_progress;// timeline diagnostics: claims reported so far
    unsigned long long windows_progress;// ... and windows (STATS builds)
};

enum CounterIdx {
    kCntClaims = 0, kCntFailedClaims, kCntFlushes, kCntRefills, kCntIntraSteals, kCntInterSteals,
    kCntStealAttempts, kCntChunks, kCntWindows, kCntIdleNs, kCntInterScans, kCntSpills,
    kCntTWin, kCntTProbe, kCntTClaim, kCntTTail, kCntTOut, kCntOutIters, kCntClusterSteals,
    kCntPops, kCntDeadPops, kNumCounters
};

struct KParams {
    const uint32_t* __restrict__ rp;         // n+1 (narrowed row_ptr; m < 2^32)
    const int32_t* __restrict__ col;         // m (+8 padding)
    uint32_t* bitmap;                        // {visited, leaf} word pairs: bitmap[2k] holds the
                                             // visited bits of vertices 32k..32k+31, bitmap[2k+1]
                                             // their leaf bits (one 8-byte probe = one L2 sector
                                             // returns both)
    int32_t* parent;                         // n output
    unsigned long long* cold_tb;             // n_warps: (top << 32) | bottom
    uint32_t* chunk_tab;                     // n_warps << tab_log2
    unsigned long long* pool;                // n_chunks * kChunk entries
    uint32_t* chunk_consumed;                // n_chunks
    uint32_t* chunk_next;                    // n_chunks (free-stack links)
    int* block_cold;                         // n_blocks: cumulative ColdSeg load (S14)
    Ctl* ctl;
    uint32_t n, m;
    int root;
    int tab_log2;
    uint32_t n_chunks;
    int hot_cutoff, cold_cutoff;
    int intra, inter, policy;
    int collect_stats;
    int spill;                               // demand-driven spill of oldest HotRing entries
    int spill_idle;                          // ... when at least this many warps are idle
    int inter_any;                           // any idle warp may steal inter-block (else leader of an idle block)
    unsigned int backoff_max_ns;             // idle-loop exponential backoff cap
    unsigned int backoff_min_ns;             // ... and first step
    unsigned int* timeline;                  // optional: busy-block samples (block 0 / warp 0)
    unsigned int timeline_len;
    unsigned int timeline_dt_ns;
    unsigned long long timeout_ns;
    uint32_t seed;
    uint32_t pub_batch;                      // publish the HotRing head every pub_batch pushes
    int speculate;                           // speculative claim of the child's first neighbour
    int steal_half;                          // steal max(h_s, rest/2) (resp. c_s) entries
    uint32_t ring_cap;                       // usable HotRing entries (<= H); 2 ~ one-level stack (v1)
    int leaf_skip;                           // claim children whose list is empty or [parent] in place
    unsigned long long* block_claims;        // optional: claims per block (Fig 9 task counts)
    int cluster_late;                        // cluster tier after Alg 4 instead of before it
    int steal_tries;                         // Alg 3 victims tried per idle round (best first)
    int bulk_copy;                           // flush/refill with cp.async.bulk (TMA ablation)
    uint32_t period_mask;                    // spill_period - 1
    uint32_t steal_period_mask;              // walker kernel: steal_period - 1
    int donate;                              // walker kernel: hand pushed entries to idle siblings
    const uint32_t* __restrict__ rec;        // vertex records (8 words per vertex: col[rp[v] .. +6),
                                             // rp[v], rp[v+1]; padding kFull), or null
    const int32_t* script;                   // walker STATS kernel: stack-script mode (tests), or null
    int script_len;
    int32_t* script_out;
    int script_out_len;
};

// vertex records (create time, on first use): record v = 8 words = one 32-byte
// sector: the first 6 entries of v's adjacency list (kFull past its end), then row_ptr[v] and
// row_ptr[v+1].  A walker of >= 8 lanes loads a claimed child's record with one coalesced request,
// so a list of <= 6 entries needs no dependent row_ptr -> col_idx round trip.
__global__ void dfs_records_kernel(const uint32_t* __restrict__ rp, const int32_t* __restrict__ col, uint32_t n,
                                   uint4* __restrict__ rec) {
    const size_t stride = (size_t)gridDim.x * blockDim.x;
    for (size_t v = blockIdx.x * (size_t)blockDim.x + threadIdx.x; v < n; v += stride) {
        const uint32_t s = rp[v], e = rp[v + 1];
        uint32_t w[6];
#pragma unroll
        for (int k = 0; k < 6; ++k) w[k] = s + k < e ? (uint32_t)col[s + k] : kFull;
        rec[2 * v] = make_uint4(w[0], w[1], w[2], w[3]);
        rec[2 * v + 1] = make_uint4(w[4], w[5], s, e);
    }
}

// ------------------------------------------------------------------------------------------
// small PTX helpers
// ------------------------------------------------------------------------------------------
__device__ __forceinline__ unsigned long long ld_relaxed_u64(const unsigned long long* p) {
    unsigned long long v;
    asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ uint32_t ld_relaxed_u32(const uint32_t* p) {
    uint32_t v;
    asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ int ld_relaxed_s32(const int* p) {
    int v;
    asm volatile("ld.relaxed.gpu.global.s32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void st_relaxed_u32(uint32_t* p, uint32_t v) {
    asm volatile("st.relaxed.gpu.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ unsigned long long globaltimer() {
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    return t;
}
__device__ __forceinline__ unsigned long long ld_acquire_u64(const unsigned long long* p) {
    unsigned long long v;
    asm volatile("ld.acquire.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}
// acquire side of a GPU-scope release (pairs with fence_release_gpu + the publishing atomic):
// SASS CCTL.IVALL — used only on cold paths (after a successful ColdSeg steal reservation)
__device__ __forceinline__ void fence_acquire_gpu() { asm volatile("fence.acquire.gpu;" ::: "memory"); }
__device__ __forceinline__ unsigned long long atom_cas_acquire_u64(unsigned long long* p, unsigned long long cmp,
                                                                   unsigned long long v) {
    unsigned long long r;
    asm volatile("atom.acquire.gpu.global.cas.b64 %0, [%1], %2, %3;" : "=l"(r) : "l"(p), "l"(cmp), "l"(v) : "memory");
    return r;
}
__device__ __forceinline__ unsigned long long ld_cg_u64(const unsigned long long* p) {
    unsigned long long v;
    asm volatile("ld.global.cg.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void st_cg_u64(unsigned long long* p, unsigned long long v) {
    asm volatile("st.global.cg.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
// release fence at GPU scope without the L1 invalidation (CCTL.IVALL) of __threadfence()
__device__ __forceinline__ void fence_release_gpu() { asm volatile("fence.release.gpu;" ::: "memory"); }

// predicated single-lane memory ops: one predicated instruction instead of an `if (lane == 0)`
// block, which costs a BSSY/BRA/BSYNC convergence region per use (lean step)
__device__ __forceinline__ uint32_t atom_or_if(bool p, uint32_t* a, uint32_t b) {
    uint32_t r = 0;
    asm volatile("{ .reg .pred q; setp.ne.u32 q, %1, 0; @q atom.global.or.b32 %0, [%2], %3; }"
                 : "+r"(r) : "r"((uint32_t)p), "l"(a), "r"(b) : "memory");
    return r;
}
__device__ __forceinline__ void red_or_if(bool p, uint32_t* a, uint32_t b) {
    asm volatile("{ .reg .pred q; setp.ne.u32 q, %0, 0; @q red.global.or.b32 [%1], %2; }"
                 ::"r"((uint32_t)p), "l"(a), "r"(b) : "memory");
}
__device__ __forceinline__ void st_global_if(bool p, int32_t* a, int32_t v) {
    asm volatile("{ .reg .pred q; setp.ne.u32 q, %0, 0; @q st.global.s32 [%1], %2; }"
                 ::"r"((uint32_t)p), "l"(a), "r"(v) : "memory");
}
__device__ __forceinline__ uint32_t ld_cg_if(bool p, const uint32_t* a, uint32_t dflt) {
    uint32_t r = dflt;
    asm volatile("{ .reg .pred q; setp.ne.u32 q, %1, 0; @q ld.global.cg.u32 %0, [%2]; }"
                 : "+r"(r) : "r"((uint32_t)p), "l"(a));
    return r;
}
__device__ __forceinline__ uint2 ld_cg_u2_if(bool p, const uint32_t* a, uint32_t dx, uint32_t dy) {
    uint2 r = make_uint2(dx, dy);
    asm volatile("{ .reg .pred q; setp.ne.u32 q, %2, 0; @q ld.global.cg.v2.u32 {%0, %1}, [%3]; }"
                 : "+r"(r.x), "+r"(r.y) : "r"((uint32_t)p), "l"(a));
    return r;
}
__device__ __forceinline__ uint32_t ld_nc_if(bool p, const void* a, uint32_t dflt) {
    uint32_t r = dflt;
    asm volatile("{ .reg .pred q; setp.ne.u32 q, %1, 0; @q ld.global.nc.u32 %0, [%2]; }"
                 : "+r"(r) : "r"((uint32_t)p), "l"(a));
    return r;
}

// shared-memory atomics with explicit semantics (CTA scope)
__device__ __forceinline__ uint32_t smem_addr(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ uint32_t atom_add_release_cta(uint32_t* p, uint32_t v) {
    uint32_t r;
    asm volatile("atom.release.cta.shared.add.u32 %0, [%1], %2;" : "=r"(r) : "r"(smem_addr(p)), "r"(v) : "memory");
    return r;
}
__device__ __forceinline__ uint32_t atom_add_relaxed_cta(uint32_t* p, uint32_t v) {
    uint32_t r;
    asm volatile("atom.relaxed.cta.shared.add.u32 %0, [%1], %2;" : "=r"(r) : "r"(smem_addr(p)), "r"(v) : "memory");
    return r;
}
__device__ __forceinline__ uint32_t atom_cas_acquire_cta(uint32_t* p, uint32_t cmp, uint32_t v) {
    uint32_t r;
    asm volatile("atom.acquire.cta.shared.cas.b32 %0, [%1], %2, %3;" : "=r"(r) : "r"(smem_addr(p)), "r"(cmp), "r"(v) : "memory");
    return r;
}
__device__ __forceinline__ uint32_t ld_acquire_cta(const uint32_t* p) {
    uint32_t r;
    asm volatile("ld.acquire.cta.shared.u32 %0, [%1];" : "=r"(r) : "r"(smem_addr(p)) : "memory");
    return r;
}
__device__ __forceinline__ void st_release_cta(uint32_t* p, uint32_t v) {
    asm volatile("st.release.cta.shared.u32 [%0], %1;" ::"r"(smem_addr(p)), "r"(v) : "memory");
}
__device__ __forceinline__ void atom_add_release_cta_if(bool p, uint32_t* a, uint32_t v) {
    asm volatile("{ .reg .pred q; setp.ne.u32 q, %0, 0; @q atom.release.cta.shared.add.u32 _, [%1], %2; }"
                 ::"r"((uint32_t)p), "r"(smem_addr(a)), "r"(v) : "memory");
}
__device__ __forceinline__ void st_shared_u64_if(bool p, unsigned long long* a, unsigned long long v) {
    asm volatile("{ .reg .pred q; setp.ne.u32 q, %0, 0; @q st.shared.u64 [%1], %2; }"
                 ::"r"((uint32_t)p), "r"(smem_addr(a)), "l"(v) : "memory");
}

// ---- thread-block-cluster (DSMEM) helpers for the cluster steal tier ----
// Publication for cluster-scope readers: fence.release restricted to shared::cta state (SASS
// MEMBAR.ALL.CTA + FENCE.VIEW.ASYNC.S — an unrestricted release.cluster is MEMBAR.ALL.GPU) and a
// relaxed cluster-scope atomic; the remote side pairs it with the restricted acquire fence (no
// SASS: an unrestricted acquire.cluster would invalidate the SM's L1, CCTL.IVALL).
__device__ __forceinline__ void fence_release_cta_for_cluster() {
    asm volatile("fence.release.sync_restrict::shared::cta.cluster;" ::: "memory");
}
__device__ __forceinline__ void fence_acquire_cluster_smem() {
    asm volatile("fence.acquire.sync_restrict::shared::cluster.cluster;" ::: "memory");
}
__device__ __forceinline__ void atom_add_relaxed_cluster_if(bool p, uint32_t* a, uint32_t v) {
    asm volatile("{ .reg .pred q; setp.ne.u32 q, %0, 0; @q atom.relaxed.cluster.shared.add.u32 _, [%1], %2; }"
                 ::"r"((uint32_t)p), "r"(smem_addr(a)), "r"(v) : "memory");
}
__device__ __forceinline__ uint32_t cluster_ctarank() {
    uint32_t r; asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r)); return r;
}
__device__ __forceinline__ uint32_t cluster_nctarank() {
    uint32_t r; asm volatile("mov.u32 %0, %%cluster_nctarank;" : "=r"(r)); return r;
}
// shared::cluster address of the same variable in CTA `rank` of the cluster
__device__ __forceinline__ uint32_t dsmem_map(const void* p, uint32_t rank) {
    uint32_t r; asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(r) : "r"(smem_addr(p)), "r"(rank)); return r;
}
__device__ __forceinline__ uint32_t dsmem_ld_u32(uint32_t a) {
    uint32_t v; asm volatile("ld.relaxed.cluster.shared::cluster.u32 %0, [%1];" : "=r"(v) : "r"(a) : "memory"); return v;
}
__device__ __forceinline__ unsigned long long dsmem_ld_u64(uint32_t a) {
    unsigned long long v; asm volatile("ld.shared::cluster.u64 %0, [%1];" : "=l"(v) : "r"(a) : "memory"); return v;
}
__device__ __forceinline__ uint32_t dsmem_cas_u32(uint32_t a, uint32_t cmp, uint32_t v) {
    uint32_t r;
    asm volatile("atom.relaxed.cluster.shared::cluster.cas.b32 %0, [%1], %2, %3;" : "=r"(r) : "r"(a), "r"(cmp), "r"(v) : "memory");
    return r;
}
__device__ __forceinline__ void dsmem_st_u32(uint32_t a, uint32_t v) {
    asm volatile("st.relaxed.cluster.shared::cluster.u32 [%0], %1;" ::"r"(a), "r"(v) : "memory");
}
__device__ __forceinline__ void dsmem_st_release_u32(uint32_t a, uint32_t v) {
    asm volatile("st.release.cluster.shared::cluster.u32 [%0], %1;" ::"r"(a), "r"(v) : "memory");
}
__device__ __forceinline__ void cluster_sync_all() {
    asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
}

// ---- bulk async copies (cp.async.bulk, the TMA engine's non-tensor path) for the optional
// bulk flush/refill (dfs_options.bulk_copy; the paper's TMA ablation) ----
__device__ __forceinline__ void bulk_s2g(void* g, const void* sm, uint32_t bytes) {
    asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;"
                 ::"l"(g), "r"(smem_addr(sm)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void bulk_commit_wait() {
    asm volatile("cp.async.bulk.commit_group;\n\tcp.async.bulk.wait_group 0;" ::: "memory");
}
__device__ __forceinline__ void bulk_g2s(void* sm, const void* g, uint32_t bytes, uint64_t* mbar) {
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                 ::"r"(smem_addr(sm)), "l"(g), "r"(bytes), "r"(smem_addr(mbar)) : "memory");
}
__device__ __forceinline__ void fence_proxy_async_smem() { asm volatile("fence.proxy.async.shared::cta;" ::: "memory"); }
__device__ __forceinline__ void fence_proxy_async_global() { asm volatile("fence.proxy.async.global;" ::: "memory"); }
__device__ __forceinline__ void mbar_init(uint64_t* m) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_addr(m)) : "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t* m, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_addr(m)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* m, uint32_t parity) {
    asm volatile("{ .reg .pred p; W: mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1; @!p bra W; }"
                 ::"r"(smem_addr(m)), "r"(parity) : "memory");
}

__device__ __forceinline__ unsigned long long pack_entry(uint32_t v, uint32_t i) {
    return (unsigned long long)v | ((unsigned long long)i << 32);
}
__device__ __forceinline__ uint32_t entry_v(unsigned long long e) { return (uint32_t)e; }
__device__ __forceinline__ uint32_t entry_i(unsigned long long e) { return (uint32_t)(e >> 32); }

__device__ __forceinline__ uint32_t xorshift32(uint32_t& s) {
    s ^= s << 13; s ^= s >> 17; s ^= s << 5;
    return s;
}

// packed HotRing control word: (head << 16) | tail, 16-bit counters (H <= 2^15)
__device__ __forceinline__ uint32_t ht_head(uint32_t x) { return x >> 16; }
__device__ __forceinline__ uint32_t ht_tail(uint32_t x) { return x & 0xFFFFu; }
__device__ __forceinline__ int ht_rest(uint32_t x) { return (int)(int16_t)(uint16_t)((x >> 16) - (x & 0xFFFFu)); }

// ------------------------------------------------------------------------------------------
// shared-memory control block (one per CTA)
// ------------------------------------------------------------------------------------------
struct SmemCtl {
    uint32_t ht[kMaxWarps];                // HotRing (head << 16) | tail; atomics only
    volatile uint32_t tailf[kMaxWarps];    // 16-bit: slots below tailf are free for reuse
    uint32_t lock[kMaxWarps];              // per-warp lock for tail-side ops (thieves, flush)
    unsigned int warp_mask;                // 1 = warp active
    unsigned int lbusy;                    // warps of this block holding work + registered thieves
    unsigned long long t_start;            // globaltimer at kernel start (watchdog, timeline)
    volatile int done;                     // block-local copy of ctl->done
    uint32_t inter_token;                  // one idle warp per block scans other blocks at a time
    uint64_t mbar[kMaxWarps];              // per-warp mbarrier of the bulk refill (bulk_copy)
    uint32_t mbar_phase[kMaxWarps];        // ... and the parity of its next wait (not a register:
                                           // the 128-wide step runs at the 64-register cap)
    unsigned long long cnt[kMaxWarps][kNumCounters]; // per-warp stats counters (collect_stats)
};

__device__ __forceinline__ void smem_lock(uint32_t* l) {
    while (atom_cas_acquire_cta(l, 0u, 1u) != 0u) { }
}
__device__ __forceinline__ bool smem_trylock(uint32_t* l) { return atom_cas_acquire_cta(l, 0u, 1u) == 0u; }
__device__ __forceinline__ void smem_unlock(uint32_t* l) { st_release_cta(l, 0u); }

// ------------------------------------------------------------------------------------------
// chunk pool: tagged lock-free free stack + bump allocator
// ------------------------------------------------------------------------------------------
// pool_alloc reads the link chunk_next[idx] written by the pool_free that pushed idx: the head
// is read with acquire semantics (pairs with pool_free's fence.release + CAS), so the link read
// is ordered after it; a failed CAS returns the new head, also with acquire semantics.
__device__ __forceinline__ uint32_t pool_alloc(const KParams& P) {
    Ctl* c = P.ctl;
    unsigned long long old = ld_acquire_u64(&c->free_head);
    for (;;) {
        uint32_t idx = (uint32_t)old;
        if (idx == kEmptySlot) break;
        uint32_t nxt = ld_relaxed_u32(&P.chunk_next[idx]);
        unsigned long long nw = ((unsigned long long)((uint32_t)(old >> 32) + 1u) << 32) | nxt;
        unsigned long long got = atom_cas_acquire_u64(&c->free_head, old, nw);
        if (got == old) return idx;
        old = got;
    }
    uint32_t b = atomicAdd(&c->pool_bump, 1u);
    return b < P.n_chunks ? b : kEmptySlot;
}

__device__ __forceinline__ void pool_free(const KParams& P, uint32_t idx) {
    Ctl* c = P.ctl;
    unsigned long long old = ld_relaxed_u64(&c->free_head);
    for (;;) {
        st_relaxed_u32(&P.chunk_next[idx], (uint32_t)old);
        fence_release_gpu();
        unsigned long long nw = ((unsigned long long)((uint32_t)(old >> 32) + 1u) << 32) | idx;
        unsigned long long got = atomicCAS(&c->free_head, old, nw);
        if (got == old) return;
        old = got;
    }
}

__device__ __forceinline__ void raise_error(const KParams& P, int code) {
    atomicCAS(&P.ctl->status, 0, code);
    __threadfence();
    atomicExch(&P.ctl->done, 1u);
}

// bulk flush / refill copies (bulk_copy = 1), compiled only into the BULK instantiations of the
// traversal kernel: inlined into the default kernels they made the 128-wide kernel's hot loop 16%
// slower on RMAT (instruction footprint), and out of line the call ABI forced spills.
// A contiguous piece of a flush or refill is split at the ring wrap and at ColdSeg chunk ends;
// when ring slot and ColdSeg position have equal parity, lane 0 moves the piece's 16-byte-aligned
// middle with one cp.async.bulk and the lanes copy the rest.
template <int H>
__device__ __forceinline__ void bulk_flush_copy(unsigned long long* ring, uint32_t t, uint32_t top, uint32_t kf,
                                             const uint32_t* tab, uint32_t tmask, unsigned long long* pool,
                                             int lane) {
    fence_proxy_async_smem();                         // generic ring writes -> async proxy
    uint32_t r = t, c = top, left = kf;
    bool any_bulk = false;
    while (left) {
        const uint32_t a = H - (r & (H - 1)), b = kChunk - (c & (kChunk - 1));
        const uint32_t L = left < a ? (left < b ? left : b) : (a < b ? a : b);
        const uint32_t ch = ld_relaxed_u32(&tab[(c >> kChunkLog2) & tmask]);
        unsigned long long* gp = pool + ((size_t)ch << kChunkLog2) + (c & (kChunk - 1));
        const unsigned long long* sp = ring + (r & (H - 1));
        uint32_t head = 0, body = 0;
        if (((r ^ c) & 1u) == 0) { head = r & 1u; if (head > L) head = L; body = (L - head) & ~1u; }
        if (body && lane == 0) { bulk_s2g(gp + head, sp + head, body * 8u); any_bulk = true; }
        for (uint32_t q = lane; q < L; q += 32u)
            if (q < head || q >= head + body) st_cg_u64(gp + q, sp[q]);
        r += L; c += L; left -= L;
    }
    if (lane == 0 && any_bulk) { bulk_commit_wait(); fence_proxy_async_global(); }
    __syncwarp();
}

template <int H>
__device__ __forceinline__ void bulk_refill_copy(unsigned long long* ring, uint32_t head0, uint32_t base, uint32_t k,
                                              const uint32_t* tab, uint32_t tmask, const unsigned long long* pool,
                                              int lane, uint64_t* mbar, uint32_t* phase) {
    uint32_t tx = 0;
    for (int pass = 0; pass < 2; ++pass) {            // pass 0: count the bulk bytes, pass 1: issue
        uint32_t r = head0, c = base, left = k;
        if (pass == 1 && tx && lane == 0) mbar_expect_tx(mbar, tx);
        while (left) {
            const uint32_t a = H - (r & (H - 1)), b = kChunk - (c & (kChunk - 1));
            const uint32_t L = left < a ? (left < b ? left : b) : (a < b ? a : b);
            uint32_t head = 0, body = 0;
            if (((r ^ c) & 1u) == 0) { head = r & 1u; if (head > L) head = L; body = (L - head) & ~1u; }
            if (pass == 0) {
                tx += body * 8u;
            } else {
                const uint32_t ch = ld_relaxed_u32(&tab[(c >> kChunkLog2) & tmask]);
                const unsigned long long* gp = pool + ((size_t)ch << kChunkLog2) + (c & (kChunk - 1));
                unsigned long long* sp = ring + (r & (H - 1));
                if (body && lane == 0) bulk_g2s(sp + head, gp + head, body * 8u, mbar);
                for (uint32_t q = lane; q < L; q += 32u)
                    if (q < head || q >= head + body) sp[q] = ld_cg_u64(gp + q);
            }
            r += L; c += L; left -= L;
        }
    }
    if (tx && lane == 0) {
        mbar_wait(mbar, *phase);
        *phase ^= 1u;
    }
    __syncwarp();
}

// ------------------------------------------------------------------------------------------
// The persistent traversal kernel.
//   H   = HotRing entries per warp (power of two, <= 2^15)
//   VEC = neighbours per lane per window (1: 32-wide window; 4: 128-wide, 128-bit loads)
//   WMAX = max warps per block (launch bounds: 32 -> 64 registers, 16 -> 128 registers)
//   STATS = compile the diagnostic counters in
//   BULK = flush/refill with cp.async.bulk (dfs_options.bulk_copy; the paper's TMA variant)
//   CL  = compile the cluster (DSMEM) steal tier in: HotRing publication becomes cluster-visible
//         and idle warps steal from the HotRings of the other CTAs of their thread-block cluster
// Launched with blockDim.x = 32 * W (W <= WMAX) and dynamic shared memory
// sizeof(SmemCtl) (16-byte padded) + W * H * 8 bytes.
// ------------------------------------------------------------------------------------------
template <int H, int VEC, int WMAX, bool STATS, bool CL, bool BULK>
__global__ void __launch_bounds__(32 * WMAX, 1) dfs_persistent_kernel(const KParams P) {
    static_assert((H & (H - 1)) == 0 && H >= 64 && H <= 32768, "H must be a power of two in [64, 2^15]");
    static_assert(VEC == 1 || VEC == 4, "VEC is 1 or 4");
    constexpr uint32_t kBatch = H / 2;              // flush batch (reading S10)
    constexpr uint32_t kWin = 32u * VEC;            // positions per window
    constexpr int kHeadLanes = VEC == 1 ? 8 : 16;   // lanes fetched before a window's end is known
#ifndef DFS_PF_LANES128
#define DFS_PF_LANES128 0
#endif
    // lanes whose candidates' row_ptr pairs are loaded with the probes: the first 8 positions of
    // a 32-wide window; none for 128-wide windows (round 2: on RMAT-24 those speculative loads were
    // 15% of the L2 sector requests and most missed — 0 lanes: 9.76 -> 8.88 ms, DRAM reads 6.46 ->
    // 5.00 GB, profiles/r02/ab/pf_width_rmat.jsonl; DFS_PF_LANES128 = 1/2 rebuilds the old widths)
#ifndef DFS_PF_LANES32
#define DFS_PF_LANES32 8
#endif
    constexpr int kPfLanes = VEC == 1 ? DFS_PF_LANES32 : DFS_PF_LANES128;
    extern __shared__ __align__(16) unsigned char smem_raw[];
    SmemCtl& S = *reinterpret_cast<SmemCtl*>(smem_raw);
    constexpr int kCtlBytes = (sizeof(SmemCtl) + 15) & ~15;
    unsigned long long* const rings = reinterpret_cast<unsigned long long*>(smem_raw + kCtlBytes);
    // HotRing publication (owner -> thieves, lane 0 issues): a CTA-scope release, or made
    // visible to the cluster when the DSMEM steal tier is compiled in
    auto pub_add = [&](bool p, uint32_t* a, uint32_t v) {
        if constexpr (CL) { fence_release_cta_for_cluster(); atom_add_relaxed_cluster_if(p, a, v); }
        else atom_add_release_cta_if(p, a, v);
    };
    const uint32_t crank = CL ? cluster_ctarank() : 0u;     // rank in the thread-block cluster
    const uint32_t ncta = CL ? cluster_nctarank() : 1u;     // CTAs per cluster (1: tier off)

    const int lane = threadIdx.x & 31;
    const int w = threadIdx.x >> 5;
    const int W = blockDim.x >> 5;
    const int gw = blockIdx.x * W + w;
    unsigned long long* const ring = rings + (size_t)w * H;
    const uint32_t tmask = (1u << P.tab_log2) - 1u;
    uint32_t* const my_tab = P.chunk_tab + ((size_t)gw << P.tab_log2);
    const uint32_t hs = P.hot_cutoff >= 2 ? (uint32_t)P.hot_cutoff >> 1 : 1u;   // h_s (Alg 3 l.12)
    const uint32_t cs = P.cold_cutoff >= 2 ? (uint32_t)P.cold_cutoff >> 1 : 1u; // c_s (Alg 4 l.17)

    if (threadIdx.x < kMaxWarps) {
        S.ht[threadIdx.x] = 0; S.tailf[threadIdx.x] = 0; S.lock[threadIdx.x] = 0;
    }
    if (threadIdx.x == 0) {
        S.warp_mask = (blockIdx.x == 0) ? 1u : 0u; S.done = 0; S.inter_token = 0;
        S.lbusy = (blockIdx.x == 0) ? 1u : 0u;        // block 0 / warp 0 holds the root (ctl->busy = 1)
        S.t_start = globaltimer();
    }
    unsigned long long* const cnt = S.cnt[w];     // lane 0 updates its warp's counters
    if (STATS && lane < kNumCounters) cnt[lane] = 0;
    if (BULK && lane == 0) {
        mbar_init(&S.mbar[w]); S.mbar_phase[w] = 0;
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();

    // ---- per-warp state (warp-uniform registers) ----
    bool has_top = false;        // a current top entry <u, i> lives in registers
    bool have_win = false;       // nbv holds the window starting at i
    bool need_end = false;       // end must be re-read from row_ptr
    uint32_t u = 0, i = 0, end = 0;
    int nbv[VEC];                // this lane's neighbours in the current window
#pragma unroll
    for (int e = 0; e < VEC; ++e) nbv[e] = -1;
    uint32_t my_head = 0;        // owner's true HotRing head (16-bit wrap)
    uint32_t pub = 0;            // head value published in S.ht (entries in [pub, my_head) are
                                 // private: pushed/popped without synchronisation)
    bool spec_ok = false;        // speculative claim allowed on the current window (fresh child,
                                 // or a popped entry with speculate & 8)
    uint32_t par = kFull;        // parent of u when spec_ok (kFull: no position to skip)
    // speculate: bits 0-1 = mode (0 off, 1 on, 2 on for 32-wide windows), bit 2 = issue the
    // child's first window before the claim returns (32-wide), bit 3 = also claim a popped
    // entry's next position speculatively (its probe at push time saw it unvisited)
    const bool spec_on = (P.speculate & 3) == 1 || ((P.speculate & 3) == 2 && VEC == 1);
    const bool spec_pop = spec_on && (P.speculate & 8) != 0;
    const bool spec_early = spec_on && (P.speculate & 4) != 0;
    const uint32_t leaf_deg = P.leaf_skip ? 1u : 0u;   // children of degree <= this may be leaves
    uint32_t my_top = 0;         // owner copy of ColdSeg top
    uint32_t hi = 0;             // ColdSeg chunks [.., hi) mapped by this warp
    bool active = false;
    uint32_t rng = P.seed ^ (0x9E3779B9u * (uint32_t)(gw + 1));
    if (rng == 0) rng = 1;
    unsigned long long t_idle0 = 0;
    uint32_t iter = 0;
    uint32_t my_claims = 0;                      // for P.block_claims (Fig 9 task distribution)
    bool unproductive = false;                   // STATS: the top came from a pop and has not
                                                 // claimed yet (dead-pop counter, 32-wide step)
    uint32_t tl_reported = 0;                    // timeline diagnostics
    unsigned long long tl_win_reported = 0;

    if (blockIdx.x == 0 && w == 0) {
        // Alg 1 l.1-3: root claimed by the reset kernel; <root, row_ptr[root]> is our top
        has_top = true; active = true;
        u = (uint32_t)P.root; i = __ldg(P.rp + u); end = __ldg(P.rp + u + 1);
    }

    // window loader: lane holds positions base + VEC*lane + e, e < VEC (col_idx entries; one
    // 128-bit load per lane when VEC = 4).  Lanes outside [lane_lo, lanes) or past `limit` skip.
    auto load_window = [&](uint32_t base, uint32_t limit, int lanes, int* nb, int lane_lo = 0) {
        const uint32_t q = base + (uint32_t)VEC * lane;
        const bool ld = lane >= lane_lo && lane < lanes && q < limit;
        if constexpr (VEC == 4) {
            int4 x = make_int4(-1, -1, -1, -1);
            if (ld) x = __ldg(reinterpret_cast<const int4*>(P.col + q));    // col padded
            nb[0] = x.x; nb[1] = x.y; nb[2] = x.z; nb[3] = x.w;
        } else {
            nb[0] = (int)ld_nc_if(ld, P.col + q, kFull);
        }
    };
    // lanes of the current window that hold data (the rest are loaded on demand)
    int win_lanes = 32;

    // ---------------------------------------------------------------- owner stack operations
    // publish the private entries [pub, my_head) to thieves (CTA-scope release)
    auto publish = [&]() {
        if (my_head != pub) {
            pub_add(lane == 0, &S.ht[w], ((my_head - pub) & 0xFFFFu) << 16);
            pub = my_head;
        }
    };

    // flush: move up to `want` of the oldest HotRing entries to ColdSeg top, keeping at least
    // `keep` in the ring (Fig 2(e): want = batch, keep = 0 when the ring is full;
    // the demand-driven spill uses want = keep = rest/2)
    auto flush = [&](uint32_t want, uint32_t keep) -> bool {
        publish();
        uint32_t t = 0;
        if (lane == 0) { smem_lock(&S.lock[w]); t = ht_tail(ld_acquire_cta(&S.ht[w])); }
        t = __shfl_sync(kFull, t, 0);
        __syncwarp();                                 // ring entries written by lane 0 -> all lanes
        const uint32_t rest = (my_head - t) & 0xFFFFu;
        uint32_t kf = rest > keep ? rest - keep : 0u;
        if (kf > want) kf = want;
        if (kf == 0) {
            if (lane == 0) smem_unlock(&S.lock[w]);
            __syncwarp();
            return true;
        }
        // map chunks covering [my_top, my_top + kf)
        bool ok = true;
        while (ok && (unsigned long long)hi * kChunk < (unsigned long long)my_top + kf) {
            uint32_t c = 0;
            if (lane == 0) {
                c = pool_alloc(P);
                if (c != kEmptySlot) {
                    uint32_t* slot = &my_tab[hi & tmask];
                    unsigned long long spins = 0;
                    while (ld_relaxed_u32(slot) != kEmptySlot) {   // chunk hi - 2^tab_log2 still read
                        if (++spins > (1ull << 26)) { c = kEmptySlot; break; }
                        __nanosleep(64);
                    }
                    if (c != kEmptySlot) {
                        st_relaxed_u32(&P.chunk_consumed[c], 0u);
                        st_relaxed_u32(slot, c);
                    }
                }
            }
            c = __shfl_sync(kFull, c, 0);
            if (c == kEmptySlot) ok = false; else { ++hi; if (STATS && lane == 0) ++cnt[kCntChunks]; }
        }
        if (!ok) {
            if (lane == 0) { raise_error(P, kStatusENOMEM); smem_unlock(&S.lock[w]); }
            __syncwarp();
            return false;
        }
        if constexpr (BULK) {
            bulk_flush_copy<H>(ring, t, my_top, kf, my_tab, tmask, P.pool, lane);
        } else {
            // warp copy, one 8-byte entry per lane per step
            for (uint32_t q = lane; q < kf; q += 32u) {
                const unsigned long long e = ring[(t + q) & (H - 1)];
                const uint32_t p = my_top + q;
                const uint32_t c = ld_relaxed_u32(&my_tab[(p >> kChunkLog2) & tmask]);
                st_cg_u64(P.pool + ((size_t)c << kChunkLog2) + (p & (kChunk - 1)), e);
            }
        }
        fence_release_gpu();                          // every lane: its stores before the publish
        __syncwarp();
        if (lane == 0) {
            atomicAdd(&P.cold_tb[gw], (unsigned long long)kf << 32);       // publish top
            atomicAdd(&P.block_cold[blockIdx.x], (int)kf);
            // advance tail (thieves are locked out; head is ours)
            uint32_t old = ld_acquire_cta(&S.ht[w]);
            for (;;) {
                const uint32_t nw = (old & 0xFFFF0000u) | ((t + kf) & 0xFFFFu);
                const uint32_t got = atom_cas_acquire_cta(&S.ht[w], old, nw);
                if (got == old) break;
                old = got;
            }
            S.tailf[w] = (t + kf) & 0xFFFFu;
            smem_unlock(&S.lock[w]);
        }
        __syncwarp();
        my_top += kf;
        if (STATS && lane == 0) ++cnt[kCntFlushes];
        return true;
    };

    // push <v, idx> at head (Fig 2(c)); flushes first when full
    auto push = [&](uint32_t v, uint32_t idx) -> bool {
        int full = 0;
        if (lane == 0) full = ((my_head - S.tailf[w]) & 0xFFFFu) >= P.ring_cap;
        if (__shfl_sync(kFull, full, 0)) {
            if (!flush(P.ring_cap >= 2u ? P.ring_cap / 2u : 1u, 0u)) return false;
        }
        if (lane == 0) ring[my_head & (H - 1)] = pack_entry(v, idx);
        ++my_head;
        if (((my_head - pub) & 0xFFFFu) >= P.pub_batch) publish();
        return true;
    };

    // lean push (32-wide step): the ring-full test uses a register copy of tailf, refreshed only
    // when the copy says full — tailf only grows, so a stale copy is conservative; lane 0 stores
    // the entry and publishes with predicated instructions
    uint32_t tail_cache = 0;
    auto push_lean = [&](uint32_t v, uint32_t idx) -> bool {
        if (((my_head - tail_cache) & 0xFFFFu) >= P.ring_cap) {
            tail_cache = __shfl_sync(kFull, S.tailf[w], 0);
            if (((my_head - tail_cache) & 0xFFFFu) >= P.ring_cap) {
                if (!flush(P.ring_cap >= 2u ? P.ring_cap / 2u : 1u, 0u)) return false;
                tail_cache = __shfl_sync(kFull, S.tailf[w], 0);
            }
        }
        st_shared_u64_if(lane == 0, ring + (my_head & (H - 1)), pack_entry(v, idx));
        ++my_head;
        if (((my_head - pub) & 0xFFFFu) >= P.pub_batch) {
            pub_add(lane == 0, &S.ht[w], ((my_head - pub) & 0xFFFFu) << 16);
            pub = my_head;
        }
        return true;
    };

    // pop the newest HotRing entry (Fig 2(d)).  A private entry needs no synchronisation; at
    // the published head one atomic decrement resolves the race with tail-side thieves (their
    // CAS fails if the word changed)
    auto pop = [&](uint32_t& v, uint32_t& idx) -> bool {
        unsigned long long e = 0;
        int got = 0;
        if (my_head != pub) {
            if (lane == 0) e = ring[(my_head - 1u) & (H - 1)];
            e = __shfl_sync(kFull, e, 0);
            --my_head;
            v = entry_v(e); idx = entry_i(e);
            return true;
        }
        if (lane == 0) {
            const uint32_t old = atom_add_relaxed_cta(&S.ht[w], 0xFFFF0000u);   // head--
            if (ht_rest(old) >= 1) { e = ring[(ht_head(old) - 1u) & (H - 1)]; got = 1; }
            else atom_add_relaxed_cta(&S.ht[w], 0x10000u);                       // empty: undo
        }
        got = __shfl_sync(kFull, got, 0);
        if (!got) return false;
        e = __shfl_sync(kFull, e, 0);
        --my_head; --pub;
        v = entry_v(e); idx = entry_i(e);
        return true;
    };

    // refill from ColdSeg top when the HotRing is empty (Fig 2(f))
    auto refill = [&]() -> uint32_t {
        uint32_t k = 0;
        if (lane == 0) {
            unsigned long long old = ld_relaxed_u64(&P.cold_tb[gw]);
            for (;;) {
                const uint32_t bot = (uint32_t)old;
                const int avail = (int)(my_top - bot);
                if (avail <= 0) { k = 0; break; }
                k = avail < (int)kBatch ? (uint32_t)avail : kBatch;
                const unsigned long long nw = ((unsigned long long)(my_top - k) << 32) | bot;
                const unsigned long long got = atomicCAS(&P.cold_tb[gw], old, nw);
                if (got == old) break;
                old = got;
            }
        }
        k = __shfl_sync(kFull, k, 0);
        if (k == 0) return 0;
        const uint32_t base = my_top - k;
        // ring is empty (my_head == tail); place entries oldest first
        if constexpr (BULK) {
            bulk_refill_copy<H>(ring, my_head, base, k, my_tab, tmask, P.pool, lane, &S.mbar[w], &S.mbar_phase[w]);
        } else {
            for (uint32_t q = lane; q < k; q += 32u) {
                const uint32_t p = base + q;
                const uint32_t c = ld_relaxed_u32(&my_tab[(p >> kChunkLog2) & tmask]);
                ring[(my_head + q) & (H - 1)] = ld_cg_u64(P.pool + ((size_t)c << kChunkLog2) + (p & (kChunk - 1)));
            }
        }
        my_top = base;
        // release chunks that lie wholly above top + one spare chunk (never read by thieves)
        while (hi > 0 && (unsigned long long)(hi - 1) * kChunk >= (unsigned long long)my_top + kChunk) {
            if (lane == 0) {
                uint32_t* slot = &my_tab[(hi - 1) & tmask];
                const uint32_t c = ld_relaxed_u32(slot);
                st_relaxed_u32(slot, kEmptySlot);
                pool_free(P, c);
            }
            --hi;
        }
        __syncwarp();
        if (lane == 0) {
            atomicSub(&P.block_cold[blockIdx.x], (int)k);
        }
        pub_add(lane == 0, &S.ht[w], k << 16);                    // publish (ring was empty)
        my_head += k; pub = my_head;
        if (STATS && lane == 0) ++cnt[kCntRefills];
        return k;
    };

    auto set_done_local = [&]() {
        if (lane == 0) S.done = 1;
    };
    // termination counters (reading S13), lane 0 only.  A warp registers BEFORE it reserves
    // stolen work and deregisters when it holds none; the block's count going 0->1 / 1->0 adds /
    // removes the block from the global count.  When a count goes 0->1 the registering warp is an
    // inter-block thief whose victim's block is still counted, so the global count cannot reach 0
    // while any entry exists; the global increment's result is consumed before the reservation
    // is attempted (completion order).
    auto register_thief = [&]() {
        if (atomicAdd(&S.lbusy, 1u) == 0u) {
            if (atomicAdd(&P.ctl->busy, 1u) == 0xFFFFFFFFu) raise_error(P, kStatusEINTERNAL);
        }
    };
    auto deregister = [&]() {      // lane 0: leave the busy count; the last one raises done
        if (atomicSub(&S.lbusy, 1u) == 1u) {
            if (atomicSub(&P.ctl->busy, 1u) == 1u) { atomicExch(&P.ctl->done, 1u); S.done = 1; }
        }
    };

    // diagnostics: block 0 / warp 0 samples the busy-block counter every timeline_dt_ns
    unsigned int tl_next = 0;
    auto sample = [&]() {
        if (P.timeline && blockIdx.x == 0 && w == 0 && lane == 0) {
            const unsigned long long now = globaltimer() - S.t_start;
            const unsigned int slot = (unsigned int)(now / P.timeline_dt_ns);
            // timeline_len = 2 * (buffer length / 3): busy samples, claims, then (STATS) windows
            if (slot >= tl_next && slot < P.timeline_len / 2) {
                P.timeline[slot] = *(volatile unsigned int*)&P.ctl->busy + 1u;   // 0 = no sample
                P.timeline[P.timeline_len / 2 + slot] =
                    (unsigned int)*(volatile unsigned long long*)&P.ctl->claims_progress;
                if (STATS)
                    P.timeline[P.timeline_len + slot] =
                        (unsigned int)*(volatile unsigned long long*)&P.ctl->windows_progress;
                tl_next = slot + 1;
            }
        }
    };

    // cluster tier: Alg 3 over distributed shared memory — the peer HotRing with
    // max hot_rest >= hot_cutoff among the other CTAs of the thread-block cluster; same
    // reservation protocol (victim lock + CAS on the packed head/tail word), the entries move
    // SM-to-SM without touching global memory.  Returns true with the entries in our ring.
    auto cluster_steal = [&]() -> bool {
        if constexpr (CL) {
            if (!P.intra || ncta < 2) return false;
            int best = -1, bw = 0;
            uint32_t bp = 0;
            for (uint32_t d = 1; d < ncta; ++d) {
                const uint32_t pr = (crank + d) % ncta;
                int rest = -1;
                if (lane < W) rest = ht_rest(dsmem_ld_u32(dsmem_map(&S.ht[lane], pr)));
                const int b = __reduce_max_sync(kFull, rest);
                if (b > best) { best = b; bp = pr; bw = __ffs(__ballot_sync(kFull, rest == b)) - 1; }
            }
            if (best >= P.hot_cutoff) {
                if (STATS && lane == 0) ++cnt[kCntStealAttempts];
                const uint32_t rlock = dsmem_map(&S.lock[bw], bp);
                const uint32_t rht = dsmem_map(&S.ht[bw], bp);
                uint32_t ok = 0, t = 0, kst = 0;
                if (lane == 0) {
                    if (dsmem_cas_u32(rlock, 0u, 1u) == 0u) {
                        fence_acquire_cluster_smem();
                        register_thief();                        // before reserving
                        uint32_t old = dsmem_ld_u32(rht);
                        for (int tries = 0; tries < 8; ++tries) {
                            const int r = ht_rest(old);
                            if (r < P.hot_cutoff) break;
                            t = ht_tail(old);
                            kst = hs;
                            if (P.steal_half && (uint32_t)(r / 2) > kst) kst = (uint32_t)(r / 2);
                            if (kst > 32u) kst = 32u;
                            if ((int)kst > r) kst = (uint32_t)r;
                            const uint32_t nw = (old & 0xFFFF0000u) | ((t + kst) & 0xFFFFu);
                            const uint32_t got = dsmem_cas_u32(rht, old, nw);   // reserve
                            if (got == old) { ok = 1; break; }
                            old = got;
                        }
                        fence_acquire_cluster_smem();            // entries published before `old`
                        if (!ok) { dsmem_st_release_u32(rlock, 0u); deregister(); }
                    }
                }
                ok = __shfl_sync(kFull, ok, 0);
                if (ok) {
                    t = __shfl_sync(kFull, t, 0);
                    kst = __shfl_sync(kFull, kst, 0);
                    __syncwarp();                                // lane 0's acquire -> all lanes
                    if (lane < (int)kst)
                        ring[(my_head + lane) & (H - 1)] =
                            dsmem_ld_u64(dsmem_map(rings + (size_t)bw * H + ((t + lane) & (H - 1)), bp));
                    __syncwarp();
                    if (lane == 0) {
                        dsmem_st_u32(dsmem_map((const void*)&S.tailf[bw], bp), (t + kst) & 0xFFFFu);
                        dsmem_st_release_u32(rlock, 0u);        // copies done before unlock
                        atomicOr(&S.warp_mask, 1u << w);
                    }
                    pub_add(lane == 0, &S.ht[w], kst << 16);     // publish into our ring
                    __syncwarp();
                    my_head += kst; pub = my_head;
                    if (STATS && lane == 0) ++cnt[kCntClusterSteals];
                    return true;
                }
            }
        }
        return false;
    };

    // ---------------------------------------------------------------- main loop (Alg 2)
    for (;;) {
        if (has_top) {
          if constexpr (VEC == 1) {
            // ===== lean 32-wide expansion step (Alg 1 l.5-12 over one window) =====
            // Lane k holds position i + k (col_idx entry nb); positions >= end are masked.  The
            // common case — a freshly descended child whose first non-parent neighbour is
            // unvisited — runs without any lane-0 branch: the speculative claim, the parent
            // store, the ring store and the publication are predicated single instructions.
            if (!have_win || win_lanes < 32) {
                if (!have_win) {
                    if (need_end) {                                   // popped entry: end unknown
                        const uint32_t e2 = __ldg(P.rp + u + 1);
                        nbv[0] = (int)ld_nc_if(lane < kHeadLanes && i + lane < P.m, P.col + i + lane, kFull);
                        win_lanes = kHeadLanes;
                        end = e2; need_end = false;
                    } else {
                        nbv[0] = (int)ld_nc_if(i + lane < end, P.col + i + lane, kFull);
                        win_lanes = 32;
                    }
                    have_win = true;
                }
                if (win_lanes < 32) {
                    if (end > i + (uint32_t)win_lanes) {
                        const int t = (int)ld_nc_if(lane >= win_lanes && i + lane < end, P.col + i + lane, kFull);
                        if (lane >= win_lanes) nbv[0] = t;
                    }
                    win_lanes = 32;
                }
            }
            if (STATS && lane == 0) ++cnt[kCntWindows];
            const int nb = nbv[0];
            const bool valid = i + (uint32_t)lane < end;
            // long list (hubs): the next window is in flight while this one's probes resolve
            const bool have_nxt = i + 32u < end;
            const int nxt1 = (int)ld_nc_if(have_nxt && i + 32u + lane < end, P.col + i + 32u + lane, kFull);
            // speculative claim (fresh child only): the first position whose neighbour is not the
            // parent we came from is, if unvisited, exactly Alg 1's next tree edge
            const uint32_t vb = __ballot_sync(kFull, spec_ok && valid && (uint32_t)nb != par);
            const int sk = __ffs(vb) - 1;
            const uint32_t sv = vb ? (uint32_t)__shfl_sync(kFull, nb, sk & 31) : u;
            uint32_t s_old = atom_or_if(vb != 0 && lane == 0, P.bitmap + 2u * (sv >> 5), 1u << (sv & 31));
            const uint32_t s_rs = ld_nc_if(vb != 0, P.rp + sv, 0u), s_re = ld_nc_if(vb != 0, P.rp + sv + 1, 0u);
            // probe the visited bits; lanes holding the first 8 positions prefetch their
            // candidates' row_ptr pairs
            const uint2 wl = ld_cg_u2_if(valid, P.bitmap + 2u * ((uint32_t)nb >> 5), kFull, 0u);   // {visited, leaf}
            const bool pf = valid && lane < kPfLanes;
            const uint32_t prs = ld_nc_if(pf, P.rp + nb, 0u), pre = ld_nc_if(pf, P.rp + nb + 1, 0u);
            // early child window (speculate & 4): issued once the row_ptr pair arrives, before
            // the claim returns (the probes are already in flight)
            int cnb = (int)ld_nc_if(spec_early && vb != 0 && s_rs + lane < s_re, P.col + s_rs + lane, kFull);
            const bool unv = valid && !((wl.x >> (nb & 31)) & 1u) && lane != sk;   // sk is claimed either way
            const bool lf = unv && ((wl.y >> (nb & 31)) & 1u);
            bool cand = unv && !lf;
            // bulk leaf claims (leaf_skip = 2): every unvisited leaf candidate of the window is
            // claimed at once, in parallel with the claim of the next tree edge — each is exactly
            // Alg 1's descend-and-pop-back (a leaf's only in-list is u's, reading S24)
            // No other list holds a leaf and this warp is the only scanner of u's list, so the
            // probe's "unvisited" cannot change before the claim: a fire-and-forget red.or sets
            // the bit (the step does not wait for it) and the parent is u in every order.
            if (__any_sync(kFull, lf)) {
                if (STATS) unproductive = false;
                red_or_if(lf, P.bitmap + 2u * ((uint32_t)nb >> 5), 1u << (nb & 31));
                st_global_if(lf, P.parent + nb, (int32_t)u);                    // Alg 1 l.10
                if (STATS || P.block_claims || P.timeline) {
                    const uint32_t nl = __popc(__ballot_sync(kFull, lf));
                    my_claims += nl;
                    if (STATS && lane == 0) cnt[kCntClaims] += nl;
                }
            }
            s_old = __shfl_sync(kFull, s_old, 0);
            bool won = vb != 0 && !(s_old & (1u << (sv & 31)));
            uint32_t v = sv, vrs = s_rs, vre = s_re;
            int kpos = sk;
            if (won) {
                if (!spec_early) cnb = (int)ld_nc_if(vrs + lane < vre, P.col + vrs + lane, kFull);
            } else {
                if (STATS && vb && lane == 0) ++cnt[kCntFailedClaims];
                // claim the first unvisited candidate in CSR order; on a lost race try the next
                uint32_t any = __ballot_sync(kFull, cand);
                while (any) {
                    const int k = __ffs(any) - 1;
                    const uint32_t cv = (uint32_t)__shfl_sync(kFull, nb, k);
                    uint32_t crs = __shfl_sync(kFull, prs, k & (kPfLanes - 1)), cre = __shfl_sync(kFull, pre, k & (kPfLanes - 1));
                    if (k >= kPfLanes) { crs = __ldg(P.rp + cv); cre = __ldg(P.rp + cv + 1); }
                    const uint32_t bit = 1u << (cv & 31);
                    uint32_t old = atom_or_if(lane == 0, P.bitmap + 2u * (cv >> 5), bit);
                    cnb = (int)ld_nc_if(crs + lane < cre, P.col + crs + lane, kFull);   // overlaps the claim
                    old = __shfl_sync(kFull, old, 0);
                    if (!(old & bit)) { won = true; v = cv; vrs = crs; vre = cre; kpos = k; break; }
                    if (STATS && lane == 0) ++cnt[kCntFailedClaims];
                    if (lane == k) cand = false;                  // lost the race: next candidate
                    any = __ballot_sync(kFull, cand);
                }
            }
            uint32_t next_i = i + 32u;                            // u's scan resumes here
            bool advance = !won;
            if (won) {
                if (STATS) unproductive = false;
                // descend (Alg 1 l.8-11): push <u, next candidate> unless u is exhausted —
                // positions whose probe saw a claimed target stay claimed, so skipping them keeps
                // Alg 1's order — then v becomes the register top with its first window loaded
                if (STATS && lane == 0) ++cnt[kCntClaims];
                ++my_claims;
                const uint32_t later = __ballot_sync(kFull, cand && lane > kpos);
                const uint32_t ni = later ? i + (uint32_t)(__ffs(later) - 1) : i + 32u;
                st_global_if(lane == 0, P.parent + v, (int32_t)u);             // Alg 1 l.10
                // leaf skip: v's list is empty or exactly [u] — Alg 1 would descend, find
                // nothing unvisited and pop straight back to <u, ni>; stay on u instead
                if (vre - vrs <= leaf_deg && (vre == vrs || (uint32_t)__shfl_sync(kFull, cnb, 0) == u)) {
                    next_i = ni; advance = true;
                } else {
                    if (ni < end) {
                        if (!push_lean(u, ni)) goto exit_loop;
                    }
                    par = u;
                    u = v; i = vrs; end = vre; spec_ok = spec_on;
                    nbv[0] = cnb; win_lanes = 32;                      // have_win stays true
                }
            }
            if (advance) {
                // continue u's scan at next_i: shift the window down when it still overlaps
                // (leaf skip), take the prefetched next window, or pop when u is exhausted
                const uint32_t d = next_i - i;
                i = next_i;
                if (i < end && d < 32u) {
                    int x = __shfl_down_sync(kFull, nb, d);
                    const int y = (int)ld_nc_if(lane >= 32 - (int)d && i + lane < end, P.col + i + lane, kFull);
                    nbv[0] = lane >= 32 - (int)d ? y : x;
                    spec_ok = spec_on; par = kFull;               // next position: claim at once
                } else if (have_nxt) {                            // next window already loaded
                    nbv[0] = nxt1;
                    spec_ok = false;
                } else {
                    have_win = false;                             // i >= end: Alg 1 l.14: pop
                    if (STATS && lane == 0) { ++cnt[kCntPops]; if (unproductive) ++cnt[kCntDeadPops]; }
                    has_top = pop(u, i);
                    if (STATS) unproductive = true;
                    need_end = true;
                    spec_ok = spec_pop; par = kFull;
                }
            }
          } else {
            // ===== lean expansion step (Alg 1 l.5-12 over one window) =====
            // Window = positions [a, a + kWin), a = i rounded down to a multiple of VEC; lane k
            // holds positions a+VEC*k .. a+VEC*k+VEC-1 (col_idx entries); positions outside
            // [i, end) are masked.  A popped entry's window is fetched together with its end
            // offset for the first kHeadLanes lanes and completed only if the list is longer.
            // The common case — a claim that wins — runs without lane-0 branches: the claim, the
            // parent store, the ring store and the publication are predicated instructions.
            const uint32_t a = i & ~(uint32_t)(VEC - 1);
            if (!have_win || win_lanes < 32) {
                if (!have_win) {
                    if (need_end) {                                   // popped entry: end unknown
                        const uint32_t e2 = __ldg(P.rp + u + 1);
                        load_window(a, P.m, kHeadLanes, nbv);
                        win_lanes = kHeadLanes;
                        end = e2; need_end = false;
                    } else {
                        load_window(a, end, 32, nbv);
                        win_lanes = 32;
                    }
                    have_win = true;
                }
                if (win_lanes < 32) {
                    if (end > a + (uint32_t)VEC * (uint32_t)win_lanes) {
                        int tnb[VEC];
                        load_window(a, end, 32, tnb, win_lanes);
                        if (lane >= win_lanes) {
#pragma unroll
                            for (int f = 0; f < VEC; ++f) nbv[f] = tnb[f];
                        }
                    }
                    win_lanes = 32;
                }
            }
            if (STATS && lane == 0) ++cnt[kCntWindows];
            const uint32_t q0 = a + (uint32_t)VEC * lane;
            uint32_t vm = 0;                                      // valid elements of this lane
#pragma unroll
            for (int e = 0; e < VEC; ++e)
                if (q0 + e >= i && q0 + e < end) vm |= 1u << e;
            // long list (hubs): the next window is pulled into L1 while this one's probes
            // resolve (a prefetch holds no registers; the window is loaded when it is reached)
            const bool have_nxt = a + kWin < end;
#ifndef DFS_NEXTWIN_PF
#define DFS_NEXTWIN_PF 1
#endif
            if (DFS_NEXTWIN_PF && have_nxt && a + kWin + (uint32_t)VEC * lane < end)
                asm volatile("prefetch.global.L1 [%0];" ::"l"(P.col + a + kWin + (uint32_t)VEC * lane));
            // speculative claim: the first valid position whose neighbour is not the parent we
            // came from (par = kFull: none to skip) is, if unvisited, exactly Alg 1's next tree
            // edge; its claim and row_ptr pair are issued before the probes
            uint32_t sm = 0;
            if (spec_ok) {
#pragma unroll
                for (int e = 0; e < VEC; ++e)
                    if (((vm >> e) & 1u) && (uint32_t)nbv[e] != par) sm |= 1u << e;
            }
            const uint32_t vb = __ballot_sync(kFull, sm != 0);
            const int sk = __ffs(vb) - 1;
            int se = 0;
            uint32_t sv = u;
            if (vb) {
                if constexpr (VEC == 1) {
                    sv = (uint32_t)__shfl_sync(kFull, nbv[0], sk);
                } else {
                    se = __ffs(__shfl_sync(kFull, sm, sk)) - 1;
                    int pick = nbv[0];
#pragma unroll
                    for (int f = 1; f < VEC; ++f) if (se == f) pick = nbv[f];
                    sv = (uint32_t)__shfl_sync(kFull, pick, sk);
                }
            }
            // probe the visited bits; the lanes holding the first 8 positions also prefetch
            // their candidates' row_ptr pairs.  All loads are issued before the speculative
            // claim: its result may be spilled, and a spill store waits for the atomic
            uint32_t cm = 0;                                      // unvisited candidates
            uint32_t lcm = 0;                                     // ... that are leaves
            uint32_t prs[VEC], pre[VEC];
            uint2 wl[VEC];
#pragma unroll
            for (int e = 0; e < VEC; ++e) {
                const bool ok = (vm >> e) & 1u;
                const uint32_t x = (uint32_t)nbv[e];
                wl[e] = ld_cg_u2_if(ok, P.bitmap + 2u * (x >> 5), kFull, 0u);   // {visited, leaf}
                const bool pf = ok && lane < kPfLanes;
                prs[e] = ld_nc_if(pf, P.rp + x, 0u); pre[e] = ld_nc_if(pf, P.rp + x + 1, 0u);
            }
            const uint32_t s_rs = ld_nc_if(vb != 0, P.rp + sv, 0u), s_re = ld_nc_if(vb != 0, P.rp + sv + 1, 0u);
            uint32_t s_old = atom_or_if(vb != 0 && lane == 0, P.bitmap + 2u * (sv >> 5), 1u << (sv & 31));
#pragma unroll
            for (int e = 0; e < VEC; ++e) {
                const uint32_t x = (uint32_t)nbv[e];
                if (((vm >> e) & 1u) && !((wl[e].x >> (x & 31)) & 1u)) {
                    if ((wl[e].y >> (x & 31)) & 1u) lcm |= 1u << e; else cm |= 1u << e;
                }
            }
            if (lane == sk) { cm &= ~(1u << se); lcm &= ~(1u << se); }   // claimed either way
            // bulk leaf claims (leaf_skip = 2, 128-wide windows): every unvisited leaf candidate
            // of the window is claimed at once — each is exactly Alg 1's descend-and-pop-back
            // (a leaf's only in-list is u's, so its parent is u in any order)
            // (fire-and-forget red.or: no other list holds a leaf and this warp is the only
            // scanner of u's list, so the probe's "unvisited" still holds — see the 32-wide step)
            if (__any_sync(kFull, lcm != 0)) {
                uint32_t nl = 0;
#pragma unroll
                for (int e = 0; e < VEC; ++e) {
                    const bool lf = (lcm >> e) & 1u;
                    red_or_if(lf, P.bitmap + 2u * ((uint32_t)nbv[e] >> 5), 1u << (nbv[e] & 31));
                    st_global_if(lf, P.parent + nbv[e], (int32_t)u);             // Alg 1 l.10
                    nl += lf;
                }
                if (STATS || P.block_claims || P.timeline) {
                    nl = __reduce_add_sync(kFull, nl);
                    my_claims += nl;
                    if (STATS && lane == 0) cnt[kCntClaims] += nl;
                }
            }
            s_old = __shfl_sync(kFull, s_old, 0);
            bool won = vb != 0 && !(s_old & (1u << (sv & 31)));
            if (STATS && vb && !won && lane == 0) ++cnt[kCntFailedClaims];
            uint32_t v = sv, vrs = s_rs, vre = s_re;
            int kl = sk, ke = se;                                 // window slot of v
            int cnb[VEC];
            if (won) load_window(vrs & ~(uint32_t)(VEC - 1), vre, 32, cnb);
            for (;;) {
                if (won) {
                    // leaf skip: v's list is empty or exactly [u] — Alg 1 would descend, find
                    // nothing unvisited and pop straight back to <u, next>; record the tree edge
                    // and go on with u's window (its probes are still valid: claims are monotone)
                    bool leaf = vre == vrs;
                    if (P.leaf_skip && vre == vrs + 1u) {
                        int first = cnb[0];
                        if constexpr (VEC == 4) {                // selects, not a local-memory index
                            const uint32_t sel = vrs & 3u;
                            first = sel == 0u ? cnb[0] : (sel == 1u ? cnb[1] : (sel == 2u ? cnb[2] : cnb[3]));
                        }
                        leaf = (uint32_t)__shfl_sync(kFull, first, 0) == u;
                    }
                    if (!(leaf && P.leaf_skip)) break;
                    st_global_if(lane == 0, P.parent + v, (int32_t)u);     // Alg 1 l.10
                    ++my_claims;
                    if (STATS && lane == 0) ++cnt[kCntClaims];
                    won = false;
                    // only candidates after v's slot remain (those before it were taken)
                    cm = lane > kl ? cm : (lane == kl ? (cm & ~((2u << ke) - 1u)) : 0u);
                }
                // claim the first unvisited candidate in CSR order; on a lost race, the next
                const uint32_t any = __ballot_sync(kFull, cm != 0);
                if (!any) break;
                const int k = __ffs(any) - 1;
                int e = 0;
                int mine_nb = nbv[0];
                uint32_t mine_rs = prs[0], mine_re = pre[0];
                if constexpr (VEC > 1) {
                    e = __ffs(__shfl_sync(kFull, cm, k)) - 1;
#pragma unroll
                    for (int f = 1; f < VEC; ++f)
                        if (e == f) { mine_nb = nbv[f]; mine_rs = prs[f]; mine_re = pre[f]; }
                }
                const uint32_t cv = (uint32_t)__shfl_sync(kFull, mine_nb, k);
                uint32_t crs = __shfl_sync(kFull, mine_rs, k & (kPfLanes - 1));
                uint32_t cre = __shfl_sync(kFull, mine_re, k & (kPfLanes - 1));
                if (k >= kPfLanes) { crs = __ldg(P.rp + cv); cre = __ldg(P.rp + cv + 1); }
                const uint32_t bit = 1u << (cv & 31);
                uint32_t old = atom_or_if(lane == 0, P.bitmap + 2u * (cv >> 5), bit);
                load_window(crs & ~(uint32_t)(VEC - 1), cre, 32, cnb);   // overlaps the claim
                old = __shfl_sync(kFull, old, 0);
                if (!(old & bit)) { won = true; v = cv; vrs = crs; vre = cre; kl = k; ke = e; continue; }
                if (STATS && lane == 0) ++cnt[kCntFailedClaims];
                if (lane == k) cm &= ~(1u << e);                  // lost the race: next candidate
            }
            if (won) {
                // descend (Alg 1 l.8-11): push <u, next candidate> unless u is exhausted —
                // positions whose probe saw a claimed target stay claimed, so skipping them keeps
                // Alg 1's order — then v becomes the register top with its first window loaded
                if (STATS && lane == 0) ++cnt[kCntClaims];
                ++my_claims;
                const uint32_t mine = lane > kl ? cm : (lane == kl ? (cm & ~((2u << ke) - 1u)) : 0u);
                const uint32_t later = __ballot_sync(kFull, mine != 0);
                uint32_t ni = a + kWin;
                if (later) {
                    const int k2 = __ffs(later) - 1;
                    if constexpr (VEC == 1) {
                        ni = a + (uint32_t)k2;
                    } else {
                        const uint32_t m2 = __shfl_sync(kFull, mine, k2);
                        ni = a + (uint32_t)VEC * (uint32_t)k2 + (uint32_t)(__ffs(m2) - 1);
                    }
                }
                if (ni < end) {
                    if (!push_lean(u, ni)) goto exit_loop;
                }
                st_global_if(lane == 0, P.parent + v, (int32_t)u);             // Alg 1 l.10
                par = u;
                u = v; i = vrs; end = vre; spec_ok = spec_on;
                have_win = true; need_end = false; win_lanes = 32;
#pragma unroll
                for (int f = 0; f < VEC; ++f) nbv[f] = cnb[f];
            } else {
                i = a + kWin;
                spec_ok = false;
                if (have_nxt) {                                   // next window (prefetched)
                    load_window(i, end, 32, nbv);
                } else {
                    have_win = false;                             // i >= end: Alg 1 l.14: pop
                    has_top = pop(u, i);
                    need_end = true;
                    spec_ok = spec_pop; par = kFull;
                }
            }
          }   // VEC == 4 step
            // periodic work, one branch per step: diagnostics and the spill check every
            // spill_period (power of two <= 1024) steps, the done flag and the watchdog every 1024
            if ((++iter & P.period_mask) == 0) {
                if (P.timeline && lane == 0) {                    // diagnostics: claim progress
                    atomicAdd(&P.ctl->claims_progress, (unsigned long long)(my_claims - tl_reported));
                    tl_reported = my_claims;
                    if (STATS) {
                        atomicAdd(&P.ctl->windows_progress, cnt[kCntWindows] - tl_win_reported);
                        tl_win_reported = cnt[kCntWindows];
                    }
                }
                sample();
                if (P.spill) {
                    // demand-driven spill: many warps idle and a deep HotRing -> make the oldest
                    // half of it visible to other blocks (Alg 4 steals ColdSeg bottoms only)
                    uint32_t want = 0;
                    if (lane == 0) {
                        const uint32_t rest = (my_head - ht_tail(ld_acquire_cta(&S.ht[w]))) & 0xFFFFu;
                        if (rest >= 2u * (uint32_t)P.cold_cutoff) {
                            // idle warps elsewhere ~ W x (blocks with no busy warp)
                            const uint32_t busy_blocks = *(volatile unsigned int*)&P.ctl->busy;
                            if ((int)((gridDim.x - busy_blocks) * W) >= P.spill_idle) want = rest / 2;
                        }
                    }
                    want = __shfl_sync(kFull, want, 0);
                    if (want) {
                        if (!flush(want, want)) break;
                        if (STATS && lane == 0) ++cnt[kCntSpills];
                    }
                }
                if ((iter & 1023u) == 0) {
                    const int stop = __shfl_sync(kFull, (int)(*(volatile unsigned int*)&P.ctl->done), 0);
                    if (stop) { set_done_local(); break; }
                    if (__shfl_sync(kFull, (int)(globaltimer() - S.t_start > P.timeout_ns), 0)) {
                        if (lane == 0) raise_error(P, kStatusETIMEOUT);
                        set_done_local();
                        break;
                    }
                }
            }
            continue;
        }

        // ===== top exhausted and HotRing empty: refill from ColdSeg =====
        if (refill() > 0) {
            has_top = pop(u, i);
            need_end = true; have_win = false;
            spec_ok = spec_pop; par = kFull;
            continue;
        }

        // ===== idle: deregister, then steal (Alg 2 l.6-7) =====
        if (active) {
            active = false;
            if (lane == 0) {
                atomicAnd(&S.warp_mask, ~(1u << w));
                deregister();
            }
            __syncwarp();
        }
        bool got_work = false;
        uint32_t backoff = P.backoff_min_ns;
        uint32_t idle_iter = 0;
        t_idle0 = STATS ? globaltimer() : 0ull;
        while (!got_work) {
            if (__shfl_sync(kFull, S.done, 0)) goto exit_loop;
            if (w == 0) {
                if (__shfl_sync(kFull, (int)(*(volatile unsigned int*)&P.ctl->done), 0)) {
                    set_done_local();
                    goto exit_loop;
                }
            }
            // watchdog every 16th idle round (idle polling competes with busy warps for issue)
            if ((idle_iter++ & 15u) == 0 &&
                __shfl_sync(kFull, (int)(globaltimer() - S.t_start > P.timeout_ns), 0)) {
                if (lane == 0) raise_error(P, kStatusETIMEOUT);
                set_done_local();
                goto exit_loop;
            }
            // ---- Alg 3: intra-block stealing from the peer HotRing with max hot_rest ----
            // (steal_tries > 1: when the best victim is locked by another thief or drops below
            // the cutoff, try the next best instead of backing off)
            if (P.intra && W > 1) {
                int rest = -1;
                if (lane < W && lane != w) rest = ht_rest(*(volatile uint32_t*)&S.ht[lane]);
                for (int att = 0; att < P.steal_tries; ++att) {
                    const int best = __reduce_max_sync(kFull, rest);
                    if (best < P.hot_cutoff) break;
                    const int vwarp = __ffs(__ballot_sync(kFull, rest == best)) - 1;
                    if (STATS && lane == 0) ++cnt[kCntStealAttempts];
                    uint32_t ok = 0, t = 0, kst = 0;
                    if (lane == 0) {
                        if (smem_trylock(&S.lock[vwarp])) {
                            register_thief();                        // before reserving
                            uint32_t old = *(volatile uint32_t*)&S.ht[vwarp];
                            for (int tries = 0; tries < 8; ++tries) {
                                const int r = ht_rest(old);
                                if (r < P.hot_cutoff) break;
                                t = ht_tail(old);
                                kst = hs;
                                if (P.steal_half && (uint32_t)(r / 2) > kst) kst = (uint32_t)(r / 2);
                                if (kst > 32u) kst = 32u;
                                if ((int)kst > r) kst = (uint32_t)r;
                                const uint32_t nw = (old & 0xFFFF0000u) | ((t + kst) & 0xFFFFu);
                                const uint32_t got = atom_cas_acquire_cta(&S.ht[vwarp], old, nw);   // reserve
                                if (got == old) { ok = 1; break; }
                                old = got;
                            }
                            if (!ok) { smem_unlock(&S.lock[vwarp]); deregister(); }
                        }
                    }
                    ok = __shfl_sync(kFull, ok, 0);
                    if (!ok) {
                        if (lane == vwarp) rest = -1;                // next best
                        continue;
                    }
                    t = __shfl_sync(kFull, t, 0);
                    kst = __shfl_sync(kFull, kst, 0);
                    __syncwarp();                                    // lane 0's acquire -> all lanes
                    const unsigned long long* vring = rings + (size_t)vwarp * H;
                    if (lane < (int)kst) ring[(my_head + lane) & (H - 1)] = vring[(t + lane) & (H - 1)];
                    __syncwarp();
                    if (lane == 0) {
                        S.tailf[vwarp] = (t + kst) & 0xFFFFu;        // slots reusable by the owner
                        smem_unlock(&S.lock[vwarp]);
                        atomicOr(&S.warp_mask, 1u << w);             // mark active
                    }
                    pub_add(lane == 0, &S.ht[w], kst << 16);         // publish into our ring
                    __syncwarp();
                    my_head += kst; pub = my_head;
                    if (STATS && lane == 0) ++cnt[kCntIntraSteals];
                    got_work = true;
                    break;
                }
                if (got_work) break;
            }
            if (CL && !P.cluster_late && cluster_steal()) { got_work = true; break; }
            // ---- Alg 4: steal c_s entries from a remote ColdSeg bottom ----
            int token = 0;
            if (P.inter && gridDim.x > 1 &&
                (P.inter_any || (w == 0 && __shfl_sync(kFull, *(volatile unsigned int*)&S.warp_mask, 0) == 0u))) {
                // test before the CAS: most rounds find the token taken
                if (lane == 0) token = (*(volatile uint32_t*)&S.inter_token == 0u && smem_trylock(&S.inter_token)) ? 1 : 0;
                token = __shfl_sync(kFull, token, 0);
            }
            if (token) {
                const int nB = gridDim.x;
                // cumulative ColdSeg load per block (reading S14); active = load > 0
                int vb = -1;
                {
                    int nact = 0;
                    for (int b0 = 0; b0 < nB; b0 += 32) {
                        const int b = b0 + lane;
                        const bool a = b < nB && (P.inter_any || b != (int)blockIdx.x) && ld_relaxed_s32(&P.block_cold[b]) > 0;
                        nact += __popc(__ballot_sync(kFull, a));
                    }
                    if (nact > 0) {
                        uint32_t r1 = 0, r2 = 0;
                        if (lane == 0) { r1 = xorshift32(rng) % nact; r2 = xorshift32(rng) % nact; }
                        r1 = __shfl_sync(kFull, r1, 0); r2 = __shfl_sync(kFull, r2, 0);
                        if (nact > 1 && r2 == r1) r2 = (r1 + 1) % nact;
                        int pick1 = -1, pick2 = -1, load1 = 0, load2 = 0, seen = 0;
                        for (int b0 = 0; b0 < nB && (pick1 < 0 || pick2 < 0); b0 += 32) {
                            const int b = b0 + lane;
                            const int load = (b < nB && (P.inter_any || b != (int)blockIdx.x)) ? ld_relaxed_s32(&P.block_cold[b]) : 0;
                            const uint32_t m = __ballot_sync(kFull, load > 0);
                            const int c = __popc(m);
                            for (int which = 0; which < 2; ++which) {
                                const uint32_t r = which ? r2 : r1;
                                if ((which ? pick2 : pick1) < 0 && r >= (uint32_t)seen && r < (uint32_t)(seen + c)) {
                                    const int nth = __fns(m, 0, (int)(r - seen) + 1);
                                    const int ld = __shfl_sync(kFull, load, nth);
                                    if (which) { pick2 = b0 + nth; load2 = ld; } else { pick1 = b0 + nth; load1 = ld; }
                                }
                            }
                            seen += c;
                        }
                        if (P.policy == 0 || pick2 < 0) vb = pick1;             // random (Fig 9 base)
                        else vb = (load2 > load1 || (load2 == load1 && pick2 < pick1)) ? pick2 : pick1;
                    }
                }
                if (STATS && lane == 0) ++cnt[kCntInterScans];
                if (vb >= 0) {
                    // victim warp: max cold_rest = top - bottom (Alg 4 l.9-15)
                    const int WV = W;                 // all blocks have W warps
                    int rest = -1;
                    if (lane < WV) {
                        const unsigned long long word = ld_relaxed_u64(&P.cold_tb[vb * WV + lane]);
                        rest = (int)((uint32_t)(word >> 32) - (uint32_t)word);
                    }
                    const int best = __reduce_max_sync(kFull, rest);
                    if (best >= P.cold_cutoff) {
                        const int vwl = __ffs(__ballot_sync(kFull, rest == best)) - 1;
                        const int vwg = vb * WV + vwl;
                        if (STATS && lane == 0) ++cnt[kCntStealAttempts];
                        uint32_t ok = 0, bot = 0, kst = 0;
                        if (lane == 0) {
                            register_thief();
                            unsigned long long old = ld_relaxed_u64(&P.cold_tb[vwg]);
                            for (int tries = 0; tries < 4; ++tries) {
                                const uint32_t top = (uint32_t)(old >> 32), b = (uint32_t)old;
                                const int r = (int)(top - b);
                                if (r < P.cold_cutoff) break;
                                kst = cs;
                                if (P.steal_half && (uint32_t)(r / 2) > kst) kst = (uint32_t)(r / 2);
                                if (kst > 64u) kst = 64u;
                                if ((int)kst > r) kst = (uint32_t)r;
                                const unsigned long long nw = ((unsigned long long)top << 32) | (uint32_t)(b + kst);
                                const unsigned long long got = atomicCAS(&P.cold_tb[vwg], old, nw);   // reserve
                                if (got == old) { ok = 1; bot = b; break; }
                                old = got;
                            }
                            // Alg 4 l.20 threadfence: acquire after the reservation, pairing with
                            // the owner's fence.release before it published `top` (its entries
                            // and chunk-table slots are visible before we read them)
                            if (ok) fence_acquire_gpu();
                            else deregister();
                        }
                        ok = __shfl_sync(kFull, ok, 0);
                        if (ok) {
                            bot = __shfl_sync(kFull, bot, 0);
                            kst = __shfl_sync(kFull, kst, 0);
                            __syncwarp();                                // lane 0's acquire -> all lanes
                            // remote transfer (Alg 4 l.21-22): L2 loads, addresses from the CAS;
                            // the range [bot, bot+kst) may straddle two ColdSeg chunks.  A slot
                            // that is not a pool chunk (only after an error exit of its owner)
                            // is never dereferenced.
                            uint32_t* vtab = P.chunk_tab + ((size_t)vwg << P.tab_log2);
                            for (uint32_t q = lane; q < kst; q += 32u) {
                                const uint32_t p = bot + q;
                                const uint32_t c = ld_relaxed_u32(&vtab[(p >> kChunkLog2) & tmask]);
                                if (c < P.n_chunks)
                                    ring[(my_head + q) & (H - 1)] = ld_cg_u64(P.pool + ((size_t)c << kChunkLog2) + (p & (kChunk - 1)));
                                else
                                    ring[(my_head + q) & (H - 1)] = pack_entry((uint32_t)P.root, P.m);   // exhausted entry
                            }
                            __syncwarp();
                            if (lane == 0) {
                                // chunk accounting: every position below bottom is passed by
                                // exactly one steal; the thief completing a chunk frees it
                                uint32_t p = bot, left = kst;
                                while (left) {
                                    const uint32_t in_chunk = kChunk - (p & (kChunk - 1));
                                    const uint32_t part = left < in_chunk ? left : in_chunk;
                                    uint32_t* slot = &vtab[(p >> kChunkLog2) & tmask];
                                    const uint32_t c = ld_relaxed_u32(slot);
                                    if (c < P.n_chunks) {
                                        const uint32_t before = atomicAdd(&P.chunk_consumed[c], part);
                                        if (before + part == kChunk) {         // chunk fully consumed
                                            st_relaxed_u32(slot, kEmptySlot);
                                            pool_free(P, c);
                                        }
                                    }
                                    p += part; left -= part;
                                }
                                atomicSub(&P.block_cold[vb], (int)kst);
                                atomicOr(&S.warp_mask, 1u << w);               // mark w, b active
                            }
                            pub_add(lane == 0, &S.ht[w], kst << 16);           // publish into our ring
                            __syncwarp();
                            my_head += kst; pub = my_head;
                            if (STATS && lane == 0) ++cnt[kCntInterSteals];
                            if (lane == 0) smem_unlock(&S.inter_token);
                            got_work = true;
                            break;
                        }
                    }
                }
            }
            if (token && lane == 0) smem_unlock(&S.inter_token);
            if (CL && P.cluster_late && cluster_steal()) { got_work = true; break; }
            sample();
            __nanosleep(backoff);
            if (backoff < P.backoff_max_ns) backoff <<= 1;
        }
        // got work: it is in the HotRing
        if (STATS && lane == 0) cnt[kCntIdleNs] += globaltimer() - t_idle0;
        t_idle0 = 0;
        active = true;
        has_top = pop(u, i);
        need_end = true; have_win = false;
        spec_ok = spec_pop; par = kFull;
    }
exit_loop:
    __syncwarp();
    if (STATS && !active && t_idle0 && lane == 0) cnt[kCntIdleNs] += globaltimer() - t_idle0;
    // release the ColdSeg chunks still mapped by this warp so the chunk table is all-empty
    // for the next run (thieves free the chunks they fully consume).  Only after a clean
    // termination (every ColdSeg is then empty): after an error exit other warps may still
    // steal from this warp's ColdSeg, so its table stays as it is and the host re-initialises
    // the whole table before the next run (Slot::tab_dirty)
    if (__shfl_sync(kFull, lane == 0 ? (fence_acquire_gpu(), ld_relaxed_s32(&P.ctl->status)) : 0, 0) == 0) {
        const unsigned long long word = ld_relaxed_u64(&P.cold_tb[gw]);
        const uint32_t bot = (uint32_t)word;
        const uint32_t lo = bot >> kChunkLog2;     // chunks below were freed by the thieves
        for (uint32_t k = lo + lane; k < hi; k += 32) {
            uint32_t* slot = &my_tab[k & tmask];
            if (ld_relaxed_u32(slot) != kEmptySlot) st_relaxed_u32(slot, kEmptySlot);
        }
    }
    if (P.block_claims && lane == 0 && my_claims) atomicAdd(&P.block_claims[blockIdx.x], (unsigned long long)my_claims);
    if (STATS && (P.collect_stats != 2 || gw == 0)) {     // 2: the root warp's counters only
#pragma unroll
        for (int k = 0; k < kNumCounters; ++k)
            if (lane == 0 && cnt[k]) atomicAdd(&P.ctl->counters[k], cnt[k]);
        __syncwarp();
    }
    // no CTA may exit while a cluster peer can still read or lock its HotRings
    if constexpr (CL) cluster_sync_all();
}

// ------------------------------------------------------------------------------------------
// per-traversal reset (step a2) and finalize (step a9)
// ------------------------------------------------------------------------------------------
// bitmap layout: bstride = 1 (32-wide kernels) or 2 (128-wide: {visited, leaf} word pairs; the
// leaf words are copied from the graph's leaf map, or zero when bulk leaf claims are off)
__global__ void dfs_reset_kernel(uint32_t* bitmap, uint32_t nwords, uint32_t bstride, const uint32_t* leaf,
                                 unsigned long long* cold_tb,
                                 uint32_t n_warps, int* block_cold, uint32_t n_blocks, Ctl* ctl,
                                 int32_t* parent, int root, uint32_t* chunk_tab, size_t tab_words) {
    const size_t tid = blockIdx.x * (size_t)blockDim.x + threadIdx.x;
    const size_t stride = (size_t)gridDim.x * blockDim.x;
    for (size_t k = tid; k < nwords; k += stride) {
        uint32_t v = 0;
        if (k == ((uint32_t)root >> 5)) v = 1u << (root & 31);    // Alg 1 l.1: visited[root]
        if (bstride == 2) {
            reinterpret_cast<uint2*>(bitmap)[k] = make_uint2(v, leaf ? leaf[k] : 0u);
        } else {
            bitmap[k] = v;
        }
    }
    for (size_t k = tid; k < n_warps; k += stride) cold_tb[k] = 0ull;
    for (size_t k = tid; k < n_blocks; k += stride) block_cold[k] = 0;
    for (size_t k = tid; k < tab_words; k += stride) chunk_tab[k] = kEmptySlot;   // only after errors
    if (tid == 0) {
        parent[root] = -1;                                          // Alg 1 l.1: parent[root]
        ctl->busy = 1u;                                             // block 0 / warp 0 holds root
        ctl->done = 0u;
        ctl->status = 0;
        ctl->pool_bump = 0u;
        ctl->free_head = (unsigned long long)kEmptySlot;
        ctl->claims_progress = 0ull;
        ctl->windows_progress = 0ull;
        for (int k = 0; k < 24; ++k) ctl->counters[k] = 0ull;
    }
}

__global__ void dfs_finalize_kernel(const uint32_t* __restrict__ bitmap, uint32_t bstride, int32_t* parent, uint32_t n,
                                    const Ctl* ctl, int* status_acc) {
    const size_t stride = (size_t)gridDim.x * blockDim.x;
    if (blockIdx.x == 0 && threadIdx.x == 0 && ctl->status != 0) atomicMin(status_acc, ctl->status);
    for (size_t v = blockIdx.x * (size_t)blockDim.x + threadIdx.x; v < n; v += stride) {
        const uint32_t word = __ldg(bitmap + bstride * (v >> 5));
        if (!((word >> (v & 31)) & 1u)) parent[v] = -2;            // DFS_UNREACHED (reading S2)
    }
}

// visited count and TEPS numerator (sum of out-degrees of visited vertices)
__global__ void dfs_count_kernel(const uint32_t* __restrict__ bitmap, uint32_t bstride, const uint32_t* __restrict__ rp,
                                 uint32_t n, unsigned long long* out2) {
    unsigned long long nv = 0, mv = 0;
    const size_t stride = (size_t)gridDim.x * blockDim.x;
    for (size_t v = blockIdx.x * (size_t)blockDim.x + threadIdx.x; v < n; v += stride) {
        if ((__ldg(bitmap + bstride * (v >> 5)) >> (v & 31)) & 1u) { ++nv; mv += __ldg(rp + v + 1) - __ldg(rp + v); }
    }
    for (int o = 16; o > 0; o >>= 1) {
        nv += __shfl_down_sync(kFull, nv, o);
        mv += __shfl_down_sync(kFull, mv, o);
    }
    if ((threadIdx.x & 31) == 0) { atomicAdd(&out2[0], nv); atomicAdd(&out2[1], mv); }
}

// leaf map (create time, step a1).  Claiming a leaf v from u at once (bulk, out of Alg 1's
// order) is exactly Alg 1's "descend, scan, pop straight back" iff no other list can claim v and
// v's own list leads nowhere: bit v is set iff every in-edge of v (self-loops aside) comes from
// one vertex w, and v's out-list is empty or the single entry w or v.  Pass 1 finds the unique
// in-neighbour of every out-degree <= 1 vertex (kInUnset / kInMulti otherwise); pass 2 sets bits.
constexpr uint32_t kInUnset = 0xFFFFFFFFu;
constexpr uint32_t kInMulti = 0xFFFFFFFEu;
__global__ void dfs_leaf_in_kernel(const uint32_t* __restrict__ rp, const int32_t* __restrict__ col,
                                   uint32_t n, uint32_t* inn) {
    const size_t stride = (size_t)gridDim.x * blockDim.x;
    for (size_t u = blockIdx.x * (size_t)blockDim.x + threadIdx.x; u < n; u += stride) {
        for (uint32_t j = rp[u]; j < rp[u + 1]; ++j) {
            const uint32_t v = (uint32_t)col[j];
            if (v == (uint32_t)u || rp[v + 1] - rp[v] > 1u) continue;
            const uint32_t old = atomicCAS(&inn[v], kInUnset, (uint32_t)u);
            if (old != kInUnset && old != (uint32_t)u) atomicExch(&inn[v], kInMulti);
        }
    }
}
__global__ void dfs_leaf_init_kernel(const uint32_t* __restrict__ rp, const int32_t* __restrict__ col,
                                     const uint32_t* __restrict__ inn, uint32_t n, uint32_t* leaf) {
    const size_t stride = (size_t)gridDim.x * blockDim.x;
    for (size_t wd = blockIdx.x * (size_t)blockDim.x + threadIdx.x; wd < ((size_t)n + 31) / 32; wd += stride) {
        uint32_t bits = 0;
        for (uint32_t b = 0; b < 32; ++b) {
            const size_t v = wd * 32 + b;
            if (v >= n) break;
            const uint32_t deg = rp[v + 1] - rp[v];
            if (deg > 1u) continue;
            const uint32_t w = inn[v];
            if (w == kInMulti) continue;
            if (deg == 1u) {
                const uint32_t x = (uint32_t)col[rp[v]];
                if (x != (uint32_t)v && x != w && w != kInUnset) continue;
            }
            bits |= 1u << b;
        }
        leaf[wd] = bits;
    }
}

// CSR validation + narrowing of row_ptr to uint32 (step a1)
__global__ void dfs_validate_rowptr_kernel(const int64_t* __restrict__ rp64, uint32_t* rp32, int64_t n,
                                           int64_t m, int* bad) {
    // bad[0]: malformed flag; bad[1]: maximum out-degree (kernel selection)
    const size_t stride = (size_t)gridDim.x * blockDim.x;
    int64_t dmax = 0;
    for (size_t v = blockIdx.x * (size_t)blockDim.x + threadIdx.x; v <= (size_t)n; v += stride) {
        const int64_t a = rp64[v];
        bool ok = a >= 0 && a <= m;
        if (v == 0) ok = ok && a == 0;
        if (v == (size_t)n) ok = ok && a == m;
        if (v < (size_t)n) {
            const int64_t e = rp64[v + 1];
            ok = ok && e >= a;
            if (e - a > dmax) dmax = e - a;
        }
        if (!ok) atomicExch(bad, 1);
        rp32[v] = (uint32_t)a;
    }
    const int dm = __reduce_max_sync(kFull, (int)(dmax < 0x7FFFFFFF ? dmax : 0x7FFFFFFF));
    if ((threadIdx.x & 31) == 0 && dm > 0) atomicMax(bad + 1, dm);
}

__global__ void dfs_validate_col_kernel(const int32_t* __restrict__ col, int64_t m, int64_t n, int* bad) {
    const size_t stride = (size_t)gridDim.x * blockDim.x;
    for (size_t j = blockIdx.x * (size_t)blockDim.x + threadIdx.x; j < (size_t)m; j += stride) {
        const int32_t c = col[j];
        if (c < 0 || (int64_t)c >= n) atomicExch(bad, 1);
    }
}

}  // namespace b200dfs
