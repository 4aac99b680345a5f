// dfs_device.cuh — sm_100a device code of the unordered-DFS hot path.
//
// The method is DiggerBees (PPoPP '26); "P:a-b" = /root/reference/PAPER.md lines.  The kernel
// re-designs the paper's H100 kernel for B200 (DESIGN.md §"Kernels"):
//
//   * persistent grid, one 32-warp CTA per SM (subsystem 1; "1 block per SM")
//   * per-warp two-level stack (subsystem 2; §3.2, Fig 2):
//       HotRing  = circular buffer in shared memory, monotone 32-bit head/tail counters
//       ColdSeg  = per-warp virtual linear segment in global memory, backed by a chunk table
//                  and a global chunk pool (the paper's fixed n_v/n_w capacity overflows on deep
//                  graphs; reading S9)
//       flush oldest H/2 entries from tail -> ColdSeg top; refill from ColdSeg top
//   * warp-level expansion (subsystem 3; §3.3): the 32 lanes load a 32-neighbour
//     window of col_idx, probe the visited bitmap, __ballot_sync + __ffs pick the FIRST unvisited
//     neighbour in CSR order, one lane claims it with atomicOr on the bitmap word (the claim of
//     Alg 1 l.9-10 made atomic).  The current top entry lives in registers; the child's
//     row_ptr pair and its first window are loaded speculatively, overlapping the claim.
//   * intra-block stealing (subsystem 4; §3.4, Alg 3): idle warps take h_s =
//     hot_cutoff/2 entries from the TAIL of the peer HotRing with max hot_rest >= hot_cutoff,
//     under a per-warp shared-memory lock + THE-style owner/thief protocol (reading S12)
//   * inter-block stealing (subsystem 5; §3.5, Alg 4): the leader warp of an idle
//     block picks a victim block by two random choices weighted by cumulative ColdSeg load
//     (reading S14), then the victim warp with max cold_rest >= cold_cutoff, reserves c_s =
//     cold_cutoff/2 entries from the ColdSeg BOTTOM with a 64-bit CAS on the packed
//     {top,bottom} word, and copies them into its HotRing.
//   * global termination (unspecified in the paper, reading S13): a busy counter of warps that
//     hold work plus registered thieves; the atomic that brings it to 0 raises `done`.
#pragma once
#include <cstdint>

namespace b200dfs {

constexpr uint32_t kFull = 0xffffffffu;
constexpr uint32_t kEmptySlot = 0xffffffffu;
constexpr int kChunkLog2 = 11;                     // ColdSeg chunk = 2048 entries (16 KB)
constexpr uint32_t kChunk = 1u << kChunkLog2;
constexpr int kMaxWarps = 32;                      // 32-bit warp mask
constexpr int kPrefetchLanes = 8;                  // lanes that prefetch a candidate's row_ptr

// error codes written to Ctl::status (mirrors dfs_status)
constexpr int kStatusENOMEM = -2;
constexpr int kStatusETIMEOUT = -5;
constexpr int kStatusEINTERNAL = -6;

struct Ctl {
    unsigned int busy;                 // warps holding work + registered thieves (S13)
    unsigned int done;                 // set once busy reaches 0 (or on error)
    int status;                        // 0 or a negative dfs_status
    unsigned int pool_bump;            // bump allocator over the chunk pool
    unsigned long long free_head;      // tagged free-stack head: (tag << 32) | chunk id
    unsigned long long counters[16];   // stats (collect_stats)
};

enum CounterIdx {
    kCntClaims = 0, kCntFailedClaims, kCntFlushes, kCntRefills, kCntIntraSteals, kCntInterSteals,
    kCntStealAttempts, kCntChunks, kCntWindows, kNumCounters
};

struct KParams {
    const uint32_t* __restrict__ rp;         // n+1 (narrowed row_ptr; m < 2^32)
    const int32_t* __restrict__ col;         // m
    uint32_t* bitmap;                        // ceil(n/32) visited words
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
    unsigned long long timeout_ns;
    uint32_t seed;
};

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
__device__ __forceinline__ unsigned long long globaltimer() {
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    return t;
}
// 16-byte L2 (coherent) load of two stack entries
__device__ __forceinline__ void ld_cg_v2(const unsigned long long* p, unsigned long long& a,
                                         unsigned long long& b) {
    asm volatile("ld.global.cg.v2.u64 {%0, %1}, [%2];" : "=l"(a), "=l"(b) : "l"(p) : "memory");
}
__device__ __forceinline__ void st_cg_v2(unsigned long long* p, unsigned long long a,
                                         unsigned long long b) {
    asm volatile("st.global.cg.v2.u64 [%0], {%1, %2};" ::"l"(p), "l"(a), "l"(b) : "memory");
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

// ------------------------------------------------------------------------------------------
// shared-memory control block (one per CTA)
// ------------------------------------------------------------------------------------------
struct SmemCtl {
    volatile uint32_t head[kMaxWarps];    // HotRing head (next free slot); written by owner only
    volatile uint32_t tail[kMaxWarps];    // oldest entry; thieves reserve by advancing it
    volatile uint32_t tailf[kMaxWarps];   // slots below tailf are free for reuse (copy finished)
    int lock[kMaxWarps];                  // per-warp lock for tail-side operations
    unsigned int warp_mask;               // 1 = warp active
    volatile int done;                    // block-local copy of ctl->done
};

__device__ __forceinline__ void smem_lock(int* l) {
    while (atomicCAS(l, 0, 1) != 0) { }
    __threadfence_block();
}
__device__ __forceinline__ bool smem_trylock(int* l) {
    if (atomicCAS(l, 0, 1) == 0) { __threadfence_block(); return true; }
    return false;
}
__device__ __forceinline__ void smem_unlock(int* l) {
    __threadfence_block();
    atomicExch(l, 0);
}

// ------------------------------------------------------------------------------------------
// chunk pool: tagged lock-free free stack + bump allocator
// ------------------------------------------------------------------------------------------
__device__ __forceinline__ uint32_t pool_alloc(const KParams& P) {
    Ctl* c = P.ctl;
    unsigned long long old = ld_relaxed_u64(&c->free_head);
    for (;;) {
        uint32_t idx = (uint32_t)old;
        if (idx == kEmptySlot) break;
        uint32_t nxt = ld_relaxed_u32(&P.chunk_next[idx]);
        unsigned long long nw = ((unsigned long long)((uint32_t)(old >> 32) + 1u) << 32) | nxt;
        unsigned long long got = atomicCAS(&c->free_head, old, nw);
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
        asm volatile("st.relaxed.gpu.global.u32 [%0], %1;" ::"l"(&P.chunk_next[idx]), "r"((uint32_t)old) : "memory");
        __threadfence();
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

// ------------------------------------------------------------------------------------------
// The persistent traversal kernel.  H = HotRing entries per warp (power of two).
// Launched with blockDim.x = 32 * W (W <= 32) and dynamic shared memory
// sizeof(SmemCtl) (16-byte padded) + W * H * 8 bytes.
// ------------------------------------------------------------------------------------------
template <int H>
__global__ void __launch_bounds__(1024, 1) dfs_persistent_kernel(const KParams P) {
    static_assert((H & (H - 1)) == 0 && H >= 64, "H must be a power of two >= 64");
    constexpr uint32_t kBatch = H / 2;              // flush batch (reading S10)
    extern __shared__ __align__(16) unsigned char smem_raw[];
    SmemCtl& S = *reinterpret_cast<SmemCtl*>(smem_raw);
    constexpr int kCtlBytes = (sizeof(SmemCtl) + 15) & ~15;
    unsigned long long* const rings = reinterpret_cast<unsigned long long*>(smem_raw + kCtlBytes);

    const int lane = threadIdx.x & 31;
    const int w = threadIdx.x >> 5;
    const int W = blockDim.x >> 5;
    const int gw = blockIdx.x * W + w;
    unsigned long long* const ring = rings + (size_t)w * H;
    const uint32_t tmask = (1u << P.tab_log2) - 1u;
    uint32_t* const my_tab = P.chunk_tab + ((size_t)gw << P.tab_log2);
    const uint32_t hs = (uint32_t)P.hot_cutoff >> 1;        // h_s (Alg 3 l.12)
    const uint32_t cs = (uint32_t)P.cold_cutoff >> 1;       // c_s (Alg 4 l.17)

    if (threadIdx.x < kMaxWarps) {
        S.head[threadIdx.x] = 0; S.tail[threadIdx.x] = 0; S.tailf[threadIdx.x] = 0;
        S.lock[threadIdx.x] = 0;
    }
    if (threadIdx.x == 0) { S.warp_mask = (blockIdx.x == 0) ? 1u : 0u; S.done = 0; }
    __syncthreads();

    // ---- per-warp state (warp-uniform registers) ----
    bool has_top = false;        // a current top entry <u, i> lives in registers
    bool have_win = false;       // nb holds the window starting at i
    bool need_end = false;       // end must be re-read from row_ptr
    uint32_t u = 0, i = 0, end = 0;
    int nb = -1;                 // this lane's neighbour in the current window
    uint32_t my_head = 0;        // owner copy of S.head[w]
    uint32_t my_top = 0;         // owner copy of ColdSeg top
    uint32_t hi = 0;             // ColdSeg chunks [.., hi) mapped by this warp
    bool active = false;
    uint32_t rng = P.seed ^ (0x9E3779B9u * (uint32_t)(gw + 1));
    if (rng == 0) rng = 1;
    unsigned long long cnt[kNumCounters];
#pragma unroll
    for (int k = 0; k < kNumCounters; ++k) cnt[k] = 0;
    const unsigned long long t_start = globaltimer();
    uint32_t iter = 0;

    if (blockIdx.x == 0 && w == 0) {
        // Alg 1 l.1-3: root claimed by the reset kernel; <root, row_ptr[root]> is our top
        has_top = true; active = true;
        u = (uint32_t)P.root; i = __ldg(P.rp + u); end = __ldg(P.rp + u + 1);
    }

    // ---------------------------------------------------------------- owner stack operations
    // flush: move the kBatch oldest HotRing entries to ColdSeg top (Fig 2(e))
    auto flush = [&]() -> bool {
        if (lane == 0) smem_lock(&S.lock[w]);
        __syncwarp();
        const uint32_t t = __shfl_sync(kFull, S.tail[w], 0);
        // map chunks covering [my_top, my_top + kBatch)
        bool ok = true;
        while (ok && (unsigned long long)hi * kChunk < (unsigned long long)my_top + kBatch) {
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
                        P.chunk_consumed[c] = 0;
                        asm volatile("st.relaxed.gpu.global.u32 [%0], %1;" ::"l"(slot), "r"(c) : "memory");
                    }
                }
            }
            c = __shfl_sync(kFull, c, 0);
            if (c == kEmptySlot) ok = false; else { ++hi; ++cnt[kCntChunks]; }
        }
        if (!ok) {
            if (lane == 0) { raise_error(P, kStatusENOMEM); smem_unlock(&S.lock[w]); }
            __syncwarp();
            return false;
        }
        // vectorised copy: each lane moves pairs of entries (16 B); t and my_top are even
        for (uint32_t q = 2u * lane; q < kBatch; q += 64u) {
            const unsigned long long* src = ring + ((t + q) & (H - 1));
            unsigned long long a = src[0], b = src[1];
            uint32_t p = my_top + q;
            uint32_t c = ld_relaxed_u32(&my_tab[(p >> kChunkLog2) & tmask]);
            st_cg_v2(P.pool + ((size_t)c << kChunkLog2) + (p & (kChunk - 1)), a, b);
        }
        __threadfence();
        __syncwarp();
        if (lane == 0) {
            atomicAdd(&P.cold_tb[gw], (unsigned long long)kBatch << 32);   // publish top (release)
            atomicAdd(&P.block_cold[blockIdx.x], (int)kBatch);
            S.tail[w] = t + kBatch;
            S.tailf[w] = t + kBatch;
            smem_unlock(&S.lock[w]);
        }
        __syncwarp();
        my_top += kBatch;
        ++cnt[kCntFlushes];
        return true;
    };

    // push <v, idx> at head (Fig 2(c)); flushes first when full
    auto push = [&](uint32_t v, uint32_t idx) -> bool {
        if (__shfl_sync(kFull, (int)(my_head - S.tailf[w]) >= H, 0)) {
            if (!flush()) return false;
        }
        if (lane == 0) {
            ring[my_head & (H - 1)] = pack_entry(v, idx);
            __threadfence_block();
            S.head[w] = my_head + 1;
        }
        __syncwarp();
        ++my_head;
        return true;
    };

    // pop the newest HotRing entry (Fig 2(d)); THE protocol against tail-side thieves
    auto pop = [&](uint32_t& v, uint32_t& idx) -> bool {
        unsigned long long e = 0;
        int got = 0;
        if (lane == 0) {
            const uint32_t h = my_head - 1;
            S.head[w] = h;
            __threadfence_block();
            if ((int)(h - S.tail[w]) >= 0) { e = ring[h & (H - 1)]; got = 1; }
            else {
                // possible conflict with a thief (or empty): decide under the lock, where tail is
                // final — a thief may still roll its reservation back (reading S12)
                S.head[w] = h + 1;
                smem_lock(&S.lock[w]);
                if ((int)(h - S.tail[w]) >= 0) { S.head[w] = h; e = ring[h & (H - 1)]; got = 1; }
                smem_unlock(&S.lock[w]);
            }
        }
        got = __shfl_sync(kFull, got, 0);
        if (!got) return false;
        e = __shfl_sync(kFull, e, 0);
        --my_head;
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
        // ring is empty: my_head == tail (even); place entries oldest first
        for (uint32_t q = 2u * lane; q < k; q += 64u) {
            uint32_t p = base + q;
            uint32_t c = ld_relaxed_u32(&my_tab[(p >> kChunkLog2) & tmask]);
            unsigned long long a, b;
            ld_cg_v2(P.pool + ((size_t)c << kChunkLog2) + (p & (kChunk - 1)), a, b);
            unsigned long long* dst = ring + ((my_head + q) & (H - 1));
            dst[0] = a; dst[1] = b;
        }
        my_top = base;
        // release chunks that lie wholly above top + one spare chunk (never read by thieves)
        while (hi > 0 && (unsigned long long)(hi - 1) * kChunk >= (unsigned long long)my_top + kChunk) {
            if (lane == 0) {
                uint32_t* slot = &my_tab[(hi - 1) & tmask];
                uint32_t c = ld_relaxed_u32(slot);
                asm volatile("st.relaxed.gpu.global.u32 [%0], %1;" ::"l"(slot), "r"(kEmptySlot) : "memory");
                pool_free(P, c);
            }
            --hi;
        }
        __syncwarp();
        if (lane == 0) {
            atomicSub(&P.block_cold[blockIdx.x], (int)k);
            __threadfence_block();
            S.head[w] = my_head + k;
        }
        __syncwarp();
        my_head += k;
        ++cnt[kCntRefills];
        return k;
    };

    auto set_done_local = [&]() {
        if (lane == 0) S.done = 1;
    };

    // ---------------------------------------------------------------- main loop (Alg 2)
    for (;;) {
        if (has_top) {
            // ===== warp-level expansion step (Alg 1 l.5-12 over a 32-wide window) =====
            if (!have_win) {
                const uint32_t e2 = need_end ? __ldg(P.rp + u + 1) : end;
                const uint32_t idx = i + lane;
                nb = (idx < P.m) ? __ldg(P.col + idx) : -1;
                end = e2; need_end = false;
            }
            ++cnt[kCntWindows];
            const bool valid = (i + lane) < end;
            uint32_t wbits = kFull, prs = 0, pre = 0;
            if (valid) {
                wbits = __ldcg(P.bitmap + ((uint32_t)nb >> 5));
                if (lane < kPrefetchLanes) { prs = __ldg(P.rp + nb); pre = __ldg(P.rp + nb + 1); }
            }
            const bool cand = valid && !((wbits >> (nb & 31)) & 1u);
            uint32_t unv = __ballot_sync(kFull, cand);
            bool descended = false;
            while (unv) {
                const int j = __ffs(unv) - 1;                    // first unvisited in CSR order
                const uint32_t v = (uint32_t)__shfl_sync(kFull, nb, j);
                uint32_t vrs = __shfl_sync(kFull, prs, j), vre = __shfl_sync(kFull, pre, j);
                if (j >= kPrefetchLanes) { vrs = __ldg(P.rp + v); vre = __ldg(P.rp + v + 1); }
                const uint32_t bit = 1u << (v & 31);
                uint32_t old = 0;
                if (lane == 0) old = atomicOr(P.bitmap + (v >> 5), bit);          // claim
                // speculative load of the child's first window, overlapping the claim
                const uint32_t cidx = vrs + lane;
                const int cnb = (cidx < P.m) ? __ldg(P.col + cidx) : -1;
                old = __shfl_sync(kFull, old, 0);
                if (!(old & bit)) {
                    ++cnt[kCntClaims];
                    if (lane == 0) P.parent[v] = (int32_t)u;                        // Alg 1 l.10
                    const uint32_t ni = i + (uint32_t)j + 1u;
                    // Alg 1 l.8 + l.11: keep <u, ni> below the child unless u is exhausted
                    if (ni < end) {
                        if (!push(u, ni)) goto exit_loop;
                    }
                    u = v; i = vrs; end = vre; nb = cnb; have_win = true; need_end = false;
                    descended = true;
                    break;
                }
                ++cnt[kCntFailedClaims];
                unv &= unv - 1;                                   // lost the race: next candidate
            }
            if (!descended) {
                i += 32;
                have_win = false;
                if (i >= end) {                                   // Alg 1 l.14: pop
                    has_top = pop(u, i);
                    need_end = true;
                }
            }
            if ((++iter & 1023u) == 0) {
                const int stop = __shfl_sync(kFull, (int)(*(volatile unsigned int*)&P.ctl->done), 0);
                if (stop) { set_done_local(); break; }
                if (__shfl_sync(kFull, (int)(globaltimer() - t_start > P.timeout_ns), 0)) {
                    if (lane == 0) raise_error(P, kStatusETIMEOUT);
                    set_done_local();
                    break;
                }
            }
            continue;
        }

        // ===== top exhausted and HotRing empty: refill from ColdSeg =====
        if (refill() > 0) {
            has_top = pop(u, i);
            need_end = true; have_win = false;
            continue;
        }

        // ===== idle: deregister, then steal (Alg 2 l.6-7) =====
        if (active) {
            active = false;
            if (lane == 0) {
                atomicAnd(&S.warp_mask, ~(1u << w));
                if (atomicSub(&P.ctl->busy, 1u) == 1u) { atomicExch(&P.ctl->done, 1u); S.done = 1; }
            }
            __syncwarp();
        }
        bool got_work = false;
        uint32_t backoff = 32;
        while (!got_work) {
            if (__shfl_sync(kFull, S.done, 0)) goto exit_loop;
            if (w == 0) {
                if (__shfl_sync(kFull, (int)(*(volatile unsigned int*)&P.ctl->done), 0)) {
                    set_done_local();
                    goto exit_loop;
                }
            }
            if (__shfl_sync(kFull, (int)(globaltimer() - t_start > P.timeout_ns), 0)) {
                if (lane == 0) raise_error(P, kStatusETIMEOUT);
                set_done_local();
                goto exit_loop;
            }
            // ---- Alg 3: intra-block stealing from the peer HotRing with max hot_rest ----
            if (P.intra && W > 1) {
                int rest = -1;
                if (lane < W && lane != w) rest = (int)(S.head[lane] - S.tail[lane]);
                const int best = __reduce_max_sync(kFull, rest);
                if (best >= P.hot_cutoff) {
                    const int vwarp = __ffs(__ballot_sync(kFull, rest == best)) - 1;
                    ++cnt[kCntStealAttempts];
                    uint32_t ok = 0, t = 0;
                    if (lane == 0) {
                        atomicAdd(&P.ctl->busy, 1u);                 // register before reserving
                        if (smem_trylock(&S.lock[vwarp])) {
                            t = S.tail[vwarp];
                            if ((int)(S.head[vwarp] - t) >= P.hot_cutoff) {
                                S.tail[vwarp] = t + hs;              // reserve (Alg 3 l.13-15)
                                __threadfence_block();
                                if ((int)(S.head[vwarp] - (t + hs)) >= 0) ok = 1;
                                else S.tail[vwarp] = t;              // owner raced us: roll back
                            }
                            if (!ok) smem_unlock(&S.lock[vwarp]);
                        }
                        if (!ok) {
                            if (atomicSub(&P.ctl->busy, 1u) == 1u) { atomicExch(&P.ctl->done, 1u); S.done = 1; }
                        }
                    }
                    ok = __shfl_sync(kFull, ok, 0);
                    if (ok) {
                        t = __shfl_sync(kFull, t, 0);
                        const unsigned long long* vring = rings + (size_t)vwarp * H;
                        if (lane < (int)hs) ring[(my_head + lane) & (H - 1)] = vring[(t + lane) & (H - 1)];
                        __syncwarp();
                        if (lane == 0) {
                            __threadfence_block();
                            S.tailf[vwarp] = t + hs;                 // slots reusable by the owner
                            smem_unlock(&S.lock[vwarp]);
                            S.head[w] = my_head + hs;
                            atomicOr(&S.warp_mask, 1u << w);         // mark active
                        }
                        __syncwarp();
                        my_head += hs;
                        ++cnt[kCntIntraSteals];
                        got_work = true;
                        break;
                    }
                }
            }
            // ---- Alg 4: leader warp of an idle block steals from a remote ColdSeg bottom ----
            if (P.inter && w == 0 && gridDim.x > 1 &&
                __shfl_sync(kFull, *(volatile unsigned int*)&S.warp_mask, 0) == 0u) {
                const int nB = gridDim.x;
                // cumulative ColdSeg load per block (reading S14); active = load > 0
                int vb = -1;
                {
                    int nact = 0;
                    for (int b0 = 0; b0 < nB; b0 += 32) {
                        const int b = b0 + lane;
                        const bool a = b < nB && b != (int)blockIdx.x && ld_relaxed_s32(&P.block_cold[b]) > 0;
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
                            const int load = (b < nB && b != (int)blockIdx.x) ? ld_relaxed_s32(&P.block_cold[b]) : 0;
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
                if (vb >= 0) {
                    // victim warp: max cold_rest = top - bottom (Alg 4 l.9-15)
                    const int WV = W;                 // all blocks have W warps
                    int rest = -1;
                    unsigned long long word = 0;
                    if (lane < WV) {
                        word = ld_relaxed_u64(&P.cold_tb[vb * WV + lane]);
                        rest = (int)((uint32_t)(word >> 32) - (uint32_t)word);
                    }
                    const int best = __reduce_max_sync(kFull, rest);
                    if (best >= P.cold_cutoff) {
                        const int vwl = __ffs(__ballot_sync(kFull, rest == best)) - 1;
                        const int vwg = vb * WV + vwl;
                        ++cnt[kCntStealAttempts];
                        uint32_t ok = 0, bot = 0;
                        if (lane == 0) {
                            atomicAdd(&P.ctl->busy, 1u);
                            unsigned long long old = ld_relaxed_u64(&P.cold_tb[vwg]);
                            for (int tries = 0; tries < 4; ++tries) {
                                const uint32_t top = (uint32_t)(old >> 32), b = (uint32_t)old;
                                if ((int)(top - b) < P.cold_cutoff) break;
                                const unsigned long long nw = ((unsigned long long)top << 32) | (uint32_t)(b + cs);
                                const unsigned long long got = atomicCAS(&P.cold_tb[vwg], old, nw);
                                if (got == old) { ok = 1; bot = b; break; }
                                old = got;
                            }
                            if (!ok) {
                                if (atomicSub(&P.ctl->busy, 1u) == 1u) { atomicExch(&P.ctl->done, 1u); S.done = 1; }
                            }
                        }
                        ok = __shfl_sync(kFull, ok, 0);
                        if (ok) {
                            bot = __shfl_sync(kFull, bot, 0);
                            __threadfence();                                    // acquire (Alg 4 l.21)
                            uint32_t* vtab = P.chunk_tab + ((size_t)vwg << P.tab_log2);
                            uint32_t* slot = &vtab[(bot >> kChunkLog2) & tmask];
                            const uint32_t c = ld_relaxed_u32(slot);
                            const unsigned long long* src = P.pool + ((size_t)c << kChunkLog2) + (bot & (kChunk - 1));
                            if (2u * lane < cs) {
                                unsigned long long a, b;
                                ld_cg_v2(src + 2 * lane, a, b);
                                unsigned long long* dst = ring + ((my_head + 2u * lane) & (H - 1));
                                dst[0] = a; dst[1] = b;
                            }
                            __syncwarp();
                            if (lane == 0) {
                                __threadfence();
                                const uint32_t before = atomicAdd(&P.chunk_consumed[c], cs);
                                if (before + cs == kChunk) {                   // chunk fully consumed
                                    asm volatile("st.relaxed.gpu.global.u32 [%0], %1;" ::"l"(slot), "r"(kEmptySlot) : "memory");
                                    pool_free(P, c);
                                }
                                atomicSub(&P.block_cold[vb], (int)cs);
                                __threadfence_block();
                                S.head[w] = my_head + cs;
                                atomicOr(&S.warp_mask, 1u << w);               // mark w, b active
                            }
                            __syncwarp();
                            my_head += cs;
                            ++cnt[kCntInterSteals];
                            got_work = true;
                            break;
                        }
                    }
                }
            }
            __nanosleep(backoff);
            if (backoff < 2048) backoff <<= 1;
        }
        // got work: it is in the HotRing
        active = true;
        has_top = pop(u, i);
        need_end = true; have_win = false;
    }
exit_loop:
    __syncwarp();
    // release the ColdSeg chunks still mapped by this warp so the chunk table is all-empty
    // for the next run (thieves free the chunks they fully consume)
    {
        const unsigned long long word = ld_relaxed_u64(&P.cold_tb[gw]);
        const uint32_t bot = (uint32_t)word;
        const uint32_t lo = bot >> kChunkLog2;     // chunks below were freed by the thieves
        for (uint32_t k = lo + lane; k < hi; k += 32) {
            uint32_t* slot = &my_tab[k & tmask];
            const uint32_t c = ld_relaxed_u32(slot);
            if (c != kEmptySlot) {
                asm volatile("st.relaxed.gpu.global.u32 [%0], %1;" ::"l"(slot), "r"(kEmptySlot) : "memory");
            }
        }
    }
    if (P.collect_stats) {
#pragma unroll
        for (int k = 0; k < kNumCounters; ++k)
            if (lane == 0 && cnt[k]) atomicAdd(&P.ctl->counters[k], cnt[k]);
    }
}

// ------------------------------------------------------------------------------------------
// per-traversal reset (step a2) and finalize (step a9)
// ------------------------------------------------------------------------------------------
__global__ void dfs_reset_kernel(uint32_t* bitmap, uint32_t nwords, unsigned long long* cold_tb,
                                 uint32_t n_warps, int* block_cold, uint32_t n_blocks, Ctl* ctl,
                                 int32_t* parent, int root, uint32_t* chunk_tab, size_t tab_words) {
    const size_t tid = blockIdx.x * (size_t)blockDim.x + threadIdx.x;
    const size_t stride = (size_t)gridDim.x * blockDim.x;
    for (size_t k = tid; k < nwords; k += stride) {
        uint32_t v = 0;
        if (k == ((uint32_t)root >> 5)) v = 1u << (root & 31);    // Alg 1 l.1: visited[root]
        bitmap[k] = v;
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
        for (int k = 0; k < 16; ++k) ctl->counters[k] = 0ull;
    }
}

__global__ void dfs_finalize_kernel(const uint32_t* __restrict__ bitmap, int32_t* parent, uint32_t n) {
    const size_t stride = (size_t)gridDim.x * blockDim.x;
    for (size_t v = blockIdx.x * (size_t)blockDim.x + threadIdx.x; v < n; v += stride) {
        const uint32_t word = __ldg(bitmap + (v >> 5));
        if (!((word >> (v & 31)) & 1u)) parent[v] = -2;            // DFS_UNREACHED (reading S2)
    }
}

// visited count and TEPS numerator (sum of out-degrees of visited vertices)
__global__ void dfs_count_kernel(const uint32_t* __restrict__ bitmap, const uint32_t* __restrict__ rp,
                                 uint32_t n, unsigned long long* out2) {
    unsigned long long nv = 0, mv = 0;
    const size_t stride = (size_t)gridDim.x * blockDim.x;
    for (size_t v = blockIdx.x * (size_t)blockDim.x + threadIdx.x; v < n; v += stride) {
        if ((__ldg(bitmap + (v >> 5)) >> (v & 31)) & 1u) { ++nv; mv += __ldg(rp + v + 1) - __ldg(rp + v); }
    }
    for (int o = 16; o > 0; o >>= 1) {
        nv += __shfl_down_sync(kFull, nv, o);
        mv += __shfl_down_sync(kFull, mv, o);
    }
    if ((threadIdx.x & 31) == 0) { atomicAdd(&out2[0], nv); atomicAdd(&out2[1], mv); }
}

// CSR validation + narrowing of row_ptr to uint32 (step a1)
__global__ void dfs_validate_rowptr_kernel(const int64_t* __restrict__ rp64, uint32_t* rp32, int64_t n,
                                           int64_t m, int* bad) {
    const size_t stride = (size_t)gridDim.x * blockDim.x;
    for (size_t v = blockIdx.x * (size_t)blockDim.x + threadIdx.x; v <= (size_t)n; v += stride) {
        const int64_t a = rp64[v];
        bool ok = a >= 0 && a <= m;
        if (v == 0) ok = ok && a == 0;
        if (v == (size_t)n) ok = ok && a == m;
        if (v < (size_t)n) ok = ok && rp64[v + 1] >= a;
        if (!ok) atomicExch(bad, 1);
        rp32[v] = (uint32_t)a;
    }
}

__global__ void dfs_validate_col_kernel(const int32_t* __restrict__ col, int64_t m, int64_t n, int* bad) {
    const size_t stride = (size_t)gridDim.x * blockDim.x;
    for (size_t j = blockIdx.x * (size_t)blockDim.x + threadIdx.x; j < (size_t)m; j += stride) {
        const int32_t c = col[j];
        if (c < 0 || (int64_t)c >= n) atomicExch(bad, 1);
    }
}

}  // namespace b200dfs
