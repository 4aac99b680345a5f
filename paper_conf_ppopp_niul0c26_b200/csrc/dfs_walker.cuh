// dfs_walker.cuh — sub-warp walkers: the persistent traversal kernel for low-degree graphs.
//
// The warp kernel (dfs_device.cuh) gives every warp ONE walker: the 32 lanes scan a 32-position
// window of the current vertex's adjacency list (the paper's warp-level DFS, §3.3).
// On road/mesh/path graphs (average degree 2-4) 28-30 of those lanes hold nothing,
// and the traversal is bound by the number of walkers times the latency of one claim chain
// (DESIGN.md §5, §8).  Here a warp runs 32/G independent walkers of G lanes each (G = 8 or 4):
// every walker is a complete DiggerBees agent — its own top entry ⟨u, i⟩, its own HotRing in
// shared memory and ColdSeg in global memory (§3.2, Fig 2), in-order window scan with
// __ballot_sync/__ffs over its G lanes and an atomic claim of the first unvisited neighbour
// (Alg 1 order per entry, reading S4) — and the warp issues the memory operations of all its
// walkers with the same instructions.  Per-walker control flow is predicated; the rare paths
// (flush, refill, steals) run warp-cooperatively for one walker at a time.
//
// Scheduling is the paper's hierarchy with the walker as the unit: intra-block stealing (Alg 3,
// P:1067-1091) from the HotRing TAIL of the walker with max hot_rest in the CTA (siblings in the
// same warp included), inter-block stealing (Alg 4) from the ColdSeg BOTTOM of the
// walker with max cold_rest in a two-choice victim block (reading S14/S15), the same
// reservation protocols (packed head/tail word under the victim lock, reading S12; packed
// {top, bottom} CAS) and the same termination detector (reading S13, walkers instead of warps).
// "P:a-b" = /root/reference/PAPER.md lines.
#pragma once
#include "dfs_device.cuh"

namespace b200dfs {

constexpr int kMaxWalkersPerCta = 512;
// CTA size the walker kernel is compiled for (threads): 28 warps x 72 registers (round-2 sweep,
// DESIGN.md §5); the runtime launches it with at most DFS_WALKER_LB / 32 warps
#ifndef DFS_WALKER_LB
#define DFS_WALKER_LB 896
#endif
#ifndef DFS_WALKER_FULLSCAN
#define DFS_WALKER_FULLSCAN 0
#endif
constexpr int kCntDonations = kNumCounters;         // walker kernel only (Ctl::counters has 24)
constexpr int kNumWCounters = kNumCounters + 1;

struct SmemW {
    uint32_t ht[kMaxWalkersPerCta];                 // HotRing (head << 16) | tail per walker
    volatile uint32_t tailf[kMaxWalkersPerCta];     // slots below tailf are free for reuse
    uint32_t lock[kMaxWalkersPerCta];               // tail-side lock per walker (thieves, flush)
    unsigned int lbusy;                             // walkers holding work + registered thieves
    volatile int done;
    uint32_t inter_token;                           // one Alg 4 scan per CTA at a time
    unsigned long long t_start;
    unsigned long long cnt[kMaxWarps][kNumWCounters];
};

__device__ __forceinline__ uint32_t atom_add_relaxed_cta_if_ret(bool p, uint32_t* a, uint32_t v) {
    uint32_t r = 0;
    asm volatile("{ .reg .pred q; setp.ne.u32 q, %1, 0; @q atom.relaxed.cta.shared.add.u32 %0, [%2], %3; }"
                 : "+r"(r) : "r"((uint32_t)p), "r"(smem_addr(a)), "r"(v) : "memory");
    return r;
}
__device__ __forceinline__ void atom_add_relaxed_cta_if(bool p, uint32_t* a, uint32_t v) {
    asm volatile("{ .reg .pred q; setp.ne.u32 q, %0, 0; @q atom.relaxed.cta.shared.add.u32 _, [%1], %2; }"
                 ::"r"((uint32_t)p), "r"(smem_addr(a)), "r"(v) : "memory");
}
__device__ __forceinline__ unsigned long long ld_shared_u64_if(bool p, const unsigned long long* a) {
    unsigned long long r = 0;
    asm volatile("{ .reg .pred q; setp.ne.u32 q, %1, 0; @q ld.shared.u64 %0, [%2]; }"
                 : "+l"(r) : "r"((uint32_t)p), "r"(smem_addr(a)) : "memory");
    return r;
}

// ------------------------------------------------------------------------------------------
// G = lanes per walker (4 or 8), H = HotRing entries per walker (power of two).
// Launched with blockDim.x = 32 * W (W <= 32), dynamic shared memory
// sizeof(SmemW) (16-byte padded) + W * (32 / G) * H * 8 bytes.
// Stack owners are walkers: cold_tb / chunk_tab are indexed by the global walker id
// blockIdx.x * (W * 32 / G) + warp * (32 / G) + walker.
// ------------------------------------------------------------------------------------------
template <int G, int H, bool STATS, bool REC>
__global__ void __launch_bounds__(DFS_WALKER_LB, 1) dfs_walker_kernel(const KParams P) {
    static_assert(G == 2 || G == 4 || G == 8 || G == 16, "G is 2, 4, 8 or 16");
    static_assert(!REC || G >= 8, "a vertex record spans 8 lanes");
    static_assert((H & (H - 1)) == 0 && H >= 32 && H <= 1024, "H is a power of two in [32, 1024]");
    constexpr int WPW = 32 / G;                       // walkers per warp
    constexpr uint32_t GM = (1u << G) - 1u;
#ifndef DFS_WALKER_PF
#define DFS_WALKER_PF 0
#endif
    // lanes prefetching their candidates' row_ptr pairs with the probes: none (round 2 A/B:
    // path 10^8 7.21 -> 6.67 ms, batch neutral; profiles/r02/ab/walker_pf.jsonl) — a candidate
    // claim loads its pair beside the claim atomic instead
    constexpr int kPf = G < DFS_WALKER_PF ? G : DFS_WALKER_PF;
    constexpr uint32_t kStealMax = H / 4;             // entries per steal (ring space, see refill)
    extern __shared__ __align__(16) unsigned char smem_raw[];
    SmemW& S = *reinterpret_cast<SmemW*>(smem_raw);
    constexpr int kCtlBytes = (sizeof(SmemW) + 15) & ~15;
    unsigned long long* const rings = reinterpret_cast<unsigned long long*>(smem_raw + kCtlBytes);

    const int lane = threadIdx.x & 31;
    const int w = threadIdx.x >> 5;
    const int W = blockDim.x >> 5;
    const int sl = lane & (G - 1);                    // lane within the walker
    const int wk = lane / G;                          // walker within the warp
    const int base = wk * G;
    const int NWB = W * WPW;                          // walkers per CTA
    const int bk = w * WPW + wk;                      // walker within the CTA
    const int gk = blockIdx.x * NWB + bk;             // global walker id (stack owner)
    unsigned long long* const ring = rings + (size_t)bk * H;
    const uint32_t tmask = (1u << P.tab_log2) - 1u;
    uint32_t* const my_tab = P.chunk_tab + ((size_t)gk << P.tab_log2);
    const uint32_t cap = P.ring_cap < (uint32_t)H ? P.ring_cap : (uint32_t)H;
    // flush / refill batch: the paper's hot_size / 2 with capacity hot_size - 1 (Fig 2),
    // i.e. (cap + 1) / 2 — H/2 at the default cap = H
    const uint32_t batch = (cap + 1u) / 2u;
    const uint32_t hs = P.hot_cutoff >= 2 ? (uint32_t)P.hot_cutoff >> 1 : 1u;   // h_s (Alg 3 l.12)
    const uint32_t cs = P.cold_cutoff >= 2 ? (uint32_t)P.cold_cutoff >> 1 : 1u; // c_s (Alg 4 l.17)

    for (int k = threadIdx.x; k < NWB; k += blockDim.x) { S.ht[k] = 0; S.tailf[k] = 0; S.lock[k] = 0; }
    if (threadIdx.x == 0) {
        S.done = 0; S.inter_token = 0;
        S.lbusy = (blockIdx.x == 0) ? 1u : 0u;        // walker 0 of block 0 holds the root
        S.t_start = globaltimer();
    }
    unsigned long long* const cnt = S.cnt[w];
    if (STATS && lane < kNumWCounters) cnt[lane] = 0;
    __syncthreads();

    auto seg = [&](uint32_t b) -> uint32_t { return (b >> base) & GM; };
    // STATS: add the number of lanes with p to counter idx (call convergently)
    auto count = [&](int idx, bool p) {
        if constexpr (STATS) {
            const uint32_t b = __ballot_sync(kFull, p);
            if (lane == 0) cnt[idx] += __popc(b);
        }
    };

    // ---- per-walker state (uniform over the walker's G lanes) ----
    bool has_top = false, have_win = false, need_end = false, active = false;
    uint32_t u = 0, i = 0, end = 0;
    int nb = -1;                                      // this lane's neighbour: position i + sl
    uint32_t my_head = 0, pub = 0, tail_cache = 0;    // HotRing (owner view)
    uint32_t my_top = 0, hi = 0, cold_lo = 0;         // ColdSeg top, mapped chunks, "empty at" hint
    bool spec_ok = false;
    uint32_t par = kFull;
    const bool spec_on = (P.speculate & 3) != 0;
    const bool spec_pop = spec_on && (P.speculate & 8) != 0;
    const bool spec_early = spec_on && (P.speculate & 4) != 0;
    uint32_t rng = P.seed ^ (0x9E3779B9u * (uint32_t)(blockIdx.x * W + w + 1));
    if (rng == 0) rng = 1;
    uint32_t iter = 0, my_claims = 0;

    if (blockIdx.x == 0 && bk == 0) {
        // Alg 1 l.1-3: the root was claimed by the reset kernel; <root, row_ptr[root]> is our top
        has_top = true; active = true;
        u = (uint32_t)P.root; i = __ldg(P.rp + u); end = __ldg(P.rp + u + 1);
    }

    // termination counters (reading S13), called by one lane per walker
    auto register_thief = [&]() {
        if (atomicAdd(&S.lbusy, 1u) == 0u) {
            if (atomicAdd(&P.ctl->busy, 1u) == 0xFFFFFFFFu) raise_error(P, kStatusEINTERNAL);
        }
    };
    auto deregister = [&]() {
        if (atomicSub(&S.lbusy, 1u) == 1u) {
            if (atomicSub(&P.ctl->busy, 1u) == 1u) { atomicExch(&P.ctl->done, 1u); S.done = 1; }
        }
    };

    // pop the newest HotRing entry of every walker with p (Fig 2(d)); private entries need no
    // synchronisation, the published head is taken with one atomic decrement (a thief's CAS on
    // the same word then fails).  Sets has_top for those walkers.
    auto pop_if = [&](bool p) {
        const bool priv = p && my_head != pub;
        const bool atom = p && !priv;
        uint32_t old = atom_add_relaxed_cta_if_ret(atom && sl == 0, &S.ht[bk], 0xFFFF0000u);   // head--
        old = __shfl_sync(kFull, old, 0, G);
        const bool got_pub = atom && ht_rest(old) >= 1;
        atom_add_relaxed_cta_if(atom && !got_pub && sl == 0, &S.ht[bk], 0x10000u);            // empty: undo
        const bool got = priv || got_pub;
        const uint32_t slot = priv ? my_head - 1u : ht_head(old) - 1u;
        const unsigned long long e = ld_shared_u64_if(got, ring + (slot & (H - 1)));
        if (got) {
            --my_head;
            if (got_pub) --pub;
            u = entry_v(e); i = entry_i(e);
            need_end = true; have_win = false; spec_ok = spec_pop; par = kFull;
        }
        if (p) has_top = got;
        count(kCntPops, got && sl == 0);
    };

    // ---------------------------------------------------------------- warp-cooperative slow paths
    // walker k's owner registers live in lanes k*G ..; these helpers read them with shuffles and
    // write the results back into walker k's lanes

    // flush: move up to `want` of walker k's oldest HotRing entries to its ColdSeg top, keeping at
    // least `keep` (Fig 2(e))
    auto flush_walker = [&](int k, uint32_t want, uint32_t keep) -> bool {
        const int kb = w * WPW + k;
        const int kg = blockIdx.x * NWB + kb;
        unsigned long long* const kring = rings + (size_t)kb * H;
        uint32_t* const ktab = P.chunk_tab + ((size_t)kg << P.tab_log2);
        const uint32_t k_head = __shfl_sync(kFull, my_head, k * G);
        const uint32_t k_pub = __shfl_sync(kFull, pub, k * G);
        uint32_t k_top = __shfl_sync(kFull, my_top, k * G);
        uint32_t k_hi = __shfl_sync(kFull, hi, k * G);
        if (k_head != k_pub && lane == 0) atom_add_release_cta(&S.ht[kb], ((k_head - k_pub) & 0xFFFFu) << 16);
        uint32_t t = 0;
        if (lane == 0) { smem_lock(&S.lock[kb]); t = ht_tail(ld_acquire_cta(&S.ht[kb])); }
        t = __shfl_sync(kFull, t, 0);
        __syncwarp();
        const uint32_t rest = (k_head - t) & 0xFFFFu;
        uint32_t kf = rest > keep ? rest - keep : 0u;
        if (kf > want) kf = want;
        bool ok = true;
        while (kf && ok && (unsigned long long)k_hi * kChunk < (unsigned long long)k_top + kf) {
            uint32_t c = 0;
            if (lane == 0) {
                c = pool_alloc(P);
                if (c != kEmptySlot) {
                    uint32_t* slot = &ktab[k_hi & tmask];
                    unsigned long long spins = 0;
                    while (ld_relaxed_u32(slot) != kEmptySlot) {   // chunk hi - 2^tab_log2 still read
                        if (++spins > (1ull << 26)) { c = kEmptySlot; break; }
                        __nanosleep(64);
                    }
                    if (c != kEmptySlot) { st_relaxed_u32(&P.chunk_consumed[c], 0u); st_relaxed_u32(slot, c); }
                }
            }
            c = __shfl_sync(kFull, c, 0);
            if (c == kEmptySlot) ok = false; else { ++k_hi; if (STATS && lane == 0) ++cnt[kCntChunks]; }
        }
        if (!ok) {
            if (lane == 0) { raise_error(P, kStatusENOMEM); smem_unlock(&S.lock[kb]); }
            __syncwarp();
            return false;
        }
        if (kf) {
            for (uint32_t q = lane; q < kf; q += 32u) {
                const unsigned long long e = kring[(t + q) & (H - 1)];
                const uint32_t p = k_top + q;
                const uint32_t c = ld_relaxed_u32(&ktab[(p >> kChunkLog2) & tmask]);
                st_cg_u64(P.pool + ((size_t)c << kChunkLog2) + (p & (kChunk - 1)), e);
            }
            fence_release_gpu();                              // every lane: its stores before the publish
            __syncwarp();
            if (lane == 0) {
                atomicAdd(&P.cold_tb[kg], (unsigned long long)kf << 32);     // publish top
                atomicAdd(&P.block_cold[blockIdx.x], (int)kf);
                uint32_t old = ld_acquire_cta(&S.ht[kb]);
                for (;;) {                                    // advance tail (thieves locked out)
                    const uint32_t nw = (old & 0xFFFF0000u) | ((t + kf) & 0xFFFFu);
                    const uint32_t got = atom_cas_acquire_cta(&S.ht[kb], old, nw);
                    if (got == old) break;
                    old = got;
                }
                S.tailf[kb] = (t + kf) & 0xFFFFu;
            }
            if (STATS && lane == 0) ++cnt[kCntFlushes];
        }
        if (lane == 0) smem_unlock(&S.lock[kb]);
        __syncwarp();
        if (wk == k) { my_top = k_top + kf; hi = k_hi; pub = k_head; tail_cache = (t + kf) & 0xFFFFu; }
        return true;
    };

    // refill walker k's empty HotRing from its ColdSeg top (Fig 2(f)); returns the
    // number of entries moved.  Ring space: a thief may still be copying <= kStealMax slots below
    // head, so head + batch - tailf <= H holds with batch <= H/2.
    auto refill_walker = [&](int k) -> uint32_t {
        const int kb = w * WPW + k;
        const int kg = blockIdx.x * NWB + kb;
        unsigned long long* const kring = rings + (size_t)kb * H;
        uint32_t* const ktab = P.chunk_tab + ((size_t)kg << P.tab_log2);
        const uint32_t k_head = __shfl_sync(kFull, my_head, k * G);
        const uint32_t k_top = __shfl_sync(kFull, my_top, k * G);
        uint32_t k_hi = __shfl_sync(kFull, hi, k * G);
        uint32_t take = 0;
        if (lane == 0) {
            unsigned long long old = ld_relaxed_u64(&P.cold_tb[kg]);
            for (;;) {
                const uint32_t bot = (uint32_t)old;
                const int avail = (int)(k_top - bot);
                if (avail <= 0) { take = 0; break; }
                take = avail < (int)batch ? (uint32_t)avail : batch;
                const unsigned long long nw = ((unsigned long long)(k_top - take) << 32) | bot;
                const unsigned long long got = atomicCAS(&P.cold_tb[kg], old, nw);
                if (got == old) break;
                old = got;
            }
        }
        take = __shfl_sync(kFull, take, 0);
        if (take == 0) {
            if (wk == k) cold_lo = my_top;                    // empty until the next flush
            return 0;
        }
        const uint32_t nbase = k_top - take;
        for (uint32_t q = lane; q < take; q += 32u) {
            const uint32_t p = nbase + q;
            const uint32_t c = ld_relaxed_u32(&ktab[(p >> kChunkLog2) & tmask]);
            kring[(k_head + q) & (H - 1)] = ld_cg_u64(P.pool + ((size_t)c << kChunkLog2) + (p & (kChunk - 1)));
        }
        // release chunks that lie wholly above top + one spare chunk (never read by thieves)
        while (k_hi > 0 && (unsigned long long)(k_hi - 1) * kChunk >= (unsigned long long)nbase + kChunk) {
            if (lane == 0) {
                uint32_t* slot = &ktab[(k_hi - 1) & tmask];
                const uint32_t c = ld_relaxed_u32(slot);
                st_relaxed_u32(slot, kEmptySlot);
                pool_free(P, c);
            }
            --k_hi;
        }
        __syncwarp();
        if (lane == 0) {
            atomicSub(&P.block_cold[blockIdx.x], (int)take);
            atom_add_release_cta(&S.ht[kb], take << 16);     // publish (ring was empty)
        }
        __syncwarp();
        if (wk == k) { my_top = nbase; hi = k_hi; my_head = k_head + take; pub = my_head; }
        if (STATS && lane == 0) ++cnt[kCntRefills];
        return take;
    };

    // deliver kst stolen entries to the thief walkers tb (bit k = walker k of this warp; all idle,
    // deregistered, with empty rings): entry q (oldest first) goes to the (q mod nt)-th thief, so
    // one steal can feed every idle walker of the warp.  Each receiver publishes its entries
    // (CTA-scope release) and becomes active; the thief registration made before the reservation
    // counts the first receiver, the others are added to the block count (>= 1, no global update).
    // Returns the receivers.
    auto deliver = [&](uint32_t tb, uint32_t kst, auto&& load_entry) -> uint32_t {
        const int nt = __popc(tb);
        for (uint32_t it = 0; it < (kst + 31u) / 32u; ++it) {
            const uint32_t q = lane + 32u * it;
            const int tw = (int)__fns(tb, 0, (int)(q % (uint32_t)nt) + 1);
            const uint32_t th = __shfl_sync(kFull, my_head, (tw & (WPW - 1)) * G);
            if (q < kst) rings[(size_t)(w * WPW + tw) * H + ((th + q / (uint32_t)nt) & (H - 1))] = load_entry(q);
        }
        __syncwarp();
        const int rank = __popc(tb & ((1u << wk) - 1u));
        const uint32_t cntw = (((tb >> wk) & 1u) && kst > (uint32_t)rank) ? (kst - (uint32_t)rank + (uint32_t)nt - 1u) / (uint32_t)nt : 0u;
        atom_add_release_cta_if(cntw != 0 && sl == 0, &S.ht[bk], cntw << 16);
        const uint32_t nr = kst < (uint32_t)nt ? kst : (uint32_t)nt;
        if (lane == 0 && nr > 1) atomicAdd(&S.lbusy, nr - 1);
        if (cntw) { my_head += cntw; pub = my_head; active = true; }
        __syncwarp();
        uint32_t got = 0;
#pragma unroll
        for (int k = 0; k < WPW; ++k) got |= (__ballot_sync(kFull, cntw != 0) >> (k * G) & 1u) << k;
        return got;
    };

    // Alg 3 for the thief walkers tb: the walker of this CTA with max hot_rest >= hot_cutoff
    // (siblings in this warp included); reserve from its tail under its lock, copy SMEM -> SMEM
    // Victim scan: a window of 32 walkers per attempt starting at this warp's own walkers and
    // rotating through the CTA (one shared load per lane), not all of the CTA's 32 x 32/G walkers
    // as Alg 3 l.5-10 does for 32 warps: with 256 walkers per CTA the full scan was 16% of the
    // batch's instructions.  DFS_WALKER_FULLSCAN = 1 builds the full scan (A/B).
    uint32_t scan_off = 0;
    auto steal_intra = [&](uint32_t tb) -> uint32_t {
        int best = -1, bidx = -1;
        auto consider = [&](int j) {
            if (j / WPW == w && ((tb >> (j % WPW)) & 1u)) return;    // a thief itself
            const int r = ht_rest(*(volatile uint32_t*)&S.ht[j]);
            if (r > best) { best = r; bidx = j; }
        };
#if DFS_WALKER_FULLSCAN
        for (int j = lane; j < NWB; j += 32) consider(j);
#else
        if (lane < NWB) consider((int)(((uint32_t)(w * WPW) + scan_off + (uint32_t)lane) % (uint32_t)NWB));
        scan_off += 32u;
#endif
        for (int att = 0; att < P.steal_tries; ++att) {
            const int mx = __reduce_max_sync(kFull, best);
            if (mx < P.hot_cutoff) break;
            const int who = __ffs(__ballot_sync(kFull, best == mx)) - 1;
            const int vj = __shfl_sync(kFull, bidx, who);
            if (STATS && lane == 0) ++cnt[kCntStealAttempts];
            uint32_t ok = 0, t = 0, kst = 0;
            if (lane == 0 && smem_trylock(&S.lock[vj])) {
                register_thief();                            // before reserving
                uint32_t old = *(volatile uint32_t*)&S.ht[vj];
                for (int tries = 0; tries < 8; ++tries) {
                    const int r = ht_rest(old);
                    if (r < P.hot_cutoff) break;
                    t = ht_tail(old);
                    kst = hs;
                    if (P.steal_half && (uint32_t)(r / 2) > kst) kst = (uint32_t)(r / 2);
                    if (kst > kStealMax) kst = kStealMax;
                    if ((int)kst > r) kst = (uint32_t)r;
                    const uint32_t nw = (old & 0xFFFF0000u) | ((t + kst) & 0xFFFFu);
                    const uint32_t got = atom_cas_acquire_cta(&S.ht[vj], old, nw);   // reserve
                    if (got == old) { ok = 1; break; }
                    old = got;
                }
                if (!ok) { smem_unlock(&S.lock[vj]); deregister(); }
            }
            ok = __shfl_sync(kFull, ok, 0);
            if (!ok) {
                if (lane == who) best = -1;                  // next best
                continue;
            }
            t = __shfl_sync(kFull, t, 0);
            kst = __shfl_sync(kFull, kst, 0);
            __syncwarp();                                    // lane 0's acquire -> all lanes
            const unsigned long long* vring = rings + (size_t)vj * H;
            const uint32_t got = deliver(tb, kst, [&](uint32_t q) { return vring[(t + q) & (H - 1)]; });
            if (lane == 0) {
                S.tailf[vj] = (t + kst) & 0xFFFFu;           // slots reusable by the owner
                smem_unlock(&S.lock[vj]);
            }
            __syncwarp();
            if (STATS && lane == 0) ++cnt[kCntIntraSteals];
            return got;
        }
        return 0u;
    };

    // Alg 4 for the thief walkers tb: two-choice victim block by cumulative ColdSeg load (reading
    // S14/S15), the walker with max cold_rest >= cold_cutoff, c_s entries from its ColdSeg bottom
    auto steal_inter = [&](uint32_t tb) -> uint32_t {
        int token = 0;
        if (lane == 0) token = (*(volatile uint32_t*)&S.inter_token == 0u && smem_trylock(&S.inter_token)) ? 1 : 0;
        token = __shfl_sync(kFull, token, 0);
        if (!token) return 0u;
        uint32_t got_work = 0;
        const int nB = gridDim.x;
        int vb = -1;
        {
            int nact = 0;
            for (int b0 = 0; b0 < nB; b0 += 32) {
                const int b = b0 + lane;
                const bool a = b < nB && ld_relaxed_s32(&P.block_cold[b]) > 0;
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
                    const int load = b < nB ? ld_relaxed_s32(&P.block_cold[b]) : 0;
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
                if (P.policy == 0 || pick2 < 0) vb = pick1;
                else vb = (load2 > load1 || (load2 == load1 && pick2 < pick1)) ? pick2 : pick1;
            }
        }
        if (STATS && lane == 0) ++cnt[kCntInterScans];
        if (vb >= 0) {
            int best = -1, bidx = -1;
            for (int j = lane; j < NWB; j += 32) {
                const unsigned long long word = ld_relaxed_u64(&P.cold_tb[(size_t)vb * NWB + j]);
                const int r = (int)((uint32_t)(word >> 32) - (uint32_t)word);
                if (r > best) { best = r; bidx = j; }
            }
            const int mx = __reduce_max_sync(kFull, best);
            if (mx >= P.cold_cutoff) {
                const int who = __ffs(__ballot_sync(kFull, best == mx)) - 1;
                const int vg = vb * NWB + __shfl_sync(kFull, bidx, who);
                if (STATS && lane == 0) ++cnt[kCntStealAttempts];
                uint32_t ok = 0, bot = 0, kst = 0;
                if (lane == 0) {
                    register_thief();
                    unsigned long long old = ld_relaxed_u64(&P.cold_tb[vg]);
                    for (int tries = 0; tries < 4; ++tries) {
                        const uint32_t top = (uint32_t)(old >> 32), b = (uint32_t)old;
                        const int r = (int)(top - b);
                        if (r < P.cold_cutoff) break;
                        kst = cs;
                        if (P.steal_half && (uint32_t)(r / 2) > kst) kst = (uint32_t)(r / 2);
                        if (kst > kStealMax) kst = kStealMax;
                        if ((int)kst > r) kst = (uint32_t)r;
                        const unsigned long long nw = ((unsigned long long)top << 32) | (uint32_t)(b + kst);
                        const unsigned long long got = atomicCAS(&P.cold_tb[vg], old, nw);   // reserve
                        if (got == old) { ok = 1; bot = b; break; }
                        old = got;
                    }
                    if (ok) fence_acquire_gpu();             // Alg 4 l.20 (pairs with the owner's release)
                    else deregister();
                }
                ok = __shfl_sync(kFull, ok, 0);
                if (ok) {
                    bot = __shfl_sync(kFull, bot, 0);
                    kst = __shfl_sync(kFull, kst, 0);
                    __syncwarp();
                    uint32_t* vtab = P.chunk_tab + ((size_t)vg << P.tab_log2);
                    got_work = deliver(tb, kst, [&](uint32_t q) {
                        const uint32_t p = bot + q;
                        const uint32_t c = ld_relaxed_u32(&vtab[(p >> kChunkLog2) & tmask]);
                        return c < P.n_chunks ? ld_cg_u64(P.pool + ((size_t)c << kChunkLog2) + (p & (kChunk - 1)))
                                              : pack_entry((uint32_t)P.root, P.m);   // owner exited on an error
                    });
                    if (lane == 0) {
                        uint32_t p = bot, left = kst;
                        while (left) {                       // chunk accounting (see the warp kernel)
                            const uint32_t in_chunk = kChunk - (p & (kChunk - 1));
                            const uint32_t part = left < in_chunk ? left : in_chunk;
                            uint32_t* slot = &vtab[(p >> kChunkLog2) & tmask];
                            const uint32_t c = ld_relaxed_u32(slot);
                            if (c < P.n_chunks) {
                                const uint32_t before = atomicAdd(&P.chunk_consumed[c], part);
                                if (before + part == kChunk) { st_relaxed_u32(slot, kEmptySlot); pool_free(P, c); }
                            }
                            p += part; left -= part;
                        }
                        atomicSub(&P.block_cold[vb], (int)kst);
                    }
                    __syncwarp();
                    if (STATS && lane == 0) ++cnt[kCntInterSteals];
                }
            }
        }
        if (lane == 0) smem_unlock(&S.inter_token);
        return got_work;
    };

    // ---------------------------------------------------------------- stack-script mode (tests)
    // STATS builds only (dfs_debug_stack_script): warp 0 of block 0 drives its walkers' stack
    // operations — the same lambdas the traversal uses — through a script of 6-int records, so the
    // paper's worked examples (Figs 2 and 3) can be replayed on the real stack code.
    if constexpr (STATS) {
        if (P.script) {
            if (blockIdx.x == 0 && w == 0) {
                int oc = 0;                                   // output cursor (lane 0 writes)
                auto put = [&](int32_t x) { if (lane == 0 && oc < P.script_out_len) P.script_out[oc] = x; ++oc; };
                for (int pc = 0; pc < P.script_len; ++pc) {
                    const int32_t* r = P.script + 6 * pc;
                    const int op = r[0], k = r[1] & (WPW - 1);
                    const int kb = w * WPW + k, kg = blockIdx.x * NWB + kb;
                    uint32_t* const ktab = P.chunk_tab + ((size_t)kg << P.tab_log2);
                    unsigned long long* const kring = rings + (size_t)kb * H;
                    if (op == 0) break;
                    if (op == 1) {                            // SET k head tail top bottom
                        const uint32_t hd = (uint32_t)r[2] & 0xFFFFu, tl = (uint32_t)r[3] & 0xFFFFu;
                        const uint32_t top = (uint32_t)r[4], bot = (uint32_t)r[5];
                        uint32_t nh = 0;
                        if (lane == 0) {
                            S.ht[kb] = (hd << 16) | tl; S.tailf[kb] = tl;
                            P.cold_tb[kg] = ((unsigned long long)top << 32) | bot;
                            atomicAdd(&P.block_cold[blockIdx.x], (int)(top - bot));
                            for (uint32_t c = 0; (unsigned long long)c * kChunk < top; ++c, ++nh) {
                                const uint32_t id = pool_alloc(P);
                                st_relaxed_u32(&P.chunk_consumed[id], 0u); st_relaxed_u32(&ktab[c & tmask], id);
                            }
                        }
                        nh = __shfl_sync(kFull, nh, 0);
                        __syncwarp();
                        if (wk == k) { my_head = hd; pub = hd; tail_cache = tl; my_top = top; hi = nh; cold_lo = ~top; has_top = false; }
                    } else if (op == 2 || op == 3) {          // RING k counter v i  /  COLD k pos v i
                        if (lane == 0) {
                            const unsigned long long e = pack_entry((uint32_t)r[3], (uint32_t)r[4]);
                            const uint32_t q = (uint32_t)r[2];
                            if (op == 2) kring[q & (H - 1)] = e;
                            else P.pool[((size_t)ktab[(q >> kChunkLog2) & tmask] << kChunkLog2) + (q & (kChunk - 1))] = e;
                        }
                        __syncwarp();
                    } else if (op == 4) {                     // PUSH k v i (Fig 2(c))
                        const bool me = wk == k;
                        st_shared_u64_if(me && sl == 0, ring + (my_head & (H - 1)), pack_entry((uint32_t)r[2], (uint32_t)r[3]));
                        atom_add_release_cta_if(me && sl == 0, &S.ht[bk], 0x10000u);
                        if (me) { ++my_head; pub = my_head; }
                        __syncwarp();
                    } else if (op == 5) {                     // POP k (Fig 2(d)) -> popped (v, i) or (-1, -1)
                        pop_if(wk == k);
                        const int got = __shfl_sync(kFull, (int)has_top, k * G);
                        const uint32_t pv = __shfl_sync(kFull, u, k * G), pi = __shfl_sync(kFull, i, k * G);
                        put(got ? (int32_t)pv : -1); put(got ? (int32_t)pi : -1);
                        if (wk == k) has_top = false;
                    } else if (op == 6) {                     // FLUSH k want keep (Fig 2(e))
                        flush_walker(k, (uint32_t)r[2], (uint32_t)r[3]);
                    } else if (op == 7) {                     // REFILL k (Fig 2(f)) -> entries moved
                        put((int32_t)refill_walker(k));
                    } else if (op == 8 || op == 9) {          // STEAL_INTRA / STEAL_INTER thief-mask (Fig 3)
                        const uint32_t tb = (uint32_t)r[1] & ((1u << WPW) - 1u);
                        put((int32_t)(op == 8 ? steal_intra(tb) : steal_inter(tb)));
                    } else if (op == 10) {                    // DUMP k -> head tail top bottom
                        const uint32_t x = S.ht[kb];
                        const unsigned long long c = P.cold_tb[kg];
                        put((int32_t)ht_head(x)); put((int32_t)ht_tail(x));
                        put((int32_t)(uint32_t)(c >> 32)); put((int32_t)(uint32_t)c);
                    } else if (op == 11 || op == 12) {        // READ_RING k counter / READ_COLD k pos -> v i
                        const uint32_t q = (uint32_t)r[2];
                        const unsigned long long e = op == 11 ? kring[q & (H - 1)]
                            : P.pool[((size_t)ktab[(q >> kChunkLog2) & tmask] << kChunkLog2) + (q & (kChunk - 1))];
                        put((int32_t)entry_v(e)); put((int32_t)entry_i(e));
                    }
                    __syncwarp();
                }
            }
            return;
        }
    }

    // ---------------------------------------------------------------- main loop (Alg 2)
    for (;;) {
        if (__any_sync(kFull, has_top)) {
            const bool act = has_top;
            // ---- ring space for the one push this step may make (flush first, Fig 2(e))
            {
                bool full = act && ((my_head - tail_cache) & 0xFFFFu) >= cap;
                if (__any_sync(kFull, full)) {
                    if (full) tail_cache = S.tailf[bk];
                    full = act && ((my_head - tail_cache) & 0xFFFFu) >= cap;
                    uint32_t fb = __ballot_sync(kFull, full && sl == 0);
                    bool fail = false;
                    while (fb) {
                        const int k = (__ffs(fb) - 1) / G;
                        fb &= fb - 1;
                        if (!flush_walker(k, batch, 0u)) { fail = true; break; }
                    }
                    if (fail) goto exit_loop;
                }
            }
            // ---- window of walkers whose top came from a pop (end not yet known)
            {
                const bool lw = act && !have_win;
                const uint32_t e2 = ld_nc_if(lw && need_end, P.rp + u + 1, end);
                const int x = (int)ld_nc_if(lw && i + (uint32_t)sl < P.m, P.col + i + sl, kFull);
                if (lw) { nb = x; end = e2; need_end = false; have_win = true; }
            }
            count(kCntWindows, act && sl == 0);
            // ===== expansion step (Alg 1 l.5-12 over a G-position window), all walkers at once
            const bool valid = act && i + (uint32_t)sl < end;
            const bool have_nxt = act && i + (uint32_t)G < end;
            const int nxt = (int)ld_nc_if(have_nxt && i + (uint32_t)(G + sl) < end, P.col + i + G + sl, kFull);
            // speculative claim: the first position whose neighbour is not the parent we came from
            // is, if unvisited, exactly Alg 1's next tree edge
            const uint32_t vbs = seg(__ballot_sync(kFull, spec_ok && valid && (uint32_t)nb != par));
            const int sk = vbs ? __ffs(vbs) - 1 : -1;
            const uint32_t svx = (uint32_t)__shfl_sync(kFull, nb, sk & (G - 1), G);
            const uint32_t sv = vbs ? svx : u;
            uint32_t s_old = atom_or_if(vbs != 0 && sl == 0, P.bitmap + 2u * (sv >> 5), 1u << (sv & 31));
            // the claimed child's list: with vertex records (REC) one 32-byte load gives its
            // first 6 neighbours and its row_ptr pair — no dependent col load for
            // lists of <= 6 entries; else the row_ptr pair, then the window
            uint32_t s_rs, s_re;
            int cnb;
            if constexpr (REC) {
                const uint32_t rw = ld_nc_if(vbs != 0 && sl < 8, P.rec + 8u * sv + sl, kFull);
                s_rs = __shfl_sync(kFull, rw, 6, G); s_re = __shfl_sync(kFull, rw, 7, G);
                const int cx = (int)ld_nc_if(vbs != 0 && sl >= 6 && s_rs + sl < s_re, P.col + s_rs + sl, kFull);
                cnb = sl < 6 ? (int)rw : cx;
            } else {
                s_rs = ld_nc_if(vbs != 0, P.rp + sv, 0u); s_re = ld_nc_if(vbs != 0, P.rp + sv + 1, 0u);
            }
            // probes of the visited bits ({visited, leaf} pair: one 8-byte L2 load); without
            // records the first kPf lanes also load their candidates' row_ptr pairs
            const uint2 wl = ld_cg_u2_if(valid, P.bitmap + 2u * ((uint32_t)nb >> 5), kFull, 0u);
            const bool pf = !REC && valid && sl < kPf;
            const uint32_t prs = ld_nc_if(pf, P.rp + nb, 0u), pre = ld_nc_if(pf, P.rp + nb + 1, 0u);
            if constexpr (!REC) cnb = (int)ld_nc_if(spec_early && vbs != 0 && s_rs + sl < s_re, P.col + s_rs + sl, kFull);
            const bool unv = valid && !((wl.x >> (nb & 31)) & 1u) && sl != sk;   // sk is claimed either way
            const bool lf = unv && ((wl.y >> (nb & 31)) & 1u);
            bool cand = unv && !lf;
            // bulk leaf claims (reading S24): a leaf's only in-list is u's and this walker is its
            // only scanner, so the probe's "unvisited" still holds; fire-and-forget red.or
            if (__any_sync(kFull, lf)) {
                red_or_if(lf, P.bitmap + 2u * ((uint32_t)nb >> 5), 1u << (nb & 31));
                st_global_if(lf, P.parent + nb, (int32_t)u);                  // Alg 1 l.10
                if (P.block_claims) my_claims += __popc(seg(__ballot_sync(kFull, lf)));
                count(kCntClaims, lf);
            }
            s_old = __shfl_sync(kFull, s_old, 0, G);
            bool won = vbs != 0 && !(s_old & (1u << (sv & 31)));
            count(kCntFailedClaims, vbs != 0 && !won && sl == 0);
            uint32_t v = sv, vrs = s_rs, vre = s_re;
            int kpos = sk;
            if (!REC && !spec_early) cnb = (int)ld_nc_if(won && vrs + sl < vre, P.col + vrs + sl, kFull);
            // claim the first unvisited candidate in CSR order; on a lost race try the next (all
            // walkers that still search advance together)
            bool need = act && !won;
            for (;;) {
                const uint32_t anyc = seg(__ballot_sync(kFull, cand));
                const bool tr = need && anyc != 0;
                if (!__any_sync(kFull, tr)) break;
                const int k = anyc ? __ffs(anyc) - 1 : 0;
                const uint32_t cv = (uint32_t)__shfl_sync(kFull, nb, k, G);
                const uint32_t bit = 1u << (cv & 31);
                uint32_t crs, cre, old;
                int cw;
                if constexpr (REC) {                         // the record load overlaps the claim
                    old = atom_or_if(tr && sl == 0, P.bitmap + 2u * (cv >> 5), bit);
                    const uint32_t rw = ld_nc_if(tr && sl < 8, P.rec + 8u * cv + sl, kFull);
                    crs = __shfl_sync(kFull, rw, 6, G); cre = __shfl_sync(kFull, rw, 7, G);
                    const int cx = (int)ld_nc_if(tr && sl >= 6 && crs + sl < cre, P.col + crs + sl, kFull);
                    cw = sl < 6 ? (int)rw : cx;
                } else {
                    crs = __shfl_sync(kFull, prs, k & (kPf - 1), G); cre = __shfl_sync(kFull, pre, k & (kPf - 1), G);
                    crs = ld_nc_if(tr && k >= kPf, P.rp + cv, crs);
                    cre = ld_nc_if(tr && k >= kPf, P.rp + cv + 1, cre);
                    old = atom_or_if(tr && sl == 0, P.bitmap + 2u * (cv >> 5), bit);
                    cw = (int)ld_nc_if(tr && crs + sl < cre, P.col + crs + sl, kFull);   // overlaps the claim
                }
                old = __shfl_sync(kFull, old, 0, G);
                const bool ok = tr && !(old & bit);
                if (ok) { won = true; v = cv; vrs = crs; vre = cre; kpos = k; cnb = cw; need = false; }
                if (tr && !ok && sl == k) cand = false;      // lost the race: next candidate
                count(kCntFailedClaims, tr && !ok && sl == 0);
            }
            // ---- descend (Alg 1 l.8-11) or continue u's scan
            const uint32_t later = seg(__ballot_sync(kFull, cand && sl > kpos));
            const uint32_t ni = later ? i + (uint32_t)(__ffs(later) - 1) : i + (uint32_t)G;
            st_global_if(won && sl == 0, P.parent + v, (int32_t)u);             // Alg 1 l.10
            count(kCntClaims, won && sl == 0);
            if (P.block_claims && won) ++my_claims;
            // leaf skip: v's list is empty or exactly [u] -- Alg 1 would descend, find nothing
            // unvisited and pop straight back to <u, ni>; stay on u instead
            const int c0 = __shfl_sync(kFull, cnb, 0, G);
            const bool leafskip = won && P.leaf_skip && vre - vrs <= 1u && (vre == vrs || (uint32_t)c0 == u);
            uint32_t next_i = leafskip ? ni : i + (uint32_t)G;
            const bool advance = act && (!won || leafskip);
            const bool descend = won && !leafskip;
            // continue u's scan at next_i: shift the window down when it still overlaps (leaf
            // skip), take the loaded next window, or pop when u is exhausted
            const uint32_t d = next_i - i;
            const int src = sl + (int)d;
            const int xs = __shfl_sync(kFull, nb, src & (G - 1), G);
            const bool shift = advance && next_i < end && d < (uint32_t)G;
            const int y = (int)ld_nc_if(shift && src >= G && next_i + sl < end, P.col + next_i + sl, kFull);
            bool exhausted = false;
            if (advance) {
                i = next_i;
                if (shift) { nb = src < G ? xs : y; spec_ok = spec_on; par = kFull; }
                else if (have_nxt && d == (uint32_t)G) { nb = nxt; spec_ok = false; }
                else { exhausted = true; have_win = false; }
            }
            // push <u, ni> unless u is exhausted (positions whose probe saw a claimed target stay
            // claimed, so skipping them keeps Alg 1's order), publish at once (CTA-scope release).
            // Donation (B200 addition): while a sibling walker of this warp holds
            // nothing, the entry goes to that sibling as its top instead — a register move, no
            // ring or atomic; <u, ni> is still scanned in order by exactly one walker.  The
            // donor is registered, so the block count is >= 1 and the receiver's registration
            // needs no global update.
            bool do_push = descend && ni < end;
            if (P.donate) {
                const uint32_t pm = __ballot_sync(kFull, do_push && sl == 0);
                const uint32_t im = __ballot_sync(kFull, !act && sl == 0);
                if (pm && im) {
                    const uint32_t below = (1u << base) - 1u;
                    const int rp_ = __popc(pm & below), ri_ = __popc(im & below);
                    const bool give = do_push && rp_ < __popc(im);
                    const bool recv = !act && ri_ < __popc(pm);
                    const int srcl = recv ? (int)__fns(pm, 0, ri_ + 1) : lane;
                    const uint32_t du = __shfl_sync(kFull, u, srcl);
                    const uint32_t dni = __shfl_sync(kFull, ni, srcl);
                    const uint32_t dend = __shfl_sync(kFull, end, srcl);
                    atom_add_relaxed_cta_if(recv && !active && sl == 0, &S.lbusy, 1u);
                    count(kCntDonations, recv && sl == 0);
                    if (recv) {
                        has_top = true; active = true;
                        u = du; i = dni; end = dend;
                        have_win = false; need_end = false; spec_ok = spec_pop; par = kFull;
                    }
                    if (give) do_push = false;
                }
            }
            st_shared_u64_if(do_push && sl == 0, ring + (my_head & (H - 1)), pack_entry(u, ni));
            atom_add_release_cta_if(do_push && sl == 0, &S.ht[bk], 0x10000u);
            if (do_push) { ++my_head; pub = my_head; }
            if (descend) {
                par = u; u = v; i = vrs; end = vre; spec_ok = spec_on;
                nb = cnb; have_win = true; need_end = false;
            }
            if (__any_sync(kFull, exhausted)) pop_if(exhausted);           // Alg 1 l.14
            // ---- periodic work: demand-driven spill, done flag and watchdog
            if ((++iter & P.period_mask) == 0) {
                if (P.spill) {
                    uint32_t want = 0;
                    if (sl == 0 && has_top) {
                        const uint32_t rest = (my_head - ht_tail(ld_acquire_cta(&S.ht[bk]))) & 0xFFFFu;
                        if (rest >= 2u * (uint32_t)P.cold_cutoff) {
                            const uint32_t busy_blocks = *(volatile unsigned int*)&P.ctl->busy;
                            if ((int)((gridDim.x - busy_blocks) * NWB) >= P.spill_idle) want = rest / 2;
                        }
                    }
                    uint32_t sb = __ballot_sync(kFull, want != 0);
                    bool fail = false;
                    while (sb) {
                        const int k = (__ffs(sb) - 1) / G;
                        sb &= sb - 1;
                        const uint32_t wk_want = __shfl_sync(kFull, want, k * G);
                        if (!flush_walker(k, wk_want, wk_want)) { fail = true; break; }
                        if (STATS && lane == 0) ++cnt[kCntSpills];
                    }
                    if (fail) goto exit_loop;
                }
                if ((iter & 1023u) == 0) {
                    if (__shfl_sync(kFull, (int)(*(volatile unsigned int*)&P.ctl->done), 0)) { if (lane == 0) S.done = 1; break; }
                    if (__shfl_sync(kFull, (int)(globaltimer() - S.t_start > P.timeout_ns), 0)) {
                        if (lane == 0) { raise_error(P, kStatusETIMEOUT); S.done = 1; }
                        break;
                    }
                }
            }
        }

        // ===== walkers without a top: refill from the own ColdSeg, else steal (Alg 2 l.6-7)
        if (!__any_sync(kFull, !has_top)) continue;
        {
            uint32_t rb = __ballot_sync(kFull, !has_top && sl == 0 && my_top != cold_lo);
            uint32_t gotw = 0;
            while (rb) {
                const int k = (__ffs(rb) - 1) / G;
                rb &= rb - 1;
                if (refill_walker(k)) gotw |= GM << (k * G);
            }
            if (gotw) pop_if(((gotw >> lane) & 1u) != 0);
        }
        // newly idle walkers leave the busy count — only once their ColdSeg is empty (the refill
        // above found nothing: cold_lo == my_top); a walker whose refilled entries were all
        // stolen before its pop keeps its registration and refills again
        {
            const bool dereg = !has_top && active && my_top == cold_lo;
            if (dereg && sl == 0) deregister();
            if (dereg) active = false;
            __syncwarp();
        }
        // idle = no top and deregistered (a walker whose ColdSeg may still hold entries stays
        // registered and retries its refill on the next pass; it never steals: a thief
        // registers before it reserves, so only deregistered walkers may steal)
        const uint32_t idle_mask = __ballot_sync(kFull, !has_top && !active && sl == 0);
        if (idle_mask == 0) continue;
        uint32_t idle_w = 0;                                  // idle walkers, bit k = walker k
#pragma unroll
        for (int k = 0; k < WPW; ++k) idle_w |= ((idle_mask >> (k * G)) & 1u) << k;
        if (idle_w != (1u << WPW) - 1u) {
            // some walkers of this warp are busy: one Alg 3 steal for all idle walkers every
            // steal_period steps (the busy walkers wait for it)
            if ((iter & P.steal_period_mask) == 0 && P.intra) {
                const uint32_t got = steal_intra(idle_w);
                if (got) pop_if(((got >> wk) & 1u) != 0);
            }
            continue;
        }
        // ===== the whole warp is idle: steal with backoff until a walker has work
        {
            uint32_t backoff = P.backoff_min_ns;
            uint32_t idle_iter = 0;
            uint32_t got = 0;                                 // walkers that got work
            for (;;) {
                if (__shfl_sync(kFull, S.done, 0)) goto exit_loop;
                if (w == 0 && __shfl_sync(kFull, (int)(*(volatile unsigned int*)&P.ctl->done), 0)) {
                    if (lane == 0) S.done = 1;
                    goto exit_loop;
                }
                if ((idle_iter++ & 15u) == 0 &&
                    __shfl_sync(kFull, (int)(globaltimer() - S.t_start > P.timeout_ns), 0)) {
                    if (lane == 0) { raise_error(P, kStatusETIMEOUT); S.done = 1; }
                    goto exit_loop;
                }
                // one steal for all walkers of the warp: Alg 3, else Alg 4
                if (P.intra) got = steal_intra(idle_w);
                if (!got && P.inter && gridDim.x > 1) got = steal_inter(idle_w);
                if (got) break;
                __nanosleep(backoff);
                if (backoff < P.backoff_max_ns) backoff <<= 1;
            }
            pop_if(((got >> wk) & 1u) != 0);
        }
    }
exit_loop:
    __syncwarp();
    // release the ColdSeg chunks still mapped by each walker (clean termination only: after an
    // error other warps may still steal from them; the host then re-initialises the table)
    if (__shfl_sync(kFull, lane == 0 ? (fence_acquire_gpu(), ld_relaxed_s32(&P.ctl->status)) : 0, 0) == 0) {
        const unsigned long long word = ld_relaxed_u64(&P.cold_tb[gk]);
        const uint32_t lo = (uint32_t)word >> kChunkLog2;
        for (uint32_t k = lo + sl; k < hi; k += G) {
            uint32_t* slot = &my_tab[k & tmask];
            if (ld_relaxed_u32(slot) != kEmptySlot) st_relaxed_u32(slot, kEmptySlot);
        }
    }
    if (P.block_claims && sl == 0 && my_claims) atomicAdd(&P.block_claims[blockIdx.x], (unsigned long long)my_claims);
    if (STATS && (P.collect_stats != 2 || gk == 0)) {
#pragma unroll
        for (int k = 0; k < kNumWCounters; ++k)
            if (lane == 0 && cnt[k]) atomicAdd(&P.ctl->counters[k], cnt[k]);
        __syncwarp();
    }
}

}  // namespace b200dfs
