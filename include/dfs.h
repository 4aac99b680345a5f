/*
 * dfs.h — C ABI of the B200-native unordered-DFS library (libdfs.so).
 *
 * Operation (DiggerBees, PPoPP '26; "P:a-b" = /root/reference/PAPER.md lines):
 *   Given a CSR graph and a root r, discover every vertex reachable from r and build a DFS tree
 *   (§2.1).  Output semantics are Table 2's "DiggerBees" row: the visited
 *   set and the parent array of a valid DFS tree, lexicographic order NOT enforced ("Unordered").
 *   The traversal is the paper's hierarchical work-stealing DFS (§3) re-designed for
 *   sm_100a: a persistent kernel, per-warp two-level stacks (shared-memory HotRing + global
 *   ColdSeg, §3.2), warp-level expansion with atomic claims (§3.3), intra-block (§3.4, Alg 3)
 *   and inter-block (§3.5, Alg 4) stealing, and a global termination detector.
 *
 * Graph convention
 *   row_ptr[n+1] (int64), col_idx[m] (int32): directed out-adjacency in CSR.
 *   An undirected graph is passed with both directions.  Self loops and duplicates are allowed
 *   (a self loop is never a tree edge; for duplicates the first occurrence is the tree position).
 *   Requirements: 1 <= n <= 2^31 - 3, 0 <= m < 2^32, row_ptr[0] == 0, row_ptr non-decreasing,
 *   row_ptr[n] == m, 0 <= col_idx[j] < n.  Violations -> DFS_EINVAL.
 *
 * Output convention (parent_out, int32[n])
 *   parent_out[root] = DFS_ROOT_PARENT (-1)  (Alg 1 line 1)
 *   parent_out[v]    = DFS_UNREACHED (-2)    for every vertex not reachable from root
 *   parent_out[v]    = u                     otherwise: (u,v) is an edge and u is v's DFS-tree parent
 *   visited(v) <=> parent_out[v] != DFS_UNREACHED.  The result satisfies checks I1-I6 of
 *   DESIGN.md (scan-order-consistent DFS tree); with dfs_options.deterministic = 1 it equals
 *   Alg 1's lexicographic tree exactly.
 *
 * Memory / ownership
 *   Input and output pointers may be host or device memory (detected per call with
 *   cudaPointerGetAttributes).  dfs_graph_create COPIES the CSR to the current CUDA device; the
 *   caller keeps ownership of its arrays and may free them after the call.  The handle owns all
 *   device memory it uses (graph, visited bitmap, stack-chunk pool sized from n, counters);
 *   runs never allocate device memory, except an internal parent buffer allocated on first use
 *   when parent_out is host memory.  Output buffers are caller-allocated and fully overwritten
 *   on DFS_OK; their contents are unspecified on error.
 *
 * Synchronisation / threading
 *   Every call is synchronous: it is stream-ordered on the handle's stream (default: the legacy
 *   default stream; see dfs_set_stream) and returns after the outputs are written.  One call at
 *   a time per handle; distinct handles are independent.  All calls must be made with the
 *   handle's device current (else DFS_EDEVICE).
 *
 * Errors
 *   Functions returning int return DFS_OK (0) or a negative dfs_status.  dfs_graph_create
 *   returns NULL on failure.  dfs_last_error() returns the status of the last failing call on
 *   the calling thread.  dfs_graph_destroy(NULL) is a no-op.
 */
#ifndef B200_DFS_H
#define B200_DFS_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct dfs_graph dfs_graph;   /* opaque */

enum dfs_status {
    DFS_OK        =  0,
    DFS_EINVAL    = -1,   /* NULL pointer, bad sizes, root out of range, malformed CSR        */
    DFS_ENOMEM    = -2,   /* device allocation failed or stack-chunk pool exhausted            */
    DFS_ECUDA     = -3,   /* CUDA runtime error (launch failure, no device, ...)               */
    DFS_EDEVICE   = -4,   /* current device differs from the handle's device                   */
    DFS_ETIMEOUT  = -5,   /* traversal watchdog fired (dfs_options.timeout_ms)                 */
    DFS_EINTERNAL = -6    /* internal consistency check failed                                 */
};

#define DFS_ROOT_PARENT (-1)
#define DFS_UNREACHED   (-2)

/* Victim-block policies for inter-block stealing (Alg 4 step 1). */
enum dfs_victim_policy {
    DFS_VICTIM_RANDOM     = 0,   /* uniform random active block (Fig 9 baseline) */
    DFS_VICTIM_TWO_CHOICE = 1    /* power-of-two-choices by cumulative ColdSeg load (default) */
};

/* Tuning / ablation options.  Zero-initialise, then call dfs_options_default. */
typedef struct dfs_options {
    int32_t blocks;          /* persistent grid size; 0 = (#SMs x resident blocks per SM)          */
    int32_t warps_per_block; /* 1..32; 0 = 32                                                      */
    int32_t hot_cutoff;      /* Alg 3 threshold: steal h_s = max(1, hot_cutoff/2) entries when a peer
                                holds >= hot_cutoff (h_s <= 32); paper 32; default 1      */
    int32_t cold_cutoff;     /* Alg 4 threshold: steal c_s = max(1, cold_cutoff/2) entries (<= 64)
                                when a ColdSeg holds >= cold_cutoff; paper 64; default 1   */
    int32_t deterministic;   /* 1: one warp, no stealing: result == Alg 1 lexicographic tree       */
    int32_t intra_steal;     /* 1: enable Alg 3 (default)                                          */
    int32_t inter_steal;     /* 1: enable Alg 4 (default)                                          */
    int32_t victim_policy;   /* dfs_victim_policy; default DFS_VICTIM_TWO_CHOICE                   */
    int32_t timeout_ms;      /* watchdog; default 120000                                           */
    uint32_t seed;           /* RNG seed for victim selection                                      */
    int32_t collect_stats;   /* 1: fill the counters of dfs_stats (small overhead)                 */
    int32_t spill;           /* 1: demand-driven spill — a busy warp whose HotRing holds >=
                                2*cold_cutoff entries moves the oldest half to its ColdSeg when
                                >= spill_idle warps are idle (B200 design); default 1 */
    int32_t inter_any;       /* 1: any idle warp that finds no intra-block victim may steal
                                inter-block; 0: only the leader warp of an idle block (Alg 4,
                                P:1150-1152); default 1                                            */
    int32_t spill_idle;      /* idle-warp threshold of the spill; default 32                       */
    int32_t backoff_max_ns;  /* cap of the idle warps' exponential __nanosleep backoff; default 2048 */
    int32_t window;          /* expansion window in positions: 32 (one neighbour per lane) or 128
                                (four per lane, one 128-bit load); 0 = auto (128 iff m >= 8n)      */
    int32_t pub_batch;       /* the owner publishes its HotRing head to thieves every pub_batch
                                pushes (entries above it are private); default 1                    */
    int32_t speculate;       /* bits 0-1: 1 = claim a freshly descended child's first non-parent
                                neighbour in parallel with the visited probes; 0 = off; 2 = on for
                                32-wide windows only.  bit 2: load the claimed child's first
                                32-wide window as soon as its row_ptr pair arrives, before the
                                claim's result (discarded if the claim fails).  bit 3: also claim
                                a popped entry's next
                                position speculatively (its probe saw it unvisited when the entry
                                was pushed).  Default 2|4|8                                          */
    int32_t steal_half;      /* 1 (default): a thief takes max(h_s, rest/2) <= 32 HotRing entries
                                (resp. max(c_s, rest/2) <= 64 ColdSeg entries); 0: exactly h_s/c_s
                                as in Alg 3/4                                                       */
    int32_t concurrency;     /* batches: number of traversals run concurrently on the GPU, each on
                                its own stream and a 1/concurrency share of the SMs (SURVEY
                                §8(f)-2); 0 = auto (8, capped by the number of roots; a single
                                dfs_run is always 1; at most 16).  Slots beyond the first allocate
                                their scratch on first use.                                        */
    int32_t ring_cap;        /* usable HotRing entries (0 = all 256); 2 makes every push spill: the
                                "one-level stack" of the paper's v1 (Fig 8)            */
    int32_t backoff_min_ns;  /* first __nanosleep of an idle warp's backoff; default 32           */
    int32_t max_pool_chunks; /* fault injection: cap on ColdSeg chunks a traversal may use (0 = the
                                whole pool); exhausting it returns DFS_ENOMEM                      */
    int32_t reserved0;       /* must be 0 (was eager_siblings: claiming every later unvisited
                                neighbour of a window at once — measured slower, removed)          */
    int32_t leaf_skip;       /* 1: a claimed child whose list is empty or holds only its parent is
                                finished in place — Alg 1 would descend and pop straight back — so
                                the parent's window scan continues without a push/pop round trip.
                                2 (default): in addition, every window claims all its unvisited
                                leaf candidates at once (leaf map built at create: all in-edges
                                from one vertex w, out-list empty, [w] or [v]; S24).
                                0: always descend                                                  */
    int32_t cluster;         /* cluster steal tier: 2, 4 or 8 = launch the persistent
                                grid as thread-block clusters of that many CTAs; an idle warp that
                                finds no Alg 3 victim in its own CTA steals from the HotRings of the
                                other CTAs of its cluster through distributed shared memory (same
                                reservation protocol as Alg 3) before trying Alg 4.  The grid is
                                rounded down to whole co-resident clusters.  0 = off; 1 = the
                                cluster build launched as clusters of one CTA (diagnostic: the
                                cost of cluster-visible publication alone)                       */
    int32_t cluster_late;    /* 1: an idle warp tries the cluster tier after Alg 4 instead of
                                between Alg 3 and Alg 4                                            */
    int32_t steal_tries;     /* Alg 3 victims an idle warp tries per round, best first: when the
                                max-hot_rest victim is locked by another thief (or falls below
                                hot_cutoff) it moves on to the next best; 1 = Alg 3 as written;
                                default 8                                                          */
    int32_t bulk_copy;       /* 1: flush and refill move the 16-byte-aligned part of each piece with
                                cp.async.bulk (shared->global, resp. global->shared completing on a
                                per-warp mbarrier) — the paper's TMA variant;
                                0: warp-wide 8-byte copies.  Default 1.  Ignored when cluster >= 1
                                (the cluster build has no bulk variant)                            */
    int32_t spill_period;    /* a busy warp checks the spill condition every spill_period expansion
                                steps (power of two <= 1024; 0 = 32)                               */
    int32_t l2_persist_mb;   /* > 0: set the device's persisting-L2 limit to this many MB (capped by
                                cudaDevAttrMaxPersistingL2CacheSize; device-wide) and launch the
                                traversal with an access-policy window that keeps row_ptr persisting
                                in L2 while col_idx streams.  0 (default) = auto: 64 MB with
                                128-wide windows (A/B on B200: RMAT-24 -4.8%, road/path neutral),
                                else off; -1 = off.  The limit stays set after the handle is gone  */
    int32_t walker_lanes;    /* lanes per walker: 32 = the warp kernel (one walker per warp, windows of
                                `window` positions); 16, 8, 4 or 2 = the sub-warp walker kernel (32/L
                                independent walkers per warp, each with its own HotRing/ColdSeg and
                                an L-position window); 0 = auto: 4-lane walkers on
                                low-degree graphs (m <= 4n, max degree <= 16) for batches with
                                several traversals in flight and for path-like graphs (m < 2.2n),
                                else the warp kernel.  deterministic, cluster >= 1 and window = 128
                                use the warp kernel                                                */
    int32_t steal_period;    /* walker kernel: an idle walker in a warp that still has busy walkers
                                tries one Alg 3 steal (for all idle walkers of the warp) every
                                steal_period steps (power of two <= 1024; 0 = 16)                  */
    int32_t donate;          /* walker kernel: 1 (default) = a walker about to push an entry while a
                                sibling walker of its warp holds nothing hands the entry to that
                                sibling instead; 0 = always push                    */
    int32_t records;         /* walker kernel with >= 8 lanes: 1 = read a claimed child's list
                                through its 32-byte vertex record (first 6 neighbours + its
                                row_ptr pair; built once per handle on first use, 32 bytes per
                                vertex of device memory; DESIGN.md §4 — measured slower); 0
                                (default) = row_ptr then col_idx                                   */
} dfs_options;

typedef struct dfs_stats {
    float   kernel_ms;       /* device time of reset + traversal + finalize (CUDA events)          */
    float   traversal_ms;    /* device time of the persistent traversal kernel alone               */
    int32_t blocks, warps_per_block;
    int64_t n_visited;       /* |visited|                                                          */
    int64_t m_visited;       /* sum of out-degrees of visited vertices (TEPS numerator)            */
    /* counters (collect_stats = 1) */
    int64_t claims, failed_claims, flushes, refills, intra_steals, inter_steals, steal_attempts,
            chunks_allocated, windows;
    int64_t idle_ns;         /* sum over warps of time spent idle (stealing / waiting)             */
    int64_t inter_scans;     /* inter-block victim-selection rounds                                */
    int64_t spills;          /* demand-driven spills                                               */
    /* SM-cycle breakdown of the expansion step summed over windows (collect_stats; diagnostics):
       wait for the window data, wait for the probes, wait for the speculative claim, rest */
    int64_t cyc_window, cyc_probe, cyc_claim, cyc_tail;
    int64_t cyc_outside;     /* cycles between consecutive expansion steps of a busy warp (pops,
                                flushes, spills, periodic checks)                                  */
    /* optional, caller-owned host array of 2*num_roots int64 (NULL = not wanted): per-root
       (n_visited, m_visited) of a batch, in root order */
    int64_t *root_counts;
    /* optional, caller-owned host array of `blocks` int64 (NULL = not wanted; single traversals):
       claims (tree vertices discovered) per block — the task distribution of Fig 9 */
    int64_t *block_claims;
    int64_t cluster_steals;  /* steals through distributed shared memory (cluster tier)           */
    int64_t pops;            /* 32-wide step: entries popped after a list was exhausted            */
    int64_t dead_pops;       /* ... of which found nothing left to claim (every remaining target
                                was claimed after the entry was pushed)                            */
    int64_t donations;       /* walker kernel: entries handed to idle sibling walkers             */
    int32_t walker_lanes;    /* kernel that ran: 32 = warp kernel, else lanes per walker          */
    int32_t window;          /* warp kernel window (32 or 128)                                    */
} dfs_stats;

void dfs_options_default(dfs_options *opt);

/* Create a graph handle on the current CUDA device (copies and validates the CSR).
 * Returns NULL on failure (see dfs_last_error). */
dfs_graph *dfs_graph_create(const int64_t *row_ptr, const int32_t *col_idx, int64_t n, int64_t m);

/* One unordered DFS from root (Alg 2 skeleton P:249-286 with §3's hierarchy).  parent_out: n
 * int32, host or device.  Default options. */
int dfs_run(dfs_graph *g, int32_t root, int32_t *parent_out);

/* num_roots independent traversals; row i of parents_out (num_roots x n, row-major, host or
 * device) receives the result for roots[i] (roots: host or device; repeated roots are allowed,
 * each row is its own traversal).  num_roots = 0 is a no-op returning DFS_OK (roots and
 * parents_out may then be NULL); num_roots < 0 or a NULL array otherwise: DFS_EINVAL.
 * North-star batch entry; multi-GPU batches partition roots across processes above this call. */
int dfs_run_batch(dfs_graph *g, const int32_t *roots, int32_t num_roots, int32_t *parents_out);

/* dfs_run with explicit options (may be NULL = defaults) and optional stats (may be NULL). */
int dfs_run_ex(dfs_graph *g, int32_t root, int32_t *parent_out, const dfs_options *opt,
               dfs_stats *stats);

/* Batch with explicit options; stats (may be NULL) accumulates over the batch. */
int dfs_run_batch_ex(dfs_graph *g, const int32_t *roots, int32_t num_roots, int32_t *parents_out,
                     const dfs_options *opt, dfs_stats *stats);

/* Stream all subsequent calls on this handle are ordered on (a cudaStream_t; NULL = legacy
 * default stream). */
int dfs_set_stream(dfs_graph *g, void *cuda_stream);

/* n, m, device ordinal of a handle (any pointer may be NULL). */
int dfs_graph_info(const dfs_graph *g, int64_t *n, int64_t *m, int32_t *device);

/* Number of this library's kernels launched on the handle since creation (reset, traversal,
 * finalize, ...): the bench's "gpu_launches" count. */
int64_t dfs_launch_count(const dfs_graph *g);

/* Diagnostics: busy-warp timeline.  dfs_debug_timeline(g, len, dt_ns, NULL) enables sampling
 * every dt_ns (block 0 / warp 0) into a device buffer of len entries for subsequent runs, in three
 * regions of t = len/3 entries: entry k < t = busy blocks + 1 (0 = no sample), entry t + k = claims
 * reported so far, entry 2t + k = expansion windows reported so far (collect_stats runs only; busy
 * warps report every period); calling it again with the same len and a host buffer `out` copies the
 * last run's samples out and clears them; len = 0 disables. */
int dfs_debug_timeline(dfs_graph *g, uint32_t len, uint32_t dt_ns, uint32_t *out);

/* Diagnostics / tests: run a script of stack operations on the walkers of warp 0, block 0 of the
 * sub-warp walker kernel (lanes = 16, 8, 4 or 2 lanes per walker), using the kernel's own HotRing,
 * ColdSeg and steal code (the paper's worked examples, Figs 2 and 3, are replayed this
 * way by tests/test_gpu_stack_script.py).  script: n_ops records of 6 int32 {op, a, b, c, d, e}:
 *   0 END; 1 SET w head tail top bottom (maps ColdSeg chunks for [0, top)); 2 RING w counter v i;
 *   3 COLD w pos v i; 4 PUSH w v i; 5 POP w -> (v, i) or (-1, -1); 6 FLUSH w want keep;
 *   7 REFILL w -> entries moved; 8 STEAL_INTRA thief-walker-mask -> receivers mask;
 *   9 STEAL_INTER thief-walker-mask -> receivers mask; 10 DUMP w -> head tail top bottom;
 *   11 READ_RING w counter -> (v, i); 12 READ_COLD w pos -> (v, i).
 * Outputs are appended to out[0 .. out_len) (host memory).  opt supplies cutoffs, steal_half,
 * ring_cap, ...; the handle's scratch is re-initialised before its next traversal. */
int dfs_debug_stack_script(dfs_graph *g, int32_t lanes, const int32_t *script, int32_t n_ops,
                           int32_t *out, int32_t out_len, const dfs_options *opt);

void dfs_graph_destroy(dfs_graph *g);

int dfs_last_error(void);
const char *dfs_strerror(int code);

#ifdef __cplusplus
}
#endif
#endif /* B200_DFS_H */
