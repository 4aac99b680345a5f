/* span_sim.c — an idealised model of the parallel unordered DFS ("span").
 *
 * W walkers advance in lock-step ticks.  In one tick every busy walker performs one expansion
 * step of the paper's warp-level DFS on its top entry <u, i>: scan u's list from i
 * for the first unvisited neighbour (Alg 1 l.5-12, at most 32 positions = one window), claim it
 * and push it, or pop when u's list is exhausted.  An idle walker steals half of the entries at
 * the BOTTOM of a victim's stack (the heavier of two random walkers, Alg 3/4's two-choice rule,
 * P:1067-1180) and becomes busy `delay` ticks later.  There is no memory system: a tick stands
 * for the latency of one dependent expansion step, so (ticks x measured step latency) is the
 * time the schedule needs, and ticks at W -> infinity is the DFS's critical path (span).
 *
 * It also prints the BFS eccentricity of the root: no traversal that builds a tree from the root
 * can finish in fewer sequential claims (a vertex at distance d needs a claimed neighbour at
 * distance d-1), whatever its order.
 *
 * Input: rp.bin (int64 row_ptr[n+1]) and col.bin (int32 col_idx[m]) in the current directory
 * (scripts/span_sim.py writes them).  Not part of the product: a planning/analysis tool.
 *
 * usage: span_sim root W [delay=0] [half=1]
 */
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>

typedef struct { uint32_t u, i; } Ent;
typedef struct { Ent *s; int64_t lo, hi, cap; int64_t ready; } Stk;

static uint64_t rs = 88172645463325252ULL;
static inline uint64_t xr(void) { rs ^= rs << 13; rs ^= rs >> 7; rs ^= rs << 17; return rs; }

static void *xmalloc(size_t b) { void *p = malloc(b); if (!p) { fprintf(stderr, "oom\n"); exit(1); } return p; }

int main(int argc, char **argv)
{
    if (argc < 3) { fprintf(stderr, "usage: span_sim root W [delay] [half]\n"); return 2; }
    const int64_t root = atoll(argv[1]);
    const int W = atoi(argv[2]);
    const int64_t delay = argc > 3 ? atoll(argv[3]) : 0;
    const int half = argc > 4 ? atoi(argv[4]) : 1;
    FILE *f = fopen("rp.bin", "rb");
    if (!f) { perror("rp.bin"); return 1; }
    fseek(f, 0, SEEK_END);
    const int64_t n = ftell(f) / 8 - 1;
    rewind(f);
    int64_t *rp = xmalloc((size_t)(n + 1) * 8);
    if (fread(rp, 8, (size_t)n + 1, f) != (size_t)n + 1) return 1;
    fclose(f);
    const int64_t m = rp[n];
    int32_t *col = xmalloc((size_t)m * 4 + 4);
    f = fopen("col.bin", "rb");
    if (!f || fread(col, 4, (size_t)m, f) != (size_t)m) return 1;
    fclose(f);

    /* BFS eccentricity of the root */
    int32_t *dist = xmalloc((size_t)n * 4), *q = xmalloc((size_t)n * 4);
    for (int64_t v = 0; v < n; ++v) dist[v] = -1;
    int64_t qh = 0, qt = 0, ecc = 0;
    dist[root] = 0; q[qt++] = (int32_t)root;
    while (qh < qt) {
        const int32_t u = q[qh++];
        for (int64_t j = rp[u]; j < rp[u + 1]; ++j) {
            const int32_t v = col[j];
            if (dist[v] < 0) { dist[v] = dist[u] + 1; if (dist[v] > ecc) ecc = dist[v]; q[qt++] = v; }
        }
    }
    const int64_t reach = qt;
    free(dist); free(q);

    uint8_t *vis = calloc((size_t)n, 1);
    Stk *S = calloc((size_t)W, sizeof(Stk));
    for (int w = 0; w < W; ++w) { S[w].cap = 256; S[w].s = xmalloc(256 * sizeof(Ent)); }
    vis[root] = 1;
    S[0].s[0] = (Ent){(uint32_t)root, (uint32_t)rp[root]};
    S[0].hi = 1;
    int64_t claims = 1, tick = 0, busy_sum = 0, steps = 0;
    for (;;) {
        int64_t nb = 0;
        for (int w = 0; w < W; ++w) {
            Stk *st = &S[w];
            if (st->hi <= st->lo || st->ready > tick) continue;
            ++nb; ++steps;
            Ent *t = &st->s[st->hi - 1];
            const int64_t e = rp[t->u + 1];
            int64_t j = t->i;
            int claimed = 0;
            for (int k = 0; k < 32 && j < e; ++k, ++j) {
                const int32_t v = col[j];
                if (!vis[v]) {
                    vis[v] = 1; ++claims; t->i = (uint32_t)(j + 1); claimed = 1;
                    if (st->hi == st->cap) {
                        const int64_t c = st->hi - st->lo;
                        if (st->lo > c) { memmove(st->s, st->s + st->lo, (size_t)c * sizeof(Ent)); st->lo = 0; st->hi = c; }
                        else { st->cap *= 2; st->s = realloc(st->s, (size_t)st->cap * sizeof(Ent)); }
                    }
                    st->s[st->hi++] = (Ent){(uint32_t)v, (uint32_t)rp[v]};
                    break;
                }
            }
            if (!claimed) { if (j >= e) st->hi--; else t->i = (uint32_t)j; }
        }
        int any = 0;
        for (int w = 0; w < W; ++w) {
            Stk *st = &S[w];
            if (st->hi > st->lo) { any = 1; continue; }
            st->lo = st->hi = 0;
            int best = -1;
            int64_t bl = 0;
            for (int k = 0; k < 2; ++k) {
                const int v = (int)(xr() % (uint64_t)W);
                const int64_t l = S[v].hi - S[v].lo;
                if (l > bl) { bl = l; best = v; }
            }
            if (best < 0 || bl < 2) continue;
            const int64_t take = half ? bl / 2 : 1;
            Stk *vs = &S[best];
            if (st->cap < take) { st->cap = take * 2; st->s = realloc(st->s, (size_t)st->cap * sizeof(Ent)); }
            memcpy(st->s, vs->s + vs->lo, (size_t)take * sizeof(Ent));
            vs->lo += take; st->hi = take; st->ready = tick + 1 + delay;
            any = 1;
        }
        ++tick; busy_sum += nb;
        if (!any) break;
    }
    printf("{\"root\": %lld, \"walkers\": %d, \"steal_delay\": %lld, \"ticks\": %lld, \"claims\": %lld, "
           "\"reach\": %lld, \"steps\": %lld, \"work_bound_ticks\": %lld, \"busy_mean\": %.1f, \"bfs_ecc\": %lld}\n",
           (long long)root, W, (long long)delay, (long long)tick, (long long)claims, (long long)reach,
           (long long)steps, (long long)(steps / W), (double)busy_sum / (double)tick, (long long)ecc);
    return 0;
}
