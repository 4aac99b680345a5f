/*
 * graphgen.c — seeded synthetic CSR generators shared by the oracle side and the CUDA side.
 *
 * This module holds NO part of the DFS method's arithmetic (no traversal, no claim, no stack);
 * it only builds input graphs.  It is the one module both tests/bench legs import (the
 * "seeded input generators" exception of the build rules).  Recipes: DESIGN.md §"Input recipe",
 * shapes after the paper's workloads (road/mesh DIMACS10 graphs P:1342-1359, Table 4 P:1893-1907;
 * power-law SNAP/LAW graphs) and BASELINE.json configs C1-C5.
 *
 * All generated graphs are symmetric (both directions stored), adjacency lists sorted ascending,
 * with no self loops and no duplicates unless a generator says otherwise.
 * Randomness: counter-based splitmix64 so results are independent of the thread count.
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#ifdef _OPENMP
#include <omp.h>
#endif

typedef struct gg_graph {
    int64_t n, m;
    int64_t *row_ptr;   /* n+1 */
    int32_t *col;       /* m   */
} gg_graph;

/* ---------------------------------------------------------------- RNG (counter based) */
static inline uint64_t splitmix64(uint64_t x)
{
    x += 0x9E3779B97F4A7C15ULL;
    x = (x ^ (x >> 30)) * 0xBF58476D1CE4E5B9ULL;
    x = (x ^ (x >> 27)) * 0x94D049BB133111EBULL;
    return x ^ (x >> 31);
}
static inline uint64_t rng_at(uint64_t seed, uint64_t stream, uint64_t k)
{
    return splitmix64(splitmix64(seed ^ (stream * 0xD1B54A32D192ED03ULL)) + k * 0x9E3779B97F4A7C15ULL);
}
/* sequential generator */
typedef struct { uint64_t s; } rng_t;
static inline uint64_t rng_next(rng_t *r) { r->s += 0x9E3779B97F4A7C15ULL; uint64_t x = r->s;
    x = (x ^ (x >> 30)) * 0xBF58476D1CE4E5B9ULL; x = (x ^ (x >> 27)) * 0x94D049BB133111EBULL; return x ^ (x >> 31); }
static inline uint64_t rng_below(rng_t *r, uint64_t bound) { return (uint64_t)(((__uint128_t)rng_next(r) * bound) >> 64); }
static inline double rng_unit(rng_t *r) { return (double)(rng_next(r) >> 11) * (1.0 / 9007199254740992.0); }

/* ---------------------------------------------------------------- helpers */
static gg_graph *gg_alloc(int64_t n, int64_t m)
{
    gg_graph *g = (gg_graph *)calloc(1, sizeof(gg_graph));
    if (!g) return NULL;
    g->n = n; g->m = m;
    g->row_ptr = (int64_t *)malloc(((size_t)n + 1) * sizeof(int64_t));
    g->col = (int32_t *)malloc((size_t)(m > 0 ? m : 1) * sizeof(int32_t));
    if (!g->row_ptr || !g->col) { free(g->row_ptr); free(g->col); free(g); return NULL; }
    return g;
}

void gg_destroy(gg_graph *g) { if (g) { free(g->row_ptr); free(g->col); free(g); } }
int64_t gg_n(const gg_graph *g) { return g->n; }
int64_t gg_m(const gg_graph *g) { return g->m; }
void gg_export(const gg_graph *g, int64_t *row_ptr, int32_t *col)
{
    memcpy(row_ptr, g->row_ptr, ((size_t)g->n + 1) * sizeof(int64_t));
    if (g->m) memcpy(col, g->col, (size_t)g->m * sizeof(int32_t));
}

static int cmp_i32(const void *a, const void *b)
{
    int32_t x = *(const int32_t *)a, y = *(const int32_t *)b;
    return (x > y) - (x < y);
}

/* insertion sort for short lists, qsort otherwise */
static void sort_list(int32_t *a, int64_t len)
{
    if (len < 24) {
        for (int64_t i = 1; i < len; ++i) {
            int32_t x = a[i]; int64_t j = i - 1;
            while (j >= 0 && a[j] > x) { a[j + 1] = a[j]; --j; }
            a[j + 1] = x;
        }
    } else qsort(a, (size_t)len, sizeof(int32_t), cmp_i32);
}

/* Build a CSR from an edge list.  symmetrize: store both (u,v) and (v,u).  Lists are sorted;
 * dedup removes repeated entries; drop_self removes self loops. */
gg_graph *gg_from_edges(int64_t n, int64_t ne, const int32_t *src, const int32_t *dst,
                        int symmetrize, int dedup, int drop_self)
{
    int64_t *deg = (int64_t *)calloc((size_t)n + 1, sizeof(int64_t));
    if (!deg) return NULL;
    for (int64_t e = 0; e < ne; ++e) {
        if (drop_self && src[e] == dst[e]) continue;
        deg[src[e] + 1]++;
        if (symmetrize) deg[dst[e] + 1]++;
    }
    for (int64_t v = 0; v < n; ++v) deg[v + 1] += deg[v];
    int64_t total = deg[n];
    int32_t *tmp = (int32_t *)malloc((size_t)(total > 0 ? total : 1) * sizeof(int32_t));
    int64_t *fill = (int64_t *)malloc((size_t)n * sizeof(int64_t));
    if (!tmp || !fill) { free(deg); free(tmp); free(fill); return NULL; }
    memcpy(fill, deg, (size_t)n * sizeof(int64_t));
    for (int64_t e = 0; e < ne; ++e) {
        if (drop_self && src[e] == dst[e]) continue;
        tmp[fill[src[e]]++] = dst[e];
        if (symmetrize) tmp[fill[dst[e]]++] = src[e];
    }
    free(fill);
    int64_t *newdeg = (int64_t *)calloc((size_t)n + 1, sizeof(int64_t));
    if (!newdeg) { free(deg); free(tmp); return NULL; }
    #pragma omp parallel for schedule(dynamic, 4096)
    for (int64_t v = 0; v < n; ++v) {
        int32_t *a = tmp + deg[v];
        int64_t len = deg[v + 1] - deg[v];
        sort_list(a, len);
        int64_t k = len;
        if (dedup && len > 1) {
            k = 1;
            for (int64_t i = 1; i < len; ++i) if (a[i] != a[k - 1]) a[k++] = a[i];
        }
        newdeg[v + 1] = k;
    }
    for (int64_t v = 0; v < n; ++v) newdeg[v + 1] += newdeg[v];
    gg_graph *g = gg_alloc(n, newdeg[n]);
    if (!g) { free(deg); free(tmp); free(newdeg); return NULL; }
    memcpy(g->row_ptr, newdeg, ((size_t)n + 1) * sizeof(int64_t));
    #pragma omp parallel for schedule(dynamic, 4096)
    for (int64_t v = 0; v < n; ++v)
        memcpy(g->col + newdeg[v], tmp + deg[v], (size_t)(newdeg[v + 1] - newdeg[v]) * sizeof(int32_t));
    free(deg); free(tmp); free(newdeg);
    return g;
}

/* ---------------------------------------------------------------- C1: 2-D grid */
/* W x H 4-neighbour grid, id = row*W + col, ascending adjacency (up, left, right, down). */
gg_graph *gg_grid(int64_t W, int64_t H)
{
    int64_t n = W * H;
    int64_t m = 2 * ((W - 1) * H + W * (H - 1));
    gg_graph *g = gg_alloc(n, m);
    if (!g) return NULL;
    int64_t k = 0;
    for (int64_t r = 0; r < H; ++r)
        for (int64_t c = 0; c < W; ++c) {
            int64_t v = r * W + c;
            g->row_ptr[v] = k;
            if (r > 0) g->col[k++] = (int32_t)(v - W);
            if (c > 0) g->col[k++] = (int32_t)(v - 1);
            if (c + 1 < W) g->col[k++] = (int32_t)(v + 1);
            if (r + 1 < H) g->col[k++] = (int32_t)(v + W);
        }
    g->row_ptr[n] = k;
    return g;
}

/* ---------------------------------------------------------------- C2: road-maze */
static int64_t uf_find(int64_t *p, int64_t x)
{
    while (p[x] != x) { p[x] = p[p[x]]; x = p[x]; }
    return x;
}

/* Random spanning tree of the W x H grid (randomised Kruskal over shuffled grid edges) plus each
 * remaining grid edge kept with probability extra*n/#remaining (extra = 0.2 -> avg degree 2.4).
 * Row-major ids.  Deep, narrow DFS like DIMACS10 road graphs (euro_osm). */
gg_graph *gg_road(int64_t W, int64_t H, uint64_t seed, double extra)
{
    int64_t n = W * H;
    int64_t ng = (W - 1) * H + W * (H - 1);
    int32_t *eu = (int32_t *)malloc((size_t)ng * sizeof(int32_t));
    int32_t *ev = (int32_t *)malloc((size_t)ng * sizeof(int32_t));
    int64_t *par = (int64_t *)malloc((size_t)n * sizeof(int64_t));
    uint8_t *intree = (uint8_t *)calloc((size_t)ng, 1);
    if (!eu || !ev || !par || !intree) { free(eu); free(ev); free(par); free(intree); return NULL; }
    int64_t k = 0;
    for (int64_t r = 0; r < H; ++r)
        for (int64_t c = 0; c < W; ++c) {
            int64_t v = r * W + c;
            if (c + 1 < W) { eu[k] = (int32_t)v; ev[k] = (int32_t)(v + 1); ++k; }
            if (r + 1 < H) { eu[k] = (int32_t)v; ev[k] = (int32_t)(v + W); ++k; }
        }
    rng_t rng = { seed };
    for (int64_t i = ng - 1; i > 0; --i) {           /* Fisher-Yates */
        int64_t j = (int64_t)rng_below(&rng, (uint64_t)i + 1);
        int32_t t = eu[i]; eu[i] = eu[j]; eu[j] = t;
        t = ev[i]; ev[i] = ev[j]; ev[j] = t;
    }
    for (int64_t v = 0; v < n; ++v) par[v] = v;
    int64_t ntree = 0;
    for (int64_t e = 0; e < ng; ++e) {
        int64_t a = uf_find(par, eu[e]), b = uf_find(par, ev[e]);
        if (a != b) { par[a] = b; intree[e] = 1; ++ntree; }
    }
    free(par);
    int64_t nrem = ng - ntree;
    double p = nrem > 0 ? extra * (double)n / (double)nrem : 0.0;
    int64_t kept = 0;
    for (int64_t e = 0; e < ng; ++e) {
        int keep = intree[e] || rng_unit(&rng) < p;
        if (keep) { eu[kept] = eu[e]; ev[kept] = ev[e]; ++kept; }
    }
    free(intree);
    gg_graph *g = gg_from_edges(n, kept, eu, ev, 1, 1, 1);
    free(eu); free(ev);
    return g;
}

/* ---------------------------------------------------------------- C3: RMAT / Kronecker */
/* Graph500-style Kronecker generator: scale, edge factor ef, quadrant probabilities (A,B,C,D),
 * 2^scale * ef generated edges, random vertex permutation, symmetrised, dedup, no self loops. */
gg_graph *gg_rmat(int scale, int64_t ef, double A, double B, double C, uint64_t seed)
{
    int64_t n = (int64_t)1 << scale;
    int64_t ne = n * ef;
    int32_t *src = (int32_t *)malloc((size_t)ne * sizeof(int32_t));
    int32_t *dst = (int32_t *)malloc((size_t)ne * sizeof(int32_t));
    int32_t *perm = (int32_t *)malloc((size_t)n * sizeof(int32_t));
    if (!src || !dst || !perm) { free(src); free(dst); free(perm); return NULL; }
    const uint64_t tA = (uint64_t)(A * 4294967296.0);
    const uint64_t tAB = (uint64_t)((A + B) * 4294967296.0);
    const uint64_t tABC = (uint64_t)((A + B + C) * 4294967296.0);
    #pragma omp parallel for schedule(static)
    for (int64_t e = 0; e < ne; ++e) {
        uint32_t u = 0, v = 0;
        for (int l = 0; l < scale; l += 2) {
            uint64_t r = rng_at(seed, 1, (uint64_t)e * 16 + (uint64_t)(l >> 1));
            for (int h = 0; h < 2 && l + h < scale; ++h) {
                uint64_t x = (r >> (32 * h)) & 0xFFFFFFFFULL;
                int bu = 0, bv = 0;
                if (x < tA) { }
                else if (x < tAB) bv = 1;
                else if (x < tABC) bu = 1;
                else { bu = 1; bv = 1; }
                u = (u << 1) | (uint32_t)bu; v = (v << 1) | (uint32_t)bv;
            }
        }
        src[e] = (int32_t)u; dst[e] = (int32_t)v;
    }
    for (int64_t v = 0; v < n; ++v) perm[v] = (int32_t)v;
    rng_t rng = { seed ^ 0xABCDEF12345ULL };
    for (int64_t i = n - 1; i > 0; --i) {
        int64_t j = (int64_t)rng_below(&rng, (uint64_t)i + 1);
        int32_t t = perm[i]; perm[i] = perm[j]; perm[j] = t;
    }
    #pragma omp parallel for schedule(static)
    for (int64_t e = 0; e < ne; ++e) { src[e] = perm[src[e]]; dst[e] = perm[dst[e]]; }
    free(perm);
    gg_graph *g = gg_from_edges(n, ne, src, dst, 1, 1, 1);
    free(src); free(dst);
    return g;
}

/* ---------------------------------------------------------------- C4a: path + chords */
/* Path 0-1-...-(n-1) plus nchords uniform random chords {u,v} with |u-v| > 1, dedup. */
gg_graph *gg_path_chords(int64_t n, int64_t nchords, uint64_t seed)
{
    int64_t ne = (n - 1) + nchords;
    int32_t *src = (int32_t *)malloc((size_t)(ne > 0 ? ne : 1) * sizeof(int32_t));
    int32_t *dst = (int32_t *)malloc((size_t)(ne > 0 ? ne : 1) * sizeof(int32_t));
    if (!src || !dst) { free(src); free(dst); return NULL; }
    int64_t k = 0;
    for (int64_t i = 0; i + 1 < n; ++i) { src[k] = (int32_t)i; dst[k] = (int32_t)(i + 1); ++k; }
    rng_t rng = { seed };
    for (int64_t c = 0; c < nchords && n > 3; ) {
        int64_t u = (int64_t)rng_below(&rng, (uint64_t)n), v = (int64_t)rng_below(&rng, (uint64_t)n);
        if (u - v <= 1 && v - u <= 1) continue;
        src[k] = (int32_t)u; dst[k] = (int32_t)v; ++k; ++c;
    }
    gg_graph *g = gg_from_edges(n, k, src, dst, 1, 1, 1);
    free(src); free(dst);
    return g;
}

/* ---------------------------------------------------------------- C4b: caterpillar */
/* Spine 0..S-1 (a path); spine vertex s carries L leaves with ids S + s*L + k (> every spine id,
 * so CSR order descends the spine first).  A tree: its spanning tree is unique. */
gg_graph *gg_caterpillar(int64_t S, int64_t L)
{
    int64_t n = S + S * L;
    int64_t m = 2 * (n - 1);
    gg_graph *g = gg_alloc(n, m);
    if (!g) return NULL;
    int64_t k = 0;
    for (int64_t s = 0; s < S; ++s) {
        g->row_ptr[s] = k;
        if (s > 0) g->col[k++] = (int32_t)(s - 1);
        if (s + 1 < S) g->col[k++] = (int32_t)(s + 1);
        for (int64_t l = 0; l < L; ++l) g->col[k++] = (int32_t)(S + s * L + l);
    }
    for (int64_t s = 0; s < S; ++s)
        for (int64_t l = 0; l < L; ++l) {
            g->row_ptr[S + s * L + l] = k;
            g->col[k++] = (int32_t)s;
        }
    g->row_ptr[n] = k;
    return g;
}

/* ---------------------------------------------------------------- small shapes for tests */
gg_graph *gg_random(int64_t n, int64_t ne, uint64_t seed, int symmetric, int allow_self, int allow_dup)
{
    int32_t *src = (int32_t *)malloc((size_t)(ne > 0 ? ne : 1) * sizeof(int32_t));
    int32_t *dst = (int32_t *)malloc((size_t)(ne > 0 ? ne : 1) * sizeof(int32_t));
    if (!src || !dst) { free(src); free(dst); return NULL; }
    rng_t rng = { seed };
    for (int64_t e = 0; e < ne; ++e) {
        src[e] = (int32_t)rng_below(&rng, (uint64_t)n);
        dst[e] = (int32_t)rng_below(&rng, (uint64_t)n);
    }
    gg_graph *g = gg_from_edges(n, ne, src, dst, symmetric, !allow_dup, !allow_self);
    free(src); free(dst);
    return g;
}


/* ---------------------------------------------------------------- Matrix Market input */
/* Read a Matrix Market coordinate file (pattern / real / integer; general / symmetric) as a CSR
 * graph: entry (i, j) (1-based) is the directed edge i-1 -> j-1; symmetric files store both
 * directions (the artifact converts SuiteSparse .mtx files to CSR).  Self loops and
 * duplicates are dropped (the SuiteSparse graphs are simple).  Returns NULL on parse errors. */
#include <stdio.h>
#include <ctype.h>
gg_graph *gg_read_mtx(const char *path, int force_symmetric)
{
    FILE *f = fopen(path, "r");
    if (!f) return NULL;
    char line[1024];
    if (!fgets(line, sizeof line, f)) { fclose(f); return NULL; }
    for (char *c = line; *c; ++c) *c = (char)tolower((unsigned char)*c);
    if (strncmp(line, "%%matrixmarket", 14) != 0 || !strstr(line, "coordinate")) { fclose(f); return NULL; }
    const int symmetric = force_symmetric || strstr(line, "symmetric") != NULL || strstr(line, "hermitian") != NULL;
    const int pattern = strstr(line, "pattern") != NULL;
    const int cplx = strstr(line, "complex") != NULL;
    do {
        if (!fgets(line, sizeof line, f)) { fclose(f); return NULL; }
    } while (line[0] == '%');
    long long rows = 0, cols = 0, nnz = 0;
    if (sscanf(line, "%lld %lld %lld", &rows, &cols, &nnz) != 3 || rows <= 0 || cols <= 0 || nnz < 0) { fclose(f); return NULL; }
    const int64_t n = rows > cols ? rows : cols;
    int32_t *src = (int32_t *)malloc((size_t)(nnz > 0 ? nnz : 1) * sizeof(int32_t));
    int32_t *dst = (int32_t *)malloc((size_t)(nnz > 0 ? nnz : 1) * sizeof(int32_t));
    if (!src || !dst) { free(src); free(dst); fclose(f); return NULL; }
    int64_t k = 0;
    while (k < nnz && fgets(line, sizeof line, f)) {
        if (line[0] == '%' || line[0] == '\n') continue;
        long long a = 0, b = 0;
        if (sscanf(line, "%lld %lld", &a, &b) != 2 || a < 1 || b < 1 || a > n || b > n) { free(src); free(dst); fclose(f); return NULL; }
        (void)pattern; (void)cplx;                 /* values are ignored: the graph is the pattern */
        src[k] = (int32_t)(a - 1); dst[k] = (int32_t)(b - 1); ++k;
    }
    fclose(f);
    if (k != nnz) { free(src); free(dst); return NULL; }
    gg_graph *g = gg_from_edges(n, k, src, dst, symmetric, 1, 1);
    free(src); free(dst);
    return g;
}

/* Write a CSR graph as a general pattern Matrix Market file (1-based). */
int gg_write_mtx(const char *path, int64_t n, const int64_t *row_ptr, const int32_t *col)
{
    FILE *f = fopen(path, "w");
    if (!f) return -1;
    fprintf(f, "%%%%MatrixMarket matrix coordinate pattern general\n%lld %lld %lld\n",
            (long long)n, (long long)n, (long long)row_ptr[n]);
    for (int64_t u = 0; u < n; ++u)
        for (int64_t j = row_ptr[u]; j < row_ptr[u + 1]; ++j)
            fprintf(f, "%lld %lld\n", (long long)u + 1, (long long)col[j] + 1);
    fclose(f);
    return 0;
}
