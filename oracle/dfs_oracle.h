/*
 * dfs_oracle.h — CPU oracle for unordered DFS (DiggerBees, PPoPP '26).
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and the
 * cpu_baseline / --impl reference legs of bench.py may load this library.
 * It shares no code, header, table or helper with the CUDA path
 * (paper_conf_ppopp_niul0c26_b200/csrc, include/dfs.h); neither includes the other.
 *
 * Citations "P:a-b" are /root/reference/PAPER.md line ranges.
 *
 * Graph convention (both sides agree by DESIGN.md, not by shared code):
 *   CSR out-adjacency, row_ptr[n+1] (int64), column_idx[m] (int32)   (§2.1)
 *   parent[root] = -1 (Alg 1 l.1); unreached vertices = -2 (reading S2).
 */
#ifndef DFS_ORACLE_H
#define DFS_ORACLE_H
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define ORACLE_ROOT_PARENT (-1)
#define ORACLE_UNREACHED   (-2)

/* Alg 1 verbatim: serial stack-based DFS.  Fills parent[n].
 * Returns the number of visited vertices, or -1 on invalid arguments / OOM. */
int64_t oracle_dfs(int64_t n, const int64_t *row_ptr, const int32_t *column_idx,
                   int32_t root, int32_t *parent);

/* Textbook BFS reachability from root (second, independent routine used by I4).
 * visited[n] gets 0/1.  Returns the number reached or -1. */
int64_t oracle_reach(int64_t n, const int64_t *row_ptr, const int32_t *column_idx,
                     int32_t root, uint8_t *visited);

/* Result of oracle_check_tree.  ok_* : 1 = holds, 0 = violated, -1 = not checked. */
typedef struct {
    int32_t ok_i1;          /* root: parent[r] = -1, no other -1, values in {-2,-1} ∪ [0,n) */
    int32_t ok_i2;          /* every visited v != r has a visited parent p with (p,v) in E */
    int32_t ok_i3;          /* parent pointers reach r from every visited v (acyclic) */
    int32_t ok_i4;          /* visited set == BFS reach set of r */
    int32_t ok_i5;          /* closure: (u,v) in E, u visited => v visited */
    int32_t ok_i6;          /* scan-order consistency (reading S1) */
    int32_t ok_i7;          /* classical DFS tree (some child order; only back/forward/right-to-left cross) */
    int32_t pad;
    int64_t n_visited;      /* |{v : parent[v] != -2}| */
    int64_t m_visited;      /* sum of outdeg over visited vertices (TEPS numerator, reading S6) */
    int64_t n_cross;        /* I7: number of non-tree CSR entries that are cross edges violating the order
                               (undirected: cross edges; -1 when I7 not computed) */
    int64_t bad_vertex;     /* first offending vertex for the first failed check, else -1 */
} oracle_check_result;

/* Flags for oracle_check_tree. */
#define ORACLE_CHECK_I7            1  /* compute I7 */
#define ORACLE_CHECK_UNDIRECTED    2  /* caller asserts the graph is symmetric: I7 = "no cross edge" */

/* Exact integer validation of a candidate parent array (tolerance 0).
 * Returns 1 if I1-I6 (and I7 when requested) all hold, 0 if any fails, -1 on bad args / OOM.
 * Later checks that depend on earlier ones are reported -1 when an earlier one fails. */
int oracle_check_tree(int64_t n, const int64_t *row_ptr, const int32_t *column_idx,
                      int32_t root, const int32_t *parent, int flags,
                      oracle_check_result *res);

#ifdef __cplusplus
}
#endif
#endif
