/* oracle.h -- TEST INFRASTRUCTURE ONLY.
 *
 * Plain, slow, single-threaded CPU oracle for the graphB+ balancing path
 * (Alabandi, Tesic, Rusnak, Burtscher, SC'21; /root/reference/PAPER.md).
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
 * --impl reference legs may load it.  It shares no code, header, table or
 * constant generator with the CUDA library (include/graphb.h,
 * paper_conf_sc_alabanditrb21_b200/csrc); the two meet only at the seeded
 * input generators (graphgen/).
 *
 * Every function states the PAPER.md passage it writes out; readings of
 * silent or ambiguous passages are listed in DESIGN.md "Readings".
 */
#ifndef GRAPHB_ORACLE_H
#define GRAPHB_ORACLE_H
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define OR_OK      0
#define OR_EINVAL -1
#define OR_ENOMEM -3
#define OR_EUNBAL -5 /* internal check failed: Sigma_T not balanced */

typedef struct or_graph or_graph;

/* --- counter-based hash (reading R4: SplitMix64 finaliser) ---- */
uint64_t or_mix64(uint64_t z);
uint64_t or_splitmix64_next(uint64_t *state);
uint64_t or_tkey(uint64_t seed, int64_t t);
uint64_t or_rkey(uint64_t seed, int64_t t, int64_t comp);
uint32_t or_pscore(uint64_t seed, int64_t t, int32_t a, int32_t b);

/* --- graph ------------------------------------------------------------- */
int  or_build(int64_t n, int64_t m, const int64_t *row_ptr, const int32_t *col,
              const int8_t *sign, or_graph **out);
void or_free(or_graph *g);
int64_t or_n(const or_graph *g);
int64_t or_m(const or_graph *g);
int64_t or_ncomp(const or_graph *g);
/* edge list indexed by eid (rank of (min,max)); u < v; neg = 1 if sigma = -1 */
void or_edges(const or_graph *g, int32_t *u, int32_t *v, int8_t *neg);
/* comp[v] = component rank (by minimum vertex); coff[ncomp+1]; cverts[n] */
void or_components(const or_graph *g, int32_t *comp, int64_t *coff, int32_t *cverts);

/* --- one tree ---------------------------------------------------------- */
/* Alg. 2 sampler M = BFS (L116-L123, L130): hashed roots + min-hash parents. */
int or_bfs_tree(const or_graph *g, uint64_t seed, int64_t t,
                int32_t *parent, int32_t *dist, int32_t *peid);
/* Alg. 1 (L96-L108) on a caller tree: flip[e] = 1 iff the fundamental cycle
 * of non-tree edge e is negative.  sumk = sum of cycle lengths, ncyc = number
 * of non-tree edges.  Returns OR_EINVAL if parent is not a spanning forest
 * with one root per component. */
int or_balance_tree(const or_graph *g, const int32_t *parent, uint8_t *flip,
                    uint64_t *sumk, int64_t *ncyc, int32_t *maxdepth);
/* Alg. 3 steps 1-2 (L182-L189) by a sequential pre-order walk. */
int or_preorder(const or_graph *g, const int32_t *parent, int32_t *pre, int32_t *size);
/* Harary bipartition of Sigma_T the paper's way (L224): drop negative edges,
 * CCs, collapse, BFS, even/odd levels.  side[v] in {0,1}; delta2[v] = 2*delta
 * (L144: 2 larger side, 1 tie, 0 smaller side), per connected component. */
int or_harary(const or_graph *g, const uint8_t *flip, uint8_t *side, uint8_t *delta2);

/* Signature of the nearest balanced state with switch set flip[0..m)
 * (SURVEY §8 f.2): XOR over switched e of mix64(e ^ 0x5851F42D4C957F2D). */
uint64_t or_state_signature(const uint8_t *flip, int64_t m);

/* --- frustration cloud (Alg. 2 over trees t_begin, t_begin+stride, ... < t_end)
 * cnt[e] += flip_t(e); agree[v] += delta2_t(v);
 * stats (may be NULL): per processed tree {sumk, ncyc, maxdepth, state signature}. */
int or_balance(const or_graph *g, int64_t t_begin, int64_t t_end, int64_t stride,
               uint64_t seed, uint32_t *cnt, uint32_t *agree, uint64_t *stats);

/* Alg. 2 with M = random: a uniformly random spanning forest by Wilson's
 * algorithm with per-vertex random stacks (reading R17); order 0/1 starts the
 * walks in ascending/descending vertex order (the result must not depend on
 * it).  parent[root] = -1; pops[v] (optional) = times v's stack was popped. */
uint64_t or_wdraw(uint64_t seed, int64_t t, int32_t u, uint32_t j);
int or_wilson_tree(const or_graph *g, uint64_t seed, int64_t t, int order,
                   int32_t *parent, uint32_t *pops);

/* Alg. 2 with M = DFS (reading R18): scan of u's neighbours starts at
 * or_dstart(seed,t,u) mod deg(u) and wraps around; parent[root] = -1. */
uint64_t or_dstart(uint64_t seed, int64_t t, int32_t u);
int or_dfs_tree(const or_graph *g, uint64_t seed, int64_t t, int32_t *parent);

/* or_balance with the sampler chosen: 0 = BFS (R4), 1 = uniform (Wilson),
 * 2 = DFS (R18). */
int or_balance_m(const or_graph *g, int64_t t_begin, int64_t t_end, int64_t stride,
                 uint64_t seed, int sampler, uint32_t *cnt, uint32_t *agree, uint64_t *stats);

#ifdef __cplusplus
}
#endif
#endif
