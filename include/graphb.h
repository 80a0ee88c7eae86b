/* graphb.h -- C ABI of the B200-native graphB+ balancing hot path.
 *
 * What it computes (PAPER.md = /root/reference/PAPER.md, Alabandi et al.,
 * "Discovering and Balancing Fundamental Cycles in Large Signed Graphs", SC'21):
 *
 *   Alg. 2 (L125-L138): for k sampled spanning trees T of Sigma (method M =
 *     BFS, L116-L123, "random BFS trees" L479), find the nearest balanced state
 *     Sigma_T (Alg. 1 L96-L108, computed the graphB+ way, Alg. 3 L176-L202 with
 *     the labels of Alg. 4) and form its Harary bipartition (L224);
 *   L144: status(v) = (1/|T|) sum_T delta_T(v), delta = 1 / 0.5 / 0;
 *   L248: count per vertex over the trees and reduce.
 *
 * Outputs are integer counters over the trees:
 *   edge_flip_counts[e] = #trees in which the sign of undirected edge e is
 *                         switched (Alg. 1; tree edges never are),
 *   vertex_agree[v]     = sum_T 2*delta_T(v) (half-units: 2 larger Harary side,
 *                         1 tie, 0 smaller side), so status(v) = agree/(2T).
 *
 * Conventions:
 *   - m counts undirected edges; the CSR has 2m slots (Table 1, R2).
 *   - eid(u,v) = rank of (min(u,v), max(u,v)) in lexicographic order.
 *   - The tree of index t is defined by (graph, seed, t) only (reading R4;
 *     the paper samples "random BFS trees", L479, and gives no rule).  With
 *     mix64 = the SplitMix64 output function (z ^= z>>30; z *= 0xBF58476D1CE4E5B9;
 *     z ^= z>>27; z *= 0x94D049BB133111EB; z ^= z>>31, all mod 2^64) and
 *     G = 0x9E3779B97F4A7C15:
 *       tkey(seed,t)  = mix64(seed + G*(t+1))
 *       root of component C (components ranked by their smallest vertex) =
 *         C's vertices in ascending order [mix64(tkey ^ 0xD1B54A32D192ED03*(C+1)) mod |C|]
 *       dist = BFS distance from the roots (level-synchronous BFS, L116, L123)
 *       parent(w) = the neighbour u with dist(u) = dist(w) - 1 minimising the
 *         pair (pscore(u,w), u), where pscore(u,w) = high 32 bits of
 *         mix64(tkey + G*(min(u,w)*2^32 + max(u,w))) (original vertex ids;
 *         ties to the smaller u).
 *     Disconnected inputs are forests (R3).
 *   - A non-tree edge gets the sign that makes its fundamental cycle even
 *     (L214): flip(e) = (#negative tree edges on the path + neg(e)) mod 2 (R1).
 *
 * All calls return GB_OK (0) or a negative gb_err and set gb_last_error().
 * Not thread-safe; one loaded graph per process, on the CUDA device current at
 * gb_load_csr time.  Every step runs in the library's sm_100a kernels; there
 * is no CPU fallback: without a usable CUDA device calls return GB_ECUDA.
 */
#ifndef GRAPHB_H
#define GRAPHB_H
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

enum gb_err {
    GB_OK = 0,
    GB_EINVAL = -1, /* invalid argument or input graph                     */
    GB_ESTATE = -2, /* no graph loaded                                     */
    GB_ENOMEM = -3, /* device or host allocation failed                    */
    GB_ECUDA = -4   /* CUDA runtime error (message in gb_last_error)       */
};

/* Load a signed graph Sigma = (G, sigma) (one compact
 * CSR, allocated once).  Host arrays, borrowed for the call and copied:
 *   row_ptr [n+1] int64, row_ptr[0] = 0, non-decreasing, row_ptr[n] = 2m
 *   col_idx [2m]  int32, each row strictly increasing (sorted, no duplicates),
 *                 no self loops, 0 <= col < n
 *   sign    [2m]  int8, each +1 or -1, sign(u,v) == sign(v,u) (symmetric)
 * Limits: 1 <= n < 2^31, 2m < 2^32.  Returns GB_EINVAL on any violation (also
 * NULL pointers with m > 0).  A second call replaces the loaded graph. */
int gb_load_csr(int64_t n, int64_t m, const int64_t *row_ptr,
                const int32_t *col_idx, const int8_t *sign);

/* Alg. 2 over trees t = 0 .. num_trees-1 (0 <= num_trees <= 2^30-1).
 * Host outputs, caller-allocated, written in full on success, untouched on
 * error: out_edge_flip_counts [m] indexed by eid, out_vertex_agree [n].
 * num_trees == 0 writes zeros. */
int gb_balance(int64_t num_trees, uint64_t seed,
               uint32_t *out_edge_flip_counts, uint32_t *out_vertex_agree);

/* Release all device and host state.  Idempotent. */
void gb_free(void);

/* ---- extensions (sharding, tests, measurement) -------------------------- */

/* Trees t_begin, t_begin+t_stride, ... < t_end (the tree sharding of L248).
 * DEVICE outputs on the loaded graph's device, ACCUMULATED (+=):
 *   d_edge_cnt [m] int32, d_vertex_agree [n] int32.
 * cuda_stream: a cudaStream_t to run on (NULL = the library's own stream).
 * Asynchronous with respect to the host: the call enqueues its kernels on
 * the stream and returns without synchronising (its statistics are read back
 * by the next gb_get_stats / gb_tree_stats / gb_cloud_states, which wait for
 * the stream).  Calls share the library's tree workspace: issue successive
 * calls on one stream, or synchronise between streams.  The first call on a
 * new graph or batch size allocates (cudaMalloc, which synchronises). */
int gb_balance_range(int64_t t_begin, int64_t t_end, int64_t t_stride, uint64_t seed,
                     int32_t *d_edge_cnt, int32_t *d_vertex_agree, void *cuda_stream);

/* One tree, every stage copied back to host arrays (any pointer may be NULL):
 *   parent[n] (-1 at roots), dist[n] (BFS level), pre[n] (pre-order ID,
 *   Alg. 3 step 1; any valid pre-order of T -- sibling order is not fixed,
 *   R5), size[n] (subtree size, Alg. 4), flip[m] (0/1 by eid),
 *   sum_cycle_len (sum over non-tree edges of the fundamental-cycle length,
 *   counting e itself; L230), num_cycles (= m - n + #components, L112). */
int gb_tree_debug(int64_t t, uint64_t seed, int32_t *parent, int32_t *dist,
                  int32_t *pre, int32_t *size, uint8_t *flip,
                  uint64_t *sum_cycle_len, int64_t *num_cycles);

/* Alg. 3 on a caller tree (host parent[n], -1 at roots): returns flip[m] and
 * the cycle statistics.  GB_EINVAL unless parent is a spanning forest of the
 * loaded graph with exactly one root per connected component. */
int gb_balance_given_tree(const int32_t *parent, uint8_t *flip,
                          uint64_t *sum_cycle_len, int64_t *num_cycles);

/* Options (before gb_balance*): "batch" trees per batch (0 = auto; at most
 * 128, the multi-source BFS width -- larger values are clamped to 128),
 * "cycle_group" trees per cycle-kernel pass (0 = auto), "walk"
 * (0 = two-ended interval walk, 1 = Alg. 3 descent with warp ballots,
 * 2 = the paper's partitioned two-word tree-edge lists (L238-L244) with a
 * linear scan, 3 = pre-order climb: of the two current vertices the one with
 * the larger pre climbs, 4-byte parent words indexed by pre), "desc_linear"
 * (walk 1: 1 = linear int4 ballot rounds over the child starts, 0 = 32-ary
 * pivots), "walk_ept" (walk 0: 1, 2 or 4 edges per thread),
 * "timing" (1 = record per-phase CUDA events), "sub" (trees per labelling launch, 0 = auto), "msprof" (see gb_msbfs_profile),
 * "recpass" (walk 0: 1 = pre-indexed records scattered in a pass after the
 * top-down pass, 0 = inside it), "jump" (walk 0: 1, 2 or 4 tree levels per
 * ancestor record of the cycle walk), "persist" (bytes of an L2 persisting
 * window over the labelling arrays, 0 = off; sets the device-wide persisting
 * L2 limit), "harary" (1 = the Harary sides of every tree come from the
 * paper's L224 procedure on the GPU -- positive-edge CCs of Sigma_T, collapse,
 * BFS level parity -- instead of the root parity pi; a slow cross-check,
 * f.2), "sampler" (Alg. 2 method M, L130: 0 = BFS trees (default, reading
 * R4), 1 = uniform random spanning trees by Wilson's algorithm with
 * per-vertex random stacks (reading R17), sampled on the GPU by parallel
 * cycle popping and processed one tree at a time; gb_tree_debug then reports
 * that tree; 2 = DFS trees with a hashed scan start per vertex, reading R18),
 * "wilson" (sampler 1: 0 = one GPU thread per tree, 1 = parallel cycle
 * popping), "push_parent" (1 = default: BFS batches of <= 16 trees choose the
 * parents of small-frontier levels while pushing -- the same R4 minimum over
 * the same candidates; 0 = always pull), "reset" (every option back to its
 * default). */
int gb_set_option(const char *key, int64_t value);

/* Statistics of the last gb_balance / gb_balance_range call (waits for its
 * stream); the totals cover every tree of the call:
 * ints[0] trees, [1] sum of cycle lengths, [2] cycles, [3] kernel launches,
 * [4] batches, [5] max tree depth, [6] batch size used, [7] cycle group used,
 * [8] edges of some Sigma_T that contradict the L224 bipartition (option
 * "harary" only; 0 means every balanced state was checked and consistent),
 * [9] trees per labelling launch, [10] trees per BFS launch.
 * phase_ms[GB_NPHASE] (valid when "timing" was 1): summed CUDA-event times.
 * Returns the number of ints written. */
#define GB_NPHASE 6
#define GB_PHASE_INIT 0   /* roots, workspace reset                      */
#define GB_PHASE_BFS 1    /* level-synchronous BFS + min-hash parents    */
#define GB_PHASE_UP 2     /* Alg. 4 bottom-up sizes (+ sibling offsets)  */
#define GB_PHASE_DOWN 3   /* Alg. 4 top-down pre-order IDs + ranges + pi */
#define GB_PHASE_CYCLE 4  /* Alg. 3 cycle traversal + balancing          */
#define GB_PHASE_ACCUM 5  /* counter accumulation + Harary agree         */
int gb_get_stats(int64_t *ints, int n_ints, double *phase_ms, int n_phase);

/* Per-tree statistics of the last gb_balance* call, for at most max_trees
 * (<= 65536 recorded) trees in processing order: out[4*i] = sum of cycle
 * lengths, out[4*i+1] = cycles, out[4*i+2] = depth, out[4*i+3] = signature of
 * the tree's nearest balanced state (XOR over switched eids e of
 * mix64(e ^ 0x5851F42D4C957F2D); equal states <=> equal signatures up to
 * 2^-64 collisions -- frustration-cloud analytics, Fig. 2 L81/L86);
 * tree_ids[i] = t.  Returns the count. */
int64_t gb_tree_stats(uint64_t *out, int64_t *tree_ids, int64_t max_trees);

/* Frustration-cloud analytics (f.2, Fig. 2 L81/L86: "5 unique states"): the
 * distinct nearest balanced states among the trees gb_tree_stats records,
 * counted on the device (hash table over the state signatures).  Writes
 * min(k, max_states) pairs sig[i] / count[i] (trees reaching that state;
 * any order) and returns k, the number of distinct states (negative
 * gb_err on failure).  sig or count may be NULL. */
int64_t gb_cloud_states(uint64_t *sig, uint64_t *count, int64_t max_states);

/* Profiling aid: with option "msprof" = 1, the multi-source BFS of the last
 * batch records %globaltimer (ns) at its phase boundaries, out[4*L + k] for
 * level L < 256: k = 0 level start, 1 end of the discovery pass, 2 end of the
 * parent pass, 3 end of the hub pass (0 = not reached).  out has 1024 entries.
 * GB_ESTATE if the option is not set. */
int gb_msbfs_profile(uint64_t *out);

/* Alg. 4 level profile of the last labelling launch (option "msprof" set):
 * out[4*L + k], level L < 256: k = 0 globaltimer (ns) at the start of level L
 * of the bottom-up pass, 1 the same for the top-down pass (level maxd + 1 =
 * the end), 2 vertices on level L summed over the launch's trees.  out has
 * 1024 entries.  GB_ESTATE if the option is not set. */
int gb_label_profile(uint64_t *out);

/* Ingest results (§8 a.1), copied to host arrays (any pointer may be NULL):
 * edge_u[m], edge_v[m] (u < v), edge_neg[m] (1 = negative) indexed by eid;
 * slot_eid[2m] (eid of every CSR slot); comp[n] (component rank, components
 * ordered by their minimum vertex). */
int gb_graph_debug(int32_t *edge_u, int32_t *edge_v, int8_t *edge_neg,
                   uint32_t *slot_eid, int32_t *comp);

/* Loaded graph: n, m, number of connected components. */
int gb_graph_info(int64_t *n, int64_t *m, int64_t *ncomp);

/* Host-only self test of the library's hash (no GPU needed): SplitMix64
 * vector and the inverse used to decode parent keys.  0 = pass. */
int gb_selftest(void);

const char *gb_last_error(void);

#ifdef __cplusplus
}
#endif
#endif
