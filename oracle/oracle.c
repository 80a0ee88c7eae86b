/* oracle.c -- TEST INFRASTRUCTURE ONLY (see oracle.h).
 *
 * A plain, slow, obviously-correct, single-threaded C implementation of what
 * the graphB+ hot path computes, written from /root/reference/PAPER.md:
 *
 *   Alg. 2 (L125-L138)  sample k spanning trees with method M = BFS,
 *   Alg. 1 (L96-L108)   for every non-tree edge e: if the fundamental cycle
 *                       T u e is negative, switch sigma(e),
 *   L224                Harary bipartition of Sigma_T (drop negative edges,
 *                       connected components, collapse, BFS, even/odd levels),
 *   L144                delta_T(v) = 1 / 0.5 / 0 (larger side / tie / smaller),
 *   L248                count per vertex (and per edge) over the trees.
 *
 * Where the method reaches a plainly defined result, this file writes the
 * definition out: the tree path of a non-tree edge is found by climbing the
 * deeper endpoint (no labels, no pre-order, no ranges -- those are the
 * graphB+ acceleration that the CUDA path implements).  Compiled with plain
 * `gcc -O2`; no threads, no SIMD intrinsics, no tricks.
 */
#include "oracle.h"

#include <stdlib.h>
#include <string.h>

struct or_graph {
    int64_t n, m;
    int64_t *row_ptr;   /* [n+1] copy of the input CSR */
    int32_t *col;       /* [2m] */
    int8_t  *sign;      /* [2m] */
    int32_t *eu, *ev;   /* [m] edge list sorted by (min,max): index = eid */
    int8_t  *eneg;      /* [m] 1 iff sigma(e) = -1 */
    int64_t *slot_eid;  /* [2m] eid of each CSR slot */
    int32_t *comp;      /* [n] component rank (ordered by minimum vertex) */
    int64_t  ncomp;
    int64_t *coff;      /* [ncomp+1] */
    int32_t *cverts;    /* [n] vertices grouped by component, ascending */
};

/* ------------------------------------------------------------------------ */
/* Hash.  DESIGN.md reading R4 (PAPER.md L479 says only "random BFS trees";
 * the seed-defined tree is the north star's re-specification):
 * the SplitMix64 finaliser, pinned by the public SplitMix64 test vector.     */
/* ------------------------------------------------------------------------ */
#define OR_GOLDEN 0x9E3779B97F4A7C15ULL

uint64_t or_mix64(uint64_t z)
{
    z ^= z >> 30;
    z *= 0xBF58476D1CE4E5B9ULL;
    z ^= z >> 27;
    z *= 0x94D049BB133111EBULL;
    z ^= z >> 31;
    return z;
}

uint64_t or_splitmix64_next(uint64_t *state)
{
    *state += OR_GOLDEN;
    return or_mix64(*state);
}

/* tkey(seed,t) = the (t+1)-th SplitMix64 output from state = seed. */
uint64_t or_tkey(uint64_t seed, int64_t t)
{
    return or_mix64(seed + OR_GOLDEN * (uint64_t)(t + 1));
}

uint64_t or_rkey(uint64_t seed, int64_t t, int64_t comp)
{
    return or_mix64(or_tkey(seed, t) ^ (0xD1B54A32D192ED03ULL * (uint64_t)(comp + 1)));
}

/* Parent score of the edge {a,b} in tree t (reading R4): the high 32 bits of
 * mix64(tkey + G * (min(a,b) * 2^32 + max(a,b))). */
uint32_t or_pscore(uint64_t seed, int64_t t, int32_t a, int32_t b)
{
    uint64_t lo = (uint64_t)(a < b ? a : b), hi = (uint64_t)(a < b ? b : a);
    return (uint32_t)(or_mix64(or_tkey(seed, t) + OR_GOLDEN * ((lo << 32) | hi)) >> 32);
}

/* ------------------------------------------------------------------------ */
/* Graph ingest: validation (DESIGN.md "Boundary" error list), the undirected
 * edge list (m = #undirected edges, Table 1 L342 reading R2), edge
 * ids = rank of (min,max), connected components (reading R3: forests are
 * accepted, one root per component).                                        */
/* ------------------------------------------------------------------------ */

/* index of value x in the sorted row u, or -1 */
static int64_t row_find(const or_graph *g, int64_t u, int32_t x)
{
    int64_t lo = g->row_ptr[u], hi = g->row_ptr[u + 1] - 1;
    while (lo <= hi) {
        int64_t mid = lo + (hi - lo) / 2;
        if (g->col[mid] == x) return mid;
        if (g->col[mid] < x) lo = mid + 1; else hi = mid - 1;
    }
    return -1;
}

/* eid of the pair (a,b): the rank of (min,max) in the sorted edge list */
static int64_t pair_eid(const or_graph *g, int32_t a, int32_t b)
{
    int32_t u = a < b ? a : b, v = a < b ? b : a;
    int64_t lo = 0, hi = g->m - 1;
    while (lo <= hi) {
        int64_t mid = lo + (hi - lo) / 2;
        if (g->eu[mid] == u && g->ev[mid] == v) return mid;
        if (g->eu[mid] < u || (g->eu[mid] == u && g->ev[mid] < v)) lo = mid + 1; else hi = mid - 1;
    }
    return -1;
}

void or_free(or_graph *g)
{
    if (!g) return;
    free(g->row_ptr); free(g->col); free(g->sign);
    free(g->eu); free(g->ev); free(g->eneg); free(g->slot_eid);
    free(g->comp); free(g->coff); free(g->cverts);
    free(g);
}

int or_build(int64_t n, int64_t m, const int64_t *row_ptr, const int32_t *col,
             const int8_t *sign, or_graph **out)
{
    *out = NULL;
    if (n < 1 || n >= ((int64_t)1 << 31) || m < 0 || !row_ptr) return OR_EINVAL;
    if (m > 0 && (!col || !sign)) return OR_EINVAL;
    if (row_ptr[0] != 0 || row_ptr[n] != 2 * m) return OR_EINVAL;
    for (int64_t u = 0; u < n; u++)
        if (row_ptr[u + 1] < row_ptr[u]) return OR_EINVAL;
    for (int64_t u = 0; u < n; u++) {
        for (int64_t j = row_ptr[u]; j < row_ptr[u + 1]; j++) {
            if (col[j] < 0 || col[j] >= n || col[j] == u) return OR_EINVAL;
            if (j > row_ptr[u] && col[j - 1] >= col[j]) return OR_EINVAL;
            if (sign[j] != 1 && sign[j] != -1) return OR_EINVAL;
        }
    }
    or_graph *g = (or_graph *)calloc(1, sizeof(or_graph));
    if (!g) return OR_ENOMEM;
    g->n = n; g->m = m;
    g->row_ptr = (int64_t *)malloc(sizeof(int64_t) * (size_t)(n + 1));
    g->col = (int32_t *)malloc(sizeof(int32_t) * (size_t)(2 * m + 1));
    g->sign = (int8_t *)malloc((size_t)(2 * m + 1));
    g->eu = (int32_t *)malloc(sizeof(int32_t) * (size_t)(m + 1));
    g->ev = (int32_t *)malloc(sizeof(int32_t) * (size_t)(m + 1));
    g->eneg = (int8_t *)malloc((size_t)(m + 1));
    g->slot_eid = (int64_t *)malloc(sizeof(int64_t) * (size_t)(2 * m + 1));
    g->comp = (int32_t *)malloc(sizeof(int32_t) * (size_t)n);
    g->coff = (int64_t *)malloc(sizeof(int64_t) * (size_t)(n + 1));
    g->cverts = (int32_t *)malloc(sizeof(int32_t) * (size_t)n);
    if (!g->row_ptr || !g->col || !g->sign || !g->eu || !g->ev || !g->eneg ||
        !g->slot_eid || !g->comp || !g->coff || !g->cverts) {
        or_free(g);
        return OR_ENOMEM;
    }
    memcpy(g->row_ptr, row_ptr, sizeof(int64_t) * (size_t)(n + 1));
    if (m) {
        memcpy(g->col, col, sizeof(int32_t) * (size_t)(2 * m));
        memcpy(g->sign, sign, (size_t)(2 * m));
    }
    /* mirror entries with equal signs */
    for (int64_t u = 0; u < n; u++)
        for (int64_t j = row_ptr[u]; j < row_ptr[u + 1]; j++) {
            int64_t k = row_find(g, col[j], (int32_t)u);
            if (k < 0 || sign[k] != sign[j]) { or_free(g); return OR_EINVAL; }
        }
    /* the edge list: rows ascending, upper entries ascending => sorted by
     * (min,max), so the position in this list is the rank = eid */
    int64_t e = 0;
    for (int64_t u = 0; u < n; u++)
        for (int64_t j = row_ptr[u]; j < row_ptr[u + 1]; j++)
            if (col[j] > u) {
                g->eu[e] = (int32_t)u; g->ev[e] = col[j]; g->eneg[e] = sign[j] < 0;
                e++;
            }
    if (e != m) { or_free(g); return OR_EINVAL; }
    for (int64_t u = 0; u < n; u++)
        for (int64_t j = row_ptr[u]; j < row_ptr[u + 1]; j++)
            g->slot_eid[j] = pair_eid(g, (int32_t)u, col[j]);
    /* components by BFS from the smallest unvisited vertex => ranked by
     * minimum vertex; members listed in ascending order afterwards */
    int32_t *queue = (int32_t *)malloc(sizeof(int32_t) * (size_t)n);
    int64_t *fill = (int64_t *)malloc(sizeof(int64_t) * (size_t)(n + 1));
    if (!queue || !fill) { free(queue); free(fill); or_free(g); return OR_ENOMEM; }
    for (int64_t v = 0; v < n; v++) g->comp[v] = -1;
    int64_t nc = 0;
    for (int64_t s = 0; s < n; s++) {
        if (g->comp[s] >= 0) continue;
        int64_t qh = 0, qt = 0;
        queue[qt++] = (int32_t)s;
        g->comp[s] = (int32_t)nc;
        while (qh < qt) {
            int32_t x = queue[qh++];
            for (int64_t j = row_ptr[x]; j < row_ptr[x + 1]; j++)
                if (g->comp[col[j]] < 0) { g->comp[col[j]] = (int32_t)nc; queue[qt++] = col[j]; }
        }
        nc++;
    }
    g->ncomp = nc;
    for (int64_t c = 0; c <= nc; c++) g->coff[c] = 0;
    for (int64_t v = 0; v < n; v++) g->coff[g->comp[v] + 1]++;
    for (int64_t c = 0; c < nc; c++) g->coff[c + 1] += g->coff[c];
    for (int64_t c = 0; c <= nc; c++) fill[c] = g->coff[c];
    for (int64_t v = 0; v < n; v++) g->cverts[fill[g->comp[v]]++] = (int32_t)v;
    free(queue); free(fill);
    *out = g;
    return OR_OK;
}

int64_t or_n(const or_graph *g) { return g->n; }
int64_t or_m(const or_graph *g) { return g->m; }
int64_t or_ncomp(const or_graph *g) { return g->ncomp; }

void or_edges(const or_graph *g, int32_t *u, int32_t *v, int8_t *neg)
{
    for (int64_t e = 0; e < g->m; e++) { u[e] = g->eu[e]; v[e] = g->ev[e]; neg[e] = g->eneg[e]; }
}

void or_components(const or_graph *g, int32_t *comp, int64_t *coff, int32_t *cverts)
{
    for (int64_t v = 0; v < g->n; v++) { comp[v] = g->comp[v]; cverts[v] = g->cverts[v]; }
    for (int64_t c = 0; c <= g->ncomp; c++) coff[c] = g->coff[c];
}

/* ------------------------------------------------------------------------ */
/* Tree sampling, Alg. 2 with M = BFS (L116-L123, L130; "random BFS trees"
 * L479).  Reading R4: the root of component C in tree t is
 * cverts_C[rkey(seed,t,C) mod |C|]; dist is the level-synchronous BFS
 * distance; parent[w] is the neighbour u with dist[u] = dist[w]-1 that
 * minimises (pscore(seed,t,u,w), u) -- the score first, the smaller vertex
 * id on an equal score.                                                     */
/* ------------------------------------------------------------------------ */
int or_bfs_tree(const or_graph *g, uint64_t seed, int64_t t,
                int32_t *parent, int32_t *dist, int32_t *peid)
{
    int64_t n = g->n;
    int32_t *queue = (int32_t *)malloc(sizeof(int32_t) * (size_t)n);
    if (!queue) return OR_ENOMEM;
    for (int64_t v = 0; v < n; v++) dist[v] = -1;
    int64_t qh = 0, qt = 0;
    for (int64_t c = 0; c < g->ncomp; c++) {
        int64_t sz = g->coff[c + 1] - g->coff[c];
        int32_t r = g->cverts[g->coff[c] + (int64_t)(or_rkey(seed, t, c) % (uint64_t)sz)];
        dist[r] = 0;
        queue[qt++] = r;
    }
    while (qh < qt) {
        int32_t x = queue[qh++];
        for (int64_t j = g->row_ptr[x]; j < g->row_ptr[x + 1]; j++)
            if (dist[g->col[j]] < 0) { dist[g->col[j]] = dist[x] + 1; queue[qt++] = g->col[j]; }
    }
    for (int64_t w = 0; w < n; w++) {
        parent[w] = -1;
        if (peid) peid[w] = -1;
        if (dist[w] == 0) continue;
        uint32_t best = 0;
        int32_t bu = -1;
        int64_t be = -1;
        for (int64_t j = g->row_ptr[w]; j < g->row_ptr[w + 1]; j++) {
            int32_t u = g->col[j];
            if (dist[u] != dist[w] - 1) continue;
            uint32_t k = or_pscore(seed, t, u, (int32_t)w);
            if (bu < 0 || k < best || (k == best && u < bu)) { best = k; bu = u; be = g->slot_eid[j]; }
        }
        parent[w] = bu;
        if (peid) peid[w] = (int32_t)be;
    }
    free(queue);
    return OR_OK;
}

/* ------------------------------------------------------------------------ */
/* Tree sampling, Alg. 2 with M = random (L130 "e.g., BFS, DFS, random";
 * L168 prior work used random spanning trees): a uniformly random spanning
 * tree by Wilson's algorithm (loop-erased random walks, reading R17).  The
 * walk's randomness is a per-vertex stack: the j-th departure from u goes to
 * N(u)[wdraw(seed,t,u,j) mod deg(u)], wdraw = mix64(tkey + W*(u*2^32 + j)).
 * Roots are the BFS sampler's (R4).  Vertices are started in ascending order
 * (order = 0) or descending order (order = 1): with fixed stacks the tree
 * does not depend on the order (the cycle-popping theorem), which the tests
 * use as a pin.  The walk overwrites nxt[u] at every departure (last-exit
 * loop erasure); pops[u] = departures from u - 1 for tree vertices.          */
/* ------------------------------------------------------------------------ */
#define OR_WMUL 0xD6E8FEB86659FD93ULL

uint64_t or_wdraw(uint64_t seed, int64_t t, int32_t u, uint32_t j)
{
    return or_mix64(or_tkey(seed, t) + OR_WMUL * (((uint64_t)(uint32_t)u << 32) | (uint64_t)j));
}

int or_wilson_tree(const or_graph *g, uint64_t seed, int64_t t, int order,
                   int32_t *parent, uint32_t *pops)
{
    int64_t n = g->n;
    uint8_t *in_tree = (uint8_t *)calloc((size_t)n + 1, 1);
    uint32_t *dep = (uint32_t *)calloc((size_t)n + 1, sizeof(uint32_t));
    int32_t *nxt = (int32_t *)malloc(sizeof(int32_t) * ((size_t)n + 1));
    if (!in_tree || !dep || !nxt) { free(in_tree); free(dep); free(nxt); return OR_ENOMEM; }
    for (int64_t v = 0; v < n; v++) nxt[v] = -1;
    for (int64_t c = 0; c < g->ncomp; c++) {
        int64_t sz = g->coff[c + 1] - g->coff[c];
        int32_t r = g->cverts[g->coff[c] + (int64_t)(or_rkey(seed, t, c) % (uint64_t)sz)];
        in_tree[r] = 1;
    }
    for (int64_t i = 0; i < n; i++) {
        int64_t v = order ? n - 1 - i : i;
        /* random walk from v until it hits the tree, remembering the last exit */
        int64_t u = v;
        while (!in_tree[u]) {
            int64_t deg = g->row_ptr[u + 1] - g->row_ptr[u];
            uint64_t k = or_wdraw(seed, t, (int32_t)u, dep[u]++) % (uint64_t)deg;
            nxt[u] = g->col[g->row_ptr[u] + (int64_t)k];
            u = nxt[u];
        }
        /* add the loop-erased path */
        for (u = v; !in_tree[u]; u = nxt[u]) in_tree[u] = 1;
    }
    for (int64_t v = 0; v < n; v++) {
        parent[v] = nxt[v];          /* -1 for the roots (never departed) */
        if (pops) pops[v] = dep[v] ? dep[v] - 1 : 0;
    }
    free(in_tree); free(dep); free(nxt);
    return OR_OK;
}

/* ------------------------------------------------------------------------ */
/* Tree sampling, Alg. 2 with M = DFS (L130), reading R18: a depth-first
 * search from the R4 root of every component (components in rank order);
 * at vertex u the neighbours are scanned from position
 * dstart(u) = mix64(tkey ^ D*(u+1)) mod deg(u) cyclically, and the first
 * unvisited one is descended into (returning to u resumes the scan).
 * parent[w] = the vertex that discovered w.                                 */
/* ------------------------------------------------------------------------ */
#define OR_DMUL 0x8CB92BA72F3D8DD7ULL

uint64_t or_dstart(uint64_t seed, int64_t t, int32_t u)
{
    return or_mix64(or_tkey(seed, t) ^ (OR_DMUL * ((uint64_t)(uint32_t)u + 1)));
}

int or_dfs_tree(const or_graph *g, uint64_t seed, int64_t t, int32_t *parent)
{
    int64_t n = g->n;
    uint8_t *seen = (uint8_t *)calloc((size_t)n + 1, 1);
    int64_t *pos = (int64_t *)calloc((size_t)n + 1, sizeof(int64_t));
    int32_t *stack = (int32_t *)malloc(sizeof(int32_t) * ((size_t)n + 1));
    if (!seen || !pos || !stack) { free(seen); free(pos); free(stack); return OR_ENOMEM; }
    for (int64_t v = 0; v < n; v++) parent[v] = -1;
    for (int64_t c = 0; c < g->ncomp; c++) {
        int64_t sz = g->coff[c + 1] - g->coff[c];
        int32_t r = g->cverts[g->coff[c] + (int64_t)(or_rkey(seed, t, c) % (uint64_t)sz)];
        int64_t top = 0;
        seen[r] = 1;
        stack[top++] = r;
        while (top > 0) {
            int32_t u = stack[top - 1];
            int64_t deg = g->row_ptr[u + 1] - g->row_ptr[u];
            if (pos[u] == deg) { top--; continue; }
            int64_t k = (int64_t)((or_dstart(seed, t, u) % (uint64_t)deg + (uint64_t)pos[u]) % (uint64_t)deg);
            pos[u]++;
            int32_t w = g->col[g->row_ptr[u] + k];
            if (!seen[w]) { seen[w] = 1; parent[w] = u; stack[top++] = w; }
        }
    }
    free(seen); free(pos); free(stack);
    return OR_OK;
}

/* depth of every vertex under parent[], checking that parent[] is a spanning
 * forest of g with exactly one root per connected component. */
static int tree_depth(const or_graph *g, const int32_t *parent, int32_t *depth, int8_t *pneg)
{
    int64_t n = g->n;
    int64_t *roots = (int64_t *)calloc((size_t)g->ncomp, sizeof(int64_t));
    if (!roots) return OR_ENOMEM;
    for (int64_t v = 0; v < n; v++) {
        depth[v] = -1;
        if (parent[v] == -1) {
            roots[g->comp[v]]++;
            pneg[v] = 0;
            continue;
        }
        if (parent[v] < 0 || parent[v] >= n) { free(roots); return OR_EINVAL; }
        int64_t j = row_find(g, v, parent[v]);
        if (j < 0) { free(roots); return OR_EINVAL; }
        pneg[v] = g->sign[j] < 0;
    }
    for (int64_t c = 0; c < g->ncomp; c++)
        if (roots[c] != 1) { free(roots); return OR_EINVAL; }
    free(roots);
    for (int64_t v = 0; v < n; v++) {
        if (depth[v] >= 0) continue;
        /* climb to a vertex of known depth or to a root */
        int64_t len = 0;
        int32_t x = (int32_t)v;
        while (depth[x] < 0 && parent[x] != -1) {
            x = parent[x];
            if (++len > n) return OR_EINVAL; /* parent[] has a cycle */
        }
        if (depth[x] < 0) depth[x] = 0; /* x is a root */
        int32_t y = (int32_t)v;
        for (int64_t i = 0; i < len; i++) { depth[y] = depth[x] + (int32_t)(len - i); y = parent[y]; }
    }
    return OR_OK;
}

/* ------------------------------------------------------------------------ */
/* Alg. 1 (L96-L108) with the fundamental cycle of L112: e together with the
 * tree path between its endpoints.  The path is found by repeatedly moving
 * the deeper endpoint to its parent until both meet (at the LCA).  c counts
 * the negative tree edges on the path.  Reading R1 (Alg. 3 L198 vs L214 /
 * Alg. 1): the cycle is negative iff c + neg(e) is odd, then sigma(e)
 * is switched, i.e. flip(e) = c XOR neg(e) and the new sign of e is (-1)^c.
 * The cycle length k counts e plus every tree edge of the path (L230 bound
 * k <= d(a)+d(b)+1).                                                         */
/* ------------------------------------------------------------------------ */
int or_balance_tree(const or_graph *g, const int32_t *parent, uint8_t *flip,
                    uint64_t *sumk, int64_t *ncyc, int32_t *maxdepth)
{
    int64_t n = g->n;
    int32_t *depth = (int32_t *)malloc(sizeof(int32_t) * (size_t)n);
    int8_t *pneg = (int8_t *)malloc((size_t)n);
    if (!depth || !pneg) { free(depth); free(pneg); return OR_ENOMEM; }
    int rc = tree_depth(g, parent, depth, pneg);
    if (rc != OR_OK) { free(depth); free(pneg); return rc; }
    uint64_t sk = 0;
    int64_t nc = 0;
    int32_t md = 0;
    for (int64_t v = 0; v < n; v++) if (depth[v] > md) md = depth[v];
    for (int64_t e = 0; e < g->m; e++) {
        int32_t u = g->eu[e], v = g->ev[e];
        flip[e] = 0;
        if (parent[v] == u || parent[u] == v) continue; /* tree edge: never switched */
        int32_t a = u, b = v;
        int c = 0;
        uint64_t k = 1;
        while (a != b) {
            if (depth[a] >= depth[b]) { c ^= pneg[a]; a = parent[a]; }
            else                      { c ^= pneg[b]; b = parent[b]; }
            k++;
        }
        flip[e] = (uint8_t)(c ^ g->eneg[e]);
        sk += k;
        nc++;
    }
    if (sumk) *sumk = sk;
    if (ncyc) *ncyc = nc;
    if (maxdepth) *maxdepth = md;
    free(depth); free(pneg);
    return OR_OK;
}

/* ------------------------------------------------------------------------ */
/* Alg. 3 steps 1-2 (L182-L189, L210-L212) as their plain definition: a
 * sequential pre-order walk; new ID = number of previously visited vertices
 * (L210); the range of tree edge p->c is [pre c, pre c + size c - 1]
 * (Alg. 4), i.e. it is given by pre and size.  Reading R5: the
 * children of a vertex are visited in ascending original id; reading R6:
 * components are walked in rank order, so pre[root_C] = coff[C].            */
/* ------------------------------------------------------------------------ */
int or_preorder(const or_graph *g, const int32_t *parent, int32_t *pre, int32_t *size)
{
    int64_t n = g->n;
    int32_t *depth = (int32_t *)malloc(sizeof(int32_t) * (size_t)n);
    int8_t *pneg = (int8_t *)malloc((size_t)n);
    int64_t *cstart = (int64_t *)calloc((size_t)(n + 1), sizeof(int64_t));
    int64_t *cfill = (int64_t *)malloc(sizeof(int64_t) * (size_t)(n + 1));
    int32_t *child = (int32_t *)malloc(sizeof(int32_t) * (size_t)n);
    int32_t *stack = (int32_t *)malloc(sizeof(int32_t) * (size_t)n);
    int32_t *order = (int32_t *)malloc(sizeof(int32_t) * (size_t)n);
    int rc = OR_ENOMEM;
    if (!depth || !pneg || !cstart || !cfill || !child || !stack || !order) goto out;
    rc = tree_depth(g, parent, depth, pneg);
    if (rc != OR_OK) goto out;
    for (int64_t v = 0; v < n; v++) if (parent[v] >= 0) cstart[parent[v] + 1]++;
    for (int64_t v = 0; v < n; v++) cstart[v + 1] += cstart[v];
    for (int64_t v = 0; v <= n; v++) cfill[v] = cstart[v];
    for (int64_t v = 0; v < n; v++) if (parent[v] >= 0) child[cfill[parent[v]]++] = (int32_t)v;
    int64_t next = 0, no = 0;
    for (int64_t c = 0; c < g->ncomp; c++) {
        int32_t root = -1;
        for (int64_t i = g->coff[c]; i < g->coff[c + 1]; i++)
            if (parent[g->cverts[i]] == -1) { root = g->cverts[i]; break; }
        int64_t sp = 0;
        stack[sp++] = root;
        while (sp > 0) {
            int32_t x = stack[--sp];
            pre[x] = (int32_t)next++;
            order[no++] = x;
            for (int64_t i = cstart[x + 1] - 1; i >= cstart[x]; i--) stack[sp++] = child[i];
        }
    }
    for (int64_t v = 0; v < n; v++) size[v] = 1;
    for (int64_t i = n - 1; i >= 0; i--) {
        int32_t x = order[i];
        if (parent[x] >= 0) size[parent[x]] += size[x];
    }
    rc = OR_OK;
out:
    free(depth); free(pneg); free(cstart); free(cfill); free(child); free(stack); free(order);
    return rc;
}

/* ------------------------------------------------------------------------ */
/* Harary bipartition of Sigma_T, the paper's procedure (L224): ignore the
 * negative edges, compute connected components, collapse each CC to a single
 * vertex, BFS the collapsed graph, even levels = one side.  Each original
 * component is bipartitioned on its own (reading R3).  delta2 = 2*delta_T(v)
 * with delta_T from L144 (1 larger side, 0.5 tie, 0 otherwise) -- reading
 * R8: integer half-units.  Returns OR_EUNBAL if Sigma_T is not balanced
 * (a negative edge inside a CC, or an odd cycle in the collapsed graph).     */
/* ------------------------------------------------------------------------ */
int or_harary(const or_graph *g, const uint8_t *flip, uint8_t *side, uint8_t *delta2)
{
    int64_t n = g->n;
    int32_t *cc = (int32_t *)malloc(sizeof(int32_t) * (size_t)n);
    int32_t *queue = (int32_t *)malloc(sizeof(int32_t) * (size_t)n);
    int32_t *lvl = (int32_t *)malloc(sizeof(int32_t) * (size_t)n);   /* per collapsed node */
    int32_t *rep = (int32_t *)malloc(sizeof(int32_t) * (size_t)n);   /* a vertex of each CC */
    int64_t *s1 = (int64_t *)calloc((size_t)g->ncomp, sizeof(int64_t));
    int rc = OR_ENOMEM;
    if (!cc || !queue || !lvl || !rep || !s1) goto out;
    /* 1. CCs of the positive part of Sigma_T */
    for (int64_t v = 0; v < n; v++) cc[v] = -1;
    int64_t ncc = 0;
    for (int64_t s = 0; s < n; s++) {
        if (cc[s] >= 0) continue;
        int64_t qh = 0, qt = 0;
        queue[qt++] = (int32_t)s;
        cc[s] = (int32_t)ncc;
        rep[ncc] = (int32_t)s;
        while (qh < qt) {
            int32_t x = queue[qh++];
            for (int64_t j = g->row_ptr[x]; j < g->row_ptr[x + 1]; j++) {
                int neg_t = (g->sign[j] < 0) ^ (flip[g->slot_eid[j]] != 0);
                if (neg_t) continue;
                if (cc[g->col[j]] < 0) { cc[g->col[j]] = (int32_t)ncc; queue[qt++] = g->col[j]; }
            }
        }
        ncc++;
    }
    /* 2-3. collapse each CC to a node and BFS the collapsed graph (node =
     * CC, edge = negative edge of Sigma_T); member lists give each CC's
     * vertices */
    {
        int64_t *mstart = (int64_t *)calloc((size_t)(ncc + 1), sizeof(int64_t));
        int64_t *mfill = (int64_t *)malloc(sizeof(int64_t) * (size_t)(ncc + 1));
        int32_t *mem = (int32_t *)malloc(sizeof(int32_t) * (size_t)n);
        if (!mstart || !mfill || !mem) { free(mstart); free(mfill); free(mem); goto out; }
        for (int64_t v = 0; v < n; v++) mstart[cc[v] + 1]++;
        for (int64_t c = 0; c < ncc; c++) mstart[c + 1] += mstart[c];
        for (int64_t c = 0; c <= ncc; c++) mfill[c] = mstart[c];
        for (int64_t v = 0; v < n; v++) mem[mfill[cc[v]]++] = (int32_t)v;
        for (int64_t c = 0; c < ncc; c++) lvl[c] = -1;
        rc = OR_OK;
        for (int64_t s = 0; s < ncc && rc == OR_OK; s++) {
            if (lvl[s] >= 0) continue;
            lvl[s] = 0;
            int64_t qh = 0, qt = 0;
            queue[qt++] = (int32_t)s;
            while (qh < qt && rc == OR_OK) {
                int32_t C = queue[qh++];
                for (int64_t i = mstart[C]; i < mstart[C + 1]; i++) {
                    int32_t x = mem[i];
                    for (int64_t j = g->row_ptr[x]; j < g->row_ptr[x + 1]; j++) {
                        int neg_t = (g->sign[j] < 0) ^ (flip[g->slot_eid[j]] != 0);
                        int32_t D = cc[g->col[j]];
                        if (!neg_t) continue;
                        if (D == C) { rc = OR_EUNBAL; break; }       /* negative edge inside a CC */
                        if (lvl[D] < 0) { lvl[D] = lvl[C] + 1; queue[qt++] = D; }
                        else if ((lvl[D] & 1) == (lvl[C] & 1)) { rc = OR_EUNBAL; break; } /* odd cycle */
                    }
                    if (rc != OR_OK) break;
                }
            }
        }
        free(mstart); free(mfill); free(mem);
        if (rc != OR_OK) goto out;
    }
    /* 4. sides and delta per original component */
    for (int64_t v = 0; v < n; v++) {
        side[v] = (uint8_t)(lvl[cc[v]] & 1);
        s1[g->comp[v]] += side[v];
    }
    for (int64_t v = 0; v < n; v++) {
        int64_t C = g->comp[v];
        int64_t sz = g->coff[C + 1] - g->coff[C];
        int64_t mine = side[v] ? s1[C] : sz - s1[C];
        int64_t other = sz - mine;
        delta2[v] = (uint8_t)(mine > other ? 2 : (mine == other ? 1 : 0));
    }
    rc = OR_OK;
out:
    free(cc); free(queue); free(lvl); free(rep); free(s1);
    return rc;
}

/* ------------------------------------------------------------------------ */
/* Frustration-cloud analytics (Fig. 2 L81/L86: the cloud is
 * the set of *unique* nearest balanced states).  A balanced state Sigma_T is
 * identified by its switch set; its signature is the XOR over switched edges
 * e of mix64(e XOR 0x5851F42D4C957F2D).  Equal states have equal signatures;
 * distinct states collide with probability 2^-64.                           */
/* ------------------------------------------------------------------------ */
uint64_t or_state_signature(const uint8_t *flip, int64_t m)
{
    uint64_t s = 0;
    for (int64_t e = 0; e < m; e++)
        if (flip[e]) s ^= or_mix64((uint64_t)e ^ 0x5851F42D4C957F2DULL);
    return s;
}

/* ------------------------------------------------------------------------ */
/* Alg. 2 (L125-L138) over the trees t_begin, t_begin+stride, ... < t_end:
 * sample T (BFS), balance (Alg. 1), Harary bipartition (L224), count per
 * edge and per vertex (L248).                                               */
/* ------------------------------------------------------------------------ */
int or_balance_m(const or_graph *g, int64_t t_begin, int64_t t_end, int64_t stride,
                 uint64_t seed, int sampler, uint32_t *cnt, uint32_t *agree, uint64_t *stats);

int or_balance(const or_graph *g, int64_t t_begin, int64_t t_end, int64_t stride,
               uint64_t seed, uint32_t *cnt, uint32_t *agree, uint64_t *stats)
{
    return or_balance_m(g, t_begin, t_end, stride, seed, 0, cnt, agree, stats);
}

/* sampler: 0 = BFS (R4), 1 = uniform (Wilson, R17), 2 = DFS (R18) */
int or_balance_m(const or_graph *g, int64_t t_begin, int64_t t_end, int64_t stride,
                 uint64_t seed, int sampler, uint32_t *cnt, uint32_t *agree, uint64_t *stats)
{
    if (stride < 1 || t_begin < 0 || t_end < t_begin) return OR_EINVAL;
    int64_t n = g->n, m = g->m;
    int32_t *parent = (int32_t *)malloc(sizeof(int32_t) * (size_t)n);
    int32_t *dist = (int32_t *)malloc(sizeof(int32_t) * (size_t)n);
    uint8_t *flip = (uint8_t *)malloc((size_t)(m + 1));
    uint8_t *side = (uint8_t *)malloc((size_t)n);
    uint8_t *delta2 = (uint8_t *)malloc((size_t)n);
    int rc = OR_ENOMEM;
    if (!parent || !dist || !flip || !side || !delta2) goto out;
    int64_t i = 0;
    for (int64_t t = t_begin; t < t_end; t += stride, i++) {
        rc = sampler == 1 ? or_wilson_tree(g, seed, t, 0, parent, NULL)
           : sampler == 2 ? or_dfs_tree(g, seed, t, parent)
                          : or_bfs_tree(g, seed, t, parent, dist, NULL);
        if (rc != OR_OK) goto out;
        uint64_t sk = 0;
        int64_t nc = 0;
        int32_t md = 0;
        rc = or_balance_tree(g, parent, flip, &sk, &nc, &md);
        if (rc != OR_OK) goto out;
        rc = or_harary(g, flip, side, delta2);
        if (rc != OR_OK) goto out;
        for (int64_t e = 0; e < m; e++) cnt[e] += flip[e];
        for (int64_t v = 0; v < n; v++) agree[v] += delta2[v];
        if (stats) {
            stats[4 * i] = sk;
            stats[4 * i + 1] = (uint64_t)nc;
            stats[4 * i + 2] = (uint64_t)md;
            stats[4 * i + 3] = or_state_signature(flip, m);
        }
    }
    rc = OR_OK;
out:
    free(parent); free(dist); free(flip); free(side); free(delta2);
    return rc;
}
