// gb_tbfs.cu -- §8 rows a.2 + a.3: hashed roots, level-synchronous BFS and
// min-hash parent selection for G trees per cooperative launch, one bitmap
// set per tree ("tree-parallel pull BFS", option bfs = 0, the default).
//
// The paper builds one BFS tree at a time with one parallel loop per level
// (§3.1; Fig. 11 "spanning tree" 6 %, L467).  The multi-source BFS of
// gb_msbfs.cu (option bfs = 1) shares each pass over the graph between 64
// trees, but then has to transpose every (vertex, tree) discovery into the
// trees' level lists in a second pass -- measured 0.41 ms of its 0.56 ms per
// C3 tree.  Here each tree keeps its own bitmaps, so the parent of a vertex
// is chosen in the same pass that discovers it:
//
//   level L -> L+1, for every vertex w not yet reached (pull, L116/L123):
//     candidates = { u in N(w) : u on level L }          (frontier bitmap test)
//     parent(w)  = argmin over candidates of (pscore(u,w), u)     (reading R4)
//
// and w is appended to the tree's level-(L+1) list (original ids, the layout
// the Alg. 4 passes stream).  While a tree's frontier is small the level
// first *pushes*: frontier vertices mark their neighbours in a bitmap and the
// pull reads only the adjacency of marked vertices (direction optimisation;
// a vertex with no frontier neighbour cannot be discovered).
//
// State per tree, one bit per internal (degree-sorted) vertex id, 1.25 MB
// each for C3 (L2-resident): vis = reached (updated as soon as a vertex is
// discovered -- every vertex is decided by exactly one warp), three frontier
// bitmaps fr(level mod 3) (fr(L) read, fr(L+1) written, fr(L-1) cleared), two
// mark bitmaps mk(level mod 2).  Per launch: fin = "reached in every tree of
// the launch", which lets a whole tile be skipped with one load.  Hubs
// (vertices with several work items) are decided by all their chunks
// together: hlev[g][h] = level + 2 once tree g discovered h (0 = not yet), so
// every chunk of a level sees the same answer.
//
#include "gb_internal.cuh"
#include "../../include/graphb.h"

#include <algorithm>

namespace gb {
namespace cg = cooperative_groups;

constexpr int kTbBms = 6;     // bitmaps per tree: vis, fr x3, mk x2
constexpr int kTbVis = 0;

struct TbParams {
    const uint32_t *brow, *badj, *borig, *bord, *brank;
    const uint2 *items;
    const int32_t *coff, *cverts;
    int64_t n, ncomp, nitems, nmulti_items, nlight0, nmulti, ls, nwords, itemwords;
    unsigned long long slots;     // 2m
    int G;
    uint32_t *bm;                 // [G][kTbBms][nwords]
    uint32_t *fin;                // [nwords] reached in every tree of the launch
    unsigned long long *hbest;    // [G][nmulti] hub parent keys (~0 = none)
    uint32_t *hpos;               // [G][nmulti] hub list positions (kNone = not discovered)
    uint32_t *hlev;               // [G][nmulti] level + 2 at which the hub was discovered (0 = not)
    const uint64_t *tkey;         // [G]
    uint32_t *qv, *parq, *pp;     // tree stride n
    uint2 *rec, *crec;
    uint4 *irec;
    uint64_t *lvl;                // [G][ls]: vertex count << 32 | degree sum, per level
    uint32_t *vbase;              // [G][ls]
    int32_t *depth, *maxd;
    int push_k;                   // push while frontier slots * push_k < unvisited slots
    unsigned long long *prof;     // option "msprof": [256][4] globaltimer per level
};

__device__ __forceinline__ uint32_t *tb_bm(const TbParams &P, int g, int k) {
    return P.bm + ((size_t)g * kTbBms + k) * (size_t)P.nwords;
}
__device__ __forceinline__ int fr_k(int L) { return 1 + (L + 3) % 3; }   // L >= -1
__device__ __forceinline__ int mk_k(int L) { return 4 + (L & 1); }

__device__ __forceinline__ bool bit_of(const uint32_t *bm, uint32_t x) {
    return (__ldcg(bm + (x >> 5)) >> (x & 31)) & 1u;
}

__device__ __forceinline__ uint32_t tb_incl_scan32(uint32_t v) {
    const int lane = threadIdx.x & 31;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
        const uint32_t y = __shfl_up_sync(0xFFFFFFFFu, v, d);
        if (lane >= d) v += y;
    }
    return v;
}

__device__ __forceinline__ unsigned long long tb_warp_min64(unsigned long long v) {
    const uint32_t hi = (uint32_t)(v >> 32);
    const uint32_t mh = __reduce_min_sync(0xFFFFFFFFu, hi);
    const uint32_t ml = __reduce_min_sync(0xFFFFFFFFu, hi == mh ? (uint32_t)v : 0xFFFFFFFFu);
    return ((unsigned long long)mh << 32) | ml;
}

// parent | neg << 31 as an internal id (keys carry the original id, R4)
__device__ __forceinline__ uint32_t tb_key_to_par(const uint32_t *brank, unsigned long long key) {
    return __ldg(brank + ((uint32_t)(key >> 1) & kIdMask)) | ((uint32_t)key << 31);
}

__device__ __forceinline__ unsigned long long tb_gtimer() {
    unsigned long long t;
    asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
    return t;
}

// ---------------------------------------------------------------------------
// roots (reading R4): root of component C in tree g = C's vertices
// (ascending)[rkey(g, C) mod |C|]; level 0 of every tree
// ---------------------------------------------------------------------------
__global__ void k_tb_roots(TbParams P) {
    const int64_t total = (int64_t)P.G * P.ncomp;
    for (int64_t x = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; x < total;
         x += (int64_t)gridDim.x * blockDim.x) {
        const int g = (int)(x / P.ncomp);
        const int64_t C = x - (int64_t)g * P.ncomp;
        const uint32_t sz = (uint32_t)(P.coff[C + 1] - P.coff[C]);
        const uint64_t rk = root_key(P.tkey[g], C);
        const uint32_t r = (uint32_t)P.cverts[P.coff[C] + (int64_t)(rk % sz)];
        const uint32_t ri = P.brank[r];
        const size_t nb = (size_t)g * P.n;
        const uint32_t deg = P.brow[ri + 1] - P.brow[ri];
        if (deg == 0) {
            // isolated vertex: a one-vertex tree, finished here (pi = 0)
            const uint32_t pre = (uint32_t)P.coff[C];
            if (P.irec) {
                P.irec[nb + ri] = make_uint4(ri, pre, 1u, 0u);
            } else {
                P.pp[nb + ri] = pre;
                P.rec[nb + pre] = make_uint2(pre, 1u);
                if (P.crec) P.crec[nb + pre] = make_uint2(0u, 0u);
            }
            continue;
        }
        const unsigned long long old = atomicAdd((unsigned long long *)(P.lvl + g * P.ls), (1ull << 32) | deg);
        const uint32_t pos = (uint32_t)(old >> 32);
        P.qv[nb + pos] = ri;
        P.parq[nb + pos] = ri;
        atomicOr(tb_bm(P, g, fr_k(0)) + (ri >> 5), 1u << (ri & 31));
        atomicOr(tb_bm(P, g, kTbVis) + (ri >> 5), 1u << (ri & 31));
    }
}

// ---------------------------------------------------------------------------
// the BFS of G trees: one cooperative kernel, per level
//   phase P (only if some tree pushes this level): the level-L list entries
//            of the pushing trees mark their unreached neighbours in mk(L);
//            grid barrier;
//   phase D  every tile not finished in all trees, every tree: unreached
//            (and, when pushing, marked) vertices look for neighbours on
//            level L, take the min-hash parent and append themselves to the
//            level-(L+1) list; grid barrier.
// ---------------------------------------------------------------------------
constexpr int kTbWarps = kBlock / 32;
constexpr int kTbHeavyQ = 32;     // heavy frontier entries queued per warp (phase P)

#define TB_PROF(slot)                                                          \
    do {                                                                       \
        if (P.prof && blockIdx.x == 0 && tid == 0 && L < 256)                  \
            P.prof[(size_t)L * 4 + (slot)] = tb_gtimer();                      \
    } while (0)

__device__ __forceinline__ void tb_mark(const TbParams &P, uint32_t who, int L, uint32_t x) {
    for (uint32_t m = who; m; m &= m - 1) {
        const int g = __ffs(m) - 1;
        const uint32_t w = x >> 5, b = 1u << (x & 31);
        if (__ldcg(tb_bm(P, g, kTbVis) + w) & b) continue;       // reached: nothing to discover
        uint32_t *mk = tb_bm(P, g, mk_k(L)) + w;
        if (!(__ldcg(mk) & b)) atomicOr(mk, b);
    }
}

__global__ void __launch_bounds__(kBlock, 4) k_tbfs(TbParams P) {
    cg::grid_group grid = cg::this_grid();
    __shared__ uint64_t s_tk[kTbMax];
    __shared__ uint32_t s_vbL[kTbMax];                // start of level L in tree g's list
    __shared__ uint32_t s_cnt[kTbMax];                // vertices on level L
    __shared__ uint32_t s_vb[kTbMax];                 // start of level L+1
    __shared__ unsigned long long s_vslots[kTbMax];   // slots of the vertices on levels <= L
    __shared__ int32_t s_depth[kTbMax];
    __shared__ uint32_t s_push;                       // bit g: tree g pushes this level
    __shared__ uint32_t s_live;                       // bit g: tree g has a non-empty level L
    __shared__ uint32_t s_hq[kTbWarps][kTbHeavyQ];    // phase P: heavy entries (internal id)
    const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
    const int G = P.G;
    const uint32_t gmask = G >= 32 ? ~0u : ((1u << G) - 1u);
    if (tid < kTbMax) {
        s_tk[tid] = tid < G ? P.tkey[tid] : 0;
        s_vbL[tid] = 0;
        s_vslots[tid] = 0;
        s_depth[tid] = 0;
    }
    const int64_t gtid = (int64_t)blockIdx.x * blockDim.x + tid;
    const int64_t nthr = (int64_t)gridDim.x * blockDim.x;
    const int64_t gwarp = gtid >> 5;
    const int64_t nwarps = nthr >> 5;
    const int64_t nit_tiles = (P.nitems + kTbWarps - 1) / kTbWarps;
    const int64_t l0 = P.nlight0 & ~31ll;             // light tiles start word-aligned
    const int64_t nl_tiles = (P.n - l0 + kBlock - 1) / kBlock;
    const int64_t ntiles = nit_tiles + nl_tiles;
    for (int L = 0;; L++) {
        __syncthreads();
        if (tid == 0) { s_push = 0; s_live = 0; }
        __syncthreads();
        if (tid < G) {
            const unsigned long long c = __ldcg((const unsigned long long *)(P.lvl + tid * P.ls + L));
            const uint32_t cnt = (uint32_t)(c >> 32), fsl = (uint32_t)c;
            s_cnt[tid] = cnt;
            s_vb[tid] = s_vbL[tid] + cnt;
            if (blockIdx.x == 0) P.vbase[tid * P.ls + L + 1] = s_vbL[tid] + cnt;
            s_vslots[tid] += fsl;
            const unsigned long long unv = P.slots - s_vslots[tid];
            if (cnt) {
                atomicOr(&s_live, 1u << tid);
                s_depth[tid] = L;
                if ((unsigned long long)fsl * (unsigned long long)P.push_k < unv) atomicOr(&s_push, 1u << tid);
            }
        }
        __syncthreads();
        const uint32_t live = s_live, push = s_push;
        if (!live) break;
        // every tree's level L + 2 counter starts at zero (L + 2 <= depth + 2 < ls)
        if (blockIdx.x == 0 && tid < G) P.lvl[tid * P.ls + L + 2] = 0;
        TB_PROF(0);
        // ---- phase P: push marks from the level-L lists ------------------
        if (push) {
            for (uint32_t m = push; m; m &= m - 1) {
                const int g = __ffs(m) - 1;
                const uint32_t cnt = s_cnt[g];
                const uint32_t *q = P.qv + (size_t)g * P.n + s_vbL[g];
                for (int64_t base = gwarp * 32; base < cnt; base += nwarps * 32) {
                    const int64_t j = base + lane;
                    uint32_t u = 0, rs = 0, re = 0;
                    bool heavy = false;
                    if (j < cnt) {
                        u = __ldg(P.brank + __ldcg(q + j));
                        rs = __ldg(P.brow + u);
                        re = __ldg(P.brow + u + 1);
                        heavy = re - rs > (uint32_t)kLight;
                        if (!heavy)
                            for (uint32_t s = rs; s < re; s++) tb_mark(P, 1u << g, L, __ldg(P.badj + s) & kIdMask);
                    }
                    const uint32_t hm = __ballot_sync(0xFFFFFFFFu, heavy);
                    if (heavy) {
                        const int at = __popc(hm & ((1u << lane) - 1u));
                        s_hq[wid][at] = u;
                    }
                    __syncwarp();
                    for (int h = 0; h < __popc(hm); h++) {
                        const uint32_t hu = s_hq[wid][h];
                        const uint32_t hs = __ldg(P.brow + hu), he = __ldg(P.brow + hu + 1);
                        for (uint32_t s = hs + lane; s < he; s += 32) tb_mark(P, 1u << g, L, __ldg(P.badj + s) & kIdMask);
                    }
                    __syncwarp();
                }
            }
            grid.sync();
        }
        TB_PROF(1);
        // ---- bookkeeping: fr(L-1) and mk(L+1) are free -> cleared ---------
        for (int g = 0; g < G; g++) {
            uint32_t *f1 = tb_bm(P, g, fr_k(L - 1));
            uint32_t *mk1 = tb_bm(P, g, mk_k(L + 1));
            for (int64_t w = gtid; w < P.nwords; w += nthr) {
                f1[w] = 0;
                mk1[w] = 0;
            }
        }
        // ---- phase D: discovery + parents ---------------------------------
        for (int64_t tile = blockIdx.x; tile < ntiles; tile += gridDim.x) {
            if (tile < nit_tiles) {
                const int64_t k = tile * kTbWarps + wid;
                if (k >= P.nitems) continue;
                const uint2 it = __ldg(P.items + k);
                const uint32_t i = it.x, s0 = it.y;
                const uint32_t ww = i >> 5, bb = 1u << (i & 31);
                if (__ldcg(P.fin + ww) & bb) continue;
                const bool multi = k < P.nmulti_items;
                // trees in which i is unreached (and marked when pushing)
                uint32_t want = 0, reached = 0;
                for (uint32_t m = live; m; m &= m - 1) {
                    const int g = __ffs(m) - 1;
                    bool ok;
                    if (multi) {
                        const uint32_t hl = __ldcg(P.hlev + (size_t)g * P.nmulti + i);
                        ok = hl == 0 || hl == (uint32_t)L + 2;
                    } else {
                        ok = !(__ldcg(tb_bm(P, g, kTbVis) + ww) & bb);
                    }
                    if (!ok) { reached |= 1u << g; continue; }
                    if ((push >> g) & 1u) ok = (__ldcg(tb_bm(P, g, mk_k(L)) + ww) & bb) != 0;
                    if (ok) want |= 1u << g;
                }
                if (want) {
                    const uint32_t rend = __ldg(P.brow + i + 1);
                    const uint32_t s1 = min(s0 + (uint32_t)kChunk, rend);
                    const uint32_t deg = rend - __ldg(P.brow + i);
                    const uint32_t ow = __ldg(P.bord + i);
                    uint32_t a[kChunk / 32];
#pragma unroll
                    for (int r = 0; r < kChunk / 32; r++) {
                        const uint32_t j = s0 + lane + 32 * r;
                        a[r] = j < s1 ? __ldg(P.badj + j) : kNone;
                    }
                    for (uint32_t m = want; m; m &= m - 1) {
                        const int g = __ffs(m) - 1;
                        const uint32_t *fr = tb_bm(P, g, fr_k(L));
                        unsigned long long key = ~0ull;
#pragma unroll
                        for (int r = 0; r < kChunk / 32; r++) {
                            if (a[r] != kNone && bit_of(fr, a[r] & kIdMask)) {
                                const uint32_t o = __ldg(P.borig + s0 + lane + 32 * r);
                                key = min(key, parent_key(s_tk[g], o, ow, a[r] >> 31));
                            }
                        }
                        key = tb_warp_min64(key);
                        if (key == ~0ull) continue;
                        reached |= 1u << g;
                        if (lane != 0) continue;
                        const size_t nb = (size_t)g * P.n;
                        unsigned long long *cnt = (unsigned long long *)(P.lvl + g * P.ls + L + 1);
                        if (!multi) {
                            atomicOr(tb_bm(P, g, kTbVis) + ww, bb);
                            atomicOr(tb_bm(P, g, fr_k(L + 1)) + ww, bb);
                            const uint32_t pos = s_vb[g] + (uint32_t)(atomicAdd(cnt, (1ull << 32) | deg) >> 32);
                            P.qv[nb + pos] = i;
                            P.parq[nb + pos] = tb_key_to_par(P.brank, key);
                        } else {
                            atomicMin(P.hbest + (size_t)g * P.nmulti + i, key);
                            if (atomicCAS(P.hlev + (size_t)g * P.nmulti + i, 0u, (uint32_t)L + 2) == 0u) {
                                atomicOr(tb_bm(P, g, kTbVis) + ww, bb);
                                atomicOr(tb_bm(P, g, fr_k(L + 1)) + ww, bb);
                                const uint32_t pos = s_vb[g] + (uint32_t)(atomicAdd(cnt, (1ull << 32) | deg) >> 32);
                                P.qv[nb + pos] = i;
                                P.hpos[(size_t)g * P.nmulti + i] = pos;
                            }
                        }
                    }
                }
                // finished trees (not live) have reached every vertex they will
                if (!multi && lane == 0 && ((reached | ~live) & gmask) == gmask) atomicOr(P.fin + ww, bb);
            } else {
                const int64_t v0 = l0 + (tile - nit_tiles) * kBlock + wid * 32;   // this warp's word
                if (v0 >= P.n) continue;
                const int64_t ww = v0 >> 5;
                const uint32_t i = (uint32_t)(v0 + lane);
                const uint32_t mine = __ballot_sync(0xFFFFFFFFu, (int64_t)i < P.n && (int64_t)i >= P.nlight0);
                const uint32_t fw = __ldcg(P.fin + ww);
                if (!(mine & ~fw)) continue;
                const bool owner = v0 >= P.nlight0;          // the boundary word is shared with items
                uint32_t deg = 0, a[kLight], ow = 0, rs = 0;
                bool loaded = false;
                uint32_t all = mine;                          // reached in every tree so far
                for (int g = 0; g < G; g++) {
                    uint32_t *vis = tb_bm(P, g, kTbVis);
                    const uint32_t vw = __ldcg(vis + ww);
                    if (!((live >> g) & 1u)) continue;        // finished tree: all reached
                    uint32_t unr = ~vw & mine;
                    if ((push >> g) & 1u) unr &= __ldcg(tb_bm(P, g, mk_k(L)) + ww);
                    uint32_t dm = 0;
                    if (unr) {
                        if (!loaded) {
                            loaded = true;
                            if ((mine >> lane) & 1u) {
                                rs = __ldg(P.brow + i);
                                deg = __ldg(P.brow + i + 1) - rs;
                                ow = __ldg(P.bord + i);
#pragma unroll
                                for (int r = 0; r < kLight; r++) a[r] = r < (int)deg ? __ldg(P.badj + rs + r) : 0u;
                            }
                        }
                        const uint32_t *fr = tb_bm(P, g, fr_k(L));
                        unsigned long long key = ~0ull;
                        if ((unr >> lane) & 1u) {
#pragma unroll
                            for (int r = 0; r < kLight; r++) {
                                if (r < (int)deg && bit_of(fr, a[r] & kIdMask)) {
                                    const uint32_t o = __ldg(P.borig + rs + r);
                                    key = min(key, parent_key(s_tk[g], o, ow, a[r] >> 31));
                                }
                            }
                        }
                        const bool disc = key != ~0ull;
                        dm = __ballot_sync(0xFFFFFFFFu, disc);
                        if (dm) {
                            const uint32_t dd = disc ? deg : 0u;
                            const uint32_t dsum = __shfl_sync(0xFFFFFFFFu, tb_incl_scan32(dd), 31);
                            const uint32_t before = __popc(dm & ((1u << lane) - 1u));
                            unsigned long long old = 0;
                            if (lane == 0) {
                                uint32_t *nx = tb_bm(P, g, fr_k(L + 1)) + ww;
                                if (owner) { vis[ww] = vw | dm; *nx = dm; }
                                else { atomicOr(vis + ww, dm); atomicOr(nx, dm); }
                                old = atomicAdd((unsigned long long *)(P.lvl + g * P.ls + L + 1),
                                                ((unsigned long long)__popc(dm) << 32) | dsum);
                            }
                            old = __shfl_sync(0xFFFFFFFFu, old, 0);
                            if (disc) {
                                const size_t nb = (size_t)g * P.n;
                                const uint32_t pos = s_vb[g] + (uint32_t)(old >> 32) + before;
                                P.qv[nb + pos] = i;
                                P.parq[nb + pos] = tb_key_to_par(P.brank, key);
                            }
                        }
                    }
                    all &= vw | dm;
                }
                if (lane == 0 && (all & ~fw)) {
                    if (owner) P.fin[ww] = fw | all;
                    else atomicOr(P.fin + ww, all);
                }
            }
        }
        TB_PROF(2);
        grid.sync();
        if (tid < G) s_vbL[tid] = s_vb[tid];
    }
    if (blockIdx.x == 0 && tid < G) {
        P.depth[tid] = s_depth[tid];
        atomicMax(P.maxd, s_depth[tid]);
    }
}

// hubs' list entries get their parents (the chunk minima are final after the
// BFS); the tables are reset for the next launch
__global__ void k_tb_fix_hubs(TbParams P) {
    const int64_t total = (int64_t)P.G * P.nmulti;
    for (int64_t x = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; x < total;
         x += (int64_t)gridDim.x * blockDim.x) {
        const int g = (int)(x / P.nmulti);
        const uint32_t pos = P.hpos[x];
        if (pos == kNone) continue;
        P.parq[(size_t)g * P.n + pos] = tb_key_to_par(P.brank, P.hbest[x]);
        P.hpos[x] = kNone;
        P.hbest[x] = ~0ull;
        P.hlev[x] = 0;
    }
}

// ---------------------------------------------------------------------------
// host side
// ---------------------------------------------------------------------------
int run_tbfs(const Graph &g, Workspace &ws, int B, const MsBfsOut &o, cudaStream_t st,
             int64_t *launches, int G, int push_k) {
    if (B < 1) { set_error("tbfs: empty batch"); return GB_EINVAL; }
    G = std::max(1, std::min(G, kTbMax));
    static int blocks = 0, blocks_dev = -1;
    if (blocks_dev != g.dev) {
        blocks_dev = g.dev;
        int per = 0;
        if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, k_tbfs, kBlock, 0) != cudaSuccess || per < 1)
            per = 1;
        blocks = per * g.num_sms;
    }
    const int64_t nwords = (g.n + 31) / 32;
    for (int b0 = 0; b0 < B; b0 += G) {
        TbParams P;
        P.brow = g.brow; P.badj = g.badj; P.borig = g.borig; P.bord = g.bord; P.brank = g.brank;
        P.items = g.items; P.coff = g.coff; P.cverts = g.cverts;
        P.n = g.n; P.ncomp = g.ncomp; P.nitems = g.nitems; P.nmulti_items = g.nmulti_items;
        P.nlight0 = g.nlight0; P.nmulti = g.nmulti; P.ls = g.n + 2;
        P.nwords = nwords;
        P.itemwords = (g.nlight0 + 31) / 32;
        P.slots = (unsigned long long)g.slots;
        P.G = std::min(G, B - b0);
        P.bm = ws.tbm; P.hbest = ws.tbhbest; P.hpos = ws.tbhpos; P.hlev = ws.tbhlev;
        P.fin = ws.tbm + (size_t)kTbMax * kTbBms * nwords;
        P.prof = ws.msprof;
        const size_t nb = (size_t)b0 * g.n, lb = (size_t)b0 * P.ls;
        P.tkey = o.tkey + b0;
        P.qv = o.qv + nb; P.parq = o.parq + nb; P.pp = o.pp + nb; P.rec = o.rec + nb;
        P.crec = o.crec ? o.crec + nb : nullptr;
        P.irec = o.irec ? o.irec + nb : nullptr;
        P.lvl = o.lvl + lb; P.vbase = o.vbase + lb;
        P.depth = o.depth + b0; P.maxd = o.maxd;
        P.push_k = push_k;
        GB_CUDA_TRY(cudaMemsetAsync(ws.tbm, 0, sizeof(uint32_t) * (size_t)P.G * kTbBms * nwords, st));
        GB_CUDA_TRY(cudaMemsetAsync(P.fin, 0, sizeof(uint32_t) * (size_t)nwords, st));
        const int64_t work = (int64_t)P.G * g.ncomp;
        k_tb_roots<<<(unsigned)std::max<int64_t>(1, std::min<int64_t>((work + 255) / 256, 8192)), 256, 0, st>>>(P);
        ++*launches;
        void *args[] = {&P};
        cudaError_t e = cudaLaunchCooperativeKernel((const void *)k_tbfs, dim3(blocks), dim3(kBlock), args, 0, st);
        if (e != cudaSuccess) {
            set_error(std::string("cooperative launch (tbfs): ") + cudaGetErrorString(e));
            return GB_ECUDA;
        }
        ++*launches;
        if (g.nmulti) {
            const int64_t hw = (int64_t)P.G * g.nmulti;
            k_tb_fix_hubs<<<(unsigned)std::max<int64_t>(1, std::min<int64_t>((hw + 255) / 256, 4096)), 256, 0, st>>>(P);
            ++*launches;
        }
    }
    GB_CUDA_TRY(cudaGetLastError());
    return GB_OK;
}

}  // namespace gb
