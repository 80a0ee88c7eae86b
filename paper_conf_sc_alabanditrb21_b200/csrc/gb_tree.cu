// gb_tree.cu -- §8 rows a.2-a.5 and a.9: per batch of B trees,
//   a.2 hashed roots + level-synchronous BFS distances,
//   a.3 min-hash parent selection (folded into the BFS expansion),
//   a.4 Alg. 4 bottom-up subtree sizes (L270-L278),
//   a.5 Alg. 4 top-down pre-order IDs and ranges (L279-L291) + root parity pi,
// all B trees advancing level by level inside persistent cooperative kernels
// (one grid-wide barrier per level for the whole batch, no host round trip).
//
// Frontier expansion is slot-balanced: every queued vertex carries the prefix
// of its level's degrees, so a warp takes 32 consecutive adjacency slots of
// the level at a time (whatever vertices they belong to) and finds each
// slot's owner with a 5-step shuffle search over 32 queue entries -- hubs
// (43k neighbours, Table 1) are spread over many warps and degree-1
// vertices do not waste lanes.
#include "gb_internal.cuh"
#include "../../include/graphb.h"

#include <algorithm>
#include <cstdio>
#include <cstdlib>

namespace gb {
namespace cg = cooperative_groups;

struct TreeParams {
    const uint32_t *row_ptr, *adj, *adj_eid;
    const uint2 *edges;
    const int32_t *comp, *coff, *cverts;
    int64_t n, ncomp;
    int32_t cbig;
    int B;
    int64_t ls;  // stride of lvl / vbase per tree (n + 2)
    int32_t *dist;
    uint64_t *pkey;
    unsigned long long *sz;  // packed (children so far << 32 | subtree size)
    uint32_t *qv, *qs;
    uint64_t *lvl;
    uint32_t *vbase, *pinfo, *peid, *off, *pp;
    uint2 *rec;
    uint32_t *s1;
    const uint64_t *tkey;
    int32_t *depth, *maxd;
    const int32_t *given;  // caller tree (parent ids, -1 at roots) or null
    uint32_t *cidx;        // descent variant: sibling index of each child (or null)
    uint32_t *cstart;      // descent variant: child-list start per vertex
    uint32_t *clist;       // descent variant: children pre IDs, per parent ascending
    uint2 *crec;           // descent variant: pre-indexed {cstart, #children}
    unsigned long long *visited;  // [B] vertices reached (given-tree validation)
    unsigned long long *dbg;      // debug counters (GB_CHECK) or null
};

__device__ __forceinline__ uint32_t lanemask_lt() {
    uint32_t m;
    asm("mov.u32 %0, %%lanemask_lt;" : "=r"(m));
    return m;
}

__device__ __forceinline__ uint32_t warp_incl_scan32(uint32_t v) {
    const int lane = threadIdx.x & 31;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
        uint32_t y = __shfl_up_sync(0xFFFFFFFFu, v, d);
        if (lane >= d) v += y;
    }
    return v;
}

// ---------------------------------------------------------------------------
// batch reset + roots (a.2)
// ---------------------------------------------------------------------------
__global__ void k_batch_prep(TreeParams P) {
    int b = blockIdx.x * blockDim.x + threadIdx.x;
    if (b < P.B) {
        P.lvl[b * P.ls + 0] = 0;
        P.lvl[b * P.ls + 1] = 0;
        P.vbase[b * P.ls + 0] = 0;
        P.depth[b] = 0;
        if (P.visited) P.visited[b] = 0;
    }
    if (b == 0) *P.maxd = 0;
}

// root of component C in tree b: cverts_C[rkey mod |C|] (reading R4)
__device__ __forceinline__ void place_root(const TreeParams &P, int b, int64_t C, uint32_t r) {
    const size_t nb = (size_t)b * P.n;
    P.dist[nb + r] = 0;
    P.sz[nb + r] = 1;
    P.pinfo[nb + r] = kNone;
    P.peid[nb + r] = kNone;
    P.off[nb + r] = 0;
    uint32_t deg = P.row_ptr[r + 1] - P.row_ptr[r];
    uint32_t pre = (uint32_t)P.coff[C];
    if (deg == 0) {
        // isolated vertex: a one-vertex tree, finished here (pi = 0)
        P.pp[nb + r] = pre;
        P.rec[nb + pre] = make_uint2(pre, 1u);
        if (P.visited) atomicAdd(P.visited + b, 1ull);
        return;
    }
    unsigned long long old = atomicAdd((unsigned long long *)(P.lvl + b * P.ls), (1ull << 32) | deg);
    uint32_t pos = (uint32_t)(old >> 32);
    P.qv[nb + pos] = r;
    P.qs[nb + pos] = (uint32_t)old;
}

__global__ void k_roots(TreeParams P) {
    int64_t total = (int64_t)P.B * P.ncomp;
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < total;
         i += (int64_t)gridDim.x * blockDim.x) {
        int b = (int)(i / P.ncomp);
        int64_t C = i - (int64_t)b * P.ncomp;
        uint32_t sz = (uint32_t)(P.coff[C + 1] - P.coff[C]);
        uint64_t rk = root_key(P.tkey[b], C);
        uint32_t r = (uint32_t)P.cverts[P.coff[C] + (int64_t)(rk % sz)];
        place_root(P, b, C, r);
    }
}

// caller-given tree: its roots (parent == -1); one tree (b = 0)
__global__ void k_roots_given(TreeParams P) {
    for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < P.n;
         v += (int64_t)gridDim.x * blockDim.x)
        if (P.given[v] == -1) place_root(P, 0, P.comp[v], (uint32_t)v);
}

// ---------------------------------------------------------------------------
// a.2 + a.3: level-synchronous BFS of all B trees
// ---------------------------------------------------------------------------
struct LevelTable {
    uint32_t vb[kMaxBatch];
    uint32_t nv[kMaxBatch];
    unsigned long long soff[kMaxBatch + 1];
};

// expand the slots [s0, s1) of level L of tree b (one warp)
__device__ __forceinline__ void expand_range(const TreeParams &P, int b, int L, uint32_t s0,
                                             uint32_t s1, uint32_t vb, uint32_t nv, uint64_t tk) {
    const int lane = threadIdx.x & 31;
    const size_t nb = (size_t)b * P.n;
    const uint32_t *qs = P.qs + nb + vb;
    const uint32_t *qv = P.qv + nb + vb;
    // owner of slot s0: the largest q with qs[q] <= s0
    uint32_t q = 0;
    if (lane == 0) {
        uint32_t lo = 0, hi = nv;
        while (hi - lo > 1) {
            uint32_t mid = lo + ((hi - lo) >> 1);
            if (__ldcg(qs + mid) <= s0) lo = mid; else hi = mid;
        }
        q = lo;
    }
    q = __shfl_sync(0xFFFFFFFFu, q, 0);
    const uint32_t lmask = lanemask_lt();
    unsigned long long *lvl_next = (unsigned long long *)(P.lvl + b * P.ls + L + 1);
    for (uint32_t s = s0; s < s1; s += 32) {
        const uint32_t qi = q + lane;
        const bool qok = qi < nv;
        const uint32_t myqs = qok ? __ldcg(qs + qi) : 0xFFFFFFFFu;
        const uint32_t myw = qok ? __ldcg(qv + qi) : 0u;
        const uint32_t myrp = qok ? __ldg(P.row_ptr + myw) : 0u;
        const uint32_t sl = s + lane;
        int idx = 0;
#pragma unroll
        for (int st = 16; st; st >>= 1) {
            uint32_t v = __shfl_sync(0xFFFFFFFFu, myqs, idx + st);
            if (v <= sl) idx += st;
        }
        const uint32_t w = __shfl_sync(0xFFFFFFFFu, myw, idx);
        const uint32_t j = __shfl_sync(0xFFFFFFFFu, myrp, idx) + (sl - __shfl_sync(0xFFFFFFFFu, myqs, idx));
        const bool act = sl < s1;
        bool disc = false;
        uint32_t x = 0, deg = 0;
        if (act && P.dbg) {
            if (j < __ldg(P.row_ptr + w) || j >= __ldg(P.row_ptr + w + 1)) {
                unsigned long long k = atomicAdd(P.dbg + 2, 1ull);
                if (k < 4) {
                    unsigned long long *r = P.dbg + 8 + 8 * k;
                    r[0] = b; r[1] = L; r[2] = s; r[3] = q; r[4] = idx; r[5] = sl;
                    r[6] = nv; r[7] = s0 | ((unsigned long long)s1 << 32);
                }
            }
            if (__ldcg(P.dist + nb + w) != L) atomicAdd(P.dbg + 3, 1ull);
        }
        if (act) {
            x = __ldg(P.adj + j) & kIdMask;
            int32_t *dp = P.dist + nb + x;
            if (P.given) {
                // caller tree: follow tree edges only (parent(x) == w)
                if (P.given[x] == (int32_t)w) {
                    disc = true;
                    *dp = L + 1;
                    P.peid[nb + x] = __ldg(P.adj_eid + j);
                }
            } else {
                int32_t dx = __ldcg(dp);
                if (dx == kInf) {
                    int32_t old = atomicCAS(dp, kInf, L + 1);
                    if (old == kInf) disc = true; else dx = old;
                }
                // a neighbour one level up is a parent candidate of w (a.3)
                if (!disc && dx == L - 1) {
                    uint32_t e = __ldg(P.adj_eid + j);
                    atomicMin((unsigned long long *)(P.pkey + nb + w), edge_key(tk, e));
                }
            }
            if (disc) deg = __ldg(P.row_ptr + x + 1) - __ldg(P.row_ptr + x);
        }
        const uint32_t dm = __ballot_sync(0xFFFFFFFFu, disc);
        if (dm) {
            const uint32_t incl = warp_incl_scan32(deg);
            const uint32_t total = __shfl_sync(0xFFFFFFFFu, incl, 31);
            const int leader = __ffs(dm) - 1;
            unsigned long long old = 0;
            if (lane == leader)
                old = atomicAdd(lvl_next, ((unsigned long long)__popc(dm) << 32) | total);
            old = __shfl_sync(0xFFFFFFFFu, old, leader);
            if (disc) {
                uint32_t pos = vb + nv + (uint32_t)(old >> 32) + __popc(dm & lmask);
                P.qv[nb + pos] = x;
                P.qs[nb + pos] = (uint32_t)old + (incl - deg);
                if (!P.given) P.pkey[nb + x] = ~0ull;
                P.sz[nb + x] = 1;
            }
        }
        // next window starts at slot s+32: its owner is the last loaded entry
        // with qs <= s+32, or the entry right after the window
        const uint32_t nxt = s + 32;
        const uint32_t cnt = __popc(__ballot_sync(0xFFFFFFFFu, myqs <= nxt));
        uint32_t nq = q + cnt - 1;
        if (cnt == 32 && nxt < s1 && q + 32 < nv && __ldcg(qs + q + 32) <= nxt) nq = q + 32;
        q = nq;
    }
}

__global__ void __launch_bounds__(kBlock) k_bfs(TreeParams P) {
    cg::grid_group grid = cg::this_grid();
    __shared__ LevelTable T;
    __shared__ uint64_t s_tkey[kMaxBatch];
    __shared__ int32_t s_depth[kMaxBatch];
    __shared__ int s_more;
    const int B = P.B;
    const int64_t gwarp = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
    if (threadIdx.x < B) {
        T.vb[threadIdx.x] = 0;
        s_tkey[threadIdx.x] = P.tkey[threadIdx.x];
        s_depth[threadIdx.x] = 0;
    }
    for (int L = 0;; L++) {
        __syncthreads();
        if (threadIdx.x < B) {
            unsigned long long c = __ldcg((const unsigned long long *)(P.lvl + threadIdx.x * P.ls + L));
            T.nv[threadIdx.x] = (uint32_t)(c >> 32);
            T.soff[threadIdx.x + 1] = (uint32_t)c;
        }
        __syncthreads();
        if (threadIdx.x == 0) {
            T.soff[0] = 0;
            for (int b = 0; b < B; b++) T.soff[b + 1] += T.soff[b];
        }
        if (blockIdx.x == 0 && threadIdx.x < B) {
            P.lvl[threadIdx.x * P.ls + L + 2] = 0;
            P.vbase[threadIdx.x * P.ls + L + 1] = T.vb[threadIdx.x] + T.nv[threadIdx.x];
        }
        __syncthreads();
        const unsigned long long W = T.soff[B];
        const unsigned long long chunk = ((W + nwarps - 1) / nwarps + 31) & ~31ull;
        const unsigned long long g0 = (unsigned long long)gwarp * chunk;
        const unsigned long long g1 = min(W, g0 + chunk);
        for (int b = 0; b < B && g0 < g1; b++) {
            const unsigned long long t0 = T.soff[b], t1 = T.soff[b + 1];
            if (t1 <= g0 || t0 >= g1) continue;
            expand_range(P, b, L, (uint32_t)(max(g0, t0) - t0), (uint32_t)(min(g1, t1) - t0),
                         T.vb[b], T.nv[b], s_tkey[b]);
        }
        grid.sync();
        if (threadIdx.x == 0) s_more = 0;
        __syncthreads();
        if (threadIdx.x < B) {
            unsigned long long c = __ldcg((const unsigned long long *)(P.lvl + threadIdx.x * P.ls + L + 1));
            T.vb[threadIdx.x] += T.nv[threadIdx.x];
            if (c >> 32) {
                s_depth[threadIdx.x] = L + 1;
                atomicOr(&s_more, 1);
            }
        }
        __syncthreads();
        if (!s_more) break;
    }
    if (blockIdx.x == 0 && threadIdx.x < B) {
        P.depth[threadIdx.x] = s_depth[threadIdx.x];
        atomicMax(P.maxd, s_depth[threadIdx.x]);
        if (P.visited) atomicAdd(P.visited + threadIdx.x, (unsigned long long)T.vb[threadIdx.x]);
    }
}

// ---------------------------------------------------------------------------
// per-level item tables shared by the bottom-up and top-down passes
// ---------------------------------------------------------------------------
__device__ __forceinline__ void load_level(const TreeParams &P, int L, LevelTable &T,
                                           const int32_t *s_depth) {
    if (threadIdx.x < P.B) {
        int b = threadIdx.x;
        uint32_t nv = 0;
        if (L <= s_depth[b]) nv = (uint32_t)(__ldcg((const unsigned long long *)(P.lvl + b * P.ls + L)) >> 32);
        T.nv[b] = nv;
        T.vb[b] = __ldcg(P.vbase + b * P.ls + L);
        T.soff[b + 1] = nv;
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        T.soff[0] = 0;
        for (int b = 0; b < P.B; b++) T.soff[b + 1] += T.soff[b];
    }
    __syncthreads();
}

__device__ __forceinline__ int tree_of(const LevelTable &T, int B, unsigned long long i) {
    int lo = 0, hi = B;  // soff[lo] <= i < soff[hi]
    while (hi - lo > 1) {
        int mid = (lo + hi) >> 1;
        if (T.soff[mid] <= i) lo = mid; else hi = mid;
    }
    return lo;
}

// Warp-aggregated 64-bit atomicAdd of v into *addr; returns the value each
// lane would have seen with its own atomicAdd in some serial order.  Lanes
// adding to the same address in one contiguous run of lanes share one atomic
// (the children of a hub arrive in runs); everything else adds on its own.
__device__ __forceinline__ unsigned long long aggregated_add(unsigned long long *addr,
                                                             unsigned long long v, bool valid) {
    const int lane = threadIdx.x & 31;
    const unsigned long long k = valid ? (unsigned long long)addr : ~(unsigned long long)lane;
    const uint32_t peers = __match_any_sync(0xFFFFFFFFu, k);
    const int leader = __ffs(peers) - 1;
    const uint32_t run = peers >> leader;
    const bool contiguous = (run & (run + 1)) == 0;
    unsigned long long res = 0;
    if (__all_sync(0xFFFFFFFFu, contiguous)) {
        unsigned long long incl = v;
#pragma unroll
        for (int d = 1; d < 32; d <<= 1) {
            unsigned long long y = __shfl_up_sync(0xFFFFFFFFu, incl, d);
            if (lane - d >= leader) incl += y;
        }
        const int tail = 31 - __clz(peers);
        unsigned long long old = 0;
        if (lane == tail && valid) old = atomicAdd(addr, incl);
        old = __shfl_sync(0xFFFFFFFFu, old, tail);
        res = old + incl - v;
    } else if (valid) {
        res = atomicAdd(addr, v);
    }
    return res;
}

// ---------------------------------------------------------------------------
// a.4: Alg. 4 bottom-up pass (L273-L278).  Levels D..1; every vertex decodes
// its parent from the minimum edge key, then adds its final subtree size to
// its parent's count with an atomic add (L256).  The value returned by that
// add is 1 + the sizes of the siblings added before it: exactly the offset of
// this child's range inside its parent's (Alg. 4 L282-L288 with "earlier
// children" = earlier atomic adds, reading R5).
// ---------------------------------------------------------------------------
__global__ void __launch_bounds__(kBlock) k_bottom_up(TreeParams P) {
    cg::grid_group grid = cg::this_grid();
    __shared__ LevelTable T;
    __shared__ uint64_t s_tkey[kMaxBatch];
    __shared__ int32_t s_depth[kMaxBatch];
    const int B = P.B;
    if (threadIdx.x < B) {
        s_tkey[threadIdx.x] = P.tkey[threadIdx.x];
        s_depth[threadIdx.x] = __ldcg(P.depth + threadIdx.x);
    }
    __syncthreads();
    const int maxd = __ldcg(P.maxd);
    const int lane = threadIdx.x & 31;
    const int64_t gwarp = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int L = maxd; L >= 1; L--) {
        load_level(P, L, T, s_depth);
        const unsigned long long total = T.soff[B];
        for (unsigned long long wb = (unsigned long long)gwarp * 32; wb < total;
             wb += (unsigned long long)nwarps * 32) {
            const unsigned long long i = wb + lane;
            const bool valid = i < total;
            int b = 0;
            uint32_t w = 0, p = 0, sz = 0;
            size_t nb = 0;
            if (valid) {
                b = tree_of(T, B, i);
                nb = (size_t)b * P.n;
                w = __ldcg(P.qv + nb + T.vb[b] + (uint32_t)(i - T.soff[b]));
                uint32_t e = P.given ? __ldcg(P.peid + nb + w)
                                     : edge_of_key(s_tkey[b], __ldcg((const unsigned long long *)(P.pkey + nb + w)));
                uint2 ed = __ldg(P.edges + e);
                const uint32_t v2 = ed.y & kIdMask;
                p = (ed.x == w) ? v2 : ed.x;
                P.pinfo[nb + w] = p | (ed.y & kNegBit);
                P.peid[nb + w] = e;
                sz = (uint32_t)__ldcg(P.sz + nb + w);
            }
            // one add counts the child and its size: the old value is
            // (sibling index, 1 + sizes of the earlier siblings)
            const unsigned long long o =
                aggregated_add(P.sz + nb + p, (1ull << 32) | sz, valid);
            if (valid) {
                P.off[nb + w] = (uint32_t)o;
                if (P.cidx) P.cidx[nb + w] = (uint32_t)(o >> 32);
            }
        }
        grid.sync();
    }
}

// ---------------------------------------------------------------------------
// a.5: Alg. 4 top-down pass (L279-L291): levels 0..D; pre(child) =
// pre(parent) + offset; the range of tree edge p->c is [pre c, pre c +
// size c - 1] (L285-L286); root parity pi(c) = pi(p) XOR neg(p,c) gives the
// Harary side (reading R7).  Writes the pre-indexed record
// rec[pre] = {pre(parent) | neg<<31, size} used by the cycle walk.
// ---------------------------------------------------------------------------
__global__ void __launch_bounds__(kBlock) k_top_down(TreeParams P) {
    cg::grid_group grid = cg::this_grid();
    __shared__ LevelTable T;
    __shared__ int32_t s_depth[kMaxBatch];
    __shared__ uint32_t s_big[kMaxBatch];
    const int B = P.B;
    if (threadIdx.x < B) {
        s_depth[threadIdx.x] = __ldcg(P.depth + threadIdx.x);
        s_big[threadIdx.x] = 0;
    }
    __syncthreads();
    const int maxd = __ldcg(P.maxd);
    const int64_t gtid = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    const int64_t nthr = (int64_t)gridDim.x * blockDim.x;
    for (int L = 0; L <= maxd; L++) {
        load_level(P, L, T, s_depth);
        const unsigned long long total = T.soff[B];
        for (unsigned long long i = gtid; i < total; i += nthr) {
            const int b = tree_of(T, B, i);
            const size_t nb = (size_t)b * P.n;
            const uint32_t x = __ldcg(P.qv + nb + T.vb[b] + (uint32_t)(i - T.soff[b]));
            const int32_t C = __ldg(P.comp + x);
            uint32_t pre, up, neg, pi;
            if (L == 0) {
                pre = (uint32_t)__ldg(P.coff + C);
                up = pre;
                neg = 0;
                pi = 0;
            } else {
                const uint32_t pin = __ldcg(P.pinfo + nb + x);
                const uint32_t ppp = __ldcg(P.pp + nb + (pin & kIdMask));
                up = ppp & kIdMask;
                pre = up + __ldcg(P.off + nb + x);
                neg = pin & kNegBit;
                pi = (ppp & kNegBit) ^ neg;
            }
            P.pp[nb + x] = pre | pi;
            const unsigned long long szx = __ldcg(P.sz + nb + x);
            P.rec[nb + pre] = make_uint2(up | neg, (uint32_t)szx);
            if (P.clist) {
                // Alg. 3 descent structures: the child list of x (by pre) and
                // this vertex's slot in its parent's list
                P.crec[nb + pre] = make_uint2(__ldcg(P.cstart + nb + x), (uint32_t)(szx >> 32));
                if (L > 0) {
                    const uint32_t p = __ldcg(P.pinfo + nb + x) & kIdMask;
                    P.clist[__ldcg(P.cstart + nb + p) + __ldcg(P.cidx + nb + x)] = pre;
                }
            }
            if (pi) {
                if (C == P.cbig) atomicAdd(&s_big[b], 1u);
                else atomicAdd(P.s1 + (size_t)b * P.ncomp + C, 1u);
            }
        }
        grid.sync();
    }
    __syncthreads();
    if (threadIdx.x < B && s_big[threadIdx.x])
        atomicAdd(P.s1 + (size_t)threadIdx.x * P.ncomp + P.cbig, s_big[threadIdx.x]);
}

// child count of every vertex (high half of the packed size counter), to be
// scanned in place into child-list starts (descent variant only)
__global__ void k_child_counts(TreeParams P, int64_t cnt) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < cnt;
         i += (int64_t)gridDim.x * blockDim.x)
        P.cstart[i] = (uint32_t)(P.sz[i] >> 32);
}

// debug check (GB_CHECK=1): after the BFS every vertex is reached, every
// non-root has a parent key, and the level lists hold every vertex once
__global__ void k_check_bfs(TreeParams P, unsigned long long *out) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < (int64_t)P.B * P.n;
         i += (int64_t)gridDim.x * blockDim.x) {
        int32_t d = P.dist[i];
        if (d == kInf) {
            unsigned long long k = atomicAdd(out + 0, 1ull);
            if (k < 4) {
                const int64_t bb = i / P.n, vv = i - bb * P.n;
                unsigned long long *r = out + 24 + 4 * k;
                r[0] = vv; r[1] = P.row_ptr[vv + 1] - P.row_ptr[vv];
                int32_t C = P.comp[vv];
                r[2] = (unsigned long long)(P.coff[C + 1] - P.coff[C]);
                r[3] = P.row_ptr[vv + 1] > P.row_ptr[vv] ? (unsigned long long)(uint32_t)P.dist[bb * P.n + (P.adj[P.row_ptr[vv]] & kIdMask)] : 999;
            }
        }
        else if (d > 0 && P.pkey[i] == ~0ull) atomicAdd(out + 1, 1ull);
        // BFS distances: neighbours differ by <= 1, non-roots have one at d-1
        const int64_t b = i / P.n, v = i - b * P.n;
        bool has_up = d == 0;
        for (uint32_t j = P.row_ptr[v]; j < P.row_ptr[v + 1]; j++) {
            int32_t dx = P.dist[b * P.n + (P.adj[j] & kIdMask)];
            if (dx - d > 1 || d - dx > 1) atomicAdd(out + 4, 1ull);
            if (dx == d - 1) has_up = true;
        }
        if (!has_up) atomicAdd(out + 5, 1ull);
        // queue consistency: qs[i+1] - qs[i] == deg(qv[i]) within each level
        const int32_t D = P.depth[b];
        if (v == 0) {
            for (int L = 0; L <= D; L++) {
                uint32_t vb = P.vbase[b * P.ls + L];
                unsigned long long c = P.lvl[b * P.ls + L];
                uint32_t nv = (uint32_t)(c >> 32), ns = (uint32_t)c;
                uint32_t acc = 0;
                for (uint32_t q = 0; q < nv; q++) {
                    uint32_t w = P.qv[b * P.n + vb + q];
                    if (P.qs[b * P.n + vb + q] != acc) { atomicAdd(out + 6, 1ull); break; }
                    acc += P.row_ptr[w + 1] - P.row_ptr[w];
                }
                if (acc != ns) atomicAdd(out + 7, 1ull);
            }
        }
    }
}

// ---------------------------------------------------------------------------
// host side
// ---------------------------------------------------------------------------
static int coop_blocks(const void *fn, int sms) {
    int per = 0;
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, fn, kBlock, 0) != cudaSuccess || per < 1)
        per = 1;
    return per * sms;
}

static int launch_coop(const void *fn, int blocks, TreeParams &P, cudaStream_t st) {
    void *args[] = {&P};
    cudaError_t e = cudaLaunchCooperativeKernel(fn, dim3(blocks), dim3(kBlock), args, 0, st);
    if (e != cudaSuccess) {
        set_error(std::string("cooperative launch: ") + cudaGetErrorString(e));
        return GB_ECUDA;
    }
    return GB_OK;
}

int run_batch_tree(const Graph &g, Workspace &ws, int B, const uint64_t * /*unused*/,
                   const int32_t *given_parent, cudaStream_t st, int64_t *launches,
                   cudaEvent_t *ev, bool walk_descent) {
    static int bfs_blocks = 0, up_blocks = 0, down_blocks = 0;
    if (!bfs_blocks) {
        bfs_blocks = coop_blocks((const void *)k_bfs, g.num_sms);
        up_blocks = coop_blocks((const void *)k_bottom_up, g.num_sms);
        down_blocks = coop_blocks((const void *)k_top_down, g.num_sms);
    }
    TreeParams P;
    P.row_ptr = g.row_ptr; P.adj = g.adj; P.adj_eid = g.adj_eid; P.edges = g.edges;
    P.comp = g.comp; P.coff = g.coff; P.cverts = g.cverts;
    P.n = g.n; P.ncomp = g.ncomp; P.cbig = g.cbig;
    P.B = B; P.ls = g.n + 2;
    P.dist = ws.dist; P.pkey = ws.pkey; P.sz = ws.sz; P.qv = ws.qv; P.qs = ws.qs;
    P.lvl = ws.lvl; P.vbase = ws.vbase; P.pinfo = ws.pinfo; P.peid = ws.peid; P.off = ws.off;
    P.pp = ws.pp; P.rec = ws.rec; P.s1 = ws.s1; P.tkey = ws.tkey; P.depth = ws.depth;
    P.maxd = ws.maxd; P.given = given_parent;
    P.cidx = walk_descent ? ws.cidx : nullptr;
    P.cstart = walk_descent ? ws.cstart : nullptr;
    P.clist = walk_descent ? ws.clist : nullptr;
    P.crec = walk_descent ? ws.crec : nullptr;
    P.visited = given_parent ? (unsigned long long *)ws.tstat : nullptr;
    P.dbg = nullptr;
    static unsigned long long *s_dbg = nullptr;
    if (getenv("GB_CHECK")) {
        if (!s_dbg) cudaMalloc(&s_dbg, 320);
        cudaMemsetAsync(s_dbg, 0, 320, st);
        P.dbg = s_dbg;
    }

    if (ev) GB_CUDA_TRY(cudaEventRecord(ev[0], st));
    GB_CUDA_TRY(cudaMemsetAsync(ws.dist, 0x7F, sizeof(int32_t) * (size_t)B * g.n, st));
    GB_CUDA_TRY(cudaMemsetAsync(ws.s1, 0, sizeof(uint32_t) * (size_t)B * g.ncomp, st));
    k_batch_prep<<<1, kMaxBatch, 0, st>>>(P);
    ++*launches;
    if (given_parent) {
        k_roots_given<<<(unsigned)std::min<int64_t>((g.n + 255) / 256, 4096), 256, 0, st>>>(P);
    } else {
        int64_t work = (int64_t)B * g.ncomp;
        k_roots<<<(unsigned)std::min<int64_t>((work + 255) / 256, 4096), 256, 0, st>>>(P);
    }
    ++*launches;
    GB_CUDA_TRY(cudaGetLastError());
    if (ev) GB_CUDA_TRY(cudaEventRecord(ev[1], st));
    int rc = launch_coop((const void *)k_bfs, bfs_blocks, P, st);
    if (rc) return rc;
    ++*launches;
    if (ev) GB_CUDA_TRY(cudaEventRecord(ev[2], st));
    if (getenv("GB_CHECK") && !given_parent) {
        unsigned long long *d_out = nullptr, h_out[40] = {0};
        cudaMalloc(&d_out, 320);
        cudaMemcpyAsync(d_out, P.dbg, 320, cudaMemcpyDeviceToDevice, st);
        k_check_bfs<<<1024, 256, 0, st>>>(P, d_out);
        cudaMemcpyAsync(h_out, d_out, 320, cudaMemcpyDeviceToHost, st);
        cudaStreamSynchronize(st);
        cudaFree(d_out);
        int32_t hd[kMaxBatch];
        cudaMemcpy(hd, ws.depth, 4 * B, cudaMemcpyDeviceToHost);
        fprintf(stderr, "[GB_CHECK] B=%d unreached=%llu nokey=%llu badslot=%llu badlevel=%llu "
                "distjump=%llu noup=%llu qsbad=%llu nsbad=%llu depth0=%d blocks=%d err=%s\n", B,
                h_out[0], h_out[1], h_out[2], h_out[3], h_out[4], h_out[5], h_out[6], h_out[7],
                hd[0], bfs_blocks, cudaGetErrorString(cudaGetLastError()));
        for (int k = 0; k < 4 && k < (int)h_out[0]; k++) {
            unsigned long long *r = h_out + 24 + 4 * k;
            fprintf(stderr, "   unreached v=%llu deg=%llu compsize=%llu dist(nbr0)=%lld\n", r[0], r[1], r[2], (long long)(int)r[3]);
        }
        for (int k = 0; k < 4 && k < (int)h_out[2]; k++) {
            unsigned long long *r = h_out + 8 + 8 * k;
            fprintf(stderr, "   bad: b=%llu L=%llu s=%llu q=%llu idx=%llu sl=%llu nv=%llu s0=%llu s1=%llu\n",
                    r[0], r[1], r[2], r[3], r[4], r[5], r[6], r[7] & 0xffffffffull, r[7] >> 32);
        }
    }
    rc = launch_coop((const void *)k_bottom_up, up_blocks, P, st);
    if (rc) return rc;
    ++*launches;
    if (getenv("GB_CHECK")) {
        cudaError_t e = cudaStreamSynchronize(st);
        fprintf(stderr, "[GB_CHECK] bottom_up done: %s\n", cudaGetErrorString(e));
    }
    if (walk_descent) {
        const int64_t cnt = (int64_t)B * g.n;
        k_child_counts<<<(unsigned)std::min<int64_t>((cnt + 255) / 256, 8192), 256, 0, st>>>(P, cnt);
        ++*launches;
        rc = exclusive_scan_u32(ws.cstart, ws.cstart, cnt, ws.scan_tmp, ws.scan_tmp_elems, st, launches);
        if (rc) return rc;
    }
    if (ev) GB_CUDA_TRY(cudaEventRecord(ev[3], st));
    rc = launch_coop((const void *)k_top_down, down_blocks, P, st);
    if (rc) return rc;
    ++*launches;
    if (getenv("GB_CHECK")) {
        cudaError_t e = cudaStreamSynchronize(st);
        fprintf(stderr, "[GB_CHECK] top_down done: %s\n", cudaGetErrorString(e));
    }
    return GB_OK;
}

}  // namespace gb
