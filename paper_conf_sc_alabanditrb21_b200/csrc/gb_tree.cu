// gb_tree.cu -- §8 rows a.2-a.5 and a.9: per batch of B trees,
//   a.2 hashed roots + level-synchronous BFS,
//   a.3 min-hash parent selection (folded into the BFS expansion),
//   a.4 Alg. 4 bottom-up subtree sizes (L270-L278),
//   a.5 Alg. 4 top-down pre-order IDs and ranges (L279-L291) + root parity pi,
// all B trees advancing level by level inside persistent cooperative kernels
// (one grid-wide barrier per level for the whole batch, no host round trip).
//
// Memory layout: the BFS state of a tree is one
// byte per vertex (10 MB for a 10M-vertex tree, L2-resident): 0 = unvisited,
// 0x81 + (level mod 127) = visited at a recent level, 0x80 = visited at least
// 127 levels ago.  One load answers both per-slot questions (unvisited?  one
// level up?); discovery is one atomicOr.  Everything that is
// produced and consumed in BFS order lives in *queue order* (the level lists
// qv): the parent key, the parent, the sibling offset and the subtree size,
// so the level passes stream them coalesced.  Only three arrays are indexed
// by vertex and touched at random: the subtree-size counters (bottom-up),
// the pre/pi labels (top-down, cycle walk) and the pre-indexed records.
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
    const uint32_t *row_ptr, *adj;             // original CSR (push BFS of caller trees)
    const uint32_t *brank, *bord;              // original <-> internal ids
    const uint32_t *brow;                      // degree-sorted view rows (isolated vertices)
    const int32_t *comp, *comp_i, *coff, *cverts;
    int64_t n, ncomp, nw;  // nw = state words per tree ((n + 3) / 4)
    int32_t cbig;
    int B;
    int64_t ls;  // stride of lvl / vbase per tree (n + 2)
    uint32_t *vst;  // [B][nw] byte states, 4 vertices per word
    uint32_t *qv, *qs, *qr;  // qr: row start of each queued vertex
    unsigned long long *pkeyq;
    uint64_t *lvl;
    uint32_t *vbase;
    uint32_t *size;             // subtree-size counters (walk 0), slot szi(i) of vertex i,
                                // tree stride szn (see szi)
    unsigned long long *sz64;   // vertex-indexed (children << 32 | size) (walk 1)
    uint32_t *parq, *offq, *szq, *cidxq;
    uint32_t *pp;
    uint2 *rec;
    uint4 *irec;                 // layout 0: {parent | neg, pre | pi, size, 0} by internal id
    uint32_t *prec;              // layout 2: up pre | neg by pre (pp holds pre | pi by internal id)
    uint32_t *s1;
    const uint64_t *tkey;
    int32_t *depth, *maxd;
    const int32_t *given;        // caller tree (parent ids, -1 at roots) or null
    uint32_t *cstart, *clist;    // walk 1
    uint2 *crec;                 // walk 1
    unsigned long long *visited; // [B] vertices reached (given-tree validation)
    unsigned long long *prof;    // option "msprof": [256][4] level timestamps (gb_label_profile)
    uint32_t szmask;             // (power of two >= n) - 1
    int64_t szn;                 // size counters per tree (n)
    int recpass;                 // walk 0: top-down leaves {up | neg, size} and pre in queue
                                 // order; k_rec_scatter writes rec[pre] afterwards
};

// Slot of vertex i's subtree-size counter: a multiplicative scramble of the
// id, y = i * 0x9E3779B1 mod 2^k (2^k >= n; an odd multiplier permutes
// [0, 2^k)), repeated while y >= n (cycle walking: a permutation of [0, n),
// under 2 steps on average).  Internal ids put the hubs -- the parents of
// most vertices -- next to each other, and the atomics of the bottom-up pass
// then queue on a few hot L2 sectors; scrambled, a hot counter's sector mates
// are unrelated (mostly cold) vertices (C3: bottom-up 42 -> 30 ms per 100
// trees; bit reversal over 2^k slots measured the same).
__device__ __forceinline__ uint32_t szi(const TreeParams &P, uint32_t i) {
    uint32_t y = (i * 0x9E3779B1u) & P.szmask;
    while (y >= (uint32_t)P.n) y = (y * 0x9E3779B1u) & P.szmask;
    return y;
}

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

// BFS level stamps (see the header comment)
__device__ __forceinline__ uint32_t level_stamp(int L) { return 0x81u + (uint32_t)(L % 127); }

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

// a root of the caller tree (push BFS of gb_balance_given_tree and the f.3
// samplers); r is an original id -- the push BFS walks the original CSR, and
// its level lists are translated to internal ids afterwards (k_pkey_to_parq)
__device__ __forceinline__ void place_root(const TreeParams &P, int b, int64_t C, uint32_t r) {
    const size_t nb = (size_t)b * P.n;
    atomicOr(P.vst + (size_t)b * P.nw + (r >> 2), level_stamp(0) << (8 * (r & 3)));
    const uint32_t deg = P.row_ptr[r + 1] - P.row_ptr[r];
    const uint32_t pre = (uint32_t)P.coff[C];
    if (deg == 0) {
        // isolated vertex: a one-vertex tree, finished here (pi = 0)
        const uint32_t ri = P.brank[r];
        if (P.irec) {
            P.irec[nb + ri] = make_uint4(ri, pre, 1u, 0u);
        } else {
            P.pp[nb + ri] = pre;
            if (P.prec) P.prec[nb + pre] = pre;
            else P.rec[nb + pre] = make_uint2(pre, 1u);
            if (P.crec) P.crec[nb + pre] = make_uint2(0u, 0u);
        }
        if (P.visited) atomicAdd(P.visited + b, 1ull);
        return;
    }
    unsigned long long old = atomicAdd((unsigned long long *)(P.lvl + b * P.ls), (1ull << 32) | deg);
    const uint32_t pos = (uint32_t)(old >> 32);
    P.qv[nb + pos] = r;
    P.qs[nb + pos] = (uint32_t)old;
    P.qr[nb + pos] = P.row_ptr[r];
    P.pkeyq[nb + pos] = ~0ull;
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

constexpr int kWarpBuf = 256;  // discovered vertices buffered per warp before one enqueue

// append the warp's buffered discoveries (wbuf[0..cnt): {vertex, degree, row start})
// to level L+1 with ONE atomic on the level counter, then write queue entries
__device__ __forceinline__ void flush_discoveries(const TreeParams &P, int b, uint32_t pos0,
                                                  unsigned long long *lvl_next, uint3 *wbuf,
                                                  uint32_t cnt) {
    const int lane = threadIdx.x & 31;
    __syncwarp();
    uint32_t dsum = 0;
    for (uint32_t i = lane; i < cnt; i += 32) dsum += wbuf[i].y;
#pragma unroll
    for (int d = 16; d; d >>= 1) dsum += __shfl_xor_sync(0xFFFFFFFFu, dsum, d);
    unsigned long long old = 0;
    if (lane == 0) old = atomicAdd(lvl_next, ((unsigned long long)cnt << 32) | dsum);
    old = __shfl_sync(0xFFFFFFFFu, old, 0);
    const size_t nb = (size_t)b * P.n;
    uint32_t run = (uint32_t)old;
    const uint32_t pos = pos0 + (uint32_t)(old >> 32);
    for (uint32_t c = 0; c < cnt; c += 32) {
        const uint32_t i = c + lane;
        const uint3 e = i < cnt ? wbuf[i] : make_uint3(0u, 0u, 0u);
        const uint32_t incl = warp_incl_scan32(e.y);
        if (i < cnt) {
            P.qv[nb + pos + i] = e.x;
            P.qs[nb + pos + i] = run + incl - e.y;
            P.qr[nb + pos + i] = e.z;
            P.pkeyq[nb + pos + i] = ~0ull;
        }
        run += __shfl_sync(0xFFFFFFFFu, incl, 31);
    }
    __syncwarp();
}

// expand the slots [s0, s1) of level L of tree b (one warp)
__device__ __forceinline__ void expand_range(const TreeParams &P, int b, int L, uint32_t s0,
                                             uint32_t s1, uint32_t vb, uint32_t nv, uint64_t tk,
                                             uint3 *wbuf) {
    const int lane = threadIdx.x & 31;
    const size_t nb = (size_t)b * P.n;
    const uint32_t *qs = P.qs + nb + vb;
    const uint32_t *qv = P.qv + nb + vb;
    const uint32_t *qr = P.qr + nb + vb;
    uint32_t *vst = P.vst + (size_t)b * P.nw;
    const uint32_t st_prev = level_stamp(L + 126);  // = stamp(L - 1) for L >= 1
    const uint32_t st_next = level_stamp(L + 1);
    unsigned long long *pk = P.pkeyq + nb + vb;
    // owner of slot s0: the largest q with qs[q] <= s0
    uint32_t q = 0;
    if (lane == 0) {
        uint32_t lo = 0, hi = nv;
        while (hi - lo > 1) {
            const uint32_t mid = lo + ((hi - lo) >> 1);
            if (__ldcg(qs + mid) <= s0) lo = mid; else hi = mid;
        }
        q = lo;
    }
    q = __shfl_sync(0xFFFFFFFFu, q, 0);
    const uint32_t lmask = lanemask_lt();
    unsigned long long *lvl_next = (unsigned long long *)(P.lvl + b * P.ls + L + 1);
    uint32_t nbuf = 0;  // warp-uniform fill of wbuf
    for (uint32_t s = s0; s < s1; s += 32) {
        const uint32_t qi = q + lane;
        const bool qok = qi < nv;
        const uint32_t myqs = qok ? __ldcg(qs + qi) : 0xFFFFFFFFu;
        const uint32_t myw = qok ? __ldcg(qv + qi) : 0u;
        const uint32_t myrp = qok ? __ldcg(qr + qi) : 0u;
        const uint32_t sl = s + lane;
        int idx = 0;
#pragma unroll
        for (int st = 16; st; st >>= 1) {
            const uint32_t v = __shfl_sync(0xFFFFFFFFu, myqs, idx + st);
            if (v <= sl) idx += st;
        }
        const uint32_t w = __shfl_sync(0xFFFFFFFFu, myw, idx);
        const uint32_t j = __shfl_sync(0xFFFFFFFFu, myrp, idx) + (sl - __shfl_sync(0xFFFFFFFFu, myqs, idx));
        const bool act = sl < s1;
        bool disc = false;
        uint32_t x = 0, deg = 0, neg = 0, rs = 0;
        unsigned long long key = ~0ull;
        if (act) {
            const uint32_t a = __ldg(P.adj + j);
            x = a & kIdMask;
            neg = a >> 31;
            const uint32_t word = x >> 2, sh = 8 * (x & 3);
            if (P.given) {
                // caller tree: follow tree edges only (parent(x) == w)
                if (P.given[x] == (int32_t)w) {
                    disc = true;
                    atomicOr(vst + word, st_next << sh);
                }
            } else {
                const uint32_t st = (__ldcg(vst + word) >> sh) & 0xFFu;
                if (st == 0) {
                    disc = !((atomicOr(vst + word, st_next << sh) >> sh) & 0xFFu);
                } else if (L > 0 && st == st_prev) {
                    // a neighbour one level up is a parent candidate of w (a.3)
                    key = parent_key(tk, x, w, neg);
                }
            }
            if (disc) {
                rs = __ldg(P.row_ptr + x);
                deg = __ldg(P.row_ptr + x + 1) - rs;
            }
        }
        if (!P.given && __any_sync(0xFFFFFFFFu, key != ~0ull)) {
            // segmented minimum over the lanes of one owner, one atomic per run
            const uint32_t oi = q + idx;
            const uint32_t prev = __shfl_up_sync(0xFFFFFFFFu, oi, 1);
            const uint32_t starts = __ballot_sync(0xFFFFFFFFu, lane == 0 || prev != oi);
            const int leader = 31 - __clz(starts & (lmask | (1u << lane)));
#pragma unroll
            for (int d = 1; d < 32; d <<= 1) {
                const unsigned long long y = __shfl_up_sync(0xFFFFFFFFu, key, d);
                if (lane - d >= leader) key = min(key, y);
            }
            const bool tail = lane == 31 || ((starts >> (lane + 1)) & 1u);
            if (tail && key != ~0ull) atomicMin(pk + oi, key);
        }
        const uint32_t dm = __ballot_sync(0xFFFFFFFFu, disc);
        if (dm) {
            if (P.given) {
                // caller trees: enqueue directly (the parent key is the caller's)
                const uint32_t incl = warp_incl_scan32(deg);
                const uint32_t total = __shfl_sync(0xFFFFFFFFu, incl, 31);
                const int leader = __ffs(dm) - 1;
                unsigned long long old = 0;
                if (lane == leader)
                    old = atomicAdd(lvl_next, ((unsigned long long)__popc(dm) << 32) | total);
                old = __shfl_sync(0xFFFFFFFFu, old, leader);
                if (disc) {
                    const uint32_t pos = vb + nv + (uint32_t)(old >> 32) + __popc(dm & lmask);
                    P.qv[nb + pos] = x;
                    P.qs[nb + pos] = (uint32_t)old + (incl - deg);
                    P.qr[nb + pos] = rs;
                    P.pkeyq[nb + pos] = ((unsigned long long)w << 1) | neg;
                }
            } else {
                const uint32_t k = __popc(dm);
                if (nbuf + k > (uint32_t)kWarpBuf) {
                    flush_discoveries(P, b, vb + nv, lvl_next, wbuf, nbuf);
                    nbuf = 0;
                }
                if (disc) wbuf[nbuf + __popc(dm & lmask)] = make_uint3(x, deg, rs);
                nbuf += k;
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
    if (nbuf) flush_discoveries(P, b, vb + nv, lvl_next, wbuf, nbuf);
}

__global__ void __launch_bounds__(kBlock, 6) k_bfs(TreeParams P) {
    cg::grid_group grid = cg::this_grid();
    __shared__ LevelTable T;
    __shared__ uint64_t s_tkey[kMaxBatch];
    __shared__ int32_t s_depth[kMaxBatch];
    __shared__ int s_more;
    __shared__ uint3 s_wbuf[kBlock / 32][kWarpBuf];
    const int B = P.B;
    const int64_t gtid = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    const int64_t nthr = (int64_t)gridDim.x * blockDim.x;
    const int64_t gwarp = gtid >> 5;
    const int64_t nwarps = nthr >> 5;
    if (threadIdx.x < B) {
        T.vb[threadIdx.x] = 0;
        s_tkey[threadIdx.x] = P.tkey[threadIdx.x];
        s_depth[threadIdx.x] = 0;
    }
    for (int L = 0;; L++) {
        __syncthreads();
        if (threadIdx.x < B) {
            const unsigned long long c = __ldcg((const unsigned long long *)(P.lvl + threadIdx.x * P.ls + L));
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
        // level L+1 compares against stamp(L) == stamp(L-127): retire the
        // vertices of level L-127 (deep graphs only) so the stamps stay exact
        if (L >= 127) {
            for (int b = 0; b < B; b++) {
                const uint32_t r0 = __ldcg(P.vbase + b * P.ls + (L - 127));
                const uint32_t r1 = __ldcg(P.vbase + b * P.ls + (L - 126));
                for (int64_t i = r0 + gtid; i < (int64_t)r1; i += nthr) {
                    const uint32_t x = __ldcg(P.qv + (size_t)b * P.n + i);
                    atomicAnd(P.vst + (size_t)b * P.nw + (x >> 2), ~(0x7Fu << (8 * (x & 3))));
                }
            }
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
                         T.vb[b], T.nv[b], s_tkey[b], s_wbuf[threadIdx.x >> 5]);
        }
        grid.sync();
        if (threadIdx.x == 0) s_more = 0;
        __syncthreads();
        if (threadIdx.x < B) {
            const unsigned long long c = __ldcg((const unsigned long long *)(P.lvl + threadIdx.x * P.ls + L + 1));
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
        const int b = threadIdx.x;
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

// independent vertices per thread in the level passes (measured: 4)
#ifndef GB_ILP_UP
#define GB_ILP_UP 4
#endif
#ifndef GB_ILP_DOWN
#define GB_ILP_DOWN 4
#endif

// Levels with at most kSolo vertices (the first and last levels of a BFS
// tree) are processed by block 0 alone: consecutive small levels are
// separated by __syncthreads instead of grid barriers, and the other blocks
// skip them (a grid barrier is kept only where a large level follows or
// precedes).  kSoloLevels bounds the depth for which the level totals are
// tabulated in shared memory.
constexpr unsigned long long kSolo = 1024;
constexpr int kSoloLevels = 64;

__device__ __forceinline__ bool level_tables(const TreeParams &P, int maxd, const int32_t *s_depth,
                                             unsigned long long *s_tot) {
    if (maxd >= kSoloLevels) return false;
    for (int L = threadIdx.x; L <= maxd; L += blockDim.x) {
        unsigned long long t = 0;
        for (int b = 0; b < P.B; b++)
            if (L <= s_depth[b]) t += __ldcg((const unsigned long long *)(P.lvl + b * P.ls + L)) >> 32;
        s_tot[L] = t;
    }
    __syncthreads();
    return true;
}

__device__ __forceinline__ unsigned long long gtimer_ns() {
    unsigned long long t;
    asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
    return t;
}

// queue-order streams of the level passes: read / written once per pass, so
// (option GB_LABEL_HINT) they are marked evict_first and leave L2 to the one
// random-access label array of the pass
#ifdef GB_LABEL_HINT
#define GB_QLD(ptr) ld_hint((ptr), qpol)
#define GB_QST(ptr, val) st_hint((ptr), (val), qpol)
#define GB_QPOL const uint64_t qpol = l2_stream_policy()
#else
#define GB_QLD(ptr) __ldcg(ptr)
#define GB_QST(ptr, val) (*(ptr) = (val))
#define GB_QPOL
#endif

__device__ __forceinline__ int tree_of(const LevelTable &T, int B, unsigned long long i) {
    int lo = 0, hi = B;  // soff[lo] <= i < soff[hi]
    while (hi - lo > 1) {
        const int mid = (lo + hi) >> 1;
        if (T.soff[mid] <= i) lo = mid; else hi = mid;
    }
    return lo;
}

// Warp-aggregated atomicAdd of v into *addr; returns the value each lane
// would have seen with its own atomicAdd in some serial order.  Lanes adding
// to the same address in one contiguous run of lanes share one atomic (the
// children of a hub arrive in runs); everything else adds on its own.
template <typename T>
__device__ __forceinline__ T aggregated_add(T *addr, T v, bool valid) {
    const int lane = threadIdx.x & 31;
    const unsigned long long k = valid ? (unsigned long long)addr : ~(unsigned long long)lane;
    const uint32_t peers = __match_any_sync(0xFFFFFFFFu, k);
    const int leader = __ffs(peers) - 1;
    const uint32_t run = peers >> leader;
    const bool contiguous = (run & (run + 1)) == 0;
    T res = 0;
    if (__all_sync(0xFFFFFFFFu, contiguous)) {
        T incl = v;
#pragma unroll
        for (int d = 1; d < 32; d <<= 1) {
            const T y = __shfl_up_sync(0xFFFFFFFFu, incl, d);
            if (lane - d >= leader) incl += y;
        }
        const int tail = 31 - __clz(peers);
        T old = 0;
        if (lane == tail && valid) old = atomicAdd(addr, incl);
        old = __shfl_sync(0xFFFFFFFFu, old, tail);
        res = old + incl - v;
    } else if (valid) {
        res = atomicAdd(addr, v);
    }
    return res;
}

// ---------------------------------------------------------------------------
// a.4: Alg. 4 bottom-up pass (L273-L278).  Levels D..1, items in queue order;
// every vertex adds its final subtree size to its parent's count with an
// atomic add (L256).  The value returned by that add is 1 + the sizes of the
// siblings added before it: exactly the offset of this child's range inside
// its parent's (Alg. 4, "earlier children" = earlier atomic adds,
// reading R5).  With walk 1 the same 64-bit add also counts the children, so
// the sibling index matches the pre order.
// ---------------------------------------------------------------------------
template <bool kDescent>
__global__ void __launch_bounds__(kBlock) k_bottom_up(TreeParams P) {
    cg::grid_group grid = cg::this_grid();
    __shared__ LevelTable T;
    __shared__ int32_t s_depth[kMaxBatch];
    const int B = P.B;
    if (threadIdx.x < B) s_depth[threadIdx.x] = __ldcg(P.depth + threadIdx.x);
    __syncthreads();
    const int maxd = __ldcg(P.maxd);
    const int lane = threadIdx.x & 31;
    __shared__ unsigned long long s_tot[kSoloLevels];
    const bool solo_ok = level_tables(P, maxd, s_depth, s_tot);
    for (int L = maxd; L >= 1; L--) {
        load_level(P, L, T, s_depth);
        const unsigned long long total = T.soff[B];
        if (P.prof && blockIdx.x == 0 && threadIdx.x == 0 && L < 256) {
            P.prof[4 * L] = gtimer_ns();
            P.prof[4 * L + 2] = total;
        }
        const bool solo = solo_ok && total <= kSolo;
        const int64_t gwarp = solo ? (int64_t)(threadIdx.x >> 5) : ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
        const int64_t nwarps = solo ? (int64_t)(blockDim.x >> 5) : ((int64_t)gridDim.x * blockDim.x) >> 5;
        const int64_t gtid = solo ? (int64_t)threadIdx.x : (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
        const int64_t nthr = solo ? (int64_t)blockDim.x : (int64_t)gridDim.x * blockDim.x;
        if (!solo || blockIdx.x == 0) {
        if constexpr (!kDescent) {
            // kILP independent vertices per thread: their queue words, their
            // own sizes and the adds to their parents are in flight together
            constexpr int kILP = GB_ILP_UP;
            GB_QPOL;
            for (unsigned long long base = gtid; base < total; base += kILP * nthr) {
                size_t qi[kILP], nbk[kILP], sbk[kILP];
                uint32_t w[kILP], p[kILP], sz[kILP];
                bool ok[kILP];
#pragma unroll
                for (int k = 0; k < kILP; k++) {
                    const unsigned long long i = base + (unsigned long long)k * nthr;
                    ok[k] = i < total;
                    if (ok[k]) {
                        const int b = tree_of(T, B, i);
                        nbk[k] = (size_t)b * P.n;
                        sbk[k] = (size_t)b * P.szn;
                        qi[k] = nbk[k] + T.vb[b] + (uint32_t)(i - T.soff[b]);
                        w[k] = GB_QLD(P.qv + qi[k]);
                        p[k] = GB_QLD(P.parq + qi[k]) & kIdMask;
                    }
                }
#pragma unroll
                for (int k = 0; k < kILP; k++)
                    if (ok[k]) sz[k] = 1 + __ldcg(P.size + sbk[k] + szi(P, w[k]));
#pragma unroll
                for (int k = 0; k < kILP; k++) {
                    if (ok[k]) {
                        const uint32_t o = atomicAdd(P.size + sbk[k] + szi(P, p[k]), sz[k]);
                        GB_QST(P.offq + qi[k], 1 + o);
                        GB_QST(P.szq + qi[k], sz[k]);
                    }
                }
            }
        } else {
        for (unsigned long long wb = (unsigned long long)gwarp * 32; wb < total;
             wb += (unsigned long long)nwarps * 32) {
            const unsigned long long i = wb + lane;
            const bool valid = i < total;
            size_t nb = 0, qi = 0, sb = 0;
            uint32_t w = 0, p = 0, sz = 0, neg = 0;
            if (valid) {
                const int b = tree_of(T, B, i);
                nb = (size_t)b * P.n;
                sb = (size_t)b * P.szn;
                qi = nb + T.vb[b] + (uint32_t)(i - T.soff[b]);
                w = __ldcg(P.qv + qi);
                const uint32_t pq = __ldcg(P.parq + qi);
                p = pq & kIdMask;
                neg = pq & kNegBit;
                // counters hold the sum of the children's sizes: size = 1 + that
                sz = 1 + (kDescent ? (uint32_t)__ldcg(P.sz64 + nb + w)
                                   : __ldcg(P.size + sb + szi(P, w)));
            }
            if (kDescent) {
                const unsigned long long o =
                    aggregated_add<unsigned long long>(P.sz64 + nb + p, (1ull << 32) | sz, valid);
                if (valid) {
                    P.offq[qi] = 1 + (uint32_t)o;
                    P.cidxq[qi] = (uint32_t)(o >> 32);
                }
            } else {
                const uint32_t o = aggregated_add<uint32_t>(P.size + sb + szi(P, p), sz, valid);
                if (valid) P.offq[qi] = 1 + o;
            }
            if (valid) P.szq[qi] = sz;
        }
        }
        }
        if (L > 1) {
            if (solo && s_tot[L - 1] <= kSolo) __syncthreads();
            else grid.sync();
        }
    }
    if (P.prof && blockIdx.x == 0 && threadIdx.x == 0) P.prof[0] = gtimer_ns();
}

// ---------------------------------------------------------------------------
// a.5: Alg. 4 top-down pass (L279-L291): levels 0..D, items in queue order;
// pre(child) = pre(parent) + offset; the range of tree edge p->c is
// [pre c, pre c + size c - 1] (L285-L286); the root parity pi(c) = pi(p) XOR
// neg(p,c) gives the Harary side (reading R7).  Writes the pre-indexed record
// rec[pre] = {pre(parent) | neg<<31, size} used by the cycle walk.
// ---------------------------------------------------------------------------
template <bool kDescent>
__global__ void __launch_bounds__(kBlock, 4) k_top_down(TreeParams P) {
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
    const bool one_comp = P.ncomp == 1;
    __shared__ unsigned long long s_tot[kSoloLevels];
    const bool solo_ok = level_tables(P, maxd, s_depth, s_tot);
    for (int L = 0; L <= maxd; L++) {
        load_level(P, L, T, s_depth);
        const unsigned long long total = T.soff[B];
        if (P.prof && blockIdx.x == 0 && threadIdx.x == 0 && L < 255) P.prof[4 * L + 1] = gtimer_ns();
        const bool solo = solo_ok && total <= kSolo;
        const int64_t gtid = solo ? (int64_t)threadIdx.x : (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
        const int64_t nthr = solo ? (int64_t)blockDim.x : (int64_t)gridDim.x * blockDim.x;
        // barrier after level L: block-local between two small levels
        const bool local_sync = solo && L < maxd && s_tot[L + 1] <= kSolo;
        if (solo && blockIdx.x != 0) {
            if (L < maxd && !local_sync) grid.sync();
            continue;
        }
        if (!kDescent && L > 0) {
            // kILP independent vertices per thread per iteration: their queue
            // words, then their parents' labels, are in flight together
            constexpr int kILP = GB_ILP_DOWN;
            GB_QPOL;
            for (unsigned long long base = gtid; base < total; base += kILP * nthr) {
                size_t qi[kILP], nbk[kILP];
                uint32_t x[kILP], pq[kILP], off[kILP], szx[kILP], ppp[kILP];
                int bk[kILP];
#pragma unroll
                for (int k = 0; k < kILP; k++) {
                    const unsigned long long i = base + (unsigned long long)k * nthr;
                    bk[k] = -1;
                    if (i < total) {
                        bk[k] = tree_of(T, B, i);
                        nbk[k] = (size_t)bk[k] * P.n;
                        qi[k] = nbk[k] + T.vb[bk[k]] + (uint32_t)(i - T.soff[bk[k]]);
                        x[k] = GB_QLD(P.qv + qi[k]);
                        pq[k] = GB_QLD(P.parq + qi[k]);
                        off[k] = GB_QLD(P.offq + qi[k]);
                        szx[k] = GB_QLD(P.szq + qi[k]);
                    }
                }
#pragma unroll
                for (int k = 0; k < kILP; k++)
                    if (bk[k] >= 0)
                        ppp[k] = P.irec ? __ldcg(reinterpret_cast<const uint32_t *>(P.irec + nbk[k] + (pq[k] & kIdMask)) + 1)
                                        : __ldcg(P.pp + nbk[k] + (pq[k] & kIdMask));
#pragma unroll
                for (int k = 0; k < kILP; k++) {
                    if (bk[k] < 0) continue;
                    const uint32_t up = ppp[k] & kIdMask, neg = pq[k] & kNegBit;
                    const uint32_t pre = up + off[k];
                    const uint32_t pi = (ppp[k] & kNegBit) ^ neg;
                    if (P.irec) {
                        // layout 0: the record by internal id, complete here
                        P.irec[nbk[k] + x[k]] = make_uint4(pq[k], pre | pi, szx[k], 0u);
                    } else if (P.prec) {
                        // layout 2: pre | pi by internal id, the parent word by pre
                        P.pp[nbk[k] + x[k]] = pre | pi;
                        P.prec[nbk[k] + pre] = up | neg;
                    } else if (P.recpass) {
                        P.pp[nbk[k] + x[k]] = pre | pi;
                        GB_QST(P.parq + qi[k], up | neg);
                        GB_QST(P.offq + qi[k], pre);
                    } else {
                        P.pp[nbk[k] + x[k]] = pre | pi;
                        P.rec[nbk[k] + pre] = make_uint2(up | neg, szx[k]);
                    }
                    if (pi) {
                        const int32_t C = one_comp ? 0 : __ldg(P.comp_i + x[k]);
                        if (C == P.cbig) atomicAdd(&s_big[bk[k]], 1u);
                        else atomicAdd(P.s1 + (size_t)bk[k] * P.ncomp + C, 1u);
                    }
                }
            }
            if (L < maxd) {
                if (local_sync) __syncthreads();
                else grid.sync();
            }
            continue;
        }
        for (unsigned long long i = gtid; i < total; i += nthr) {
            const int b = tree_of(T, B, i);
            const size_t nb = (size_t)b * P.n;
            const size_t qi = nb + T.vb[b] + (uint32_t)(i - T.soff[b]);
            const uint32_t x = __ldcg(P.qv + qi);
            uint32_t pre, up, neg, pi, p = 0, szx;
            if (L == 0) {
                const int32_t C = one_comp ? 0 : __ldg(P.comp_i + x);
                pre = (uint32_t)__ldg(P.coff + C);
                up = pre;
                neg = 0;
                pi = 0;
                szx = 1 + (kDescent ? (uint32_t)__ldcg(P.sz64 + nb + x)
                                    : __ldcg(P.size + (size_t)b * P.szn + szi(P, x)));
            } else {
                const uint32_t pq = __ldcg(P.parq + qi);
                p = pq & kIdMask;
                const uint32_t ppp = P.irec ? __ldcg(reinterpret_cast<const uint32_t *>(P.irec + nb + p) + 1)
                                            : __ldcg(P.pp + nb + p);
                up = ppp & kIdMask;
                pre = up + __ldcg(P.offq + qi);
                neg = pq & kNegBit;
                pi = (ppp & kNegBit) ^ neg;
                szx = __ldcg(P.szq + qi);
            }
            if (!kDescent && P.irec) {
                P.irec[nb + x] = make_uint4(L == 0 ? x : (p | neg), pre | pi, szx, 0u);
            } else if (!kDescent && P.prec) {
                P.pp[nb + x] = pre | pi;
                P.prec[nb + pre] = up | neg;
            } else if (!kDescent && P.recpass) {
                P.pp[nb + x] = pre | pi;
                P.parq[qi] = up | neg;
                P.offq[qi] = pre;
                P.szq[qi] = szx;
            } else {
                P.pp[nb + x] = pre | pi;
                P.rec[nb + pre] = make_uint2(up | neg, szx);
            }
            if (kDescent) {
                // Alg. 3 descent structures: the child list of x (by pre) and
                // this vertex's slot in its parent's list
                P.crec[nb + pre] = make_uint2(__ldcg(P.cstart + nb + x),
                                              (uint32_t)(__ldcg(P.sz64 + nb + x) >> 32));
                if (L > 0) P.clist[__ldcg(P.cstart + nb + p) + __ldcg(P.cidxq + qi)] = pre;
            }
            if (pi) {
                const int32_t C = one_comp ? 0 : __ldg(P.comp_i + x);
                if (C == P.cbig) atomicAdd(&s_big[b], 1u);
                else atomicAdd(P.s1 + (size_t)b * P.ncomp + C, 1u);
            }
        }
        if (L < maxd) {
            if (local_sync) __syncthreads();
            else grid.sync();
        }
    }
    if (P.prof && blockIdx.x == 0 && threadIdx.x == 0 && maxd + 1 < 256) P.prof[4 * (maxd + 1) + 1] = gtimer_ns();
    __syncthreads();
    if (threadIdx.x < B && s_big[threadIdx.x])
        atomicAdd(P.s1 + (size_t)threadIdx.x * P.ncomp + P.cbig, s_big[threadIdx.x]);
}

// walk 0, option "recpass": the pre-indexed records of every queued vertex,
// rec[pre] = {pre(parent) | neg << 31, size}, scattered in one pass with no
// level order (the top-down pass left them in queue order).  Keeping this
// 8-byte scatter out of the level passes leaves their random-access working
// set at one 4-byte label array per tree.
__global__ void k_rec_scatter(TreeParams P) {
    const int b = blockIdx.y;
    const size_t nb = (size_t)b * P.n;
    const uint32_t cnt = __ldcg(P.vbase + b * P.ls + __ldcg(P.depth + b) + 1);
    // the queue-order streams are read once (evict_first); the records stay
    // in L2 until their sectors are complete (evict_last): measured 39.0 ->
    // 37.5 ms per 100 C3 trees for the whole top-down phase
    const uint64_t stream = l2_stream_policy(), keep = l2_keep_policy();
    for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < cnt; i += gridDim.x * blockDim.x) {
        const uint32_t pre = ld_hint(P.offq + nb + i, stream);
        st_hint(P.rec + nb + pre, make_uint2(ld_hint(P.parq + nb + i, stream), ld_hint(P.szq + nb + i, stream)), keep);
    }
}

// child count of every vertex (high half of the packed counter), scanned in
// place into child-list starts (walk 1 only)
__global__ void k_child_counts(TreeParams P, int64_t cnt) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < cnt;
         i += (int64_t)gridDim.x * blockDim.x)
        P.cstart[i] = (uint32_t)(P.sz64[i] >> 32);
}

// caller trees (push BFS): parent keys -> parent | neg << 31 in queue order,
// and the level lists translated to internal ids (the labelling passes' and
// the walk's index space); level-0 entries (roots) point at themselves
__global__ void k_pkey_to_parq(TreeParams P, const unsigned long long *pkeyq) {
    const int64_t cnt = (int64_t)P.vbase[P.depth[0] + 1];
    const int64_t nroots = (int64_t)P.vbase[1];
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < cnt;
         i += (int64_t)gridDim.x * blockDim.x) {
        const uint32_t vi = P.brank[P.qv[i]];
        P.qv[i] = vi;
        if (i < nroots) {
            P.parq[i] = vi;
        } else {
            const unsigned long long k = pkeyq[i];
            P.parq[i] = P.brank[(uint32_t)(k >> 1) & kIdMask] | ((uint32_t)k << 31);
        }
    }
}

// ---------------------------------------------------------------------------
// debug views of one tree (b = 0): parent / dist / size by vertex
// ---------------------------------------------------------------------------
__global__ void k_debug_tree(TreeParams P, int32_t *parent, int32_t *dist, int32_t *size, int32_t *pre) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < P.n;
         i += (int64_t)gridDim.x * blockDim.x) {
        const uint32_t v = P.bord[i];   // labels live in internal ids; outputs by original id
        parent[v] = -1;
        dist[v] = 0;
        if (P.brow[i + 1] == P.brow[i]) {
            // isolated vertex: a one-vertex tree (labels not stored per tree)
            size[v] = 1;
            pre[v] = P.coff[P.comp_i[i]];
            continue;
        }
        size[v] = 1 + (P.sz64 ? (int32_t)(uint32_t)P.sz64[i] : (int32_t)P.size[szi(P, (uint32_t)i)]);
        pre[v] = (int32_t)((P.irec ? P.irec[i].y : P.pp[i]) & kIdMask);
    }
}

__global__ void k_debug_tree_scatter(TreeParams P, int64_t nqueued, int32_t *parent, int32_t *dist) {
    const int D = P.depth[0];
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < nqueued;
         i += (int64_t)gridDim.x * blockDim.x) {
        int lo = 0, hi = D + 1;  // vbase[lo] <= i < vbase[hi]
        while (hi - lo > 1) {
            const int mid = (lo + hi) >> 1;
            if ((int64_t)P.vbase[mid] <= i) lo = mid; else hi = mid;
        }
        const uint32_t v = P.bord[P.qv[i]];
        dist[v] = lo;
        parent[v] = lo == 0 ? -1 : (int32_t)P.bord[P.parq[i] & kIdMask];
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

// trees b0 .. b0+B-1 of the workspace
static TreeParams make_params(const Graph &g, Workspace &ws, int B, const int32_t *given,
                              bool descent, int b0 = 0) {
    TreeParams P;
    P.row_ptr = g.row_ptr; P.adj = g.adj;
    P.brank = g.brank; P.bord = g.bord; P.brow = g.brow;
    P.comp = g.comp; P.comp_i = g.comp_i; P.coff = g.coff; P.cverts = g.cverts;
    P.n = g.n; P.ncomp = g.ncomp; P.nw = (g.n + 3) / 4; P.cbig = g.cbig;
    P.B = B; P.ls = g.n + 2;
    P.vst = ws.vst; P.qv = ws.qv; P.qs = ws.qs; P.qr = ws.qr; P.pkeyq = ws.pkeyq;
    P.lvl = ws.lvl; P.vbase = ws.vbase;
    P.size = descent ? nullptr : ws.size;
    P.szn = g.n;
    P.szmask = (uint32_t)(size_slots(g.n) - 1);
    P.sz64 = descent ? ws.sz64 : nullptr;
    P.parq = ws.parq; P.offq = ws.offq; P.szq = ws.szq;
    P.cidxq = descent ? ws.cidxq : nullptr;
    P.pp = ws.pp; P.rec = ws.rec; P.s1 = ws.s1; P.tkey = ws.tkey; P.depth = ws.depth;
    P.irec = (ws.irec_layout && !descent) ? ws.irec : nullptr;
    P.prec = descent ? nullptr : ws.prec;
    P.maxd = ws.maxd; P.given = given;
    P.cstart = descent ? ws.cstart : nullptr;
    P.clist = descent ? ws.clist : nullptr;
    P.crec = descent ? ws.crec : nullptr;
    P.visited = given ? ws.visited : nullptr;
    P.recpass = 0;
    P.prof = ws.msprof ? ws.msprof + 1024 : nullptr;
    if (b0) {
        const size_t nb = (size_t)b0 * g.n, lb = (size_t)b0 * P.ls;
        P.qv += nb; P.parq += nb; P.offq += nb; P.szq += nb;
        if (P.pp) P.pp += nb;
        if (P.rec) P.rec += nb;
        if (P.irec) P.irec += nb;
        if (P.prec) P.prec += nb;
        if (P.size) P.size += (size_t)b0 * P.szn;
        if (P.sz64) P.sz64 += nb;
        if (P.cidxq) P.cidxq += nb;
        if (P.cstart) P.cstart += nb;
        if (P.crec) P.crec += nb;
        P.lvl += lb; P.vbase += lb;
        P.s1 += (size_t)b0 * g.ncomp;
        P.tkey += b0; P.depth += b0;
        P.vst = nullptr; P.qs = nullptr; P.qr = nullptr; P.pkeyq = nullptr;
    }
    return P;
}

// option "persist": an L2 persisting access-policy window over the one
// random-access array of the next launch (0 = off)
static int set_window(cudaStream_t st, void *base, size_t bytes, size_t persist) {
    if (!persist) return GB_OK;
    cudaStreamAttrValue a = {};
    a.accessPolicyWindow.base_ptr = base;
    a.accessPolicyWindow.num_bytes = base ? std::min(bytes, persist) : 0;
    a.accessPolicyWindow.hitRatio = 1.0f;
    a.accessPolicyWindow.hitProp = cudaAccessPropertyPersisting;
    a.accessPolicyWindow.missProp = cudaAccessPropertyStreaming;
    GB_CUDA_TRY(cudaStreamSetAttribute(st, cudaStreamAttributeAccessPolicyWindow, &a));
    return GB_OK;
}

int run_batch_tree(const Graph &g, Workspace &ws, int B, const int32_t *given_parent,
                   cudaStream_t st, int64_t *launches, cudaEvent_t *ev, bool descent, int sub,
                   int recpass, size_t persist, int sampler) {
    if (descent || ws.irec_layout || ws.prec) recpass = 0;
    // co-resident grid sizes, recomputed when the device changes
    static int bfs_blocks = 0, up_blocks[2] = {0, 0}, down_blocks[2] = {0, 0}, blocks_dev = -1;
    if (blocks_dev != g.dev) {
        blocks_dev = g.dev;
        bfs_blocks = coop_blocks((const void *)k_bfs, g.num_sms);
        up_blocks[0] = coop_blocks((const void *)k_bottom_up<false>, g.num_sms);
        up_blocks[1] = coop_blocks((const void *)k_bottom_up<true>, g.num_sms);
        down_blocks[0] = coop_blocks((const void *)k_top_down<false>, g.num_sms);
        down_blocks[1] = coop_blocks((const void *)k_top_down<true>, g.num_sms);
    }
    if (sub < 1 || sub > B) sub = B;
    TreeParams P = make_params(g, ws, B, given_parent, descent);
    if (ev) GB_CUDA_TRY(cudaEventRecord(ev[0], st));
    GB_CUDA_TRY(cudaMemsetAsync(ws.s1, 0, sizeof(uint32_t) * (size_t)B * g.ncomp, st));
    if (descent) GB_CUDA_TRY(cudaMemsetAsync(ws.sz64, 0, sizeof(unsigned long long) * (size_t)B * g.n, st));
    else GB_CUDA_TRY(cudaMemsetAsync(ws.size, 0, sizeof(uint32_t) * (size_t)B * g.n, st));
    k_batch_prep<<<1, kMaxBatch, 0, st>>>(P);
    ++*launches;
    // f.3: a uniform random spanning tree (B = 1), then the caller-tree path
    const bool sampled = sampler == 1 && !given_parent;
    if (sampled) {
        if (ev) GB_CUDA_TRY(cudaEventRecord(ev[1], st));
        if (!ws.wparent) GB_CUDA_TRY(cudaMalloc(&ws.wparent, sizeof(int32_t) * (size_t)g.n));
        int rc = run_wilson(g, ws, st, launches, ws.wparent, nullptr);
        if (rc) return rc;
        given_parent = ws.wparent;
        P.given = given_parent;
        P.visited = ws.visited;
    }
    if (given_parent) {
        // a caller tree (B = 1): push BFS along its parent edges
        GB_CUDA_TRY(cudaMemsetAsync(ws.vst, 0, sizeof(uint32_t) * (size_t)P.nw, st));
        k_roots_given<<<(unsigned)std::min<int64_t>((g.n + 255) / 256, 4096), 256, 0, st>>>(P);
        ++*launches;
        GB_CUDA_TRY(cudaGetLastError());
        if (ev && !sampled) GB_CUDA_TRY(cudaEventRecord(ev[1], st));
        int rc = launch_coop((const void *)k_bfs, bfs_blocks, P, st);
        if (rc) return rc;
        ++*launches;
        k_pkey_to_parq<<<(unsigned)std::min<int64_t>((g.n + 255) / 256, 4096), 256, 0, st>>>(P, ws.pkeyq);
        ++*launches;
    } else {
        if (ev) GB_CUDA_TRY(cudaEventRecord(ev[1], st));
        MsBfsOut o;
        o.qv = ws.qv; o.parq = ws.parq; o.pp = ws.pp; o.rec = ws.rec;
        o.irec = (ws.irec_layout && !descent) ? ws.irec : nullptr;
        o.prec = descent ? nullptr : ws.prec;
        o.crec = descent ? ws.crec : nullptr;
        o.lvl = ws.lvl; o.vbase = ws.vbase; o.depth = ws.depth; o.maxd = ws.maxd; o.tkey = ws.tkey;
        int rc = run_msbfs(g, ws, B, o, st, launches);
        if (rc) return rc;
    }
    GB_CUDA_TRY(cudaGetLastError());
    if (ev) GB_CUDA_TRY(cudaEventRecord(ev[2], st));
    // Alg. 4 on sub-batches of `sub` trees (their random-access arrays stay
    // L2-resident): all bottom-up passes, then all top-down passes
    for (int b0 = 0; b0 < B; b0 += sub) {
        TreeParams Q = make_params(g, ws, std::min(sub, B - b0), given_parent, descent, b0);
        if (!descent && set_window(st, Q.size, sizeof(uint32_t) * (size_t)Q.B * g.n, persist)) return GB_ECUDA;
        int rc = descent ? launch_coop((const void *)k_bottom_up<true>, up_blocks[1], Q, st)
                         : launch_coop((const void *)k_bottom_up<false>, up_blocks[0], Q, st);
        if (rc) return rc;
        ++*launches;
    }
    if (descent) {
        const int64_t cnt = (int64_t)B * g.n;
        k_child_counts<<<(unsigned)std::min<int64_t>((cnt + 255) / 256, 8192), 256, 0, st>>>(P, cnt);
        ++*launches;
        int rc = exclusive_scan_u32(ws.cstart, ws.cstart, cnt, ws.scan_tmp, ws.scan_tmp_elems, st, launches);
        if (rc) return rc;
    }
    if (ev) GB_CUDA_TRY(cudaEventRecord(ev[3], st));
    for (int b0 = 0; b0 < B; b0 += sub) {
        TreeParams Q = make_params(g, ws, std::min(sub, B - b0), given_parent, descent, b0);
        Q.recpass = recpass;
        if (set_window(st, Q.pp, sizeof(uint32_t) * (size_t)Q.B * g.n, persist)) return GB_ECUDA;
        int rc = descent ? launch_coop((const void *)k_top_down<true>, down_blocks[1], Q, st)
                         : launch_coop((const void *)k_top_down<false>, down_blocks[0], Q, st);
        if (rc) return rc;
        ++*launches;
        if (recpass) {
            if (set_window(st, Q.rec, sizeof(uint2) * (size_t)Q.B * g.n, persist)) return GB_ECUDA;
            const unsigned gx = (unsigned)std::max<int64_t>(1, std::min<int64_t>((g.n + 255) / 256,
                                                                                 (int64_t)g.num_sms * 8 / Q.B + 1));
            k_rec_scatter<<<dim3(gx, Q.B), 256, 0, st>>>(Q);
            ++*launches;
        }
    }
    if (set_window(st, nullptr, 0, persist)) return GB_ECUDA;
    return GB_OK;
}

int debug_tree_views(const Graph &g, Workspace &ws, bool descent, int32_t *d_parent,
                     int32_t *d_dist, int32_t *d_size, int32_t *d_pre, cudaStream_t st) {
    TreeParams P = make_params(g, ws, 1, nullptr, descent);
    int32_t depth = 0;
    GB_CUDA_TRY(cudaMemcpyAsync(&depth, ws.depth, sizeof(int32_t), cudaMemcpyDeviceToHost, st));
    GB_CUDA_TRY(cudaStreamSynchronize(st));
    uint32_t nq = 0;
    GB_CUDA_TRY(cudaMemcpyAsync(&nq, ws.vbase + depth + 1, sizeof(uint32_t), cudaMemcpyDeviceToHost, st));
    GB_CUDA_TRY(cudaStreamSynchronize(st));
    k_debug_tree<<<256, 256, 0, st>>>(P, d_parent, d_dist, d_size, d_pre);
    k_debug_tree_scatter<<<256, 256, 0, st>>>(P, nq, d_parent, d_dist);
    GB_CUDA_TRY(cudaGetLastError());
    GB_CUDA_TRY(cudaStreamSynchronize(st));
    return GB_OK;
}

}  // namespace gb
