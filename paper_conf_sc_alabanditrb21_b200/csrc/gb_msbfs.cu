// gb_msbfs.cu -- §8 rows a.2 + a.3 for a batch of B <= 128 sampled trees at
// once: hashed roots, level-synchronous BFS and min-hash parent selection.
//
// The paper builds one BFS tree at a time (§3.1, Fig. 11 "spanning tree"
// 6 %) and rejects one-tree-per-thread for memory and locality on a 12 GB
// Titan V (L250).  Here the B trees of a batch share every pass over the
// graph (§8 a.9, multi-source BFS): each vertex carries a 128-bit word with
// one bit per tree (two 64-bit halves, interleaved: trees 0-63, 64-127) --
//   vis[v]  trees that have reached v,
//   F_L[v]  trees in which v is on level L (the frontier),
// plus two bitmaps with one bit per vertex: "F_L[v] != 0" (the frontier
// bitmap, 1.25 MB for 10 M vertices: L2-resident, it gates every frontier
// word gather) and "vis[v] == all trees" (finished vertices are skipped
// without touching their words).
//
// Level L -> L+1 is a *pull* over the unfinished vertices:
//   new(w) = OR_{u in N(w), F_L[u] != 0} F_L[u]  AND NOT vis(w),
// one read of w's adjacency serving all B trees.  For every tree t in new(w)
// the parent of w is the neighbour u with bit t in F_L[u] (one level up)
// minimising parent_key(t, u, w) (reading R4).  Discoveries go to the
// per-tree level lists (qv, parq) as internal ids: the labelling passes and
// the cycle walk index their per-tree arrays by the degree-sorted ids, so the
// parents -- mostly hubs and other high-degree vertices -- share a small hot
// region of each array.
//
// Work mapping (degree-sorted internal ids, gb_ingest.cu):
//   light vertices (degree <= kLight): one lane per vertex;
//   heavier vertices: warp work items of <= kChunk slots, lanes stride the
//     slots, lane l keeps the best key of trees l and l+32;
//   multi-chunk vertices (degree > kChunk, the hubs of Table 1's max degree
//     column): partial ORs and partial minima of all their chunks are merged
//     with global atomics (phase C, only when one of them discovered
//     something on this level).
#include "gb_internal.cuh"
#include "../../include/graphb.h"

#include <algorithm>
#include <cstdlib>

namespace gb {
namespace cg = cooperative_groups;

constexpr int kMsMaxBlocks = 2048;   // capacity of the per-block count table
constexpr int kPPTrees = 16;         // push-parent levels: batches of <= 16 trees
#ifndef GB_PP_DIV
#define GB_PP_DIV 64
#endif

struct MsParams {
    const uint32_t *brow, *badj, *borig, *bord, *brank;
    const uint2 *items;
    const int32_t *coff, *cverts, *bigc, *comp_i;
    int64_t nbig, niso;
    int64_t n, ncomp, nitems, nmulti_items, nlight0, nmulti, ls, nwords, itemwords;
    int B;
    unsigned long long full0, full1;   // the "every tree" masks of the two halves
    unsigned long long *vis, *fr, *hacc, *hbest;   // vis, fr, hacc: [n][2] (half h at 2u + h); hbest [nmulti][128]
    uint32_t *fbm;     // [3][nwords] frontier bitmaps (level L % 3)
    uint32_t *fullbm;  // [nwords] finished vertices
    uint32_t *tb;      // [2][nwords] "has a neighbour on the frontier" (push levels)
    uint32_t *fcnt;    // [3] vertices on the frontier of level L (mod 3); [3] vertices finished
    int64_t push_div;  // a level pushes first while frontier * push_div <= unfinished vertices
    int32_t *flag;
    unsigned long long *pnew;   // push-parent levels: [n] trees discovering the vertex (or null)
    unsigned long long *pbest;  // push-parent levels: [n][kPPTrees] best parent keys (~0 = none)
    int pp_from;                // first level that may use them
    uint32_t *mscnt;   // [128][kMsMaxBlocks] discoveries per tree per block (phase A)
    const uint64_t *tkey;
    uint32_t *qv, *parq, *pp;
    uint2 *rec, *crec;
    uint4 *irec;
    uint32_t *prec;
    uint64_t *lvl;
    uint32_t *vbase;
    int32_t *depth, *maxd;
    unsigned long long *prof;   // optional: globaltimer at phase boundaries (block 0)
};

__device__ __forceinline__ unsigned long long gtimer() {
    unsigned long long t;
    asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
    return t;
}
#define MS_PROF(slot)                                                        \
    do {                                                                     \
        if (P.prof && blockIdx.x == 0 && tid == 0 && L < 256)                \
            P.prof[(size_t)L * 4 + (slot)] = gtimer();                       \
    } while (0)

constexpr int kMsWarps = kBlock / 32;

__device__ __forceinline__ uint32_t warp_incl_scan32(uint32_t v) {
    const int lane = threadIdx.x & 31;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
        const uint32_t y = __shfl_up_sync(0xFFFFFFFFu, v, d);
        if (lane >= d) v += y;
    }
    return v;
}

__device__ __forceinline__ unsigned long long warp_or64(unsigned long long v) {
#pragma unroll
    for (int d = 16; d; d >>= 1) v |= __shfl_xor_sync(0xFFFFFFFFu, v, d);
    return v;
}

__device__ __forceinline__ bool bm_test(const uint32_t *bm, uint32_t u) {
    return (__ldcg(bm + (u >> 5)) >> (u & 31)) & 1u;
}

// the two halves of a vertex's 128-bit tree mask
struct W2 {
    unsigned long long a, b;   // trees 0-63, 64-127
};
// S = words per vertex: 2 (batches of 65..128 trees, interleaved halves) or 1
// (<= 64 trees: the round-1 layout, 8-byte loads)
template <int S>
__device__ __forceinline__ W2 ld2(const unsigned long long *p) {
    if constexpr (S == 1) {
        return W2{__ldcg(p), 0ull};
    } else {
        const uint4 v = __ldcg(reinterpret_cast<const uint4 *>(p));
        return W2{(unsigned long long)v.x | ((unsigned long long)v.y << 32),
                  (unsigned long long)v.z | ((unsigned long long)v.w << 32)};
    }
}
template <int S>
__device__ __forceinline__ void st2(unsigned long long *p, W2 w) {
    if constexpr (S == 1) {
        *p = w.a;
    } else {
        *reinterpret_cast<uint4 *>(p) = make_uint4((uint32_t)w.a, (uint32_t)(w.a >> 32), (uint32_t)w.b,
                                                   (uint32_t)(w.b >> 32));
    }
}

// half h of the frontier word of u (0 unless u is on the current level in
// some tree)
template <int S>
__device__ __forceinline__ unsigned long long fr_word(const unsigned long long *F, const uint32_t *bm,
                                                      uint32_t u, int h) {
    return bm_test(bm, u) ? __ldcg(F + S * (size_t)u + h) : 0ull;
}
// both halves (one 16-byte load when S = 2)
template <int S>
__device__ __forceinline__ W2 fr_word2(const unsigned long long *F, const uint32_t *bm, uint32_t u) {
    return bm_test(bm, u) ? ld2<S>(F + S * (size_t)u) : W2{0ull, 0ull};
}

// level-(L+1) entry `pos` of tree t: the vertex and its parent | neg << 31,
// both as internal (degree-sorted) ids -- the index space of the labelling
// passes and the walk.  Keys and `par` carry the parent's original id (the
// min-hash rule R4 is defined on original ids), translated here.
__device__ __forceinline__ void ms_emit(const MsParams &P, int t, uint32_t pos, uint32_t vi,
                                        unsigned long long key) {
    const size_t o = (size_t)t * P.n + pos;
    P.qv[o] = vi;
    P.parq[o] = __ldg(P.brank + ((uint32_t)(key >> 1) & kIdMask)) | ((uint32_t)key << 31);
}

__device__ __forceinline__ void ms_emit_par(const MsParams &P, int t, uint32_t pos, uint32_t vi,
                                            uint32_t par) {
    const size_t o = (size_t)t * P.n + pos;
    P.qv[o] = vi;
    P.parq[o] = __ldg(P.brank + (par & kIdMask)) | (par & kNegBit);
}

// OR of the frontier words over the slots [s0, s1) (one warp, lanes stride)
template <int S>
__device__ __forceinline__ W2 ms_chunk_or(const MsParams &P, const unsigned long long *F,
                                          const uint32_t *bm, uint32_t s0, uint32_t s1) {
    const int lane = threadIdx.x & 31;
    W2 acc{0ull, 0ull};
    uint32_t j = s0 + lane;
    for (; j + 96 < s1; j += 128) {
        const uint32_t a0 = __ldg(P.badj + j) & kIdMask, a1 = __ldg(P.badj + j + 32) & kIdMask;
        const uint32_t a2 = __ldg(P.badj + j + 64) & kIdMask, a3 = __ldg(P.badj + j + 96) & kIdMask;
        const W2 w0 = fr_word2<S>(F, bm, a0), w1 = fr_word2<S>(F, bm, a1);
        const W2 w2 = fr_word2<S>(F, bm, a2), w3 = fr_word2<S>(F, bm, a3);
        acc.a |= w0.a | w1.a | w2.a | w3.a;
        acc.b |= w0.b | w1.b | w2.b | w3.b;
    }
    for (; j < s1; j += 32) {
        const W2 w = fr_word2<S>(F, bm, __ldg(P.badj + j) & kIdMask);
        acc.a |= w.a;
        acc.b |= w.b;
    }
    return W2{warp_or64(acc.a), warp_or64(acc.b)};
}

// 64-bit warp minimum as two 32-bit redux.sync reductions (lexicographic:
// the high words, then the low words of the lanes holding the high minimum)
__device__ __forceinline__ unsigned long long warp_min64(unsigned long long v) {
    const uint32_t hi = (uint32_t)(v >> 32);
    const uint32_t mh = __reduce_min_sync(0xFFFFFFFFu, hi);
    const uint32_t ml = __reduce_min_sync(0xFFFFFFFFu, hi == mh ? (uint32_t)v : 0xFFFFFFFFu);
    return ((unsigned long long)mh << 32) | ml;
}

// per-warp scratch of the parent pass (dynamic shared memory)
#ifndef GB_MS_MULTICAP
#define GB_MS_MULTICAP 512
#endif
#ifndef GB_MS_MINBLOCKS
#define GB_MS_MINBLOCKS 4
#endif
constexpr int kMultiCap = GB_MS_MULTICAP;   // multi-candidate pairs per round
struct WarpScratch {
    uint32_t ml[kMultiCap];              // multi-candidate pairs: src << 14 | tree << 8 | slot mask
    unsigned long long pk[3][32];        // parent slot index k of (vertex lane, tree), bit-planes
    uint32_t lo[kLight][32];             // candidate neighbour (original id) | neg << 31 (hashing)
    uint32_t li[kLight][32];             // the same neighbour as an internal id | neg << 31 (output)
    uint32_t ow[32];                     // original id of each lane's vertex
    uint32_t iv[32];                     // internal id of each lane's vertex (emission)
    unsigned long long best[64];         // item parents: best key per tree (of the half)
};
constexpr size_t kMsSmem = sizeof(WarpScratch) * kMsWarps;

__device__ __forceinline__ uint32_t key_to_par(unsigned long long key) {
    return ((uint32_t)(key >> 1) & kIdMask) | ((uint32_t)key << 31);
}

// 32 x 32 bit-matrix transpose across the warp: lane r holds row r (bit c =
// M[r][c]); afterwards lane c holds column c (bit r = M[r][c]).  Five rounds
// of off-diagonal block swaps.
__device__ __forceinline__ uint32_t transpose32(uint32_t x) {
    const int lane = threadIdx.x & 31;
#pragma unroll
    for (int sh = 16; sh; sh >>= 1) {
        const uint32_t m = sh == 16 ? 0x0000FFFFu : sh == 8 ? 0x00FF00FFu : sh == 4 ? 0x0F0F0F0Fu
                         : sh == 2 ? 0x33333333u : 0x55555555u;
        const uint32_t y = __shfl_xor_sync(0xFFFFFFFFu, x, sh);
        x = (lane & sh) ? ((x & ~m) | ((y & ~m) >> sh)) : ((x & m) | ((y & m) << sh));
    }
    return x;
}

// parents of the light vertices queued by a warp (lane l: internal id i,
// valid if `act`) in the trees each discovered on this level (F_{L+1}[i]).
// Per lane, c[k] = the trees in which neighbour k is one level up.  A tree
// with a single candidate takes it: its slot index k goes into three
// bit-planes (pk[j] bit t = bit j of k) with three ORs per neighbour, no
// per-tree loop.  The (vertex, tree) pairs with several candidates are listed
// and hashed one per lane (the min-hash rule, reading R4); the winner's k is
// OR-ed into the planes.  Emission is transposed: the warp's 32 discovery
// words (vertex x tree bits) are transposed so that lane t holds, for trees
// t and t + 32, the mask of vertices to append; it reserves its run of the
// tree's level list with one shared-memory add and writes its entries.
// Half h of the 128 trees (trees 64h .. 64h + 63; s_tk, s_base and s_pos
// point at the half's first tree).
template <int S>
__device__ __forceinline__ void ms_light_parents(const MsParams &P, const unsigned long long *F,
                                                 const unsigned long long *Nx, const uint32_t *bm,
                                                 uint32_t i, bool act, const uint64_t *s_tk,
                                                 const uint32_t *s_base, uint32_t *s_pos, WarpScratch &W,
                                                 int half) {
    const int lane = threadIdx.x & 31;
    unsigned long long nw = 0, s2m = 0;   // discovered trees / those with >= 2 candidates
    unsigned long long c[kLight];
    uint32_t ow = 0;
    if (act) nw = __ldcg(Nx + S * (size_t)i + half);
    if (!__any_sync(0xFFFFFFFFu, nw != 0)) return;   // nothing in this half
    if (act) {
        const uint32_t rs = __ldg(P.brow + i);
        const uint32_t deg = __ldg(P.brow + i + 1) - rs;
        ow = __ldg(P.bord + i);
        unsigned long long s1m = 0;
#pragma unroll
        for (int k = 0; k < kLight; k++) {
            c[k] = 0;
            if (k < (int)deg) {
                const uint32_t a = __ldg(P.badj + rs + k);
                c[k] = fr_word<S>(F, bm, a & kIdMask, half) & nw;
                if (c[k]) {
                    W.lo[k][lane] = __ldg(P.borig + rs + k) | (a & kNegBit);
                    W.li[k][lane] = a;
                }
                s2m |= s1m & c[k];
                s1m |= c[k];
            }
        }
    } else {
#pragma unroll
        for (int k = 0; k < kLight; k++) c[k] = 0;
    }
    W.ow[lane] = ow;
    W.iv[lane] = i;
    {   // slot-index planes of the single-candidate trees
        const unsigned long long sm = ~s2m;
        unsigned long long p0 = 0, p1 = 0, p2 = 0;
#pragma unroll
        for (int k = 0; k < kLight; k++) {
            const unsigned long long ck = c[k] & sm;
            if (k & 1) p0 |= ck;
            if (k & 2) p1 |= ck;
            if (k & 4) p2 |= ck;
        }
        W.pk[0][lane] = p0;
        W.pk[1][lane] = p1;
        W.pk[2][lane] = p2;
    }
    // several candidates: listed pairs, hashed one per lane; the winning slot
    // index goes into the planes
    const uint32_t cnt = (uint32_t)__popcll(s2m);
    const uint32_t incl = warp_incl_scan32(cnt);
    const uint32_t total = __shfl_sync(0xFFFFFFFFu, incl, 31);
    for (uint32_t r0 = 0; r0 < total; r0 += kMultiCap) {
        uint32_t off = incl - cnt;
        if (total <= kMultiCap) {
            // one round (the common case): no bounds to check
            for (unsigned long long m = s2m; m; m &= m - 1) {
                const int t = __ffsll((long long)m) - 1;
                uint32_t km = 0;
#pragma unroll
                for (int k = 0; k < kLight; k++) km |= (uint32_t)((c[k] >> t) & 1ull) << k;
                W.ml[off++] = ((uint32_t)lane << 14) | ((uint32_t)t << 8) | km;
            }
        } else {
            for (unsigned long long m = s2m; m; m &= m - 1) {
                if (off >= r0 + kMultiCap) break;
                if (off >= r0) {
                    const int t = __ffsll((long long)m) - 1;
                    uint32_t km = 0;
#pragma unroll
                    for (int k = 0; k < kLight; k++) km |= (uint32_t)((c[k] >> t) & 1ull) << k;
                    W.ml[off - r0] = ((uint32_t)lane << 14) | ((uint32_t)t << 8) | km;
                }
                off++;
            }
        }
        __syncwarp();
        const uint32_t nr = min(total - r0, (uint32_t)kMultiCap);
        for (uint32_t p = lane; p < nr; p += 32) {
            const uint32_t e = W.ml[p];
            const uint32_t src = e >> 14;
            const int t = (int)((e >> 8) & 63);
            const uint32_t o_w = W.ow[src];
            const uint64_t tk = s_tk[t];
            unsigned long long best = ~0ull;
            uint32_t bk = 0;
            for (uint32_t km = e & 0xFFu; km; km &= km - 1) {
                const uint32_t k = __ffs(km) - 1;
                const uint32_t o = W.lo[k][src];
                const unsigned long long key = parent_key(tk, o & kIdMask, o_w, o >> 31);
                if (key < best) { best = key; bk = k; }
            }
            // 32-bit shared atomics on the plane half holding bit t (the
            // 64-bit ones compile to compare-and-swap loops)
            const uint32_t bit = 1u << (t & 31), half = (uint32_t)t >> 5;
            if (bk & 1) atomicOr(reinterpret_cast<uint32_t *>(&W.pk[0][src]) + half, bit);
            if (bk & 2) atomicOr(reinterpret_cast<uint32_t *>(&W.pk[1][src]) + half, bit);
            if (bk & 4) atomicOr(reinterpret_cast<uint32_t *>(&W.pk[2][src]) + half, bit);
        }
        __syncwarp();
    }
    __syncwarp();   // planes of every lane complete
    // emission: one shared-memory reservation per tree (lane t reserves the
    // runs of trees t and t + 32, sized by the transposed discovery words);
    // lane t then lists its trees' (vertex lane, rank) pairs tree-major in
    // shared memory, and the warp writes 32 listed entries per round, one per
    // lane: consecutive lanes fill consecutive positions of a tree's level
    // list, and the rounds number the pairs, not the trees
    const uint32_t nlo = transpose32((uint32_t)nw);
    const uint32_t nhi = transpose32((uint32_t)(nw >> 32));
    uint32_t blo = 0, bhi = 0;
    if (nlo) blo = s_base[lane] + atomicAdd(&s_pos[lane], (uint32_t)__popc(nlo));
    if (nhi) bhi = s_base[lane + 32] + atomicAdd(&s_pos[lane + 32], (uint32_t)__popc(nhi));
    uint32_t *sb = reinterpret_cast<uint32_t *>(W.best);   // list start per tree of the half
    sb[lane] = blo;
    sb[lane + 32] = bhi;
    uint16_t *el = reinterpret_cast<uint16_t *>(W.ml);     // vertex lane | tree << 5 | rank << 11
    constexpr uint32_t kCap = 2 * kMultiCap;
    const uint32_t ne = (uint32_t)(__popc(nlo) + __popc(nhi));
    const uint32_t eincl = warp_incl_scan32(ne);
    const uint32_t etot = __shfl_sync(0xFFFFFFFFu, eincl, 31);
    for (uint32_t r0 = 0; r0 < etot; r0 += kCap) {
        uint32_t off = eincl - ne;
        if (etot <= kCap) {
            // one round (the common case): no bounds to check
            uint16_t *q = el + off;
            uint32_t v = (lane << 5);
            for (uint32_t m = nlo; m; m &= m - 1, v += 1u << 11) *q++ = (uint16_t)(v | (__ffs(m) - 1));
            v = ((lane + 32) << 5);
            for (uint32_t m = nhi; m; m &= m - 1, v += 1u << 11) *q++ = (uint16_t)(v | (__ffs(m) - 1));
        } else {
            uint32_t r = 0;
            for (uint32_t m = nlo; m && off < r0 + kCap; m &= m - 1, r++, off++)
                if (off >= r0) el[off - r0] = (uint16_t)((__ffs(m) - 1) | (lane << 5) | (r << 11));
            r = 0;
            for (uint32_t m = nhi; m && off < r0 + kCap; m &= m - 1, r++, off++)
                if (off >= r0) el[off - r0] = (uint16_t)((__ffs(m) - 1) | ((lane + 32) << 5) | (r << 11));
        }
        __syncwarp();
        const uint32_t nr = min(etot - r0, kCap);
        for (uint32_t p = lane; p < nr; p += 32) {
            const uint32_t e = el[p];
            const uint32_t src = e & 31u, t = (e >> 5) & 63u;
            const uint32_t k = (uint32_t)((W.pk[0][src] >> t) & 1ull) | ((uint32_t)((W.pk[1][src] >> t) & 1ull) << 1) |
                               ((uint32_t)((W.pk[2][src] >> t) & 1ull) << 2);
            const size_t o = (size_t)(t + 64 * half) * P.n + sb[t] + (e >> 11);
            P.qv[o] = W.iv[src];
            P.parq[o] = W.li[k][src];
        }
        __syncwarp();
    }
}

// parents of an item vertex whose whole adjacency fits one window (degree
// <= 32; lane = slot) in the trees `want`: trees with one candidate take it,
// the (slot, tree) pairs of the others are hashed one per lane and reduced
// with shared-memory atomicMin.  Lanes l, l + 32 get trees l, l + 32.
template <int S>
__device__ __forceinline__ void ms_item_parents(const MsParams &P, const unsigned long long *F,
                                                const uint32_t *bm, uint32_t s0, uint32_t s1,
                                                unsigned long long want, uint32_t ow,
                                                const uint64_t *s_tk, WarpScratch &W,
                                                uint32_t &p0, uint32_t &p1, int h) {
    const int lane = threadIdx.x & 31;
    uint16_t *pl = reinterpret_cast<uint16_t *>(W.ml);   // <= 32 * 64 pairs fit kMultiCap * 2
    const uint32_t j = s0 + lane;
    unsigned long long f = 0;
    uint32_t o = 0;
    if (j < s1) {
        const uint32_t a = __ldg(P.badj + j);
        f = fr_word<S>(F, bm, a & kIdMask, h) & want;
        if (f) o = __ldg(P.borig + j) | (a & kNegBit);
    }
    unsigned long long s1m = f, s2m = 0;   // trees with >= 1 / >= 2 candidates
#pragma unroll
    for (int d = 16; d; d >>= 1) {
        const unsigned long long o1 = __shfl_xor_sync(0xFFFFFFFFu, s1m, d);
        const unsigned long long o2 = __shfl_xor_sync(0xFFFFFFFFu, s2m, d);
        s2m |= o2 | (s1m & o1);
        s1m |= o1;
    }
    W.best[lane] = ~0ull;
    W.best[lane + 32] = ~0ull;
    W.lo[0][lane] = o;
    __syncwarp();
    for (unsigned long long m = f & ~s2m; m; m &= m - 1)
        W.best[__ffsll((long long)m) - 1] = ((unsigned long long)(o & kIdMask) << 1) | (o >> 31);
    const unsigned long long mm = f & s2m;
    const uint32_t cnt = (uint32_t)__popcll(mm);
    const uint32_t incl = warp_incl_scan32(cnt);
    const uint32_t total = __shfl_sync(0xFFFFFFFFu, incl, 31);
    constexpr uint32_t kCap = 2 * kMultiCap;
    for (uint32_t r0 = 0; r0 < total; r0 += kCap) {
        uint32_t off = incl - cnt;
        if (total <= kCap) {
            // one round (the common case): no bounds to check
            for (unsigned long long m = mm; m; m &= m - 1)
                pl[off++] = (uint16_t)((lane << 6) | (__ffsll((long long)m) - 1));
        } else {
            for (unsigned long long m = mm; m; m &= m - 1) {
                if (off >= r0 + kCap) break;
                if (off >= r0) pl[off - r0] = (uint16_t)((lane << 6) | (__ffsll((long long)m) - 1));
                off++;
            }
        }
        __syncwarp();
        const uint32_t nr = min(total - r0, kCap);
        for (uint32_t p = lane; p < nr; p += 32) {
            const uint32_t e = pl[p];
            const int t = (int)(e & 63);
            const uint32_t oo = W.lo[0][e >> 6];
            atomicMin(&W.best[t], parent_key(s_tk[t], oo & kIdMask, ow, oo >> 31));
        }
        __syncwarp();
    }
    p0 = key_to_par(W.best[lane]);
    p1 = key_to_par(W.best[lane + 32]);
    __syncwarp();
}

// Best parent keys of vertex ow over the slots [s0, s1) (a chunk of <= 256
// slots of a heavy vertex or a hub) for the trees in `want` (half h); lane l
// returns trees l (b0) and l + 32 (b1).  Per window of 32 slots (lane = slot)
// the (slot, tree) candidate pairs are listed tree-major in shared memory,
// hashed 32 at a time with every lane busy (the min-hash rule, reading R4),
// and reduced by a segmented warp minimum over the runs of equal trees; the
// run tails fold their minimum into the per-tree best of the chunk.
template <int S>
__device__ __forceinline__ void ms_chunk_keys(const MsParams &P, const unsigned long long *F,
                                              const uint32_t *bm, uint32_t s0, uint32_t s1,
                                              unsigned long long want, uint32_t ow, const uint64_t *s_tk,
                                              WarpScratch &W, unsigned long long &b0, unsigned long long &b1,
                                              int h) {
    const int lane = threadIdx.x & 31;
    const uint32_t lt = (1u << lane) - 1u;
    uint16_t *pl = reinterpret_cast<uint16_t *>(W.ml);   // 2 * kMultiCap pairs: lane << 6 | tree
    constexpr uint32_t kCap = 2 * kMultiCap;
    W.best[lane] = ~0ull;
    W.best[lane + 32] = ~0ull;
    __syncwarp();
    for (uint32_t base = s0; base < s1; base += 32) {
        const uint32_t j = base + lane;
        uint32_t o = 0;
        unsigned long long f = 0;
        if (j < s1) {
            const uint32_t a = __ldg(P.badj + j);
            f = fr_word<S>(F, bm, a & kIdMask, h) & want;
            if (f) o = __ldg(P.borig + j) | (a & kNegBit);
        }
        W.lo[0][lane] = o;
        unsigned long long rem = warp_or64(f);
        while (rem) {
            // list the pairs of as many trees as fit, tree-major
            uint32_t np = 0;
            for (; rem && np + 32 <= kCap; rem &= rem - 1) {
                const int t = __ffsll((long long)rem) - 1;
                const bool has = (f >> t) & 1ull;
                const uint32_t bal = __ballot_sync(0xFFFFFFFFu, has);
                if (has) pl[np + __popc(bal & lt)] = (uint16_t)((lane << 6) | t);
                np += __popc(bal);
            }
            __syncwarp();
            for (uint32_t r0 = 0; r0 < np; r0 += 32) {
                const uint32_t p = r0 + lane;
                const bool valid = p < np;
                const uint32_t e = valid ? pl[p] : 0u;
                const int t = valid ? (int)(e & 63) : 64 + lane;   // unique for idle lanes
                unsigned long long key = ~0ull;
                if (valid) {
                    const uint32_t oo = W.lo[0][e >> 6];
                    key = parent_key(s_tk[t], oo & kIdMask, ow, oo >> 31);
                }
                // segmented inclusive minimum over runs of equal t
                const int tprev = __shfl_up_sync(0xFFFFFFFFu, t, 1);
                const uint32_t starts = __ballot_sync(0xFFFFFFFFu, lane == 0 || tprev != t);
                const int leader = 31 - __clz(starts & (lt | (1u << lane)));
#pragma unroll
                for (int d = 1; d < 32; d <<= 1) {
                    const unsigned long long y = __shfl_up_sync(0xFFFFFFFFu, key, d);
                    if (lane - d >= leader) key = min(key, y);
                }
                const bool tail = lane == 31 || ((starts >> (lane + 1)) & 1u);
                if (valid && tail) W.best[t] = min(W.best[t], key);   // one tail per tree per round
                __syncwarp();
            }
        }
        __syncwarp();
    }
    b0 = W.best[lane];
    b1 = W.best[lane + 32];
    __syncwarp();
}

// position (0-based) of the r-th set bit of m
__device__ __forceinline__ int select_bit64(unsigned long long m, int r) {
    int pos = 0;
    uint32_t x = (uint32_t)m;
    int c = __popc(x);
    if (r >= c) { r -= c; x = (uint32_t)(m >> 32); pos = 32; }
    c = __popc(x & 0xFFFFu); if (r >= c) { r -= c; x >>= 16; pos += 16; }
    c = __popc(x & 0xFFu);   if (r >= c) { r -= c; x >>= 8;  pos += 8; }
    c = __popc(x & 0xFu);    if (r >= c) { r -= c; x >>= 4;  pos += 4; }
    c = __popc(x & 0x3u);    if (r >= c) { r -= c; x >>= 2;  pos += 2; }
    if (r >= (int)(x & 1u)) pos += 1;
    return pos;
}

// ---------------------------------------------------------------------------
// roots (reading R4): root of component C in tree b = C's vertices
// (ascending)[rkey(b, C) mod |C|]; level 0 of every tree
// ---------------------------------------------------------------------------
template <int S>
__global__ void k_ms_roots(MsParams P) {
    // single-vertex components (the isolated vertices, internal ids
    // [n - niso, n)): their one-vertex trees are identical in every tree --
    // reached in all trees at level 0, never on a frontier, labels pre =
    // coff[C], pi = 0, size 1 (read from the component table wherever needed)
    for (int64_t i = P.n - P.niso + blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < P.n;
         i += (int64_t)gridDim.x * blockDim.x) {
        st2<S>(P.vis + S * i, W2{P.full0, P.full1});
        if (!P.irec) {
            // layout 1 (walks 1, 2, option jump) reads pre-indexed records of
            // every vertex: the one-vertex trees' records, per tree
            const uint32_t pre = (uint32_t)P.coff[P.comp_i[i]];
            for (int b = 0; b < P.B; b++) {
                const size_t nb = (size_t)b * P.n;
                P.pp[nb + i] = pre;
                if (P.prec) P.prec[nb + pre] = pre;
                else P.rec[nb + pre] = make_uint2(pre, 1u);
                if (P.crec) P.crec[nb + pre] = make_uint2(0u, 0u);
            }
        }
    }
    // ... and finished from the start: their "finished" bits are set (the
    // discovery passes skip them) and counted once
    if (P.niso > 0) {
        const int64_t i0 = P.n - P.niso;
        for (int64_t w = (i0 >> 5) + blockIdx.x * (int64_t)blockDim.x + threadIdx.x; w < P.nwords;
             w += (int64_t)gridDim.x * blockDim.x) {
            uint32_t m = ~0u;
            if ((w << 5) < i0) m &= ~0u << (uint32_t)(i0 - (w << 5));
            if (((w + 1) << 5) > P.n) m &= ~0u >> (uint32_t)(((w + 1) << 5) - P.n);
            atomicOr(P.fullbm + w, m);
        }
        if (blockIdx.x == 0 && threadIdx.x == 0) P.fcnt[3] = (uint32_t)P.niso;
    }
    const int64_t total = (int64_t)P.B * P.nbig;
    for (int64_t x = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; x < total;
         x += (int64_t)gridDim.x * blockDim.x) {
        const int b = (int)(x / P.nbig);
        const int64_t C = P.bigc[x - (int64_t)b * P.nbig];
        const uint32_t sz = (uint32_t)(P.coff[C + 1] - P.coff[C]);
        const uint64_t rk = root_key(P.tkey[b], C);
        const uint32_t r = (uint32_t)P.cverts[P.coff[C] + (int64_t)(rk % sz)];
        const uint32_t ri = P.brank[r];
        const unsigned long long bit = 1ull << (b & 63);
        const int h = b >> 6;
        atomicOr(P.vis + S * (size_t)ri + h, bit);
        const size_t nb = (size_t)b * P.n;
        const unsigned long long old = atomicAdd((unsigned long long *)(P.lvl + b * P.ls), 1ull << 32);
        const uint32_t pos = (uint32_t)(old >> 32);
        P.qv[nb + pos] = ri;
        P.parq[nb + pos] = ri;
        atomicOr(P.fr + S * (size_t)ri + h, bit);
        atomicOr(P.fbm + (ri >> 5), 1u << (ri & 31));
    }
}

// push-parent levels: candidate (u -> x) of the frontier vertex u (trees fu,
// original id ou) through adjacency slot j (a = badj[j])
__device__ __forceinline__ void pp_push(const MsParams &P, unsigned long long fu, uint32_t ou,
                                        uint32_t a, uint32_t j, const uint64_t *s_tk) {
    const uint32_t x = a & kIdMask;
    const unsigned long long want = fu & ~__ldcg(P.vis + x);
    if (!want) return;
    atomicOr(P.pnew + x, want);
    const uint32_t ox = __ldg(P.borig + j);
    for (unsigned long long m = want; m; m &= m - 1) {
        const int t = __ffsll((long long)m) - 1;
        atomicMin(P.pbest + (size_t)x * kPPTrees + t, parent_key(s_tk[t], ou, ox, a >> 31));
    }
}

// push-parent levels: the entry of vertex i in tree t (its best key, then the
// slot is reset for the next use)
__device__ __forceinline__ void pp_emit(const MsParams &P, int t, uint32_t i, const uint32_t *s_base,
                                        uint32_t *s_pos) {
    unsigned long long *slot = P.pbest + (size_t)i * kPPTrees + t;
    const unsigned long long key = __ldcg(slot);
    *slot = ~0ull;
    ms_emit(P, t, s_base[t] + atomicAdd(&s_pos[t], 1u), i, key);
}

// ---------------------------------------------------------------------------
// the BFS: one cooperative kernel.  Per level L:
//   phase A  every block pulls over its tiles (static: tile k -> block
//            k mod grid): new(w), vis, F_{L+1}, the bitmaps; per-tree
//            discovery counts in shared memory, published per block;
//   -- grid barrier --
//   phase B  each block's offset in every tree's level-(L+1) list = the
//            counts of the blocks before it; the same tiles again: the
//            parents of the discoveries (light vertices: one (vertex, tree)
//            pair per lane), written to the level lists; hubs' partial minima;
//   -- grid barrier --
//   phase C  (only if a hub discovered something) hubs' parents appended,
//            then one more barrier.
// ---------------------------------------------------------------------------
template <int S>
__global__ void __launch_bounds__(kBlock, GB_MS_MINBLOCKS) k_msbfs(MsParams P) {
    cg::grid_group grid = cg::this_grid();
    __shared__ uint64_t s_tk[kMsBatch];
    __shared__ uint32_t s_cnt[kMsBatch], s_pos[kMsBatch], s_base[kMsBatch];
    __shared__ uint32_t s_vbase[kMsBatch], s_vb[kMsBatch];
    __shared__ int32_t s_depth[kMsBatch];
    __shared__ int s_more;
    extern __shared__ __align__(16) unsigned char s_dyn[];
    WarpScratch &W = reinterpret_cast<WarpScratch *>(s_dyn)[threadIdx.x >> 5];
    __shared__ uint32_t s_q[kMsWarps][64];           // discovered light vertices (phase B)
    uint32_t qn = 0;                                  // warp-uniform fill of s_q
    const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
    const int B = P.B;
    if (tid < kMsBatch) {
        s_tk[tid] = tid < B ? P.tkey[tid] : 0;
        s_cnt[tid] = 0;
        s_pos[tid] = 0;
        s_base[tid] = 0;
        s_vbase[tid] = 0;
        s_depth[tid] = 0;
    }
    const int64_t gtid = (int64_t)blockIdx.x * blockDim.x + tid;
    const int64_t gwarp = gtid >> 5;
    const int64_t nthr = (int64_t)gridDim.x * blockDim.x;
    const int64_t nwarps = nthr >> 5;
    const int64_t nit_tiles = (P.nitems + kMsWarps - 1) / kMsWarps;
    const int64_t l0 = P.nlight0 & ~31ll;   // light tiles start word-aligned
    const int64_t nl_tiles = (P.n - l0 + kBlock - 1) / kBlock;
    const int64_t ntiles = nit_tiles + nl_tiles;
    const W2 full{P.full0, P.full1};
    const uint32_t nblk = gridDim.x;
    __shared__ uint32_t s_fc, s_ff;
    for (int L = 0;; L++) {
        const unsigned long long *F = P.fr + (size_t)(L & 1) * S * P.n;
        unsigned long long *Nx = P.fr + (size_t)((L + 1) & 1) * S * P.n;
        const uint32_t *bm = P.fbm + (size_t)(L % 3) * P.nwords;
        uint32_t *nbm = P.fbm + (size_t)((L + 1) % 3) * P.nwords;
        uint32_t *cbm = P.fbm + (size_t)((L + 2) % 3) * P.nwords;   // free: cleared for L+2
        __syncthreads();
        if (tid < B) {
            const uint32_t c = (uint32_t)(__ldcg((const unsigned long long *)(P.lvl + tid * P.ls + L)) >> 32);
            s_vb[tid] = s_vbase[tid] + c;   // start of level L+1 in tree tid's list
            if (blockIdx.x == 0) P.vbase[tid * P.ls + L + 1] = s_vb[tid];
        }
        // words written with atomics next level (items, the boundary word)
        for (int64_t w = gtid; w < P.itemwords; w += nthr) cbm[w] = 0;
        if (tid == 0) { s_fc = 0; s_ff = 0; }
        if (blockIdx.x == 0 && tid == 0) P.fcnt[(L + 2) % 3] = 0;
        __syncthreads();
        // Direction optimisation: while the frontier is small (the first
        // levels), push from it first -- every frontier vertex marks its
        // neighbours in tbc -- so that the pull below reads the adjacency of
        // marked vertices only (nothing else can be discovered).  Heavy
        // vertices push through their work items (<= 256 slots per warp).
        // level 0: one root per tree in every component with >= 2 vertices
        const uint32_t fc = L == 0 ? (uint32_t)(((int64_t)B * P.nbig < P.n) ? (int64_t)B * P.nbig : P.n)
                                   : __ldcg(P.fcnt + L % 3);
        const int64_t unfinished = P.n - (int64_t)__ldcg(P.fcnt + 3);
        // batches that can take the push-parent path also push whenever the
        // frontier is small against the whole graph (the last levels, where
        // a pull still walks every tile for a few unfinished vertices)
        const bool ppcap = S == 1 && P.pbest != nullptr && B <= kPPTrees && L >= P.pp_from;
        const bool push = (int64_t)fc * P.push_div <= unfinished || (ppcap && (int64_t)fc * GB_PP_DIV <= P.n);
        // Push-parent levels (batches of <= 16 trees): the push itself
        // discovers -- new(x) |= F_L(u) & ~vis(x) -- and selects the parents:
        // every (frontier vertex u, neighbour x, tree t) candidate takes part
        // in an atomicMin of parent_key(t, u, x) (reading R4: the same
        // minimum over the same candidates), so phases A and B read one word
        // per marked vertex instead of scanning its adjacency (on RMAT the
        // marked hubs hold millions of slots)
        const bool pp = ppcap && push;
        uint32_t *tbc = P.tb + (size_t)(L & 1) * P.nwords;
        if (push) {
            // the work items of frontier vertices: for batches of <= 16 trees
            // a warp tests 32 items at a time and walks the chunks of those
            // on the frontier (RMAT: a few frontier vertices among millions of
            // hub chunks); larger batches take one item per warp and round
            // (measured ~2 % faster on C2 / C4, whose push levels are the first)
            if (!(S == 1 && B <= kPPTrees)) {
                for (int64_t k = gwarp; k < P.nitems; k += nwarps) {
                    const uint2 it = __ldg(P.items + k);
                    if (!bm_test(bm, it.x)) continue;
                    const uint32_t s1 = min(it.y + (uint32_t)kChunk, __ldg(P.brow + it.x + 1));
                    for (uint32_t j = it.y + lane; j < s1; j += 32) {
                        const uint32_t x = __ldg(P.badj + j) & kIdMask;
                        atomicOr(tbc + (x >> 5), 1u << (x & 31));
                    }
                }
            } else
            for (int64_t k0 = gwarp * 32; k0 < P.nitems; k0 += nwarps * 32) {
                const int64_t kk = k0 + lane;
                const uint2 itl = kk < P.nitems ? __ldg(P.items + kk) : make_uint2(0u, 0u);
                for (uint32_t fm = __ballot_sync(0xFFFFFFFFu, kk < P.nitems && bm_test(bm, itl.x)); fm;
                     fm &= fm - 1) {
                    const int src = __ffs(fm) - 1;
                    const uint2 it = make_uint2(__shfl_sync(0xFFFFFFFFu, itl.x, src),
                                                __shfl_sync(0xFFFFFFFFu, itl.y, src));
                    const uint32_t s1 = min(it.y + (uint32_t)kChunk, __ldg(P.brow + it.x + 1));
                    const unsigned long long fu = pp ? __ldcg(F + it.x) : 0ull;
                    const uint32_t ou = pp ? __ldg(P.bord + it.x) : 0u;
                    for (uint32_t j = it.y + lane; j < s1; j += 32) {
                        const uint32_t a = __ldg(P.badj + j), x = a & kIdMask;
                        atomicOr(tbc + (x >> 5), 1u << (x & 31));
                        if (pp) pp_push(P, fu, ou, a, j, s_tk);
                    }
                }
            }
            for (int64_t w = (P.nlight0 >> 5) + gwarp; w < P.nwords; w += nwarps) {
                uint32_t word = __ldcg(bm + w);
                if ((w << 5) < P.nlight0) word &= ~0u << (uint32_t)(P.nlight0 - (w << 5));   // item vertices done above
                if (!((word >> lane) & 1u)) continue;
                const uint32_t u = (uint32_t)(w * 32 + lane);
                const uint32_t rs = __ldg(P.brow + u), re = __ldg(P.brow + u + 1);
                const unsigned long long fu = pp ? __ldcg(F + u) : 0ull;
                const uint32_t ou = pp ? __ldg(P.bord + u) : 0u;
                for (uint32_t j = rs; j < re; j++) {
                    const uint32_t a = __ldg(P.badj + j), x = a & kIdMask;
                    atomicOr(tbc + (x >> 5), 1u << (x & 31));
                    if (pp) pp_push(P, fu, ou, a, j, s_tk);
                }
            }
            grid.sync();
        }
        MS_PROF(0);
        // ---------------- phase A: discoveries --------------------------------
        // per-lane discovery counts of trees lane, lane + 32, lane + 64, lane + 96
        // (summed over the warp's tiles, added to the block's table once)
        uint32_t a_cnt0 = 0, a_cnt1 = 0, a_cnt2 = 0, a_cnt3 = 0;
        if (pp) {
            // push-parent level: every marked vertex reads its discoveries
            // from pnew; a warp owns whole 32-vertex words (the same static
            // mapping in phase B), so no hub chunk or adjacency is visited
            for (int64_t w = (int64_t)blockIdx.x * kMsWarps + wid; w < P.nwords;
                 w += (int64_t)gridDim.x * kMsWarps) {
                const uint32_t i = (uint32_t)(w * 32 + lane);
                const uint32_t tw = __ldcg(tbc + w), fw = __ldcg(P.fullbm + w);
                unsigned long long nwv = 0;
                bool nowfull = false;
                if ((int64_t)i < P.n && ((tw >> lane) & 1u) && !((fw >> lane) & 1u)) {
                    const unsigned long long pn = __ldcg(P.pnew + i);
                    if (pn) {
                        P.pnew[i] = 0ull;
                        const unsigned long long vis = __ldcg(P.vis + S * (size_t)i);
                        nwv = pn & ~vis;
                        if (nwv) {
                            const unsigned long long nv = vis | nwv;
                            P.vis[S * (size_t)i] = nv;
                            Nx[S * (size_t)i] = nwv;
                            nowfull = nv == full.a;
                        }
                    }
                }
                const uint32_t fb = __ballot_sync(0xFFFFFFFFu, nwv != 0);
                if (fb) a_cnt0 += __popc(transpose32((uint32_t)nwv));   // <= 16 trees
                const uint32_t nf = __ballot_sync(0xFFFFFFFFu, nowfull);
                if (lane == 0) {
                    if (fb) atomicAdd(&s_fc, (uint32_t)__popc(fb));
                    if (nf) atomicAdd(&s_ff, (uint32_t)__popc(nf));
                    nbm[w] = fb;
                    if (nf) P.fullbm[w] = fw | nf;
                }
            }
        } else
        for (int64_t tile = blockIdx.x; tile < ntiles; tile += gridDim.x) {
            if (tile < nit_tiles) {
                const int64_t k = tile * kMsWarps + wid;
                if (k < P.nitems) {
                    const uint2 it = __ldg(P.items + k);
                    const uint32_t i = it.x, s0 = it.y;
                    if (bm_test(P.fullbm, i)) continue;
                    if (push && !bm_test(tbc, i)) continue;
                    const uint32_t s1 = min(s0 + (uint32_t)kChunk, __ldg(P.brow + i + 1));
                    const bool multi = k < P.nmulti_items;
                    const W2 vis = ld2<S>(P.vis + S * (size_t)i);
                    W2 part = ms_chunk_or<S>(P, F, bm, s0, s1);
                    part.a &= ~vis.a;
                    part.b &= ~vis.b;
                    if (multi) {
                        if ((part.a | part.b) && lane == 0) {
                            if (part.a) atomicOr(P.hacc + S * (size_t)i, part.a);
                            if (part.b) atomicOr(P.hacc + S * (size_t)i + 1, part.b);
                            P.flag[L & 1] = 1;
                        }
                    } else if (part.a | part.b) {
                        if (lane == 0) {
                            st2<S>(Nx + S * (size_t)i, part);
                            const W2 nv{vis.a | part.a, vis.b | part.b};
                            st2<S>(P.vis + S * (size_t)i, nv);
                            atomicOr(nbm + (i >> 5), 1u << (i & 31));
                            if (nv.a == full.a && nv.b == full.b) {
                                atomicOr(P.fullbm + (i >> 5), 1u << (i & 31));
                                atomicAdd(&s_ff, 1u);
                            }
                        }
                        a_cnt0 += (uint32_t)(part.a >> lane) & 1u;
                        a_cnt1 += (uint32_t)(part.a >> (lane + 32)) & 1u;
                        a_cnt2 += (uint32_t)(part.b >> lane) & 1u;
                        a_cnt3 += (uint32_t)(part.b >> (lane + 32)) & 1u;
                        if (lane == 0) atomicAdd(&s_fc, 1u);
                    }
                }
            } else {
                const int64_t v0 = l0 + (tile - nit_tiles) * kBlock + wid * 32;   // this warp's word
                if (v0 >= P.n) continue;
                const uint32_t i = (uint32_t)(v0 + lane);
                const bool mine = (int64_t)i < P.n && (int64_t)i >= P.nlight0;
                const uint32_t fw = __ldcg(P.fullbm + (v0 >> 5));
                const uint32_t tw = push ? __ldcg(tbc + (v0 >> 5)) : ~0u;
                W2 nw{0ull, 0ull};
                bool nowfull = false;
                if (mine && !((fw >> lane) & 1u) && ((tw >> lane) & 1u)) {
                    const W2 vis = ld2<S>(P.vis + S * (size_t)i);
                    const uint32_t rs = __ldg(P.brow + i);
                    const uint32_t deg = __ldg(P.brow + i + 1) - rs;
                    W2 acc{0ull, 0ull};
#pragma unroll
                    for (int k = 0; k < kLight; k++)
                        if (k < (int)deg) {
                            const W2 w = fr_word2<S>(F, bm, __ldg(P.badj + rs + k) & kIdMask);
                            acc.a |= w.a;
                            acc.b |= w.b;
                        }
                    nw = W2{acc.a & ~vis.a, acc.b & ~vis.b};
                    const W2 nv{vis.a | nw.a, vis.b | nw.b};
                    if (nw.a | nw.b) {
                        st2<S>(P.vis + S * (size_t)i, nv);
                        st2<S>(Nx + S * (size_t)i, nw);
                    }
                    nowfull = nv.a == full.a && nv.b == full.b;
                }
                const uint32_t fb = __ballot_sync(0xFFFFFFFFu, (nw.a | nw.b) != 0);
                if (fb) {
                    // per-tree discovery counts: transpose the warp's 32 words
                    // so that lane t counts trees t, t + 32, t + 64, t + 96
                    const uint32_t c0 = __popc(transpose32((uint32_t)nw.a));
                    const uint32_t c1 = __popc(transpose32((uint32_t)(nw.a >> 32)));
                    a_cnt0 += c0;
                    a_cnt1 += c1;
                    if (__any_sync(0xFFFFFFFFu, nw.b != 0)) {
                        const uint32_t c2 = __popc(transpose32((uint32_t)nw.b));
                        const uint32_t c3 = __popc(transpose32((uint32_t)(nw.b >> 32)));
                        a_cnt2 += c2;
                        a_cnt3 += c3;
                    }
                }
                const uint32_t nf = __ballot_sync(0xFFFFFFFFu, nowfull);
                if (lane == 0 && fb) atomicAdd(&s_fc, (uint32_t)__popc(fb));
                if (lane == 0 && nf) atomicAdd(&s_ff, (uint32_t)__popc(nf));
                if (lane == 0) {
                    if (v0 >= P.nlight0) {
                        nbm[v0 >> 5] = fb;
                        if (nf) P.fullbm[v0 >> 5] = fw | nf;
                    } else {   // boundary word shared with item vertices
                        if (fb) atomicOr(nbm + (v0 >> 5), fb);
                        if (nf) atomicOr(P.fullbm + (v0 >> 5), nf);
                    }
                }
            }
        }
        if (a_cnt0) atomicAdd(&s_cnt[lane], a_cnt0);
        if (a_cnt1) atomicAdd(&s_cnt[lane + 32], a_cnt1);
        if (a_cnt2) atomicAdd(&s_cnt[lane + 64], a_cnt2);
        if (a_cnt3) atomicAdd(&s_cnt[lane + 96], a_cnt3);
        __syncthreads();
        if (tid < kMsBatch) {
            P.mscnt[(size_t)tid * kMsMaxBlocks + blockIdx.x] = s_cnt[tid];
            s_cnt[tid] = 0;
        }
        if (tid == 0 && s_fc) atomicAdd(P.fcnt + (L + 1) % 3, s_fc);
        if (tid == 0 && s_ff) atomicAdd(P.fcnt + 3, s_ff);
        grid.sync();
        MS_PROF(1);
        // ---------------- phase B: parents ------------------------------------
        // this block's offsets: counts of the blocks before it (warp per tree)
        for (int t = wid; t < B; t += kMsWarps) {
            const uint32_t *row = P.mscnt + (size_t)t * kMsMaxBlocks;
            uint32_t before = 0, all = 0;
            // eight independent loads in flight per lane (the counts of up to
            // 2048 blocks: a dependent chain here was ~40 us per level)
            for (uint32_t b0 = 0; b0 < nblk; b0 += 256) {
                uint32_t c[8];
#pragma unroll
                for (int k = 0; k < 8; k++) {
                    const uint32_t b = b0 + 32 * k + lane;
                    c[k] = b < nblk ? __ldcg(row + b) : 0u;
                }
#pragma unroll
                for (int k = 0; k < 8; k++) {
                    all += c[k];
                    if (b0 + 32 * k + lane < blockIdx.x) before += c[k];
                }
            }
#pragma unroll
            for (int d = 16; d; d >>= 1) {
                before += __shfl_xor_sync(0xFFFFFFFFu, before, d);
                all += __shfl_xor_sync(0xFFFFFFFFu, all, d);
            }
            if (lane == 0) {
                s_base[t] = s_vb[t] + before;
                s_pos[t] = 0;
                if (blockIdx.x == 0) P.lvl[t * P.ls + L + 1] = (uint64_t)all << 32;
            }
        }
        __syncthreads();
        if (pp) {
            for (int64_t w = (int64_t)blockIdx.x * kMsWarps + wid; w < P.nwords;
                 w += (int64_t)gridDim.x * kMsWarps) {
                const uint32_t fb = __ldcg(nbm + w);
                if ((fb >> lane) & 1u) {
                    const uint32_t i = (uint32_t)(w * 32 + lane);
                    for (unsigned long long m = __ldcg(Nx + S * (size_t)i); m; m &= m - 1)
                        pp_emit(P, __ffsll((long long)m) - 1, i, s_base, s_pos);
                }
            }
        } else
        for (int64_t tile = blockIdx.x; tile < ntiles; tile += gridDim.x) {
            if (tile < nit_tiles) {
                const int64_t k = tile * kMsWarps + wid;
                if (k < P.nitems && k >= P.nmulti_items) {
                    const uint2 it = __ldg(P.items + k);
                    const uint32_t i = it.x;
                    if (!bm_test(nbm, i)) continue;
                    const W2 nw2 = ld2<S>(Nx + S * (size_t)i);
                    const uint32_t s1 = min(it.y + (uint32_t)kChunk, __ldg(P.brow + i + 1));
                    const uint32_t ow = __ldg(P.bord + i);
                    for (int h = 0; h < 2; h++) {
                        const unsigned long long nw = h ? nw2.b : nw2.a;
                        if (!nw) continue;   // warp-uniform
                        const int tb = 64 * h;
                        uint32_t p0, p1;
                        if (s1 - it.y <= 32) {
                            ms_item_parents<S>(P, F, bm, it.y, s1, nw, ow, s_tk + tb, W, p0, p1, h);
                        } else {
                            unsigned long long b0, b1;
                            ms_chunk_keys<S>(P, F, bm, it.y, s1, nw, ow, s_tk + tb, W, b0, b1, h);
                            p0 = key_to_par(b0);
                            p1 = key_to_par(b1);
                        }
                        if ((nw >> lane) & 1ull)
                            ms_emit_par(P, tb + lane, s_base[tb + lane] + atomicAdd(&s_pos[tb + lane], 1u), i, p0);
                        if ((nw >> (lane + 32)) & 1ull)
                            ms_emit_par(P, tb + lane + 32,
                                        s_base[tb + lane + 32] + atomicAdd(&s_pos[tb + lane + 32], 1u), i, p1);
                    }
                }
            } else {
                // light vertices: the warp queues its discovered vertices and
                // processes them 32 at a time (one per lane)
                const int64_t v0 = l0 + (tile - nit_tiles) * kBlock + wid * 32;
                if (v0 >= P.n) continue;
                uint32_t fb = __ldcg(nbm + (v0 >> 5));
                if (v0 < P.nlight0) fb &= ~0u << (uint32_t)(P.nlight0 - v0);   // item lanes are not ours
                if (!fb) continue;
                if ((fb >> lane) & 1u) s_q[wid][qn + __popc(fb & ((1u << lane) - 1u))] = (uint32_t)(v0 + lane);
                qn += __popc(fb);
                if (qn >= 32) {
                    __syncwarp();
                    const uint32_t i = s_q[wid][lane];
                    const uint32_t rest = s_q[wid][32 + lane];
                    __syncwarp();
                    s_q[wid][lane] = rest;
                    qn -= 32;
                    ms_light_parents<S>(P, F, Nx, bm, i, true, s_tk, s_base, s_pos, W, 0);
                    if (B > 64) ms_light_parents<S>(P, F, Nx, bm, i, true, s_tk + 64, s_base + 64, s_pos + 64, W, 1);
                }
            }
        }
        __syncwarp();
        if (qn) {
            ms_light_parents<S>(P, F, Nx, bm, s_q[wid][lane], lane < qn, s_tk, s_base, s_pos, W, 0);
            if (B > 64)
                ms_light_parents<S>(P, F, Nx, bm, s_q[wid][lane], lane < qn, s_tk + 64, s_base + 64, s_pos + 64, W, 1);
        }
        qn = 0;
        // the push bitmap of level L + 1 starts empty
        for (int64_t w = gtid; w < P.nwords; w += nthr) P.tb[(size_t)((L + 1) & 1) * P.nwords + w] = 0;
        // hubs: partial minima of every chunk
        const bool multi = P.nmulti_items > 0 && *(volatile int32_t *)(P.flag + (L & 1)) != 0;
        if (multi) {
            for (int64_t k = gwarp; k < P.nmulti_items; k += nwarps) {
                const uint2 it = __ldg(P.items + k);
                const uint32_t hi = it.x;
                const W2 want2 = ld2<S>(P.hacc + S * (size_t)hi);
                if (!(want2.a | want2.b)) continue;
                const uint32_t e1 = min(it.y + (uint32_t)kChunk, __ldg(P.brow + hi + 1));
                for (int h = 0; h < 2; h++) {
                    const unsigned long long want = h ? want2.b : want2.a;
                    if (!want) continue;
                    unsigned long long b0, b1;
                    ms_chunk_keys<S>(P, F, bm, it.y, e1, want, __ldg(P.bord + hi), s_tk + 64 * h, W, b0, b1, h);
                    if (b0 != ~0ull) atomicMin(P.hbest + (size_t)hi * kMsBatch + 64 * h + lane, b0);
                    if (b1 != ~0ull) atomicMin(P.hbest + (size_t)hi * kMsBatch + 64 * h + lane + 32, b1);
                }
            }
        }
        if (blockIdx.x == 0 && tid == 0) P.flag[(L + 1) & 1] = 0;
        grid.sync();
        MS_PROF(2);
        // ---------------- phase C: hubs -----------------------------------------
        if (multi) {
            for (int64_t hi = gwarp; hi < P.nmulti; hi += nwarps) {
                const W2 want2 = ld2<S>(P.hacc + S * (size_t)hi);
                if (!(want2.a | want2.b)) continue;
#pragma unroll
                for (int q = 0; q < 4; q++) {
                    const int t = lane + 32 * q;
                    const unsigned long long want = q < 2 ? want2.a : want2.b;
                    if ((want >> (t & 63)) & 1ull) {
                        unsigned long long *slot = P.hbest + (size_t)hi * kMsBatch + t;
                        const unsigned long long key = __ldcg(slot);
                        *slot = ~0ull;
                        const unsigned long long old =
                            atomicAdd((unsigned long long *)(P.lvl + t * P.ls + L + 1), 1ull << 32);
                        ms_emit(P, t, s_vb[t] + (uint32_t)(old >> 32), (uint32_t)hi, key);
                    }
                }
                __syncwarp();
                if (lane == 0) {
                    atomicAdd(P.fcnt + (L + 1) % 3, 1u);
                    const W2 v0 = ld2<S>(P.vis + S * (size_t)hi);
                    const W2 vis{v0.a | want2.a, v0.b | want2.b};
                    st2<S>(P.vis + S * (size_t)hi, vis);
                    st2<S>(Nx + S * (size_t)hi, want2);
                    st2<S>(P.hacc + S * (size_t)hi, W2{0ull, 0ull});
                    atomicOr(nbm + (hi >> 5), 1u << (hi & 31));
                    if (vis.a == full.a && vis.b == full.b) {
                        atomicOr(P.fullbm + (hi >> 5), 1u << (hi & 31));
                        atomicAdd(P.fcnt + 3, 1u);
                    }
                }
            }
            grid.sync();
        }
        MS_PROF(3);
        // ---------------- next level or done --------------------------------
        if (tid == 0) s_more = 0;
        __syncthreads();
        if (tid < B) {
            const uint32_t cc = (uint32_t)(__ldcg((const unsigned long long *)(P.lvl + tid * P.ls + L + 1)) >> 32);
            if (cc) {
                s_depth[tid] = L + 1;
                atomicOr(&s_more, 1);
            }
            s_vbase[tid] = s_vb[tid];
        }
        __syncthreads();
        if (!s_more) break;
    }
    if (blockIdx.x == 0 && tid < B) {
        P.depth[tid] = s_depth[tid];
        atomicMax(P.maxd, s_depth[tid]);
    }
}

// ---------------------------------------------------------------------------
// host side
// ---------------------------------------------------------------------------
int run_msbfs(const Graph &g, Workspace &ws, int B, const MsBfsOut &o, cudaStream_t st,
              int64_t *launches) {
    if (B < 1 || B > kMsBatch) { set_error("msbfs: batch out of range"); return GB_EINVAL; }
    // co-resident grid size, recomputed when the device changes (SM count)
    const int S = B > 64 ? 2 : 1;   // words per vertex
    const void *kern = S == 2 ? (const void *)k_msbfs<2> : (const void *)k_msbfs<1>;
    static int blocks[2] = {0, 0}, blocks_dev = -1;
    if (blocks_dev != g.dev) {
        blocks_dev = g.dev;
        for (int k = 0; k < 2; k++) {
            const void *f = k ? (const void *)k_msbfs<2> : (const void *)k_msbfs<1>;
            int per = 0;
            GB_CUDA_TRY(cudaFuncSetAttribute(f, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kMsSmem));
            if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, f, kBlock, kMsSmem) != cudaSuccess || per < 1)
                per = 1;
            blocks[k] = std::min(per * g.num_sms, kMsMaxBlocks);
        }
    }
    MsParams P;
    P.brow = g.brow; P.badj = g.badj; P.borig = g.borig; P.bord = g.bord; P.brank = g.brank;
    P.items = g.items; P.coff = g.coff; P.cverts = g.cverts;
    P.bigc = g.bigc; P.nbig = g.nbig; P.niso = g.niso; P.comp_i = g.comp_i;
    P.n = g.n; P.ncomp = g.ncomp; P.nitems = g.nitems; P.nmulti_items = g.nmulti_items;
    P.nlight0 = g.nlight0; P.nmulti = g.nmulti; P.ls = g.n + 2;
    P.nwords = (g.n + 31) / 32;
    P.itemwords = (g.nlight0 + 31) / 32;
    P.B = B;
    P.full0 = B >= 64 ? ~0ull : ((1ull << B) - 1);
    P.full1 = B >= 128 ? ~0ull : B > 64 ? ((1ull << (B - 64)) - 1) : 0ull;
    P.vis = ws.vis; P.fr = ws.fr; P.hacc = ws.hacc; P.hbest = ws.hbest;
    P.fbm = ws.fbm; P.fullbm = ws.fbm + 3 * P.nwords;
    P.tb = ws.fbm + 4 * P.nwords;
    P.fcnt = reinterpret_cast<uint32_t *>(ws.msflag + 4);
    P.push_div = 32;   // measured on C3: 32 and 128 equal (bfs 59.0 ms / 100 trees), 8 worse (61.3)
    P.flag = ws.msflag; P.mscnt = ws.mscnt;
    P.pnew = nullptr; P.pbest = nullptr;
    // level 0 pulls: its frontier is one root per tree in every component of
    // >= 2 vertices (RMAT-26: ~10 M pushes), measured C5 bfs 242.6 vs 238.2 ms
    P.pp_from = 1;
    if (S == 1 && B <= kPPTrees && ws.pp_ok && !ws.pp_nomem) {
        // push-parent state, allocated once (all-zero / all-ones between uses)
        if (!ws.pbest) {
            size_t fr = 0, tot = 0;
            const size_t need = sizeof(unsigned long long) * (size_t)g.n * (kPPTrees + 1);
            if (cudaMemGetInfo(&fr, &tot) == cudaSuccess && fr > 2 * need) {
                GB_CUDA_TRY(cudaMalloc(&ws.pnew, sizeof(unsigned long long) * (size_t)g.n));
                GB_CUDA_TRY(cudaMalloc(&ws.pbest, sizeof(unsigned long long) * (size_t)g.n * kPPTrees));
                GB_CUDA_TRY(cudaMemsetAsync(ws.pnew, 0, sizeof(unsigned long long) * (size_t)g.n, st));
                GB_CUDA_TRY(cudaMemsetAsync(ws.pbest, 0xFF, sizeof(unsigned long long) * (size_t)g.n * kPPTrees, st));
            } else {
                ws.pp_nomem = true;
            }
        }
        P.pnew = ws.pnew;
        P.pbest = ws.pbest;
    }
    P.tkey = o.tkey; P.qv = o.qv; P.parq = o.parq; P.pp = o.pp; P.rec = o.rec; P.crec = o.crec; P.irec = o.irec; P.prec = o.prec;
    P.lvl = o.lvl; P.vbase = o.vbase; P.depth = o.depth; P.maxd = o.maxd;
    P.prof = ws.msprof;
    GB_CUDA_TRY(cudaMemsetAsync(ws.vis, 0, sizeof(unsigned long long) * S * (size_t)g.n, st));
    GB_CUDA_TRY(cudaMemsetAsync(ws.fr, 0, sizeof(unsigned long long) * S * (size_t)g.n, st));
    GB_CUDA_TRY(cudaMemsetAsync(ws.fbm, 0, sizeof(uint32_t) * 6 * (size_t)P.nwords, st));
    GB_CUDA_TRY(cudaMemsetAsync(ws.msflag, 0, sizeof(int32_t) * 8, st));
    const int64_t work = std::max<int64_t>((int64_t)B * g.nbig, g.niso);
    const unsigned rgrid = (unsigned)std::max<int64_t>(1, std::min<int64_t>((work + 255) / 256, 8192));
    if (S == 2) k_ms_roots<2><<<rgrid, 256, 0, st>>>(P);
    else k_ms_roots<1><<<rgrid, 256, 0, st>>>(P);
    ++*launches;
    void *args[] = {&P};
    cudaError_t e = cudaLaunchCooperativeKernel(kern, dim3(blocks[S - 1]), dim3(kBlock), args, kMsSmem, st);
    if (e != cudaSuccess) {
        set_error(std::string("cooperative launch (msbfs): ") + cudaGetErrorString(e));
        return GB_ECUDA;
    }
    ++*launches;
    return GB_OK;
}

}  // namespace gb
