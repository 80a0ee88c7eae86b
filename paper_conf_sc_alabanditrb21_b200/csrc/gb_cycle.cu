// gb_cycle.cu -- §8 rows a.6-a.8:
//   a.6 cycle traversal + balancing (Alg. 3),
//   a.7 Harary majority and per-vertex agree (L144, L224, L248),
//   a.8 accumulation without contended atomics.
//
// Cycle walk.  The labels of Alg. 4 make "x is an ancestor of y" an interval
// test: pre x <= pre y <= pre x + size x - 1 (L212: the range of the edge
// into x).  Two walks are provided; both traverse every edge of the
// fundamental cycle exactly once, XOR its negative bits and count its length:
//
//  walk 0 (two-ended, §8 f.1): one thread per non-tree edge (u,v).  u climbs
//   while it is not an ancestor of v, v climbs while it is not an ancestor of
//   u; both stop at the LCA.  Each step is one 8-byte gather of the
//   pre-indexed record {parent pre | neg, size}; the two climbs are
//   independent, so every thread keeps two loads in flight.
//  walk 1 (Alg. 3 as written, §8 a.6): u climbs to the LCA through parent
//   edges (the inverse range of L212), then the warp descends from the LCA to
//   v: at each vertex the child whose range contains pre v is found with a
//   coalesced load of up to 32 sorted child starts and one __ballot_sync
//   (32-ary pivot rounds for hubs), L214.
//
// Either way: c = XOR of the negative tree edges; the non-tree edge gets the
// sign (-1)^c, i.e. flip = c XOR neg(e) (reading R1).  No synchronization is
// needed: the tree is read-only and every non-tree edge has one writer (L309).
#include "gb_internal.cuh"
#include "../../include/graphb.h"

#include <algorithm>

namespace gb {

struct CycleParams {
    const uint2 *edges;    // [m] {u, v | neg<<31} by eid, internal ids (the labels' index space)
    int64_t n, m;
    const uint32_t *pp;    // [B][n] pre | pi<<31
    const uint2 *rec;      // [B][n] pre-indexed {up | neg<<31, size}                (layout 1)
    const uint4 *irec;     // [B][n] by internal id {parent | neg, pre | pi, size, 0} (layout 0)
    const uint32_t *prec;  // [B][n] pre-indexed parent word up | neg<<31       (layout 2)
    const uint2 *crec;     // [B][n] pre-indexed {child-list start, #children}
    const uint32_t *clist; // children pre IDs, per parent ascending
    uint32_t *fbits;       // [B][words]
    unsigned long long *tstat;  // [B][3] {sum cycle length, cycles, state signature}
    int64_t words;
    int b0, G;             // trees b0 .. b0+G-1 of the batch
    int linear;            // walk 1: child search by linear int4 ballot rounds (1) or 32-ary pivots (0)
    const uint32_t *tbase; // walk 2: [n+1] start of each vertex's tree-edge list (pre order)
    const uint32_t *tnbr;  // walk 2: [2n] neighbour (pre id) of each tree-edge record
    const uint2 *trng;     // walk 2: [2n] {begin | inverted<<31, end | neg<<31} (L238)
    uint2 *jrec;           // [G][n][K] K-level ancestor records (walk 0, option "jump" = K > 1)
};

constexpr int kCycleBlock = 256;
constexpr int kMaxGroup = 64;

// f.2: signature of a nearest balanced state = XOR over its switched edges of
// mix64(e ^ K) (order-free, so each warp reduces its 32 edges on its own)
constexpr uint64_t kSigSalt = 0x5851F42D4C957F2Dull;

__device__ __forceinline__ void warp_stats(int lane, int g, uint32_t k, bool cyc, bool flip,
                                           int64_t e, unsigned long long *s_k,
                                           unsigned long long *s_c, unsigned long long *s_sig) {
    uint32_t kk = k, cc = cyc ? 1u : 0u;
    unsigned long long sig = flip ? mix64((uint64_t)e ^ kSigSalt) : 0ull;
#pragma unroll
    for (int d = 16; d; d >>= 1) {
        kk += __shfl_xor_sync(0xFFFFFFFFu, kk, d);
        cc += __shfl_xor_sync(0xFFFFFFFFu, cc, d);
        sig ^= __shfl_xor_sync(0xFFFFFFFFu, sig, d);
    }
    if (lane == 0) {
        if (cc) {
            atomicAdd(&s_k[g], (unsigned long long)kk);
            atomicAdd(&s_c[g], (unsigned long long)cc);
        }
        if (sig) atomicXor(&s_sig[g], sig);
    }
}

// the same from per-thread sums over many edges (one reduction per kernel)
__device__ __forceinline__ void warp_stats_sum(int lane, int g, unsigned long long ks, uint32_t cs,
                                               unsigned long long sig, unsigned long long *s_k,
                                               unsigned long long *s_c, unsigned long long *s_sig) {
#pragma unroll
    for (int d = 16; d; d >>= 1) {
        ks += __shfl_xor_sync(0xFFFFFFFFu, ks, d);
        cs += __shfl_xor_sync(0xFFFFFFFFu, cs, d);
        sig ^= __shfl_xor_sync(0xFFFFFFFFu, sig, d);
    }
    if (lane == 0) {
        if (cs) {
            atomicAdd(&s_k[g], ks);
            atomicAdd(&s_c[g], (unsigned long long)cs);
        }
        if (sig) atomicXor(&s_sig[g], sig);
    }
}

__device__ __forceinline__ void flush_stats(const CycleParams &P, const unsigned long long *s_k,
                                            const unsigned long long *s_c,
                                            const unsigned long long *s_sig) {
    for (int i = threadIdx.x; i < P.G; i += blockDim.x) {
        unsigned long long *t = P.tstat + 3 * (P.b0 + i);
        if (s_c[i]) {
            atomicAdd(t, s_k[i]);
            atomicAdd(t + 1, s_c[i]);
        }
        if (s_sig[i]) atomicXor(t + 2, s_sig[i]);
    }
}

// &base[i] as one mad.wide.u32 (i * 16 + base): the compiler otherwise widens
// and masks the 31-bit id in 64-bit arithmetic (six instructions per step)
__device__ __forceinline__ const uint4 *rec_at(const uint4 *base, uint32_t i) {
    const uint4 *p;
    asm("mad.wide.u32 %0, %1, 16, %2;" : "=l"(p) : "r"(i), "l"(base));
    return p;
}

__device__ __forceinline__ bool is_anc(uint32_t a, uint32_t size_a, uint32_t t) {
    return (t - a) < size_a;  // a <= t <= a + size_a - 1 (unsigned wrap for t < a)
}

// one warp = 32 consecutive edges (one flip word per tree)
__global__ void __launch_bounds__(kCycleBlock) k_cycles_two_ended(CycleParams P) {
    __shared__ unsigned long long s_k[kMaxGroup], s_c[kMaxGroup], s_sig[kMaxGroup];
    for (int i = threadIdx.x; i < P.G; i += blockDim.x) { s_k[i] = 0; s_c[i] = 0; s_sig[i] = 0; }
    __syncthreads();
    const int lane = threadIdx.x & 31;
    const int64_t gw = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t word = gw; word < P.words; word += nw) {
        const int64_t e = word * 32 + lane;
        const bool valid = e < P.m;
        uint2 ed = valid ? __ldg(P.edges + e) : make_uint2(0, 0);
        const uint32_t u = ed.x, v = ed.y & kIdMask, nege = ed.y >> 31;
        for (int g = 0; g < P.G; g++) {
            const size_t nb = (size_t)(P.b0 + g) * P.n;
            const uint2 *rec = P.rec + nb;
            uint32_t flip = 0, k = 0;
            bool cyc = false;
            if (valid) {
                const uint32_t x0 = __ldg(P.pp + nb + u) & kIdMask;
                const uint32_t y0 = __ldg(P.pp + nb + v) & kIdMask;
                uint2 rx = __ldg(rec + x0), ry = __ldg(rec + y0);
                // tree edge iff one endpoint is the other's parent (simple graph)
                if ((rx.x & kIdMask) != y0 && (ry.x & kIdMask) != x0) {
                    cyc = true;
                    uint32_t x = x0, y = y0, c = 0;
                    k = 1;
                    bool ax = is_anc(x, rx.y, y0), ay = is_anc(y, ry.y, x0);
                    while (!(ax && ay)) {
                        if (!ax) {
                            c ^= rx.x;
                            x = rx.x & kIdMask;
                            rx = __ldg(rec + x);
                            k++;
                            ax = is_anc(x, rx.y, y0);
                        }
                        if (!ay) {
                            c ^= ry.x;
                            y = ry.x & kIdMask;
                            ry = __ldg(rec + y);
                            k++;
                            ay = is_anc(y, ry.y, x0);
                        }
                    }
                    flip = (c >> 31) ^ nege;
                }
            }
            const uint32_t bits = __ballot_sync(0xFFFFFFFFu, flip != 0);
            if (lane == 0) P.fbits[(size_t)(P.b0 + g) * P.words + word] = bits;
            // per-tree cycle statistics and state signature
            warp_stats(lane, g, k, cyc, flip != 0, e, s_k, s_c, s_sig);
        }
    }
    __syncthreads();
    flush_stats(P, s_k, s_c, s_sig);
}

// Walk 3 (layout 2): pre-order climb.  Ancestors precede their descendants
// in pre order (pre c = pre p + offset, offset >= 1, Alg. 4), so of
// two distinct vertices of one tree the one with the larger pre is not an
// ancestor of the other: it lies strictly below their LCA, and climbing it is
// always a step of the fundamental cycle; the two climbs meet exactly at the
// LCA.  Only the pre labels steer the walk (the range ends are not read), and
// a step is one 4-byte gather of prec[pre] = pre(parent) | neg<<31: the two
// per-tree arrays (pp by internal id, prec by pre, 8 bytes per vertex) are
// the walk's whole random-access working set.
__global__ void __launch_bounds__(kCycleBlock) k_cycles_pclimb(CycleParams P) {
    __shared__ unsigned long long s_k[kMaxGroup], s_c[kMaxGroup], s_sig[kMaxGroup];
    for (int i = threadIdx.x; i < P.G; i += blockDim.x) { s_k[i] = 0; s_c[i] = 0; s_sig[i] = 0; }
    __syncthreads();
    const int lane = threadIdx.x & 31;
    const int64_t gw = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t word = gw; word < P.words; word += nw) {
        const int64_t e = word * 32 + lane;
        const bool valid = e < P.m;
        uint2 ed = valid ? __ldg(P.edges + e) : make_uint2(0, 0);
        const uint32_t u = ed.x, v = ed.y & kIdMask, nege = ed.y >> 31;
        for (int g = 0; g < P.G; g++) {
            const size_t nb = (size_t)(P.b0 + g) * P.n;
            const uint32_t *pp = P.pp + nb, *prec = P.prec + nb;
            uint32_t flip = 0, k = 0;
            bool cyc = false;
            if (valid) {
                uint32_t x = __ldg(pp + u) & kIdMask, y = __ldg(pp + v) & kIdMask;
                uint32_t rx = __ldg(prec + x), ry = __ldg(prec + y);
                // tree edge iff one endpoint is the other's parent (simple graph)
                if ((rx & kIdMask) != y && (ry & kIdMask) != x) {
                    cyc = true;
                    uint32_t c = 0;
                    k = 1;
                    while (x != y) {
                        if (x > y) {
                            c ^= rx;
                            x = rx & kIdMask;
                            if (x != y) rx = __ldg(prec + x);
                        } else {
                            c ^= ry;
                            y = ry & kIdMask;
                            if (x != y) ry = __ldg(prec + y);
                        }
                        k++;
                    }
                    flip = (c >> 31) ^ nege;
                }
            }
            const uint32_t bits = __ballot_sync(0xFFFFFFFFu, flip != 0);
            if (lane == 0) P.fbits[(size_t)(P.b0 + g) * P.words + word] = bits;
            warp_stats(lane, g, k, cyc, flip != 0, e, s_k, s_c, s_sig);
        }
    }
    __syncthreads();
    flush_stats(P, s_k, s_c, s_sig);
}

// Layout 0 (default): the same two-ended walk over records indexed by
// internal vertex id, {parent | neg<<31, pre | pi<<31, size}.  The endpoints'
// records are the first two loads (no separate label lookup), the tree-edge
// test is on the parent words, and a climb step is one 16-byte gather; the
// ancestors the climbs share (hubs and other high-degree vertices, internal
// ids at the front) sit in a dense, L2-hot region.
__global__ void __launch_bounds__(kCycleBlock, 8) k_cycles_irec(CycleParams P) {
    __shared__ unsigned long long s_k[kMaxGroup], s_c[kMaxGroup], s_sig[kMaxGroup];
    for (int i = threadIdx.x; i < P.G; i += blockDim.x) { s_k[i] = 0; s_c[i] = 0; s_sig[i] = 0; }
    __syncthreads();
    const int lane = threadIdx.x & 31;
    const int64_t gw = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
    // tree by tree (the G trees of a cycle group re-read the edge list from
    // L2); a tree's cycle statistics are summed per thread and reduced across
    // the warp once, not per 32-edge word
    for (int g = 0; g < P.G; g++) {
        const uint4 *rec = P.irec + (size_t)(P.b0 + g) * P.n;
        uint32_t *fb = P.fbits + (size_t)(P.b0 + g) * P.words;
        unsigned long long a_k = 0, a_sig = 0;
        uint32_t a_c = 0;
        for (int64_t word = gw; word < P.words; word += nw) {
            const int64_t e = word * 32 + lane;
            uint32_t flip = 0;
            if (e < P.m) {
                const uint2 ed = __ldg(P.edges + e);
                const uint32_t u = ed.x, v = ed.y & kIdMask;
                uint4 rx = __ldg(rec_at(rec, u)), ry = __ldg(rec_at(rec, v));
                // tree edge iff one endpoint is the other's parent (simple graph)
                if ((rx.x & kIdMask) != v && (ry.x & kIdMask) != u) {
                    const uint32_t px = rx.y & kIdMask, py = ry.y & kIdMask;
                    uint32_t c = 0, k = 1;
                    bool ax = is_anc(px, rx.z, py), ay = is_anc(py, ry.z, px);
                    while (!(ax && ay)) {
                        if (!ax) {
                            c ^= rx.x;
                            rx = __ldg(rec_at(rec, rx.x & kIdMask));
                            k++;
                            ax = is_anc(rx.y & kIdMask, rx.z, py);
                        }
                        if (!ay) {
                            c ^= ry.x;
                            ry = __ldg(rec_at(rec, ry.x & kIdMask));
                            k++;
                            ay = is_anc(ry.y & kIdMask, ry.z, px);
                        }
                    }
                    flip = (c >> 31) ^ (ed.y >> 31);
                    a_k += k;
                    a_c++;
                    if (flip) a_sig ^= mix64((uint64_t)e ^ kSigSalt);
                }
            }
            const uint32_t bits = __ballot_sync(0xFFFFFFFFu, flip != 0);
            if (lane == 0) fb[word] = bits;
        }
        warp_stats_sum(lane, g, a_k, a_c, a_sig, s_k, s_c, s_sig);
    }
    __syncthreads();
    flush_stats(P, s_k, s_c, s_sig);
}

// The same walk with EPT edges per thread (EPT consecutive 32-edge words per
// warp), their climbs interleaved: 2 * EPT independent gathers in flight per
// thread, and a lane idles only once all its edges are done (the cycle
// lengths of one edge vary a lot; the sum over EPT edges less so).
template <int EPT>
__global__ void __launch_bounds__(kCycleBlock) k_cycles_irec_m(CycleParams P) {
    __shared__ unsigned long long s_k[kMaxGroup], s_c[kMaxGroup], s_sig[kMaxGroup];
    for (int i = threadIdx.x; i < P.G; i += blockDim.x) { s_k[i] = 0; s_c[i] = 0; s_sig[i] = 0; }
    __syncthreads();
    const int lane = threadIdx.x & 31;
    const int64_t gw = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t w0 = gw * EPT; w0 < P.words; w0 += nw * EPT) {
        uint32_t u[EPT], v[EPT], nege[EPT];
        bool valid[EPT];
#pragma unroll
        for (int j = 0; j < EPT; j++) {
            const int64_t e = (w0 + j) * 32 + lane;
            valid[j] = w0 + j < P.words && e < P.m;
            const uint2 ed = valid[j] ? __ldg(P.edges + e) : make_uint2(0, 0);
            u[j] = ed.x;
            v[j] = ed.y & kIdMask;
            nege[j] = ed.y >> 31;
        }
        for (int g = 0; g < P.G; g++) {
            const uint4 *rec = P.irec + (size_t)(P.b0 + g) * P.n;
            uint4 rx[EPT], ry[EPT];
            uint32_t px[EPT], py[EPT], c[EPT], k[EPT];
            bool ax[EPT], ay[EPT], cyc[EPT];
#pragma unroll
            for (int j = 0; j < EPT; j++) {
                rx[j] = valid[j] ? __ldg(rec_at(rec, u[j])) : make_uint4(0, 0, 1, 0);
                ry[j] = valid[j] ? __ldg(rec_at(rec, v[j])) : make_uint4(0, 0, 1, 0);
            }
#pragma unroll
            for (int j = 0; j < EPT; j++) {
                // tree edge iff one endpoint is the other's parent (simple graph)
                cyc[j] = valid[j] && (rx[j].x & kIdMask) != v[j] && (ry[j].x & kIdMask) != u[j];
                px[j] = rx[j].y & kIdMask;
                py[j] = ry[j].y & kIdMask;
                c[j] = 0;
                k[j] = cyc[j] ? 1u : 0u;
                ax[j] = !cyc[j] || is_anc(px[j], rx[j].z, py[j]);
                ay[j] = !cyc[j] || is_anc(py[j], ry[j].z, px[j]);
            }
            for (;;) {
                bool more = false;
#pragma unroll
                for (int j = 0; j < EPT; j++) {
                    if (!ax[j]) {
                        c[j] ^= rx[j].x;
                        rx[j] = __ldg(rec_at(rec, rx[j].x & kIdMask));
                        k[j]++;
                    }
                    if (!ay[j]) {
                        c[j] ^= ry[j].x;
                        ry[j] = __ldg(rec_at(rec, ry[j].x & kIdMask));
                        k[j]++;
                    }
                }
#pragma unroll
                for (int j = 0; j < EPT; j++) {
                    if (!ax[j]) ax[j] = is_anc(rx[j].y & kIdMask, rx[j].z, py[j]);
                    if (!ay[j]) ay[j] = is_anc(ry[j].y & kIdMask, ry[j].z, px[j]);
                    more |= !(ax[j] && ay[j]);
                }
                if (!more) break;
            }
#pragma unroll
            for (int j = 0; j < EPT; j++) {
                const uint32_t flip = cyc[j] ? (c[j] >> 31) ^ nege[j] : 0u;
                const uint32_t bits = __ballot_sync(0xFFFFFFFFu, flip != 0);
                if (lane == 0 && w0 + j < P.words) P.fbits[(size_t)(P.b0 + g) * P.words + w0 + j] = bits;
                warp_stats(lane, g, k[j], cyc[j], flip != 0, (w0 + j) * 32 + lane, s_k, s_c, s_sig);
            }
        }
    }
    __syncthreads();
    flush_stats(P, s_k, s_c, s_sig);
}

// ---------------------------------------------------------------------------
// K-level records for the two-ended walk (option "jump"): jrec[x][j] =
// rec[a_j(x)], a_0 = x, a_{j+1} = parent of a_j (the root is its own parent).
// Built by one streaming pass in pre order -- consecutive pre IDs share most
// ancestors, so the gathers of rec[a_j] hit L1/L2 -- and written as full
// 32-byte sectors.  A climb step then still visits every tree edge of the
// cycle (its sign and range are in the record) but one gather serves K
// levels: the dependent-load chain of a cycle shrinks by a factor of K.
// ---------------------------------------------------------------------------
template <int K>
__global__ void k_build_jump(const uint2 *__restrict__ rec, uint2 *__restrict__ jrec, int64_t n) {
    const int g = blockIdx.y;
    const uint2 *r = rec + (size_t)g * n;
    uint4 *out = reinterpret_cast<uint4 *>(jrec + (size_t)g * n * K);
    for (int64_t x = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; x < n;
         x += (int64_t)gridDim.x * blockDim.x) {
        uint2 a[K];
        a[0] = __ldg(r + x);
#pragma unroll
        for (int j = 1; j < K; j++) a[j] = __ldg(r + (a[j - 1].x & kIdMask));
#pragma unroll
        for (int j = 0; j < K; j += 2) out[x * (K / 2) + j / 2] = make_uint4(a[j].x, a[j].y, a[j + 1].x, a[j + 1].y);
    }
}

template <int K>
__device__ __forceinline__ void load_jump(const uint2 *jrec, uint32_t x, uint2 (&a)[K]) {
    const uint4 *p = reinterpret_cast<const uint4 *>(jrec + (size_t)x * K);
#pragma unroll
    for (int j = 0; j < K; j += 2) {
        const uint4 q = __ldg(p + j / 2);
        a[j] = make_uint2(q.x, q.y);
        a[j + 1] = make_uint2(q.z, q.w);
    }
}

// one step up from a[0] (the current vertex); the window shifts by one and is
// refilled from the new vertex's record once it is used up
template <int K>
__device__ __forceinline__ void climb_step(const uint2 *jrec, uint2 (&a)[K], int &left, uint32_t &x,
                                           uint32_t &c) {
    c ^= a[0].x;
    x = a[0].x & kIdMask;
    if (--left == 0) {
        load_jump<K>(jrec, x, a);
        left = K;
    } else {
#pragma unroll
        for (int j = 0; j + 1 < K; j++) a[j] = a[j + 1];
    }
}

template <int K>
__global__ void __launch_bounds__(kCycleBlock) k_cycles_jump(CycleParams P) {
    __shared__ unsigned long long s_k[kMaxGroup], s_c[kMaxGroup], s_sig[kMaxGroup];
    for (int i = threadIdx.x; i < P.G; i += blockDim.x) { s_k[i] = 0; s_c[i] = 0; s_sig[i] = 0; }
    __syncthreads();
    const int lane = threadIdx.x & 31;
    const int64_t gw = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t word = gw; word < P.words; word += nw) {
        const int64_t e = word * 32 + lane;
        const bool valid = e < P.m;
        uint2 ed = valid ? __ldg(P.edges + e) : make_uint2(0, 0);
        const uint32_t u = ed.x, v = ed.y & kIdMask, nege = ed.y >> 31;
        for (int g = 0; g < P.G; g++) {
            const size_t nb = (size_t)(P.b0 + g) * P.n;
            const uint2 *jr = P.jrec + (size_t)g * P.n * K;
            uint32_t flip = 0, k = 0;
            bool cyc = false;
            if (valid) {
                const uint32_t x0 = __ldg(P.pp + nb + u) & kIdMask;
                const uint32_t y0 = __ldg(P.pp + nb + v) & kIdMask;
                uint2 ax[K], ay[K];
                load_jump<K>(jr, x0, ax);
                load_jump<K>(jr, y0, ay);
                // tree edge iff one endpoint is the other's parent (simple graph)
                if ((ax[0].x & kIdMask) != y0 && (ay[0].x & kIdMask) != x0) {
                    cyc = true;
                    uint32_t x = x0, y = y0, c = 0;
                    int lx = K, ly = K;
                    k = 1;
                    bool fx = is_anc(x, ax[0].y, y0), fy = is_anc(y, ay[0].y, x0);
                    while (!(fx && fy)) {
                        if (!fx) {
                            climb_step<K>(jr, ax, lx, x, c);
                            k++;
                            fx = is_anc(x, ax[0].y, y0);
                        }
                        if (!fy) {
                            climb_step<K>(jr, ay, ly, y, c);
                            k++;
                            fy = is_anc(y, ay[0].y, x0);
                        }
                    }
                    flip = (c >> 31) ^ nege;
                }
            }
            const uint32_t bits = __ballot_sync(0xFFFFFFFFu, flip != 0);
            if (lane == 0) P.fbits[(size_t)(P.b0 + g) * P.words + word] = bits;
            warp_stats(lane, g, k, cyc, flip != 0, e, s_k, s_c, s_sig);
        }
    }
    __syncthreads();
    flush_stats(P, s_k, s_c, s_sig);
}

// Alg. 3 as written: lane-parallel climb to the LCA, then warp-cooperative
// descents from the LCA to v, one lane's cycle at a time.
__global__ void __launch_bounds__(kCycleBlock) k_cycles_descent(CycleParams P) {
    __shared__ unsigned long long s_k[kMaxGroup], s_c[kMaxGroup], s_sig[kMaxGroup];
    for (int i = threadIdx.x; i < P.G; i += blockDim.x) { s_k[i] = 0; s_c[i] = 0; s_sig[i] = 0; }
    __syncthreads();
    const int lane = threadIdx.x & 31;
    const int64_t gw = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t word = gw; word < P.words; word += nw) {
        const int64_t e = word * 32 + lane;
        const bool valid = e < P.m;
        uint2 ed = valid ? __ldg(P.edges + e) : make_uint2(0, 0);
        const uint32_t u = ed.x, v = ed.y & kIdMask, nege = ed.y >> 31;
        for (int g = 0; g < P.G; g++) {
            const size_t nb = (size_t)(P.b0 + g) * P.n;
            const uint2 *rec = P.rec + nb;
            const uint2 *crec = P.crec + nb;
            uint32_t c = 0, k = 0, x = 0, y0 = 0;
            bool cyc = false;
            if (valid) {
                const uint32_t x0 = __ldg(P.pp + nb + u) & kIdMask;
                y0 = __ldg(P.pp + nb + v) & kIdMask;
                uint2 rx = __ldg(rec + x0), ry = __ldg(rec + y0);
                if ((rx.x & kIdMask) != y0 && (ry.x & kIdMask) != x0) {
                    cyc = true;
                    k = 1;
                    x = x0;
                    // the parent edge's range is the complement of x's range
                    // (L212): follow it while pre v is outside x's range
                    while (!is_anc(x, rx.y, y0)) {
                        c ^= rx.x;
                        x = rx.x & kIdMask;
                        rx = __ldg(rec + x);
                        k++;
                    }
                }
            }
            // descents: the whole warp serves one lane's cycle at a time
            uint32_t pending = __ballot_sync(0xFFFFFFFFu, cyc && x != y0);
            while (pending) {
                const int src = __ffs(pending) - 1;
                pending &= pending - 1;
                uint32_t cx = __shfl_sync(0xFFFFFFFFu, x, src);
                const uint32_t ty = __shfl_sync(0xFFFFFFFFu, y0, src);
                uint32_t cpar = 0, steps = 0;
                while (cx != ty) {
                    // children of cx: clist[cs .. cs+nc), ascending pre; find
                    // the last child start <= ty (its range holds ty)
                    const uint2 cr = __ldg(crec + cx);
                    uint32_t lo = cr.x, cnt = cr.y;
                    if (P.linear) {
                        // linear ballot rounds over the sorted child starts,
                        // four per lane with one 16-byte load (128 per round):
                        // the round that holds the first start > ty decides
                        const uint32_t a0 = lo & ~3u, end = lo + cnt;
                        for (uint32_t base = a0;; base += 128) {
                            const uint32_t q = base + 4 * lane;
                            uint4 v4 = make_uint4(~0u, ~0u, ~0u, ~0u);
                            if (q < end) v4 = __ldg(reinterpret_cast<const uint4 *>(P.clist + q));
                            // positions outside [lo, end) never count
                            const bool b0 = q >= lo && q < end && v4.x <= ty;
                            const bool b1 = q + 1 >= lo && q + 1 < end && v4.y <= ty;
                            const bool b2 = q + 2 >= lo && q + 2 < end && v4.z <= ty;
                            const bool b3 = q + 3 >= lo && q + 3 < end && v4.w <= ty;
                            const uint32_t m0 = __ballot_sync(0xFFFFFFFFu, b0), m1 = __ballot_sync(0xFFFFFFFFu, b1);
                            const uint32_t m2 = __ballot_sync(0xFFFFFFFFu, b2), m3 = __ballot_sync(0xFFFFFFFFu, b3);
                            const uint32_t tot = __popc(m0) + __popc(m1) + __popc(m2) + __popc(m3);
                            const uint32_t avail = min(end, base + 128) - max(lo, base);
                            if (tot < avail || base + 128 >= end) {
                                // sorted: the starts <= ty are a prefix; the child is the last of them
                                const uint32_t before = max(lo, base) - lo;
                                lo = lo + before + tot - 1;
                                cnt = 1;
                                break;
                            }
                        }
                        const uint32_t ch = __ldg(P.clist + lo);
                        cpar ^= __ldg(rec + ch).x;   // neg bit of the edge into ch
                        cx = ch;
                        steps++;
                        continue;
                    }
                    while (cnt > 32) {
                        const uint32_t step = (cnt + 31) >> 5;
                        const uint32_t pos = lane * step;
                        const uint32_t pv = pos < cnt ? __ldg(P.clist + lo + pos) : 0xFFFFFFFFu;
                        const uint32_t bal = __ballot_sync(0xFFFFFFFFu, pv <= ty);
                        const uint32_t h = 31 - __clz(bal);
                        const uint32_t nlo = h * step;
                        cnt = min(step, cnt - nlo);
                        lo += nlo;
                    }
                    const uint32_t cv = lane < cnt ? __ldg(P.clist + lo + lane) : 0xFFFFFFFFu;
                    const uint32_t bal = __ballot_sync(0xFFFFFFFFu, cv <= ty);
                    const uint32_t ch = __shfl_sync(0xFFFFFFFFu, cv, 31 - __clz(bal));
                    cpar ^= __ldg(rec + ch).x;   // neg bit of the edge into ch
                    cx = ch;
                    steps++;
                }
                if (lane == src) { c ^= cpar; k += steps; }
            }
            const uint32_t flip = cyc ? ((c >> 31) ^ nege) : 0u;
            const uint32_t bits = __ballot_sync(0xFFFFFFFFu, flip != 0);
            if (lane == 0) P.fbits[(size_t)(P.b0 + g) * P.words + word] = bits;
            warp_stats(lane, g, k, cyc, flip != 0, e, s_k, s_c, s_sig);
        }
    }
    __syncthreads();
    flush_stats(P, s_k, s_c, s_sig);
}

// ---------------------------------------------------------------------------
// walk 2 (§8 f.1): the paper's own traversal data structure (§3.2.1-3.2.2,
// L238-L244).  Per tree, in pre-order ID space, every vertex x has a
// partitioned tree-edge list with the parent edge first, then the child edges
// (ascending); each edge is two words (L238): begin | inverted << 31 and
// end | sign << 31, next to the neighbour id.  The parent edge's range is x's
// own subtree range, inverted (L212: it leads to every ID outside it).  The
// walk is Alg. 3 as written (L190-L201): from v_src, scan the list for the
// edge whose (possibly inverted) range holds v_dst, count its sign, move,
// until v_dst -- one thread per non-tree edge, as the paper's lane per
// non-tree edge (L307), reading record pairs with 16-byte loads.
// ---------------------------------------------------------------------------
__global__ void k_paper_counts(const uint2 *__restrict__ crec, int64_t n, uint32_t *__restrict__ tcnt) {
    for (int64_t x = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; x <= n;
         x += (int64_t)gridDim.x * blockDim.x)
        tcnt[x] = x < n ? 1u + __ldg(&crec[x].y) : 0u;   // parent slot + children
}

// thread per pre ID x: the parent-edge record of x's own list, and the record
// of edge parent(x) -> x in the parent's list (its position = x's rank among
// the sorted children, found by binary search)
__global__ void k_paper_fill(const uint2 *__restrict__ rec, const uint2 *__restrict__ crec,
                             const uint32_t *__restrict__ clist, const uint32_t *__restrict__ tbase,
                             int64_t n, uint32_t *__restrict__ tnbr, uint2 *__restrict__ trng) {
    for (int64_t xi = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; xi < n;
         xi += (int64_t)gridDim.x * blockDim.x) {
        const uint32_t x = (uint32_t)xi;
        const uint2 r = __ldg(rec + x);
        const uint32_t up = r.x & kIdMask, neg = r.x & kNegBit, end = x + r.y - 1;
        const uint32_t s = __ldg(tbase + x);
        if (up == x) {   // a root: no parent edge; an empty range that never matches
            tnbr[s] = x;
            trng[s] = make_uint2(1u, 0u);
            continue;
        }
        tnbr[s] = up;
        trng[s] = make_uint2(x | kNegBit, end | neg);          // inverted: everything outside x's subtree
        const uint2 cp = __ldg(crec + up);
        uint32_t lo = 0, hi = cp.y;                              // clist[cp.x + lo] <= x < clist[cp.x + hi]
        while (hi - lo > 1) {
            const uint32_t mid = (lo + hi) >> 1;
            if (__ldg(clist + cp.x + mid) <= x) lo = mid; else hi = mid;
        }
        const uint32_t sp = __ldg(tbase + up) + 1 + lo;
        tnbr[sp] = x;
        trng[sp] = make_uint2(x, end | neg);
    }
}

__device__ __forceinline__ bool paper_hit(uint2 w, uint32_t y) {
    const uint32_t b = w.x & kIdMask, e = w.y & kIdMask;
    const bool in = (y - b) <= (e - b) && b <= e;
    return in != (bool)(w.x >> 31);
}

__global__ void __launch_bounds__(kCycleBlock) k_cycles_paper(CycleParams P) {
    __shared__ unsigned long long s_k[kMaxGroup], s_c[kMaxGroup], s_sig[kMaxGroup];
    for (int i = threadIdx.x; i < P.G; i += blockDim.x) { s_k[i] = 0; s_c[i] = 0; s_sig[i] = 0; }
    __syncthreads();
    const int lane = threadIdx.x & 31;
    const int64_t gw = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
    const size_t nb = (size_t)P.b0 * P.n;
    const uint2 *rec = P.rec + nb;
    for (int64_t word = gw; word < P.words; word += nw) {
        const int64_t e = word * 32 + lane;
        const bool valid = e < P.m;
        uint2 ed = valid ? __ldg(P.edges + e) : make_uint2(0, 0);
        const uint32_t u = ed.x, v = ed.y & kIdMask, nege = ed.y >> 31;
        uint32_t flip = 0, k = 0;
        bool cyc = false;
        if (valid) {
            uint32_t x = __ldg(P.pp + nb + u) & kIdMask;
            const uint32_t y = __ldg(P.pp + nb + v) & kIdMask;
            // tree edge iff one endpoint is the other's parent (simple graph)
            if ((__ldg(rec + x).x & kIdMask) != y && (__ldg(rec + y).x & kIdMask) != x) {
                cyc = true;
                uint32_t c = 0;
                k = 1;
                while (x != y) {
                    const uint32_t s0 = __ldg(P.tbase + x), s1 = __ldg(P.tbase + x + 1);
                    uint32_t s = s0 & ~1u;
                    bool found = false;
                    for (; s < s1; s += 2) {
                        const uint4 two = __ldg(reinterpret_cast<const uint4 *>(P.trng + s));
                        if (s >= s0 && paper_hit(make_uint2(two.x, two.y), y)) { found = true; break; }
                        if (s + 1 < s1 && paper_hit(make_uint2(two.z, two.w), y)) { s++; found = true; break; }
                    }
                    if (!found) { k = 0; break; }   // cannot happen on a valid tree; no endless loop
                    c ^= __ldg(P.trng + s).y;                 // the sign bit of the traversed edge
                    x = __ldg(P.tnbr + s);
                    k++;
                }
                flip = (c >> 31) ^ nege;
            }
        }
        const uint32_t bits = __ballot_sync(0xFFFFFFFFu, flip != 0);
        if (lane == 0) P.fbits[(size_t)P.b0 * P.words + word] = bits;
        warp_stats(lane, 0, k, cyc, flip != 0, e, s_k, s_c, s_sig);
    }
    __syncthreads();
    flush_stats(P, s_k, s_c, s_sig);
}

// ---------------------------------------------------------------------------
// a.8: per batch, edge_cnt[e] += sum_b flip_b(e) (one coalesced RMW per edge
// per batch; the B flip words of a 32-edge group are warp-broadcast loads)
// and a.7: agree[v] += sum_b 2*delta_b(v), delta from the root-parity sides:
// side(v) = pi(v); per component s1 = #{pi = 1}, s0 = |C| - s1 (L144, L224).
// ---------------------------------------------------------------------------
__global__ void k_accumulate_edges(const uint32_t *__restrict__ fbits, int64_t words, int64_t m,
                                   int B, int32_t *__restrict__ cnt) {
    for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < m;
         e += (int64_t)gridDim.x * blockDim.x) {
        const int64_t w = e >> 5;
        const uint32_t sh = (uint32_t)(e & 31);
        int32_t s = 0;
        for (int b = 0; b < B; b++) s += (__ldg(fbits + (size_t)b * words + w) >> sh) & 1u;
        if (s) cnt[e] += s;
    }
}

// (labels in internal ids i; the counter of the original vertex bord[i])
__global__ void k_accumulate_agree(const uint32_t *__restrict__ pp, int ps, const uint32_t *__restrict__ s1,
                                   const int32_t *__restrict__ comp_i, const int32_t *__restrict__ coff,
                                   const uint32_t *__restrict__ bord,
                                   int64_t n, int64_t ncomp, int B, int32_t *__restrict__ agree) {
    for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < n;
         v += (int64_t)gridDim.x * blockDim.x) {
        const int32_t C = __ldg(comp_i + v);
        const uint32_t cs = (uint32_t)(__ldg(coff + C + 1) - __ldg(coff + C));
        int32_t d = 0;
        if (cs == 1) {
            // a single-vertex component is its own larger side in every tree
            // (its labels are not stored per tree)
            agree[__ldg(bord + v)] += 2 * B;
            continue;
        }
        for (int b = 0; b < B; b++) {
            const uint32_t ones = __ldg(s1 + (size_t)b * ncomp + C);
            const uint32_t mine = (__ldg(pp + ((size_t)b * n + v) * ps) >> 31) ? ones : cs - ones;
            const uint32_t other = cs - mine;
            d += mine > other ? 2 : (mine == other ? 1 : 0);
        }
        agree[__ldg(bord + v)] += d;
    }
}

static unsigned grid_cap(int64_t work, int threads, int sms, int per_sm) {
    int64_t b = (work + threads - 1) / threads;
    int64_t cap = (int64_t)sms * per_sm;
    return (unsigned)std::max<int64_t>(1, std::min(b, cap));
}

int run_batch_cycles(const Graph &g, Workspace &ws, int B, int group, int walk,
                     cudaStream_t st, int64_t *launches, int jump, int linear, int ept) {
    CycleParams P;
    const bool descent = walk == 1, paper = walk == 2;
    if (walk == 3 && !ws.prec) { set_error("walk 3 needs layout 2"); return GB_EINVAL; }
    if (walk != 0 || !ws.jrec) jump = 1;
    P.jrec = ws.jrec;
    P.edges = g.edges_i; P.n = g.n; P.m = g.m;
    P.pp = ws.pp; P.rec = ws.rec; P.crec = ws.crec; P.clist = ws.clist;
    P.irec = ws.irec;
    P.prec = ws.prec;
    P.linear = linear;
    P.tbase = nullptr; P.tnbr = nullptr; P.trng = nullptr;
    const bool irec = ws.irec_layout && walk == 0;
    if (irec) jump = 1;
    P.fbits = ws.fbits; P.tstat = ws.tstat;
    P.words = (g.m + 31) / 32;
    if (P.words == 0) return GB_OK;
    if (paper) group = 1;   // one tree's lists at a time
    group = std::max(1, std::min(group, kMaxGroup));
    if (paper && !ws.ptbase) {
        GB_CUDA_TRY(cudaMalloc(&ws.ptbase, sizeof(uint32_t) * (size_t)(2 * (g.n + 1))));
        GB_CUDA_TRY(cudaMalloc(&ws.ptnbr, sizeof(uint32_t) * (size_t)(2 * g.n + 2)));
        GB_CUDA_TRY(cudaMalloc(&ws.ptrng, sizeof(uint2) * (size_t)(2 * g.n + 2)));
    }
    for (int b0 = 0; b0 < B; b0 += group) {
        P.b0 = b0;
        P.G = std::min(group, B - b0);
        unsigned grid = grid_cap(P.words * 32, kCycleBlock, g.num_sms, 8);
        if (jump > 1) {
            const unsigned bx = grid_cap(g.n, 256, g.num_sms, std::max(1, 8 / P.G));
            if (jump == 2) k_build_jump<2><<<dim3(bx, P.G), 256, 0, st>>>(ws.rec + (size_t)b0 * g.n, ws.jrec, g.n);
            else k_build_jump<4><<<dim3(bx, P.G), 256, 0, st>>>(ws.rec + (size_t)b0 * g.n, ws.jrec, g.n);
            ++*launches;
        }
        if (paper) {
            // the paper's partitioned tree-edge lists of tree b0 (pre order)
            const size_t nb = (size_t)b0 * g.n;
            uint32_t *tcnt = ws.ptbase + (g.n + 1);
            const unsigned gx = grid_cap(g.n + 1, 256, g.num_sms, 8);
            k_paper_counts<<<gx, 256, 0, st>>>(ws.crec + nb, g.n, tcnt);
            int rc = exclusive_scan_u32(tcnt, ws.ptbase, g.n + 1, ws.scan_tmp, ws.scan_tmp_elems, st, launches);
            if (rc) return rc;
            k_paper_fill<<<gx, 256, 0, st>>>(ws.rec + nb, ws.crec + nb, ws.clist, ws.ptbase, g.n, ws.ptnbr, ws.ptrng);
            *launches += 2;
            P.tbase = ws.ptbase; P.tnbr = ws.ptnbr; P.trng = ws.ptrng;
            k_cycles_paper<<<grid, kCycleBlock, 0, st>>>(P);
        }
        else if (irec && ept == 2) k_cycles_irec_m<2><<<grid_cap(P.words * 16, kCycleBlock, g.num_sms, 8), kCycleBlock, 0, st>>>(P);
        else if (irec && ept == 4) k_cycles_irec_m<4><<<grid_cap(P.words * 8, kCycleBlock, g.num_sms, 8), kCycleBlock, 0, st>>>(P);
        else if (irec) k_cycles_irec<<<grid, kCycleBlock, 0, st>>>(P);
        else if (walk == 3) k_cycles_pclimb<<<grid, kCycleBlock, 0, st>>>(P);
        else if (descent) k_cycles_descent<<<grid, kCycleBlock, 0, st>>>(P);
        else if (jump == 2) k_cycles_jump<2><<<grid, kCycleBlock, 0, st>>>(P);
        else if (jump == 4) k_cycles_jump<4><<<grid, kCycleBlock, 0, st>>>(P);
        else k_cycles_two_ended<<<grid, kCycleBlock, 0, st>>>(P);
        ++*launches;
    }
    GB_CUDA_TRY(cudaGetLastError());
    return GB_OK;
}

int run_batch_accumulate(const Graph &g, Workspace &ws, int B, int32_t *d_cnt, int32_t *d_agree,
                         cudaStream_t st, int64_t *launches) {
    const int64_t words = (g.m + 31) / 32;
    if (g.m) {
        k_accumulate_edges<<<grid_cap(g.m, 256, g.num_sms, 16), 256, 0, st>>>(ws.fbits, words, g.m, B, d_cnt);
        ++*launches;
    }
    k_accumulate_agree<<<grid_cap(g.n, 256, g.num_sms, 16), 256, 0, st>>>(
        label_words(ws), label_stride(ws), ws.s1, g.comp_i, g.coff, g.bord, g.n, g.ncomp, B, d_agree);
    ++*launches;
    GB_CUDA_TRY(cudaGetLastError());
    return GB_OK;
}

}  // namespace gb
