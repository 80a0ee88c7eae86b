// gb_ingest.cu -- §8 row a.1: CSR ingest with per-edge ids (once per load).
//
// one compact CSR holds Sigma; L238: 1-bit sign flags packed
// next to the 31-bit ids; L333: the paper keeps only the LCC -- here forests
// are accepted (reading R3), so connected components are labelled once.
//
// Everything runs on the device: validation (sorted simple symmetric rows,
// signs +-1 and symmetric), edge ids eid(u,v) = rank of (min,max) (the rank
// of an upper slot is ebase[u] + its position among row u's upper slots),
// packed adjacency words, the edge table, and connected components (hook to
// the smaller root + pointer jumping, so each root is its component's
// minimum vertex and components rank by minimum vertex).
#include "gb_internal.cuh"
#include "../../include/graphb.h"


#include <algorithm>
#include <vector>

namespace gb {

// ---------------------------------------------------------------------------
// Exclusive scan of uint32 (wrapping), three kernels: tile reduce, scan of the
// tile sums in one CTA, tile scan + offset.
// ---------------------------------------------------------------------------
constexpr int kScanThreads = 256;
constexpr int kScanItems = 8;
constexpr int kScanTile = kScanThreads * kScanItems;

__device__ __forceinline__ uint32_t warp_incl_scan(uint32_t v) {
    const int lane = threadIdx.x & 31;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
        uint32_t y = __shfl_up_sync(0xFFFFFFFFu, v, d);
        if (lane >= d) v += y;
    }
    return v;
}

// block-wide exclusive scan of one value per thread; returns the block total
__device__ __forceinline__ uint32_t block_excl_scan(uint32_t v, uint32_t &excl) {
    __shared__ uint32_t wsum[32];
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    uint32_t incl = warp_incl_scan(v);
    if (lane == 31) wsum[wid] = incl;
    __syncthreads();
    if (wid == 0) {
        uint32_t s = lane < (int)(blockDim.x >> 5) ? wsum[lane] : 0;
        s = warp_incl_scan(s);
        wsum[lane] = s;
    }
    __syncthreads();
    uint32_t base = wid ? wsum[wid - 1] : 0;
    uint32_t total = wsum[(blockDim.x >> 5) - 1];
    excl = base + incl - v;
    __syncthreads();
    return total;
}

__global__ void k_scan_reduce(const uint32_t *__restrict__ in, int64_t count,
                              uint32_t *__restrict__ part) {
    int64_t base = (int64_t)blockIdx.x * kScanTile;
    uint32_t s = 0;
#pragma unroll
    for (int i = 0; i < kScanItems; i++) {
        int64_t k = base + (int64_t)threadIdx.x * kScanItems + i;
        if (k < count) s += in[k];
    }
    uint32_t ex;
    uint32_t tot = block_excl_scan(s, ex);
    if (threadIdx.x == 0) part[blockIdx.x] = tot;
}

__global__ void k_scan_partials(uint32_t *part, int64_t nparts) {
    __shared__ uint32_t carry;
    if (threadIdx.x == 0) carry = 0;
    __syncthreads();
    for (int64_t b = 0; b < nparts; b += blockDim.x) {
        int64_t k = b + threadIdx.x;
        uint32_t v = k < nparts ? part[k] : 0;
        uint32_t ex;
        uint32_t tot = block_excl_scan(v, ex);
        if (k < nparts) part[k] = carry + ex;
        __syncthreads();
        if (threadIdx.x == 0) carry += tot;
        __syncthreads();
    }
}

__global__ void k_scan_down(const uint32_t *__restrict__ in, uint32_t *__restrict__ out,
                            int64_t count, const uint32_t *__restrict__ part) {
    int64_t base = (int64_t)blockIdx.x * kScanTile + (int64_t)threadIdx.x * kScanItems;
    uint32_t v[kScanItems];
    uint32_t s = 0;
#pragma unroll
    for (int i = 0; i < kScanItems; i++) {
        v[i] = (base + i < count) ? in[base + i] : 0;
        s += v[i];
    }
    uint32_t ex;
    block_excl_scan(s, ex);
    uint32_t run = part[blockIdx.x] + ex;
#pragma unroll
    for (int i = 0; i < kScanItems; i++) {
        if (base + i < count) out[base + i] = run;
        run += v[i];
    }
}

size_t scan_tmp_elems(int64_t count) { return (size_t)((count + kScanTile - 1) / kScanTile) + 1; }

int exclusive_scan_u32(const uint32_t *in, uint32_t *out, int64_t count, uint32_t *tmp,
                       size_t tmp_elems, cudaStream_t st, int64_t *launches) {
    if (count <= 0) return GB_OK;
    int64_t nb = (count + kScanTile - 1) / kScanTile;
    if ((size_t)nb > tmp_elems) { set_error("scan workspace too small"); return GB_ENOMEM; }
    k_scan_reduce<<<(unsigned)nb, kScanThreads, 0, st>>>(in, count, tmp);
    k_scan_partials<<<1, 1024, 0, st>>>(tmp, nb);
    k_scan_down<<<(unsigned)nb, kScanThreads, 0, st>>>(in, out, count, tmp);
    *launches += 3;
    GB_CUDA_TRY(cudaGetLastError());
    return GB_OK;
}

// ---------------------------------------------------------------------------
// Stable LSD radix sort of (key, value) pairs, 8-bit digits (used twice at
// ingest: vertices grouped by component, and the degree-sorted view).  One
// warp owns a tile of 256 consecutive elements: pass 1 counts the tile's
// digits, an exclusive scan over the digit-major count matrix gives every
// (digit, tile) its output run, pass 2 walks the tile in order, 32 elements
// at a time, ranking equal digits with __match_any_sync -- stable.
// ---------------------------------------------------------------------------
constexpr int kRsWarps = 8;
constexpr int kRsTile = 256;      // elements per warp tile

__device__ __forceinline__ uint32_t rs_digit(uint32_t k, int shift, uint32_t flip) {
    return ((k >> shift) & 255u) ^ flip;
}

__global__ void k_rs_hist(const uint32_t *__restrict__ keys, int64_t n, int shift, uint32_t flip,
                          uint32_t *__restrict__ hist, int64_t ntiles) {
    __shared__ uint32_t h[kRsWarps][256];
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    for (int d = lane; d < 256; d += 32) h[wid][d] = 0;
    __syncwarp();
    const int64_t tile = (int64_t)blockIdx.x * kRsWarps + wid;
    if (tile >= ntiles) return;
    const int64_t base = tile * kRsTile;
    for (int c = 0; c < kRsTile / 32; c++) {
        const int64_t i = base + c * 32 + lane;
        if (i < n) atomicAdd(&h[wid][rs_digit(__ldg(keys + i), shift, flip)], 1u);
    }
    __syncwarp();
    for (int d = lane; d < 256; d += 32) hist[(int64_t)d * ntiles + tile] = h[wid][d];
}

__global__ void k_rs_scatter(const uint32_t *__restrict__ kin, const uint32_t *__restrict__ vin,
                             uint32_t *__restrict__ kout, uint32_t *__restrict__ vout, int64_t n,
                             int shift, uint32_t flip, const uint32_t *__restrict__ off, int64_t ntiles) {
    __shared__ uint32_t run[kRsWarps][256];
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    const int64_t tile = (int64_t)blockIdx.x * kRsWarps + wid;
    if (tile >= ntiles) return;      // warp-uniform
    for (int d = lane; d < 256; d += 32) run[wid][d] = __ldg(off + (int64_t)d * ntiles + tile);
    __syncwarp();
    const uint32_t lt = (1u << lane) - 1u;
    const int64_t base = tile * kRsTile;
    for (int c = 0; c < kRsTile / 32; c++) {
        const int64_t i = base + c * 32 + lane;
        const bool valid = i < n;
        const uint32_t k = valid ? __ldg(kin + i) : 0u;
        const uint32_t d = rs_digit(k, shift, flip);
        const uint32_t peers = __match_any_sync(0xFFFFFFFFu, valid ? d : 0x100u + (uint32_t)lane);
        const uint32_t b = valid ? run[wid][d] : 0u;
        __syncwarp();
        if (valid) {
            const uint32_t pos = b + __popc(peers & lt);
            kout[pos] = k;
            vout[pos] = __ldg(vin + i);
            if (lane == __ffs(peers) - 1) run[wid][d] = b + __popc(peers);
        }
        __syncwarp();
    }
}

// temporaries: 2n (ping-pong keys / values) + 256 * ceil(n / 256) (counts)
size_t radix_tmp_elems(int64_t n) { return (size_t)(2 * n + 256 * ((n + kRsTile - 1) / kRsTile) + 64); }

// keys_in -> keys_out, vals_in -> vals_out over key bits [0, bits), stable;
// descending order of keys if `desc` (equal keys keep their input order)
static int radix_sort_pairs(const uint32_t *kin, uint32_t *kout, const uint32_t *vin, uint32_t *vout,
                            int64_t n, int bits, bool desc, uint32_t *tmp, uint32_t *scan_tmp,
                            size_t scan_elems, cudaStream_t st, int64_t *launches) {
    if (n <= 0) return GB_OK;
    const int64_t ntiles = (n + kRsTile - 1) / kRsTile;
    uint32_t *ktmp = tmp, *vtmp = tmp + n, *hist = tmp + 2 * n;
    const int passes = std::max(1, (bits + 7) / 8);
    const uint32_t flip = desc ? 255u : 0u;
    const unsigned blocks = (unsigned)((ntiles + kRsWarps - 1) / kRsWarps);
    const uint32_t *ks = kin, *vs = vin;
    for (int p = 0; p < passes; p++) {
        const bool to_out = ((passes - 1 - p) % 2) == 0;
        uint32_t *kd = to_out ? kout : ktmp, *vd = to_out ? vout : vtmp;
        k_rs_hist<<<blocks, kRsWarps * 32, 0, st>>>(ks, n, 8 * p, flip, hist, ntiles);
        int rc = exclusive_scan_u32(hist, hist, 256 * ntiles, scan_tmp, scan_elems, st, launches);
        if (rc) return rc;
        k_rs_scatter<<<blocks, kRsWarps * 32, 0, st>>>(ks, vs, kd, vd, n, 8 * p, flip, hist, ntiles);
        *launches += 2;
        ks = kd;
        vs = vd;
    }
    GB_CUDA_TRY(cudaGetLastError());
    return GB_OK;
}

// ---------------------------------------------------------------------------
// Validation + edge ids
// ---------------------------------------------------------------------------
enum : uint32_t {
    kErrRowPtr = 1u << 0, kErrColRange = 1u << 1, kErrSelfLoop = 1u << 2,
    kErrUnsorted = 1u << 3, kErrSign = 1u << 4, kErrMirror = 1u << 5,
    kErrMirrorSign = 1u << 6,
};

__global__ void k_rowptr(const int64_t *__restrict__ rp64, int64_t n, int64_t slots,
                         uint32_t *__restrict__ rp, uint32_t *err) {
    for (int64_t u = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; u <= n;
         u += (int64_t)gridDim.x * blockDim.x) {
        int64_t a = rp64[u];
        bool bad = a < 0 || a > slots || (u < n && rp64[u + 1] < a);
        if (u == 0 && a != 0) bad = true;
        if (u == n && a != slots) bad = true;
        if (bad) atomicOr(err, kErrRowPtr);
        rp[u] = (uint32_t)(bad ? 0 : a);
    }
}

// row containing slot j: largest u with rp[u] <= j (rows may be empty)
__device__ __forceinline__ uint32_t row_of_slot(const uint32_t *__restrict__ rp, int64_t n,
                                                uint32_t j) {
    uint32_t lo = 0, hi = (uint32_t)n;  // rp[lo] <= j < rp[hi]
    while (hi - lo > 1) {
        uint32_t mid = lo + ((hi - lo) >> 1);
        if (__ldg(rp + mid) <= j) lo = mid; else hi = mid;
    }
    return lo;
}

// position of value x in the sorted row u, or kNone
__device__ __forceinline__ uint32_t find_in_row(const uint32_t *__restrict__ rp,
                                                const int32_t *__restrict__ col, uint32_t u,
                                                int32_t x) {
    uint32_t lo = __ldg(rp + u), hi = __ldg(rp + u + 1);
    while (lo < hi) {
        uint32_t mid = lo + ((hi - lo) >> 1);
        int32_t c = __ldg(col + mid);
        if (c == x) return mid;
        if (c < x) lo = mid + 1; else hi = mid;
    }
    return kNone;
}

// first slot of row u whose column exceeds u (the upper part of the row)
__global__ void k_upper(const uint32_t *__restrict__ rp, const int32_t *__restrict__ col,
                        int64_t n, uint32_t *__restrict__ uptr, uint32_t *__restrict__ upc) {
    for (int64_t u = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; u < n;
         u += (int64_t)gridDim.x * blockDim.x) {
        uint32_t lo = rp[u], hi = rp[u + 1], end = hi;
        while (lo < hi) {
            uint32_t mid = lo + ((hi - lo) >> 1);
            if (col[mid] <= (int32_t)u) lo = mid + 1; else hi = mid;
        }
        uptr[u] = lo;
        upc[u] = end - lo;
    }
}

__global__ void k_slots(const uint32_t *__restrict__ rp, const int32_t *__restrict__ col,
                        const int8_t *__restrict__ sign, int64_t n, uint64_t slots,
                        const uint32_t *__restrict__ uptr, const uint32_t *__restrict__ ebase,
                        uint32_t *__restrict__ adj, uint32_t *__restrict__ adj_eid,
                        uint2 *__restrict__ edges, uint32_t *err) {
    // a warp takes 32 consecutive slots: the rows of its first and last slot
    // by binary search over all rows, every lane's row by a search between them
    const int lane = threadIdx.x & 31;
    const uint64_t nwarp = ((uint64_t)gridDim.x * blockDim.x) >> 5;
    for (uint64_t base = ((uint64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5 << 5; base < slots;
         base += nwarp * 32) {
        const uint64_t j = base + lane;
        uint32_t r = 0;
        if (lane == 0) r = row_of_slot(rp, n, (uint32_t)base);
        if (lane == 31) r = row_of_slot(rp, n, (uint32_t)min(base + 31, slots - 1));
        const uint32_t r0 = __shfl_sync(0xFFFFFFFFu, r, 0), r1 = __shfl_sync(0xFFFFFFFFu, r, 31);
        if (j >= slots) continue;
        uint32_t u = r0, hi = r1 + 1;  // rp[u] <= j < rp[hi]
        while (hi - u > 1) {
            const uint32_t mid = u + ((hi - u) >> 1);
            if (__ldg(rp + mid) <= (uint32_t)j) u = mid; else hi = mid;
        }
        int32_t v = col[j];
        int8_t s = sign[j];
        uint32_t e = 0;
        uint32_t bad = 0;
        if (v < 0 || v >= n) bad |= kErrColRange;
        if (v == (int32_t)u) bad |= kErrSelfLoop;
        if (j > rp[u] && col[j - 1] >= v) bad |= kErrUnsorted;
        if (s != 1 && s != -1) bad |= kErrSign;
        if (!(bad & kErrColRange)) {
            uint32_t mj = find_in_row(rp, col, (uint32_t)v, (int32_t)u);
            if (mj == kNone) bad |= kErrMirror;
            else {
                if (sign[mj] != s) bad |= kErrMirrorSign;
                if (v > (int32_t)u) e = ebase[u] + ((uint32_t)j - uptr[u]);
                else e = ebase[v] + (mj - uptr[v]);
            }
        }
        if (bad) { atomicOr(err, bad); continue; }
        uint32_t negb = s < 0 ? kNegBit : 0u;
        adj[j] = (uint32_t)v | negb;
        adj_eid[j] = e;
        if (v > (int32_t)u) edges[e] = make_uint2(u, (uint32_t)v | negb);
    }
}

// ---------------------------------------------------------------------------
// Connected components: hook the larger root under the smaller one, with
// pointer jumping (each final root = minimum vertex of its component).
// ---------------------------------------------------------------------------
__device__ __forceinline__ int32_t cc_find(int32_t *lab, int32_t x) {
    while (true) {
        int32_t p = ((volatile int32_t *)lab)[x];
        if (p == x) return x;
        int32_t gp = ((volatile int32_t *)lab)[p];
        if (p != gp) ((volatile int32_t *)lab)[x] = gp;
        x = p;
    }
}

__global__ void k_cc_init(int32_t *lab, int64_t n) {
    for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < n;
         v += (int64_t)gridDim.x * blockDim.x)
        lab[v] = (int32_t)v;
}

__device__ __forceinline__ void cc_hook(int32_t *lab, int32_t x, int32_t y) {
    int32_t a = cc_find(lab, x), b = cc_find(lab, y);
    while (a != b) {
        if (a < b) { int32_t t = a; a = b; b = t; }
        int32_t old = atomicCAS(lab + a, a, b);
        if (old == a) break;
        a = cc_find(lab, old);
        b = cc_find(lab, b);
    }
}

// Components in the manner of Afforest: every vertex is first hooked to its
// first two neighbours (two cheap rounds that join almost all of a large
// component), the largest component is identified from a sample, and only
// the vertices outside it hook their remaining edges.  Hooking is still
// "larger root under smaller", so every root is its component's minimum
// vertex, as with the full edge pass.
__global__ void k_cc_link(const uint32_t *__restrict__ rp, const uint32_t *__restrict__ adj, int64_t n,
                          uint32_t k, int32_t *lab) {
    for (int64_t u = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; u < n;
         u += (int64_t)gridDim.x * blockDim.x) {
        const uint32_t j = __ldg(rp + u) + k;
        if (j < __ldg(rp + u + 1)) cc_hook(lab, (int32_t)u, (int32_t)(__ldg(adj + j) & kIdMask));
    }
}

__global__ void k_cc_compress(int32_t *lab, int64_t n) {
    for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < n;
         v += (int64_t)gridDim.x * blockDim.x)
        lab[v] = cc_find(lab, (int32_t)v);
}

__global__ void k_cc_sample(int32_t *lab, int64_t n, int32_t *out, int count) {
    const int i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i < count) out[i] = cc_find(lab, (int32_t)(((uint64_t)i * 2654435761ull) % (uint64_t)n));
}

// the remaining edges (from neighbour k on) of every vertex outside component big
__global__ void k_cc_rest(const uint32_t *__restrict__ rp, const uint32_t *__restrict__ adj, int64_t n,
                          uint32_t k, int32_t big, int32_t *lab) {
    for (int64_t u = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; u < n;
         u += (int64_t)gridDim.x * blockDim.x) {
        const uint32_t e = __ldg(rp + u + 1);
        uint32_t j = __ldg(rp + u) + k;
        if (j >= e || cc_find(lab, (int32_t)u) == big) continue;
        for (; j < e; j++) cc_hook(lab, (int32_t)u, (int32_t)(__ldg(adj + j) & kIdMask));
    }
}

// final roots go to a separate array: other threads' pointer jumping may still
// write lab[] while this kernel runs
__global__ void k_cc_finish(int32_t *lab, int64_t n, uint32_t *is_root, uint32_t *root) {
    for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < n;
         v += (int64_t)gridDim.x * blockDim.x) {
        int32_t r = cc_find(lab, (int32_t)v);
        root[v] = (uint32_t)r;
        is_root[v] = (r == (int32_t)v) ? 1u : 0u;
    }
}

__global__ void k_cc_rank(const uint32_t *__restrict__ root, const uint32_t *__restrict__ rank,
                          int64_t n, int32_t *__restrict__ comp) {
    for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < n;
         v += (int64_t)gridDim.x * blockDim.x)
        comp[v] = (int32_t)rank[root[v]];
}

// Components grouped on the device: a stable radix sort of (comp, v) lists
// every component's vertices in ascending order; a component starts where the
// sorted key changes.  The largest component (ties to the smaller rank) is a
// 64-bit atomicMax of (size << 32 | ~rank).
__global__ void k_comp_keys(const int32_t *__restrict__ comp, int64_t n, uint32_t *__restrict__ keys,
                            uint32_t *__restrict__ ids) {
    for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < n;
         v += (int64_t)gridDim.x * blockDim.x) {
        keys[v] = (uint32_t)comp[v];
        ids[v] = (uint32_t)v;
    }
}

__global__ void k_comp_offsets(const uint32_t *__restrict__ skeys, int64_t n, int64_t nc,
                               int32_t *__restrict__ coff) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n;
         i += (int64_t)gridDim.x * blockDim.x) {
        const uint32_t k = skeys[i];
        if (i == 0 || skeys[i - 1] != k) coff[k] = (int32_t)i;
        if (i == 0) coff[nc] = (int32_t)n;
    }
}

__global__ void k_comp_big(const int32_t *__restrict__ coff, int64_t nc, unsigned long long *big) {
    unsigned long long best = 0;
    for (int64_t c = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; c < nc;
         c += (int64_t)gridDim.x * blockDim.x) {
        const unsigned long long sz = (unsigned long long)(coff[c + 1] - coff[c]);
        best = max(best, (sz << 32) | (0xFFFFFFFFull - (unsigned long long)c));
    }
    if (best) atomicMax(big, best);
}

__global__ void k_big_flags(const int32_t *__restrict__ coff, int64_t nc, uint32_t *__restrict__ flag) {
    for (int64_t c = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; c <= nc;
         c += (int64_t)gridDim.x * blockDim.x)
        flag[c] = c < nc && coff[c + 1] - coff[c] >= 2 ? 1u : 0u;
}

__global__ void k_big_fill(const uint32_t *__restrict__ flag, const uint32_t *__restrict__ pos, int64_t nc,
                           int32_t *__restrict__ bigc) {
    for (int64_t c = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; c < nc;
         c += (int64_t)gridDim.x * blockDim.x)
        if (flag[c]) bigc[pos[c]] = (int32_t)c;
}

// work items of the multi-source BFS: chunks of <= kChunk slots of every
// vertex heavier than kLight (internal ids 0 .. nlight0-1, degree-sorted)
__global__ void k_item_counts(const uint32_t *__restrict__ brow, int64_t nlight0, uint32_t *__restrict__ cnt) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < nlight0;
         i += (int64_t)gridDim.x * blockDim.x)
        cnt[i] = (brow[i + 1] - brow[i] + (uint32_t)kChunk - 1) / (uint32_t)kChunk;
}

__global__ void k_item_fill(const uint32_t *__restrict__ brow, const uint32_t *__restrict__ start,
                            int64_t nlight0, uint2 *__restrict__ items) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < nlight0;
         i += (int64_t)gridDim.x * blockDim.x) {
        const uint32_t s0 = brow[i], s1 = brow[i + 1];
        uint32_t o = start[i];
        for (uint32_t s = s0; s < s1; s += (uint32_t)kChunk) items[o++] = make_uint2((uint32_t)i, s);
    }
}

// ---------------------------------------------------------------------------
// Degree-sorted view for the multi-source BFS (gb_msbfs.cu)
// ---------------------------------------------------------------------------
// the edge table and the component ranks in internal ids (the tree pipeline's
// index space: hubs first, so the parents -- mostly high-degree vertices --
// cluster at the front of every per-tree label array)
__global__ void k_internal_edges(const uint2 *__restrict__ edges, const uint32_t *__restrict__ brank,
                                 int64_t m, uint2 *__restrict__ edges_i) {
    for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < m;
         e += (int64_t)gridDim.x * blockDim.x) {
        const uint2 ed = edges[e];
        edges_i[e] = make_uint2(brank[ed.x], brank[ed.y & kIdMask] | (ed.y & kNegBit));
    }
}

__global__ void k_internal_comp(const int32_t *__restrict__ comp, const uint32_t *__restrict__ bord,
                                int64_t n, int32_t *__restrict__ comp_i) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n;
         i += (int64_t)gridDim.x * blockDim.x)
        comp_i[i] = comp[bord[i]];
}

__global__ void k_degrees(const uint32_t *__restrict__ rp, int64_t n, uint32_t *__restrict__ deg,
                          uint32_t *__restrict__ ids) {
    for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < n;
         v += (int64_t)gridDim.x * blockDim.x) {
        deg[v] = rp[v + 1] - rp[v];
        ids[v] = (uint32_t)v;
    }
}

__global__ void k_view_rank(const uint32_t *__restrict__ bord, const uint32_t *__restrict__ sdeg,
                            int64_t n, uint32_t *__restrict__ brank, unsigned long long *counts) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n;
         i += (int64_t)gridDim.x * blockDim.x) {
        brank[bord[i]] = (uint32_t)i;
        const uint32_t d = sdeg[i];
        if (d > (uint32_t)kLight) atomicAdd(counts, 1ull);
        if (d > (uint32_t)kChunk) atomicAdd(counts + 1, 1ull);
        if (d == 0) atomicAdd(counts + 2, 1ull);
    }
}

__global__ void k_view_slots(const uint32_t *__restrict__ rp, const uint32_t *__restrict__ adj,
                             const uint32_t *__restrict__ brow, const uint32_t *__restrict__ bord,
                             const uint32_t *__restrict__ brank, int64_t n, uint64_t slots,
                             uint32_t *__restrict__ badj, uint32_t *__restrict__ borig) {
    for (uint64_t j = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; j < slots;
         j += (uint64_t)gridDim.x * blockDim.x) {
        const uint32_t i = row_of_slot(brow, n, (uint32_t)j);
        const uint32_t o = bord[i];
        const uint32_t x = adj[rp[o] + ((uint32_t)j - brow[i])];
        badj[j] = brank[x & kIdMask] | (x & kNegBit);
        borig[j] = x & kIdMask;
    }
}

static unsigned grid_for(int64_t work, int threads, int sms) {
    int64_t b = (work + threads - 1) / threads;
    int64_t cap = (int64_t)sms * 16;
    if (b > cap) b = cap;
    if (b < 1) b = 1;
    return (unsigned)b;
}

static const char *err_text(uint32_t f) {
    if (f & kErrRowPtr) return "row_ptr must start at 0, be non-decreasing and end at 2m";
    if (f & kErrColRange) return "column index out of range";
    if (f & kErrSelfLoop) return "self loop";
    if (f & kErrUnsorted) return "row not strictly increasing (unsorted or duplicate entry)";
    if (f & kErrSign) return "sign must be +1 or -1";
    if (f & kErrMirror) return "missing mirror entry (graph not symmetric)";
    if (f & kErrMirrorSign) return "mirror entry has a different sign";
    return "invalid graph";
}

int ingest(Graph &g, int64_t n, int64_t m, const int64_t *h_row_ptr, const int32_t *h_col,
           const int8_t *h_sign, cudaStream_t st, int64_t *launches) {
    const uint64_t slots = 2ull * (uint64_t)m;
    const int sms = g.num_sms;
    int64_t *d_rp64 = nullptr;
    int32_t *d_col = nullptr, *lab = nullptr;
    int8_t *d_sign = nullptr;
    uint32_t *d_err = nullptr, *uptr = nullptr, *upc = nullptr, *ebase = nullptr,
             *tmp = nullptr, *flag = nullptr, *rank = nullptr;
    std::vector<int32_t> smp;   // component sample (Afforest-style CC)
    int rc = GB_OK;
    uint32_t h_err = 0;
    size_t ntmp = scan_tmp_elems(std::max<int64_t>(n, 1));
    auto fail = [&](int code) { rc = code; };
#define ING_TRY(expr)                                                          \
    do {                                                                       \
        cudaError_t _e = (expr);                                               \
        if (_e != cudaSuccess) {                                               \
            set_error(std::string(#expr) + ": " + cudaGetErrorString(_e));     \
            fail(_e == cudaErrorMemoryAllocation ? GB_ENOMEM : GB_ECUDA);      \
            goto done;                                                         \
        }                                                                      \
    } while (0)
#define ING_ALLOC(ptr, slot, count)                                                         \
    do {                                                                                    \
        ptr = (decltype(ptr))arena(slot, sizeof(*ptr) * (size_t)std::max<uint64_t>((uint64_t)(count), 1)); \
        if (!ptr) { fail(GB_ENOMEM); goto done; }                                          \
    } while (0)
    ING_ALLOC(d_rp64, kArRowPtr64, n + 1);
    ING_ALLOC(d_col, kArCol, slots);
    ING_ALLOC(d_sign, kArSign, slots);
    ING_ALLOC(d_err, kArErr, 1);
    ING_ALLOC(g.row_ptr, kArRowPtr, n + 1);
    ING_ALLOC(g.adj, kArAdj, slots);
    ING_ALLOC(g.adj_eid, kArAdjEid, slots);
    ING_ALLOC(g.edges, kArEdges, m);
    ING_ALLOC(g.comp, kArComp, n);
    ING_ALLOC(g.cverts, kArCverts, n);
    ING_ALLOC(uptr, kArUptr, n);
    ING_ALLOC(upc, kArUpc, n);
    ING_ALLOC(ebase, kArEbase, n);
    ING_ALLOC(tmp, kArScanTmp, ntmp);
    ING_ALLOC(lab, kArLab, n);
    ING_ALLOC(flag, kArFlag, n);
    ING_ALLOC(rank, kArRank, n);
    ING_TRY(cudaMemcpyAsync(d_rp64, h_row_ptr, sizeof(int64_t) * (n + 1), cudaMemcpyHostToDevice, st));
    if (slots) {
        ING_TRY(cudaMemcpyAsync(d_col, h_col, sizeof(int32_t) * slots, cudaMemcpyHostToDevice, st));
        ING_TRY(cudaMemcpyAsync(d_sign, h_sign, slots, cudaMemcpyHostToDevice, st));
    }
    ING_TRY(cudaMemsetAsync(d_err, 0, sizeof(uint32_t), st));
    k_rowptr<<<grid_for(n + 1, 256, sms), 256, 0, st>>>(d_rp64, n, (int64_t)slots, g.row_ptr, d_err);
    ++*launches;
    ING_TRY(cudaMemcpyAsync(&h_err, d_err, sizeof(uint32_t), cudaMemcpyDeviceToHost, st));
    ING_TRY(cudaStreamSynchronize(st));
    if (h_err) { set_error(err_text(h_err)); fail(GB_EINVAL); goto done; }
    k_upper<<<grid_for(n, 256, sms), 256, 0, st>>>(g.row_ptr, d_col, n, uptr, upc);
    ++*launches;
    rc = exclusive_scan_u32(upc, ebase, n, tmp, ntmp, st, launches);
    if (rc) goto done;
    if (slots) {
        k_slots<<<grid_for((int64_t)slots, 256, sms), 256, 0, st>>>(
            g.row_ptr, d_col, d_sign, n, slots, uptr, ebase, g.adj, g.adj_eid, g.edges, d_err);
        ++*launches;
    }
    ING_TRY(cudaMemcpyAsync(&h_err, d_err, sizeof(uint32_t), cudaMemcpyDeviceToHost, st));
    ING_TRY(cudaStreamSynchronize(st));
    if (h_err) { set_error(err_text(h_err)); fail(GB_EINVAL); goto done; }
    // connected components
    k_cc_init<<<grid_for(n, 256, sms), 256, 0, st>>>(lab, n);
    ++*launches;
    if (m) {
        const int kSample = (int)std::min<int64_t>(1024, n);
        for (uint32_t k = 0; k < 2; k++) {
            k_cc_link<<<grid_for(n, 256, sms), 256, 0, st>>>(g.row_ptr, g.adj, n, k, lab);
            k_cc_compress<<<grid_for(n, 256, sms), 256, 0, st>>>(lab, n);
            *launches += 2;
        }
        int32_t *d_smp = reinterpret_cast<int32_t *>(flag);   // scratch until k_cc_finish
        k_cc_sample<<<(kSample + 255) / 256, 256, 0, st>>>(lab, n, d_smp, kSample);
        ++*launches;
        smp.resize(kSample);
        ING_TRY(cudaMemcpyAsync(smp.data(), d_smp, sizeof(int32_t) * kSample, cudaMemcpyDeviceToHost, st));
        ING_TRY(cudaStreamSynchronize(st));
        std::sort(smp.begin(), smp.end());
        int32_t big = smp[0];
        for (int i = 0, best = 0; i < kSample;) {
            int k = i;
            while (k < kSample && smp[k] == smp[i]) k++;
            if (k - i > best) { best = k - i; big = smp[i]; }
            i = k;
        }
        k_cc_rest<<<grid_for(n, 256, sms), 256, 0, st>>>(g.row_ptr, g.adj, n, 2, big, lab);
        ++*launches;
    }
    k_cc_finish<<<grid_for(n, 256, sms), 256, 0, st>>>(lab, n, flag, ebase);
    ++*launches;
    rc = exclusive_scan_u32(flag, rank, n, tmp, ntmp, st, launches);
    if (rc) goto done;
    k_cc_rank<<<grid_for(n, 256, sms), 256, 0, st>>>(ebase, rank, n, g.comp);
    ++*launches;
    {
        // component offsets and ascending member lists (device sort, no host pass)
        uint32_t nr[2] = {0, 0};
        ING_TRY(cudaMemcpyAsync(&nr[0], rank + (n - 1), sizeof(uint32_t), cudaMemcpyDeviceToHost, st));
        ING_TRY(cudaMemcpyAsync(&nr[1], flag + (n - 1), sizeof(uint32_t), cudaMemcpyDeviceToHost, st));
        ING_TRY(cudaStreamSynchronize(st));
        const int64_t nc = (int64_t)nr[0] + nr[1];
        uint32_t *keys = nullptr, *skeys = nullptr, *ids = nullptr;
        unsigned long long *big = nullptr;
        ING_ALLOC(keys, kArCkeys, 3 * n + 8);
        skeys = keys + n;
        ids = keys + 2 * n;
        big = (unsigned long long *)(((uintptr_t)(keys + 3 * n) + 7) & ~(uintptr_t)7);
        ING_ALLOC(g.coff, kArCoff, nc + 1);
        k_comp_keys<<<grid_for(n, 256, sms), 256, 0, st>>>(g.comp, n, keys, ids);
        ++*launches;
        int bits = 1;
        while (bits < 32 && (1ll << bits) < nc) bits++;
        uint32_t *sort_tmp = nullptr;
        ING_ALLOC(sort_tmp, kArSortTmp, radix_tmp_elems(n));
        {
            const size_t rs_scan = scan_tmp_elems(256 * ((n + 255) / 256));
            uint32_t *rs_stmp = nullptr;
            ING_ALLOC(rs_stmp, kArRsScan, rs_scan);
            rc = radix_sort_pairs(keys, skeys, ids, (uint32_t *)g.cverts, n, bits, false, sort_tmp,
                                  rs_stmp, rs_scan, st, launches);
            if (rc) goto done;
        }
        k_comp_offsets<<<grid_for(n, 256, sms), 256, 0, st>>>(skeys, n, nc, g.coff);
        ++*launches;
        ING_TRY(cudaMemsetAsync(big, 0, sizeof(unsigned long long), st));
        k_comp_big<<<grid_for(nc, 256, sms), 256, 0, st>>>(g.coff, nc, big);
        ++*launches;
        unsigned long long hb = 0;
        ING_TRY(cudaMemcpyAsync(&hb, big, sizeof(hb), cudaMemcpyDeviceToHost, st));
        ING_TRY(cudaStreamSynchronize(st));
        g.ncomp = nc;
        g.cbig = (int32_t)(0xFFFFFFFFull - (hb & 0xFFFFFFFFull));
        // components with >= 2 vertices (every tree roots each of them; a
        // single-vertex component is its own finished tree)
        uint32_t *bflag = nullptr, *bpos = nullptr;
        ING_ALLOC(bflag, kArBigFlag, 2 * nc + 2);
        bpos = bflag + nc + 1;
        k_big_flags<<<grid_for(nc + 1, 256, sms), 256, 0, st>>>(g.coff, nc, bflag);
        ++*launches;
        rc = exclusive_scan_u32(bflag, bpos, nc + 1, tmp, ntmp, st, launches);
        if (rc) goto done;
        ING_ALLOC(g.bigc, kArBigC, nc);
        k_big_fill<<<grid_for(nc, 256, sms), 256, 0, st>>>(bflag, bpos, nc, g.bigc);
        ++*launches;
        uint32_t hbig = 0;
        ING_TRY(cudaMemcpyAsync(&hbig, bpos + nc, sizeof(uint32_t), cudaMemcpyDeviceToHost, st));
        ING_TRY(cudaStreamSynchronize(st));
        g.nbig = (int64_t)hbig;
    }
    {
        // degree-sorted view: stable radix sort of the degrees (descending),
        // then the view's CSR with internal neighbour ids and original ids
        uint32_t *deg = nullptr, *sdeg = nullptr, *ids = nullptr;
        unsigned long long *cnt2 = nullptr;
        ING_ALLOC(deg, kArDeg, 3 * n + 12);
        sdeg = deg + n;
        ids = deg + 2 * n;
        cnt2 = (unsigned long long *)(((uintptr_t)(deg + 3 * n) + 7) & ~(uintptr_t)7);
        ING_ALLOC(g.brow, kArBrow, n + 1);
        ING_ALLOC(g.bord, kArBord, n);
        ING_ALLOC(g.brank, kArBrank, n);
        ING_ALLOC(g.badj, kArBadj, slots);
        ING_ALLOC(g.borig, kArBorig, slots);
        k_degrees<<<grid_for(n, 256, sms), 256, 0, st>>>(g.row_ptr, n, deg, ids);
        ++*launches;
        {
            // degrees are < n (simple graph): ceil(log2 n) key bits
            int dbits = 1;
            while (dbits < 32 && (1ll << dbits) < n) dbits++;
            uint32_t *sort_tmp = nullptr;
            ING_ALLOC(sort_tmp, kArSortTmp, radix_tmp_elems(n));
            const size_t rs_scan = scan_tmp_elems(256 * ((n + 255) / 256));
            uint32_t *rs_stmp = nullptr;
            ING_ALLOC(rs_stmp, kArRsScan, rs_scan);
            rc = radix_sort_pairs(deg, sdeg, ids, g.bord, n, dbits, true, sort_tmp, rs_stmp, rs_scan, st, launches);
            if (rc) goto done;
        }
        ING_TRY(cudaMemsetAsync(cnt2, 0, 3 * sizeof(unsigned long long), st));
        k_view_rank<<<grid_for(n, 256, sms), 256, 0, st>>>(g.bord, sdeg, n, g.brank, cnt2);
        ++*launches;
        rc = exclusive_scan_u32(sdeg, g.brow, n, tmp, ntmp, st, launches);
        if (rc) goto done;
        const uint32_t s32 = (uint32_t)slots;
        ING_TRY(cudaMemcpyAsync(g.brow + n, &s32, sizeof(uint32_t), cudaMemcpyHostToDevice, st));
        if (slots) {
            k_view_slots<<<grid_for((int64_t)slots, 256, sms), 256, 0, st>>>(
                g.row_ptr, g.adj, g.brow, g.bord, g.brank, n, slots, g.badj, g.borig);
            ++*launches;
        }
        unsigned long long hc[3] = {0, 0, 0};
        ING_TRY(cudaMemcpyAsync(hc, cnt2, sizeof(hc), cudaMemcpyDeviceToHost, st));
        ING_TRY(cudaStreamSynchronize(st));
        g.nlight0 = (int64_t)hc[0];
        g.nmulti = (int64_t)hc[1];
        g.niso = (int64_t)hc[2];          // isolated vertices: internal ids [n - niso, n)
        // work items: chunks of <= kChunk slots of every vertex heavier than kLight
        if (g.nlight0 > 0) {
            k_item_counts<<<grid_for(g.nlight0, 256, sms), 256, 0, st>>>(g.brow, g.nlight0, upc);
            ++*launches;
            rc = exclusive_scan_u32(upc, uptr, g.nlight0, tmp, ntmp, st, launches);
            if (rc) goto done;
            uint32_t hv[3] = {0, 0, 0};
            ING_TRY(cudaMemcpyAsync(&hv[0], uptr + (g.nlight0 - 1), sizeof(uint32_t), cudaMemcpyDeviceToHost, st));
            ING_TRY(cudaMemcpyAsync(&hv[1], upc + (g.nlight0 - 1), sizeof(uint32_t), cudaMemcpyDeviceToHost, st));
            if (g.nmulti < g.nlight0)
                ING_TRY(cudaMemcpyAsync(&hv[2], uptr + g.nmulti, sizeof(uint32_t), cudaMemcpyDeviceToHost, st));
            ING_TRY(cudaStreamSynchronize(st));
            g.nitems = (int64_t)hv[0] + hv[1];
            g.nmulti_items = g.nmulti < g.nlight0 ? (int64_t)hv[2] : g.nitems;
        } else {
            g.nitems = 0;
            g.nmulti_items = 0;
        }
        ING_ALLOC(g.items, kArItems, g.nitems);
        if (g.nitems) {
            k_item_fill<<<grid_for(g.nlight0, 256, sms), 256, 0, st>>>(g.brow, uptr, g.nlight0, g.items);
            ++*launches;
        }
        ING_ALLOC(g.edges_i, kArEdgesI, m);
        ING_ALLOC(g.comp_i, kArCompI, n);
        if (m) {
            k_internal_edges<<<grid_for(m, 256, sms), 256, 0, st>>>(g.edges, g.brank, m, g.edges_i);
            ++*launches;
        }
        k_internal_comp<<<grid_for(n, 256, sms), 256, 0, st>>>(g.comp, g.bord, n, g.comp_i);
        ++*launches;
        ING_TRY(cudaStreamSynchronize(st));
    }
    g.n = n;
    g.m = m;
    g.slots = slots;
done:
#undef ING_TRY
#undef ING_ALLOC
    return rc;
}

}  // namespace gb
