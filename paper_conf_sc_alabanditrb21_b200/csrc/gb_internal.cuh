// gb_internal.cuh -- shared definitions of the graphB+ B200 library (not part
// of the C ABI).  Layout of the device state is documented in DESIGN.md
// "Data layout in HBM".
#pragma once
#include <cuda_runtime.h>
#include <cooperative_groups.h>
#include <stdint.h>
#include <string>

namespace gb {

constexpr uint32_t kNegBit = 0x80000000u;   // sign bit packed next to a 31-bit id (L238)
constexpr uint32_t kIdMask = 0x7FFFFFFFu;
constexpr int32_t kInf = 0x7F7F7F7F;         // "unvisited" BFS distance (memset 0x7F)
constexpr uint32_t kNone = 0xFFFFFFFFu;
constexpr int kMaxBatch = 128;               // trees per batch (smem tables)
constexpr int kBlock = 256;                  // threads per CTA of the cooperative kernels
constexpr int kMsBatch = 128;                // trees per multi-source BFS (one bit each, two 64-bit halves)
constexpr int kLight = 8;                    // BFS: degree <= kLight -> one lane per vertex
constexpr int kChunk = 256;                  // BFS: slots per warp work item of a heavier vertex

// ---------------------------------------------------------------------------
// Counter-based hash: SplitMix64 finaliser and its inverse (R4).
// tkey(seed,t) = mix(seed + G*(t+1)); rkey = mix(tkey ^ (K*(C+1)));
// ekey = mix(tkey + G*(e+1)).  mix is a bijection on 64-bit words, so an edge
// key decodes back to the edge id: e = (unmix(key) - tkey) * G^-1 - 1.
// ---------------------------------------------------------------------------
constexpr uint64_t kGolden = 0x9E3779B97F4A7C15ull;
constexpr uint64_t kGoldenInv = 0xF1DE83E19937733Dull;
constexpr uint64_t kMul1 = 0xBF58476D1CE4E5B9ull, kMul1Inv = 0x96DE1B173F119089ull;
constexpr uint64_t kMul2 = 0x94D049BB133111EBull, kMul2Inv = 0x319642B2D24D8EC3ull;
constexpr uint64_t kRootMul = 0xD1B54A32D192ED03ull;

__host__ __device__ __forceinline__ uint64_t mix64(uint64_t z) {
    z ^= z >> 30; z *= kMul1;
    z ^= z >> 27; z *= kMul2;
    z ^= z >> 31;
    return z;
}
__host__ __device__ __forceinline__ uint64_t unmix64(uint64_t z) {
    z ^= (z >> 31) ^ (z >> 62); z *= kMul2Inv;
    z ^= (z >> 27) ^ (z >> 54); z *= kMul1Inv;
    z ^= (z >> 30) ^ (z >> 60);
    return z;
}
__host__ __device__ __forceinline__ uint64_t tree_key(uint64_t seed, int64_t t) {
    return mix64(seed + kGolden * (uint64_t)(t + 1));
}
__host__ __device__ __forceinline__ uint64_t root_key(uint64_t tkey, int64_t comp) {
    return mix64(tkey ^ (kRootMul * (uint64_t)(comp + 1)));
}
__host__ __device__ __forceinline__ uint64_t edge_key(uint64_t tkey, uint32_t e) {
    return mix64(tkey + kGolden * ((uint64_t)e + 1));
}
__host__ __device__ __forceinline__ uint32_t edge_of_key(uint64_t tkey, uint64_t key) {
    return (uint32_t)((unmix64(key) - tkey) * kGoldenInv - 1);
}

// parent key of candidate u for w (reading R4): score in the high word, then
// (u << 1 | neg): the minimum picks the lowest score, ties to the smaller u,
// and carries the winner's id and the sign of the tree edge.  score = high
// 32 bits of mix64(tkey + G * (min(u,w) << 32 | max(u,w))), original ids.
__device__ __forceinline__ unsigned long long parent_key(uint64_t tk, uint32_t u, uint32_t w,
                                                         uint32_t neg) {
    const uint64_t lo = min(u, w), hi = max(u, w);
    const uint32_t score = (uint32_t)(mix64(tk + kGolden * ((lo << 32) | hi)) >> 32);
    return ((unsigned long long)score << 32) | ((unsigned long long)u << 1) | neg;
}

// ---------------------------------------------------------------------------
// L2 eviction-priority hints (createpolicy + ld/st .L2::cache_hint): the
// per-tree label arrays gathered at random are kept (evict_last) while the
// edge table streams through (evict_first).
// ---------------------------------------------------------------------------
__device__ __forceinline__ uint64_t l2_keep_policy() {
    uint64_t p;
    asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(p));
    return p;
}
__device__ __forceinline__ uint64_t l2_stream_policy() {
    uint64_t p;
    asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
    return p;
}
__device__ __forceinline__ uint2 ld_hint(const uint2 *ptr, uint64_t pol) {
    uint2 r;
    asm volatile("ld.global.nc.L2::cache_hint.v2.u32 {%0, %1}, [%2], %3;"
                 : "=r"(r.x), "=r"(r.y) : "l"(ptr), "l"(pol));
    return r;
}
__device__ __forceinline__ uint32_t ld_hint(const uint32_t *ptr, uint64_t pol) {
    uint32_t r;
    asm volatile("ld.global.nc.L2::cache_hint.u32 %0, [%1], %2;" : "=r"(r) : "l"(ptr), "l"(pol));
    return r;
}
__device__ __forceinline__ void st_hint(uint2 *ptr, uint2 v, uint64_t pol) {
    asm volatile("st.global.L2::cache_hint.v2.u32 [%0], {%1, %2}, %3;"
                 :: "l"(ptr), "r"(v.x), "r"(v.y), "l"(pol) : "memory");
}
__device__ __forceinline__ void st_hint(uint32_t *ptr, uint32_t v, uint64_t pol) {
    asm volatile("st.global.L2::cache_hint.u32 [%0], %1, %2;" :: "l"(ptr), "r"(v), "l"(pol) : "memory");
}

// ---------------------------------------------------------------------------
// Loaded graph (device arrays; immutable after gb_load_csr).  L236: a single
// compact CSR; L238: sign bits packed next to 31-bit vertex ids.
// ---------------------------------------------------------------------------
struct Graph {
    int64_t n = 0, m = 0, ncomp = 0;
    uint64_t slots = 0;                 // 2m
    uint32_t *row_ptr = nullptr;        // [n+1]
    uint32_t *adj = nullptr;            // [2m] col | neg<<31
    uint32_t *adj_eid = nullptr;        // [2m] eid of the slot
    uint2 *edges = nullptr;             // [m] {u, v | neg<<31}, u < v, index = eid (original ids)
    // The tree pipeline (level lists, Alg. 4 labels, the cycle walk, the agree
    // accumulation) runs on the internal ids of the degree-sorted view below:
    uint2 *edges_i = nullptr;           // [m] {brank u, brank v | neg<<31}, index = eid
    int32_t *comp_i = nullptr;          // [n] component rank of internal vertex i
    int32_t *comp = nullptr;            // [n] component rank (by minimum vertex)
    int32_t *coff = nullptr;            // [ncomp+1] component offsets (pre of the root)
    int32_t *cverts = nullptr;          // [n] vertices grouped by component, ascending
    int32_t cbig = 0;                   // largest component
    int32_t *bigc = nullptr;            // [nbig] components with >= 2 vertices
    int64_t nbig = 0;
    int64_t niso = 0;                   // isolated vertices (internal ids [n - niso, n))
    // Degree-sorted view for the multi-source BFS (gb_msbfs.cu): internal ids
    // 0..n-1 order the vertices by degree, descending (ties by original id),
    // so a warp's 32 consecutive vertices have similar degrees and the hubs
    // sit at the front.  Only the BFS uses internal ids; everything it emits
    // (level lists, parents) is in original ids.
    uint32_t *brow = nullptr;           // [n+1] row pointers of the view
    uint32_t *badj = nullptr;           // [2m] internal neighbour id | neg<<31
    uint32_t *borig = nullptr;          // [2m] original neighbour id
    uint32_t *bord = nullptr;           // [n] internal -> original
    uint32_t *brank = nullptr;          // [n] original -> internal
    uint2 *items = nullptr;             // [nitems] {internal vertex, first slot}: chunks of <= kChunk
                                        // slots of the vertices with degree > kLight
    int64_t nlight0 = 0;                // first internal id with degree <= kLight
    int64_t nitems = 0;
    int64_t nmulti = 0;                 // vertices with degree > kChunk (internal ids [0, nmulti))
    int64_t nmulti_items = 0;           // their chunks (items [0, nmulti_items))
    int dev = 0;
    int num_sms = 148;
};

// Per-batch workspace for B trees (arrays are [B][n] unless noted).
// "q" = queue order (BFS level lists), "v" = vertex order, "pre" = pre order.
struct Workspace {
    int B = 0;                 // capacity in trees
    int64_t n = 0;
    uint32_t *vst = nullptr;   // [B][(n+3)/4] BFS byte states (0 / 0x80 / 0x81 + level mod 127)
    uint32_t *qv = nullptr;    // q: level lists (vertices in BFS level order)
    uint32_t *qs = nullptr;    // q: slot prefix of each queued vertex within its level
    uint32_t *qr = nullptr;    // q: CSR row start of each queued vertex
    unsigned long long *pkeyq = nullptr; // q: parent key (score<<32 | parent<<1 | neg)
    uint64_t *lvl = nullptr;   // [B][n+2] packed (vertex count << 32 | slot count) per level
    uint32_t *vbase = nullptr; // [B][n+2] start of each level in qv
    uint32_t *size = nullptr;  // v: sum of the children's subtree sizes (Alg. 4 v_cnt - 1), walk 0
    unsigned long long *sz64 = nullptr; // v: (#children << 32 | subtree size), walk 1
    uint32_t *parq = nullptr;  // q: parent id | neg(parent edge)<<31
    uint32_t *offq = nullptr;  // q: offset of the child's range inside its parent's
    uint32_t *szq = nullptr;   // q: subtree size
    uint32_t *pp = nullptr;    // v: pre | pi<<31  (pi = root-path parity)      [layout 1]
    uint2 *rec = nullptr;      // pre: {up pre | neg<<31, size}                  [layout 1]
    uint4 *irec = nullptr;     // v: {parent | neg<<31, pre | pi<<31, size, 0}   [layout 0]
    uint32_t *prec = nullptr;  // pre: up pre | neg<<31 (4 bytes)                [layout 2, walk 3]
    bool irec_layout = false;  // layout 0 (walk 0 with one level per record, the default):
                               // records indexed by internal vertex id, written by the
                               // top-down pass itself; layout 1 (walk 1, option jump):
                               // pp by vertex + records by pre order (k_rec_scatter)
    uint32_t *fbits = nullptr; // [B][ceil(m/32)] flip bitmask
    void *wbuf = nullptr;      // option "sampler" = 1, "wilson" = 1: cycle-popping state (20n bytes)
    void *wseq = nullptr;      // option "sampler" = 1, 2: [W] trees of per-thread sampler state (13n bytes each);
                               // the first 4Wn bytes are the W parent arrays
    int wseq_cap = 0;
    uint64_t *wtkey = nullptr; // [kMaxBatch] tree keys of the sampled chunk
    int32_t *wparent = nullptr;// its tree (parent, -1 at the roots)
    int32_t *hlab = nullptr;   // option "harary": [3n + 16] CC labels, CC roots, BFS levels, flag
    uint2 *jrec = nullptr;     // [G][n][K] K-level ancestor records of one cycle group (option "jump")
    int jrec_cap = 0;          // G * K the buffer holds
    // multi-source BFS state (one bit per tree of the batch, internal ids)
    unsigned long long *vis = nullptr;  // [n][2] trees that reached the vertex (two 64-tree halves)
    unsigned long long *fr = nullptr;   // [2][n][2] frontier of level L / L+1
    unsigned long long *hacc = nullptr; // [nmulti][2] discoveries of multi-chunk vertices
    unsigned long long *hbest = nullptr;// [nmulti][128] their best parent keys
    int32_t *msflag = nullptr;          // [8]: [0..1] a multi-chunk vertex discovered something,
                                        // [4..6] frontier sizes (levels mod 3)
    uint32_t *mscnt = nullptr;          // [128][2048] per-block discovery counts
    unsigned long long *msprof = nullptr;  // [256][4] BFS phase timestamps (option "msprof")
    unsigned long long *pnew = nullptr;    // push-parent levels (<= 16 trees): [n] discoveries
    unsigned long long *pbest = nullptr;   // [n][16] best parent keys (all ones between uses)
    bool pp_ok = true;                     // option "push_parent"
    bool pp_nomem = false;                 // not enough free memory for the push-parent state
    uint32_t *fbm = nullptr;            // [6][ceil(n/32)] frontier bitmaps (3), finished bitmap,
                                        // two push bitmaps (direction optimisation)
    uint32_t *s1 = nullptr;    // [B][ncomp] #vertices with pi = 1 per component
    uint64_t *tkey = nullptr;  // [kMaxBatch]
    int32_t *depth = nullptr;  // [kMaxBatch]
    unsigned long long *tstat = nullptr;   // [kMaxBatch][2] {sum cycle length, cycles}
    unsigned long long *visited = nullptr; // [kMaxBatch] vertices reached (given trees)
    int32_t *maxd = nullptr;   // [1] max depth over the batch
    // walk 1 (Alg. 3 descent)
    uint32_t *cidxq = nullptr; // q: sibling index of each child (pre order)
    uint32_t *cstart = nullptr;// v: start of the child list (global position)
    uint32_t *clist = nullptr; // [B*n] children pre IDs, grouped by parent, ascending
    uint2 *crec = nullptr;     // pre: {cstart, #children}
    // walk 2 (the paper's lists, one tree at a time)
    uint32_t *ptbase = nullptr;  // [n+1] list starts (pre order) + [n+1] counts
    uint32_t *ptnbr = nullptr;   // [2n] neighbour pre IDs
    uint2 *ptrng = nullptr;      // [2n] two-word range/sign records
    uint32_t *scan_tmp = nullptr;
    size_t scan_tmp_elems = 0;
};

// subtree-size counters per tree (walk 0): the power of two >= n (gb_tree.cu szi)
inline int64_t size_slots(int64_t n) {
    int64_t s = 2;
    while (s < n) s <<= 1;
    return s;
}

struct BatchArgs {
    int B;                 // trees in this batch
    int64_t n, m;
    int64_t ncomp;
    uint64_t slots;
};

// ---------------------------------------------------------------------------
// Error handling
// ---------------------------------------------------------------------------
void set_error(const std::string &msg);

#define GB_CUDA_TRY(expr)                                                       \
    do {                                                                         \
        cudaError_t _e = (expr);                                                 \
        if (_e != cudaSuccess) {                                                 \
            ::gb::set_error(std::string(#expr) + ": " + cudaGetErrorString(_e)); \
            return GB_ECUDA;                                                     \
        }                                                                        \
    } while (0)

// ---------------------------------------------------------------------------
// Persistent grow-only device buffers for the graph and the ingest
// temporaries: a reload of a graph that fits reuses them (no cudaMalloc /
// cudaFree per load; all dynamic memory allocated once, L236).
// ---------------------------------------------------------------------------
enum ArenaSlot {
    kArRowPtr64, kArCol, kArSign, kArErr, kArRowPtr, kArAdj, kArAdjEid, kArEdges, kArComp,
    kArCverts, kArUptr, kArUpc, kArEbase, kArScanTmp, kArLab, kArFlag, kArRank, kArCoff,
    kArBrow, kArBadj, kArBorig, kArBord, kArBrank, kArItems, kArDeg, kArSortTmp, kArCkeys,
    kArEdgesI, kArCompI, kArRsScan, kArBigFlag, kArBigC, kArSlots
};
void *arena(int slot, size_t bytes);   // nullptr on allocation failure (error set)
void arena_free_all();

// ---------------------------------------------------------------------------
// Launch helpers implemented in the .cu files
// ---------------------------------------------------------------------------
int ingest(Graph &g, int64_t n, int64_t m, const int64_t *h_row_ptr,
           const int32_t *h_col, const int8_t *h_sign, cudaStream_t st,
           int64_t *launches);

int run_batch_tree(const Graph &g, Workspace &ws, int B, const int32_t *given_parent,
                   cudaStream_t st, int64_t *launches, cudaEvent_t *ev, bool descent, int sub,
                   int recpass = 0, size_t persist = 0, int sampler = 0);

// f.3: uniform random spanning forest of tree ws.tkey[0] (Wilson by parallel
// cycle popping, gb_wilson.cu) -> parent (-1 at the roots)
int run_wilson(const Graph &g, Workspace &ws, cudaStream_t st, int64_t *launches, int32_t *parent,
               int64_t *rounds_out);
// f.3 default: W uniform spanning forests (keys ws.wtkey[0..W)), one GPU
// thread per tree, into the first W*n int32 of ws.wseq
int run_wilson_batch(const Graph &g, Workspace &ws, int W, cudaStream_t st, int64_t *launches);
// f.3: W DFS trees (reading R18), one GPU thread per tree, same output place
int run_dfs_batch(const Graph &g, Workspace &ws, int W, cudaStream_t st, int64_t *launches);

// multi-source BFS of the B <= kMsBatch sampled trees of a batch (roots, BFS
// levels, min-hash parents); fills the level lists qv / parq, lvl, vbase, depth
struct MsBfsOut {
    uint32_t *qv, *parq, *pp;
    uint2 *rec, *crec;
    uint4 *irec;
    uint32_t *prec;
    uint64_t *lvl;
    uint32_t *vbase;
    int32_t *depth, *maxd;
    const uint64_t *tkey;
};
int run_msbfs(const Graph &g, Workspace &ws, int B, const MsBfsOut &o, cudaStream_t st,
              int64_t *launches);


int debug_tree_views(const Graph &g, Workspace &ws, bool descent, int32_t *d_parent,
                     int32_t *d_dist, int32_t *d_size, int32_t *d_pre, cudaStream_t st);

// walk: 0 two-ended, 1 Alg. 3 descent over child lists, 2 the paper's
// partitioned two-word edge lists (linear scan), 3 pre-order climb (layout 2)
int run_batch_cycles(const Graph &g, Workspace &ws, int B, int group, int walk,
                     cudaStream_t st, int64_t *launches, int jump = 1, int linear = 0, int ept = 1);

int run_batch_accumulate(const Graph &g, Workspace &ws, int B, int32_t *d_cnt,
                         int32_t *d_agree, cudaStream_t st, int64_t *launches);

// the word holding pre | pi<<31 of vertex v in tree b: pp (layout 1) or the
// second word of the internal-id record (layout 0)
inline uint32_t *label_words(Workspace &ws) {
    return ws.irec_layout ? reinterpret_cast<uint32_t *>(ws.irec) + 1 : ws.pp;
}
inline int label_stride(const Workspace &ws) { return ws.irec_layout ? 4 : 1; }

// f.2: Harary sides of the B trees of a batch by the L224 procedure (replaces
// the pi bits of pp and the per-component counts s1); d_bad counts edges
// whose sign contradicts the resulting bipartition
int run_batch_harary(const Graph &g, Workspace &ws, int B, cudaStream_t st, int64_t *launches,
                     unsigned long long *d_bad);

int exclusive_scan_u32(const uint32_t *in, uint32_t *out, int64_t count, uint32_t *tmp,
                       size_t tmp_elems, cudaStream_t st, int64_t *launches);
size_t scan_tmp_elems(int64_t count);

}  // namespace gb
