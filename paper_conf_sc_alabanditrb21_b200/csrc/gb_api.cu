// gb_api.cu -- the C ABI (include/graphb.h) and host orchestration: device
// state owned from gb_load_csr to gb_free, per-batch workspaces allocated
// once (L236: "all required dynamic memory is allocated once"), batches of B
// trees driven asynchronously on one stream (§8 a.9), per-phase CUDA events
// (Fig. 11 L451-L467 breakdown), counters accumulated on the device and
// copied back once.
#include "gb_internal.cuh"
#include "../../include/graphb.h"

#include <algorithm>
#include <cstdlib>
#include <cstring>
#include <string>
#include <vector>

namespace gb {

static std::string g_err;
void set_error(const std::string &msg) { g_err = msg; }

static void *g_arena[kArSlots] = {nullptr};
static size_t g_arena_cap[kArSlots] = {0};

void *arena(int slot, size_t bytes) {
    bytes = std::max<size_t>(bytes, 256);
    if (g_arena_cap[slot] >= bytes) return g_arena[slot];
    if (g_arena[slot]) cudaFree(g_arena[slot]);
    g_arena[slot] = nullptr;
    g_arena_cap[slot] = 0;
    cudaError_t e = cudaMalloc(&g_arena[slot], bytes);
    if (e != cudaSuccess) {
        set_error(std::string("cudaMalloc (graph buffers): ") + cudaGetErrorString(e));
        g_arena[slot] = nullptr;
        return nullptr;
    }
    g_arena_cap[slot] = bytes;
    return g_arena[slot];
}

void arena_free_all() {
    for (int i = 0; i < kArSlots; i++) {
        if (g_arena[i]) cudaFree(g_arena[i]);
        g_arena[i] = nullptr;
        g_arena_cap[i] = 0;
    }
}

struct Options {
    int64_t batch = 0;       // 0 = auto
    int64_t cycle_group = 0; // 0 = auto
    int64_t walk = 0;        // 0 two-ended, 1 Alg. 3 descent (child lists), 2 the paper's edge lists (L238-L244),
                             // 3 pre-order climb (layout 2)
    int64_t desc_linear = 0; // walk 1: 1 = linear int4 ballot rounds over the child starts, 0 = 32-ary pivots
    int64_t walk_ept = 1;    // walk 0 (layout 0): edges per thread, climbed interleaved (1, 2, 4)
    int64_t timing = 0;
    int64_t sub = 0;         // trees per labelling launch (0 = auto)
    int64_t msprof = 0;      // record BFS phase timestamps (gb_msbfs_profile)
    int64_t recpass = 1;     // walk 0: pre-indexed records scattered after the top-down pass
    int64_t persist = 0;     // bytes of L2 persisting window over the labelling arrays (0 = off)
    int64_t sampler = 0;     // Alg. 2 M: 0 BFS (R4), 1 uniform spanning trees (Wilson, R17)
    int64_t wilson = 0;      // sampler 1: 0 one thread per tree (W trees at once), 1 parallel cycle popping
    int64_t harary = 0;      // 1: Harary sides by the L224 procedure (gb_harary.cu)
    int64_t jump = 1;        // walk 0: levels per ancestor record of the cycle walk (1, 2, 4)
    int64_t push_parent = 1; // BFS, batches of <= 16 trees: parents chosen while pushing small frontiers
};

struct Stats {
    int64_t trees = 0, launches = 0, batches = 0, batch_used = 0, group_used = 0, harary_bad = 0;
    int64_t sub_used = 0, bfs_group_used = 0;   // trees per labelling launch / per BFS launch
    uint64_t sumk = 0, cycles = 0;
    int64_t max_depth = 0;
    double phase_ms[GB_NPHASE] = {0};
    std::vector<uint64_t> per_tree;   // 4 per recorded tree
    std::vector<int64_t> tree_ids;
    // gb_balance_range returns without synchronising: the device-side totals,
    // per-tree records and phase events of the call are read back lazily, by
    // the first gb_get_stats / gb_tree_stats / gb_cloud_states afterwards
    bool pending = false;
    cudaStream_t stream = nullptr;
    int64_t nrec = 0;
    bool harary = false;
    std::vector<cudaEvent_t> evs;      // (GB_NPHASE + 1) per batch when "timing" is set
    double sample_ms = 0;
};

struct State {
    bool loaded = false;
    Graph g;
    Workspace ws;
    bool ws_descent = false;
    int ws_layout = -1;
    cudaStream_t stream = nullptr;
    int32_t *d_cnt = nullptr, *d_agree = nullptr;  // gb_balance's device counters
    int64_t cnt_cap_m = 0, cnt_cap_n = 0;          // their capacities (edges, vertices)
    int32_t *d_given = nullptr;                    // caller tree (gb_balance_given_tree)
    int64_t given_cap = 0;
    unsigned long long *d_visited = nullptr;       // [kMaxBatch]
    unsigned long long *d_rec_stats = nullptr;     // [kRecCap][4]
    unsigned long long *d_tot = nullptr;           // [4] sum k, cycles, max depth over every tree of the call
    unsigned long long *d_states = nullptr;        // gb_cloud_states: hash table [2 * kStateSlots]
    unsigned long long *d_hbad = nullptr;          // option "harary": violations found
    std::vector<int32_t> h_comp;
    size_t free_at_load = 0;   // device memory free after ingest (cudaMemGetInfo costs ~2 ms)
    Options opt;
    Stats st;
};
static State S;
constexpr int64_t kRecCap = 1 << 16;  // per-tree statistics kept for gb_tree_stats
constexpr int64_t kStateSlots = 2 * kRecCap;  // open-addressing table of gb_cloud_states

static void free_ws(Workspace &w) {
    void *ptrs[] = {w.vst, w.qv, w.qs, w.qr, w.pkeyq, w.lvl, w.vbase, w.size, w.sz64,
                    w.parq, w.offq, w.szq, w.pp, w.rec, w.irec, w.prec, w.fbits, w.s1, w.tkey, w.depth,
                    w.tstat, w.visited, w.maxd, w.cidxq, w.cstart, w.clist, w.crec,
                    w.scan_tmp, w.vis, w.fr, w.hacc, w.hbest, w.msflag, w.mscnt, w.fbm, w.msprof,
                    w.jrec, w.hlab, w.wbuf, w.wparent, w.wseq, w.wtkey, w.pnew, w.pbest,
                    w.ptbase, w.ptnbr, w.ptrng};
    for (void *p : ptrs) if (p) cudaFree(p);
    w = Workspace();
}

static void free_graph(Graph &g) {
    g = Graph();   // the arrays live in the persistent arena
}

// record layout: 0 = records by internal id (walk 0, one level per record),
// 1 = pp + pre-indexed records (walks 1, 2, option jump), 2 = pp + 4-byte
// pre-indexed parent words (walk 3)
static int rec_layout() {
    if (S.opt.walk == 3) return 2;
    return (S.opt.walk == 0 && S.opt.jump == 1) ? 0 : 1;
}
static bool walk_descent() { return S.opt.walk == 1 || S.opt.walk == 2; }   // need the child lists

static size_t per_tree_bytes(const Graph &g, bool descent) {
    const size_t n = (size_t)g.n;
    size_t b = 36 * n + 32 + 4 * (size_t)((g.m + 31) / 32) + 4 * (size_t)g.ncomp;
    b += rec_layout() == 0 ? 16 * n : rec_layout() == 1 ? 12 * n : 8 * n;
    if (descent) b += 24 * n;
    return b;
}

#define ALLOC(ptr, count)                                                            \
    do {                                                                             \
        cudaError_t _e = cudaMalloc((void **)&(ptr), sizeof(*(ptr)) * (size_t)std::max<int64_t>(count, 1)); \
        if (_e != cudaSuccess) {                                                     \
            set_error(std::string("cudaMalloc " #ptr ": ") + cudaGetErrorString(_e)); \
            free_ws(S.ws);                                                           \
            return _e == cudaErrorMemoryAllocation ? GB_ENOMEM : GB_ECUDA;           \
        }                                                                            \
    } while (0)

static int ensure_workspace(int B, bool descent) {
    const int layout = rec_layout();
    const bool irec = layout == 0;
    if (S.ws.B >= B && descent == S.ws_descent && layout == S.ws_layout) return GB_OK;
    B = std::max(B, S.ws.B);
    free_ws(S.ws);
    Workspace &w = S.ws;
    const Graph &g = S.g;
    const int64_t n = g.n, Bn = (int64_t)B * n, words = (g.m + 31) / 32;
    const int64_t nw = (n + 3) / 4;
    // push BFS state, used for caller-given trees only (one tree at a time)
    ALLOC(w.vst, nw);
    ALLOC(w.qs, n);
    ALLOC(w.qr, n);
    ALLOC(w.pkeyq, n);
    // multi-source BFS state (one bit per tree)
    ALLOC(w.vis, 2 * n);
    ALLOC(w.fr, 4 * n);
    ALLOC(w.hacc, 2 * std::max<int64_t>(g.nmulti, 1));
    ALLOC(w.hbest, std::max<int64_t>(g.nmulti, 1) * kMsBatch);
    ALLOC(w.msflag, 8);
    ALLOC(w.mscnt, (int64_t)kMsBatch * 2048);
    ALLOC(w.fbm, 6 * ((n + 31) / 32));
        ALLOC(w.qv, Bn);
    ALLOC(w.lvl, (int64_t)B * (n + 2));
    ALLOC(w.vbase, (int64_t)B * (n + 2));
    ALLOC(w.parq, Bn);
    ALLOC(w.offq, Bn);
    ALLOC(w.szq, Bn);
    if (irec) {
        ALLOC(w.irec, Bn);
    } else if (layout == 2) {
        ALLOC(w.pp, Bn);
        ALLOC(w.prec, Bn);
    } else {
        ALLOC(w.pp, Bn);
        ALLOC(w.rec, Bn);
    }
    w.irec_layout = irec;
    ALLOC(w.fbits, (int64_t)B * words);
    ALLOC(w.s1, (int64_t)B * g.ncomp);
    ALLOC(w.tkey, kMaxBatch);
    ALLOC(w.depth, kMaxBatch);
    ALLOC(w.tstat, 3 * kMaxBatch);
    ALLOC(w.visited, kMaxBatch);
    ALLOC(w.maxd, 1);
    if (descent) {
        ALLOC(w.sz64, Bn);
        ALLOC(w.cidxq, Bn);
        ALLOC(w.cstart, Bn);
        ALLOC(w.clist, Bn + 4);   // + 4: the 16-byte loads of walk 1's linear scan
        ALLOC(w.crec, Bn);
        w.scan_tmp_elems = scan_tmp_elems(Bn);
        ALLOC(w.scan_tmp, (int64_t)w.scan_tmp_elems);
    } else {
        ALLOC(w.size, Bn);
    }
    w.B = B;
    w.n = n;
    S.ws_descent = descent;
    S.ws_layout = layout;
    return GB_OK;
}

static int check_device() {
    int dev = -1;
    cudaError_t e = cudaGetDevice(&dev);
    if (e != cudaSuccess) {
        set_error(std::string("no usable CUDA device: ") + cudaGetErrorString(e));
        return GB_ECUDA;
    }
    int ndev = 0;
    if (cudaGetDeviceCount(&ndev) != cudaSuccess || ndev < 1) {
        set_error("no CUDA device");
        return GB_ECUDA;
    }
    return GB_OK;
}

// ---------------------------------------------------------------------------
// small device helpers
// ---------------------------------------------------------------------------
__global__ void k_tree_keys(uint64_t *tkey, int B, uint64_t seed, int64_t t0, int64_t stride) {
    int b = threadIdx.x;
    if (b < B) tkey[b] = tree_key(seed, t0 + (int64_t)b * stride);
}

__global__ void k_record_stats(const unsigned long long *tstat, const int32_t *depth, int B,
                               unsigned long long *rec, int64_t pos, int64_t cap,
                               unsigned long long *tot) {
    int b = threadIdx.x;
    if (b < B) {
        atomicAdd(tot, tstat[3 * b]);
        atomicAdd(tot + 1, tstat[3 * b + 1]);
        atomicMax(tot + 2, (unsigned long long)depth[b]);
    }
    if (b < B && pos + b < cap) {
        rec[4 * (pos + b)] = tstat[3 * b];
        rec[4 * (pos + b) + 1] = tstat[3 * b + 1];
        rec[4 * (pos + b) + 2] = (unsigned long long)depth[b];
        rec[4 * (pos + b) + 3] = tstat[3 * b + 2];
    }
}

// f.2: distinct nearest balanced states among the recorded trees.  Open
// addressing over the 64-bit state signatures (rec[4i+3]); slot = {sig, count}
// with sig 0 = empty (the signature of "no switched edge" is 0 as well, so it
// is kept in a dedicated counter, zero[0]).
__global__ void k_cloud_states(const unsigned long long *rec, int64_t k, unsigned long long *tab,
                               int64_t slots, unsigned long long *zero) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < k;
         i += (int64_t)gridDim.x * blockDim.x) {
        const unsigned long long sig = rec[4 * i + 3];
        if (sig == 0) { atomicAdd(zero, 1ull); continue; }
        int64_t h = (int64_t)(mix64(sig) & (uint64_t)(slots - 1));
        for (;;) {
            const unsigned long long prev = atomicCAS(tab + 2 * h, 0ull, sig);
            if (prev == 0 || prev == sig) { atomicAdd(tab + 2 * h + 1, 1ull); break; }
            h = (h + 1) & (slots - 1);
        }
    }
}

static int auto_batch(int64_t ntrees) {
    if (S.opt.sampler != 0) return 1;   // sampled trees go one at a time (caller-tree path)
    // the multi-source BFS holds one bit per tree in a 128-bit word
    if (S.opt.batch > 0) return (int)std::min<int64_t>(S.opt.batch, kMsBatch);
    const size_t have = S.free_at_load;
    int64_t bm = (int64_t)(0.5 * (double)have / (double)per_tree_bytes(S.g, walk_descent()));
    int64_t b = std::min<int64_t>({ntrees, (int64_t)kMsBatch, std::max<int64_t>(bm, 1)});
    return (int)std::max<int64_t>(b, 1);
}

// trees per labelling launch: small graphs label the whole batch in one
// launch; large ones a few trees at a time, so the random-access working set
// (size counters + records, 20 B per vertex and tree) stays mostly in L2 while
// the per-level grid barriers are shared (measured on C3 with internal ids,
// bottom-up + top-down per 100 trees: 1 tree 55.8 ms, 2 trees 52.4, 4 trees
// 50.8; with round 1's random original ids 1 tree was best)
static int auto_sub(int B) {
    if (S.opt.sub > 0) return (int)std::min<int64_t>(S.opt.sub, B);
    if (S.g.n >= (1 << 22)) return std::min(B, 4);
    return B;
}

static int auto_group(int B) {
    if (S.opt.cycle_group > 0) return (int)std::min<int64_t>(S.opt.cycle_group, B);
    // keep the labels of the trees walked together L2-resident (~48 MB)
    double per = (S.opt.walk == 3 ? 8.0 : 4.0 + 8.0 * (S.opt.walk == 0 ? S.opt.jump : 1)) * (double)S.g.n;
    int g = (int)std::max(1.0, std::floor(48.0e6 / per));
    return std::max(1, std::min(g, B));
}

// the whole hot path over trees t_begin, t_begin+stride, ... < t_end
static void drop_events(Stats &T) {
    for (auto e : T.evs) cudaEventDestroy(e);   // released once complete
    T.evs.clear();
}

// read back what the last balance_range left on the device (synchronises
// with its stream once)
static int finalize_stats() {
    Stats &T = S.st;
    if (!T.pending) return GB_OK;
    T.pending = false;
    GB_CUDA_TRY(cudaStreamSynchronize(T.stream));
    unsigned long long tot[4] = {0, 0, 0, 0};
    GB_CUDA_TRY(cudaMemcpy(tot, S.d_tot, sizeof(tot), cudaMemcpyDeviceToHost));
    T.sumk = tot[0];
    T.cycles = tot[1];
    T.max_depth = (int64_t)tot[2];
    T.per_tree.resize(4 * T.nrec);
    if (T.nrec)
        GB_CUDA_TRY(cudaMemcpy(T.per_tree.data(), S.d_rec_stats, sizeof(uint64_t) * 4 * T.nrec,
                               cudaMemcpyDeviceToHost));
    if (T.harary) {
        unsigned long long hb = 0;
        GB_CUDA_TRY(cudaMemcpy(&hb, S.d_hbad, sizeof(hb), cudaMemcpyDeviceToHost));
        T.harary_bad = (int64_t)hb;
    }
    for (size_t base = 0; base + GB_NPHASE < T.evs.size(); base += GB_NPHASE + 1) {
        for (int i = 0; i < GB_NPHASE; i++) {
            float ms = 0;
            cudaEventElapsedTime(&ms, T.evs[base + i], T.evs[base + i + 1]);
            T.phase_ms[i] += ms;
        }
    }
    drop_events(T);
    T.phase_ms[GB_PHASE_BFS] += T.sample_ms;
    return GB_OK;
}

static int balance_range(int64_t t_begin, int64_t t_end, int64_t stride, uint64_t seed,
                         int32_t *d_cnt, int32_t *d_agree, cudaStream_t st) {
    Stats &T = S.st;
    drop_events(T);   // an unread previous call is discarded
    T = Stats();
    T.stream = st;
    if (!S.d_rec_stats) {
        GB_CUDA_TRY(cudaMalloc(&S.d_rec_stats, sizeof(unsigned long long) * 4 * kRecCap));
        GB_CUDA_TRY(cudaMalloc(&S.d_tot, sizeof(unsigned long long) * 4));
    }
    GB_CUDA_TRY(cudaMemsetAsync(S.d_tot, 0, sizeof(unsigned long long) * 4, st));
    T.pending = true;
    const int64_t K = t_end > t_begin ? (t_end - t_begin + stride - 1) / stride : 0;
    if (K == 0) return GB_OK;
    const bool descent = walk_descent();   // walks 1 and 2 need the child lists
    int B = auto_batch(K);
    // walk 1 keeps child lists of a whole batch in one 32-bit index space
    if (descent) B = (int)std::min<int64_t>(B, std::max<int64_t>(1, ((1ll << 32) - 1) / S.g.n));
    int rc = ensure_workspace(B, descent);
    S.ws.pp_ok = S.opt.push_parent != 0;
    if (rc) return rc;
    const int G = auto_group(B);
    const int jump = S.opt.walk == 0 ? (int)S.opt.jump : 1;
    if (jump > 1 && S.ws.jrec_cap < G * jump) {
        if (S.ws.jrec) cudaFree(S.ws.jrec);
        S.ws.jrec = nullptr;
        S.ws.jrec_cap = 0;
        cudaError_t e = cudaMalloc(&S.ws.jrec, sizeof(uint2) * (size_t)G * jump * S.g.n);
        if (e != cudaSuccess) {
            set_error(std::string("cudaMalloc jrec: ") + cudaGetErrorString(e));
            S.ws.jrec = nullptr;
            return e == cudaErrorMemoryAllocation ? GB_ENOMEM : GB_ECUDA;
        }
        S.ws.jrec_cap = G * jump;
    }
    if (S.opt.msprof && !S.ws.msprof) GB_CUDA_TRY(cudaMalloc(&S.ws.msprof, sizeof(unsigned long long) * 2048));
    if (!S.opt.msprof && S.ws.msprof) { cudaFree(S.ws.msprof); S.ws.msprof = nullptr; }
    if (S.ws.msprof) GB_CUDA_TRY(cudaMemsetAsync(S.ws.msprof, 0, sizeof(unsigned long long) * 2048, st));
    T.batch_used = B;
    T.group_used = G;
    T.sub_used = auto_sub(B);
    T.bfs_group_used = S.opt.sampler != 0 ? 1 : B;
    std::vector<cudaEvent_t> &evs = T.evs;
    const bool timing = S.opt.timing != 0;
    int64_t done = 0;
    // uniform sampler: trees per sampling chunk (<= kMaxBatch, ~2 GB of walk state)
    const int64_t Wc = std::max<int64_t>(1, std::min<int64_t>({(int64_t)kMaxBatch, K,
                                             (int64_t)(2.0e9 / (13.0 * (double)S.g.n))}));
    cudaEvent_t wev[2];
    double &sample_ms = T.sample_ms;
    while (done < K) {
        const int nb = (int)std::min<int64_t>(B, K - done);
        const int64_t t0 = t_begin + done * stride;
        cudaEvent_t *ev = nullptr;
        if (timing) {
            size_t base = evs.size();
            evs.resize(base + GB_NPHASE + 1);
            for (int i = 0; i <= GB_NPHASE; i++) cudaEventCreate(&evs[base + i]);
            ev = evs.data() + base;
        }
        k_tree_keys<<<1, kMaxBatch, 0, st>>>(S.ws.tkey, nb, seed, t0, stride);
        ++T.launches;
        GB_CUDA_TRY(cudaMemsetAsync(S.ws.tstat, 0, sizeof(unsigned long long) * 3 * nb, st));
        GB_CUDA_TRY(cudaMemsetAsync(S.ws.hacc, 0, sizeof(unsigned long long) * 2 * std::max<int64_t>(S.g.nmulti, 1), st));
        GB_CUDA_TRY(cudaMemsetAsync(S.ws.hbest, 0xFF, sizeof(unsigned long long) * std::max<int64_t>(S.g.nmulti, 1) * kMsBatch, st));
        const int32_t *given = nullptr;
        if (S.opt.sampler == 2 || (S.opt.sampler == 1 && !S.opt.wilson)) {
            // uniform trees: sample the next chunk of W trees at once (one
            // thread each), then label and walk them one by one
            const int64_t j = done % Wc;
            if (j == 0) {
                const int W = (int)std::min<int64_t>(Wc, K - done);
                if (!S.ws.wtkey) GB_CUDA_TRY(cudaMalloc(&S.ws.wtkey, sizeof(uint64_t) * kMaxBatch));
                k_tree_keys<<<1, kMaxBatch, 0, st>>>(S.ws.wtkey, W, seed, t0, stride);
                ++T.launches;
                if (timing) { cudaEventCreate(&wev[0]); cudaEventCreate(&wev[1]); GB_CUDA_TRY(cudaEventRecord(wev[0], st)); }
                rc = S.opt.sampler == 2 ? run_dfs_batch(S.g, S.ws, W, st, &T.launches)
                                        : run_wilson_batch(S.g, S.ws, W, st, &T.launches);
                if (rc) return rc;
                if (timing) {
                    GB_CUDA_TRY(cudaEventRecord(wev[1], st));
                    GB_CUDA_TRY(cudaEventSynchronize(wev[1]));
                    float ms = 0;
                    cudaEventElapsedTime(&ms, wev[0], wev[1]);
                    sample_ms += ms;
                    cudaEventDestroy(wev[0]);
                    cudaEventDestroy(wev[1]);
                }
            }
            given = reinterpret_cast<const int32_t *>(S.ws.wseq) + j * S.g.n;
        }
        rc = run_batch_tree(S.g, S.ws, nb, given, st, &T.launches, ev, descent, auto_sub(nb),
                            (int)S.opt.recpass, (size_t)S.opt.persist, given ? 0 : (int)S.opt.sampler);
        if (rc) return rc;
        if (ev) GB_CUDA_TRY(cudaEventRecord(ev[4], st));
        rc = run_batch_cycles(S.g, S.ws, nb, G, (int)S.opt.walk, st, &T.launches, jump, (int)S.opt.desc_linear,
                              (int)S.opt.walk_ept);
        if (rc) return rc;
        if (ev) GB_CUDA_TRY(cudaEventRecord(ev[5], st));
        if (S.opt.harary) {
            if (!S.d_hbad) {
                GB_CUDA_TRY(cudaMalloc(&S.d_hbad, sizeof(unsigned long long)));
            }
            if (T.batches == 0) GB_CUDA_TRY(cudaMemsetAsync(S.d_hbad, 0, sizeof(unsigned long long), st));
            rc = run_batch_harary(S.g, S.ws, nb, st, &T.launches, S.d_hbad);
            if (rc) return rc;
        }
        rc = run_batch_accumulate(S.g, S.ws, nb, d_cnt, d_agree, st, &T.launches);
        if (rc) return rc;
        if (ev) GB_CUDA_TRY(cudaEventRecord(ev[6], st));
        if (done < kRecCap) {
            for (int b = 0; b < nb && done + b < kRecCap; b++) T.tree_ids.push_back(t0 + b * stride);
        }
        k_record_stats<<<1, kMaxBatch, 0, st>>>(S.ws.tstat, S.ws.depth, nb, S.d_rec_stats, done, kRecCap,
                                                S.d_tot);
        ++T.launches;
        done += nb;
        T.batches++;
    }
    GB_CUDA_TRY(cudaGetLastError());
    T.harary = S.opt.harary != 0;
    T.nrec = std::min<int64_t>(K, kRecCap);
    T.trees = K;
    return GB_OK;   // no host synchronisation (statistics are read lazily)
}

static int run_single_tree(int64_t t, uint64_t seed, const int32_t *d_given) {
    Stats &T = S.st;
    drop_events(T);
    T = Stats();
    int rc = ensure_workspace(1, walk_descent());
    if (rc) return rc;
    cudaStream_t st = S.stream;
    k_tree_keys<<<1, kMaxBatch, 0, st>>>(S.ws.tkey, 1, seed, t, 1);
    ++T.launches;
    GB_CUDA_TRY(cudaMemsetAsync(S.ws.tstat, 0, sizeof(unsigned long long) * 3, st));
    GB_CUDA_TRY(cudaMemsetAsync(S.ws.hacc, 0, sizeof(unsigned long long) * 2 * std::max<int64_t>(S.g.nmulti, 1), st));
    GB_CUDA_TRY(cudaMemsetAsync(S.ws.hbest, 0xFF, sizeof(unsigned long long) * std::max<int64_t>(S.g.nmulti, 1) * kMsBatch, st));
    const bool user_tree = d_given != nullptr;
    if (!d_given && (S.opt.sampler == 2 || (S.opt.sampler == 1 && !S.opt.wilson))) {
        if (!S.ws.wtkey) GB_CUDA_TRY(cudaMalloc(&S.ws.wtkey, sizeof(uint64_t) * kMaxBatch));
        k_tree_keys<<<1, kMaxBatch, 0, st>>>(S.ws.wtkey, 1, seed, t, 1);
        ++T.launches;
        rc = S.opt.sampler == 2 ? run_dfs_batch(S.g, S.ws, 1, st, &T.launches)
                                : run_wilson_batch(S.g, S.ws, 1, st, &T.launches);
        if (rc) return rc;
        d_given = reinterpret_cast<const int32_t *>(S.ws.wseq);
    }
    rc = run_batch_tree(S.g, S.ws, 1, d_given, st, &T.launches, nullptr, walk_descent(), 1,
                        0, 0, d_given ? 0 : (int)S.opt.sampler);
    if (rc) return rc;
    if (user_tree) {
        unsigned long long vis = 0;
        GB_CUDA_TRY(cudaMemcpyAsync(&vis, S.ws.visited, sizeof(vis), cudaMemcpyDeviceToHost, st));
        GB_CUDA_TRY(cudaStreamSynchronize(st));
        if ((int64_t)vis != S.g.n) {
            set_error("parent is not a spanning forest of the loaded graph (some vertex is not "
                      "reachable from a root through parent edges)");
            return GB_EINVAL;
        }
    }
    rc = run_batch_cycles(S.g, S.ws, 1, 1, (int)S.opt.walk, st, &T.launches, 1, (int)S.opt.desc_linear,
                          (int)S.opt.walk_ept);
    if (rc) return rc;
    GB_CUDA_TRY(cudaStreamSynchronize(st));
    return GB_OK;
}

static int copy_flips(uint8_t *flip) {
    const int64_t words = (S.g.m + 31) / 32;
    std::vector<uint32_t> fb(std::max<int64_t>(words, 1));
    if (words) GB_CUDA_TRY(cudaMemcpy(fb.data(), S.ws.fbits, 4 * words, cudaMemcpyDeviceToHost));
    for (int64_t e = 0; e < S.g.m; e++) flip[e] = (fb[e >> 5] >> (e & 31)) & 1u;
    return GB_OK;
}

static int copy_cycle_stats(uint64_t *sumk, int64_t *ncyc) {
    unsigned long long ts[2] = {0, 0};
    GB_CUDA_TRY(cudaMemcpy(ts, S.ws.tstat, sizeof(ts), cudaMemcpyDeviceToHost));
    if (sumk) *sumk = ts[0];
    if (ncyc) *ncyc = (int64_t)ts[1];
    return GB_OK;
}

}  // namespace gb

using namespace gb;

extern "C" {

const char *gb_last_error(void) { return g_err.c_str(); }

int gb_selftest(void) {
    // SplitMix64 public vector from state 0
    const uint64_t kat[3] = {0xE220A8397B1DCDAFull, 0x6E789E6AA1B965F4ull, 0x06C45D188009454Full};
    for (int i = 0; i < 3; i++)
        if (tree_key(0, i) != kat[i]) { set_error("selftest: SplitMix64 vector"); return GB_EINVAL; }
    uint64_t x = 0x0123456789ABCDEFull;
    for (int i = 0; i < 100000; i++) {
        x = x * 6364136223846793005ull + 1442695040888963407ull;
        if (unmix64(mix64(x)) != x) { set_error("selftest: unmix64"); return GB_EINVAL; }
        uint32_t e = (uint32_t)(x >> 33);
        if (edge_of_key(x, edge_key(x, e)) != e) { set_error("selftest: edge key decode"); return GB_EINVAL; }
    }
    return GB_OK;
}

// release the loaded graph and everything sized by it, but keep the stream,
// the statistics buffer and (if asked) the tree workspace for a reload
static void release_graph(bool keep_ws) {
    if (!keep_ws) {
        free_ws(S.ws);
        // gb_balance's counters and the caller-tree buffer are sized by the
        // graph; a reload of the same shape keeps them (cudaFree synchronises)
        if (S.d_cnt) cudaFree(S.d_cnt);
        if (S.d_agree) cudaFree(S.d_agree);
        if (S.d_given) cudaFree(S.d_given);
        S.d_cnt = S.d_agree = nullptr;
        S.d_given = nullptr;
        S.given_cap = 0;
        S.cnt_cap_m = S.cnt_cap_n = 0;
    }
    free_graph(S.g);
    S.loaded = false;
    S.h_comp.clear();
}

void gb_free(void) {
    drop_events(S.st);
    release_graph(false);
    arena_free_all();
    if (S.d_visited) cudaFree(S.d_visited);
    if (S.d_rec_stats) cudaFree(S.d_rec_stats);
    if (S.d_tot) cudaFree(S.d_tot);
    if (S.d_states) cudaFree(S.d_states);
    if (S.d_hbad) cudaFree(S.d_hbad);
    if (S.stream) cudaStreamDestroy(S.stream);
    Options keep = S.opt;
    S = State();
    S.opt = keep;
}

int gb_load_csr(int64_t n, int64_t m, const int64_t *row_ptr, const int32_t *col_idx,
                const int8_t *sign) {
    if (n < 1 || n >= (1ll << 31)) { set_error("n must satisfy 1 <= n < 2^31"); return GB_EINVAL; }
    if (m < 0 || 2 * m >= (1ll << 32)) { set_error("m must satisfy 0 <= 2m < 2^32"); return GB_EINVAL; }
    if (!row_ptr || (m > 0 && (!col_idx || !sign))) { set_error("NULL input array"); return GB_EINVAL; }
    if (row_ptr[0] != 0 || row_ptr[n] != 2 * m) {
        set_error("row_ptr[0] must be 0 and row_ptr[n] must equal 2m");
        return GB_EINVAL;
    }
    int rc = check_device();
    if (rc) return rc;
    int dev = 0;
    GB_CUDA_TRY(cudaGetDevice(&dev));
    // a reload on the same device keeps the tree workspace if the new graph
    // has the same shape (all dynamic memory allocated once, L236)
    const bool same_dev = S.stream != nullptr && S.g.dev == dev;
    const int64_t old_n = S.g.n, old_m = S.g.m, old_c = S.g.ncomp, old_h = S.g.nmulti;
    if (same_dev) release_graph(true); else gb_free();
    int coop = 0;
    GB_CUDA_TRY(cudaDeviceGetAttribute(&coop, cudaDevAttrCooperativeLaunch, dev));
    if (!coop) { set_error("device lacks cooperative launch"); return GB_ECUDA; }
    S.g.dev = dev;
    GB_CUDA_TRY(cudaDeviceGetAttribute(&S.g.num_sms, cudaDevAttrMultiProcessorCount, dev));
    if (!S.stream) GB_CUDA_TRY(cudaStreamCreateWithFlags(&S.stream, cudaStreamNonBlocking));
    int64_t launches = 0;
    rc = ingest(S.g, n, m, row_ptr, col_idx, sign, S.stream, &launches);
    if (rc) { gb_free(); return rc; }
    const bool same_shape = S.g.n == old_n && S.g.m == old_m && S.g.ncomp == old_c && S.g.nmulti == old_h;
    if (S.ws.B && !same_shape) free_ws(S.ws);
    if (!same_shape || !S.ws.B || !S.free_at_load) {
        // a same-shape reload keeps the workspace and the memory estimate
        size_t freeb = 0, totb = 0;
        GB_CUDA_TRY(cudaMemGetInfo(&freeb, &totb));
        S.free_at_load = freeb + (size_t)S.ws.B * per_tree_bytes(S.g, S.ws_descent);
    }
    S.loaded = true;
    S.st = Stats();
    S.st.launches = launches;
    return GB_OK;
}

int gb_graph_debug(int32_t *edge_u, int32_t *edge_v, int8_t *edge_neg, uint32_t *slot_eid,
                   int32_t *comp) {
    if (!S.loaded) { set_error("no graph loaded"); return GB_ESTATE; }
    const int64_t m = S.g.m, n = S.g.n;
    if (m && (edge_u || edge_v || edge_neg)) {
        std::vector<uint2> e(m);
        GB_CUDA_TRY(cudaMemcpy(e.data(), S.g.edges, sizeof(uint2) * m, cudaMemcpyDeviceToHost));
        for (int64_t i = 0; i < m; i++) {
            if (edge_u) edge_u[i] = (int32_t)e[i].x;
            if (edge_v) edge_v[i] = (int32_t)(e[i].y & kIdMask);
            if (edge_neg) edge_neg[i] = (int8_t)(e[i].y >> 31);
        }
    }
    if (m && slot_eid)
        GB_CUDA_TRY(cudaMemcpy(slot_eid, S.g.adj_eid, sizeof(uint32_t) * 2 * m, cudaMemcpyDeviceToHost));
    if (comp) GB_CUDA_TRY(cudaMemcpy(comp, S.g.comp, sizeof(int32_t) * n, cudaMemcpyDeviceToHost));
    return GB_OK;
}

int gb_graph_info(int64_t *n, int64_t *m, int64_t *ncomp) {
    if (!S.loaded) { set_error("no graph loaded"); return GB_ESTATE; }
    if (n) *n = S.g.n;
    if (m) *m = S.g.m;
    if (ncomp) *ncomp = S.g.ncomp;
    return GB_OK;
}

int gb_set_option(const char *key, int64_t value) {
    if (!key) { set_error("NULL option"); return GB_EINVAL; }
    if (!strcmp(key, "batch")) { if (value < 0) return GB_EINVAL; S.opt.batch = value; }
    else if (!strcmp(key, "cycle_group")) { if (value < 0) return GB_EINVAL; S.opt.cycle_group = value; }
    else if (!strcmp(key, "walk")) {
        if (value < 0 || value > 3) { set_error("walk must be 0 (two-ended), 1 (Alg. 3 descent), 2 (paper edge lists) or 3 (pre-order climb)"); return GB_EINVAL; }
        S.opt.walk = value;
    }
    else if (!strcmp(key, "desc_linear")) S.opt.desc_linear = value != 0;
    else if (!strcmp(key, "walk_ept")) {
        if (value != 1 && value != 2 && value != 4) { set_error("walk_ept must be 1, 2 or 4"); return GB_EINVAL; }
        S.opt.walk_ept = value;
    }
    else if (!strcmp(key, "push_parent")) S.opt.push_parent = value != 0;
    else if (!strcmp(key, "timing")) S.opt.timing = value != 0;
    else if (!strcmp(key, "sub")) { if (value < 0) return GB_EINVAL; S.opt.sub = value; }
    else if (!strcmp(key, "msprof")) S.opt.msprof = value != 0;
    else if (!strcmp(key, "reset")) S.opt = Options();
    else if (!strcmp(key, "harary")) S.opt.harary = value != 0;
    else if (!strcmp(key, "wilson")) S.opt.wilson = value != 0;
    else if (!strcmp(key, "sampler")) {
        if (value < 0 || value > 2) { set_error("sampler must be 0 (BFS), 1 (uniform) or 2 (DFS)"); return GB_EINVAL; }
        S.opt.sampler = value;
    }
    else if (!strcmp(key, "recpass")) S.opt.recpass = value != 0;

    else if (!strcmp(key, "jump")) {
        if (value != 1 && value != 2 && value != 4) { set_error("jump must be 1, 2 or 4"); return GB_EINVAL; }
        S.opt.jump = value;
    }
    else if (!strcmp(key, "persist")) {
        if (value < 0) return GB_EINVAL;
        if (value > 0) {
            int dev = 0, maxp = 0;
            GB_CUDA_TRY(cudaGetDevice(&dev));
            GB_CUDA_TRY(cudaDeviceGetAttribute(&maxp, cudaDevAttrMaxPersistingL2CacheSize, dev));
            value = std::min<int64_t>(value, maxp);
            GB_CUDA_TRY(cudaDeviceSetLimit(cudaLimitPersistingL2CacheSize, (size_t)value));
        }
        S.opt.persist = value;
    }
    else { set_error(std::string("unknown option ") + key); return GB_EINVAL; }
    return GB_OK;
}

int gb_balance_range(int64_t t_begin, int64_t t_end, int64_t t_stride, uint64_t seed,
                     int32_t *d_edge_cnt, int32_t *d_vertex_agree, void *cuda_stream) {
    if (!S.loaded) { set_error("no graph loaded"); return GB_ESTATE; }
    if (t_begin < 0 || t_end < t_begin || t_stride < 1 || t_end > (1ll << 30) - 1) {
        set_error("bad tree range");
        return GB_EINVAL;
    }
    if ((S.g.m > 0 && !d_edge_cnt) || !d_vertex_agree) { set_error("NULL output"); return GB_EINVAL; }
    cudaStream_t st = cuda_stream ? (cudaStream_t)cuda_stream : S.stream;
    return balance_range(t_begin, t_end, t_stride, seed, d_edge_cnt, d_vertex_agree, st);
}

int gb_balance(int64_t num_trees, uint64_t seed, uint32_t *out_edge_flip_counts,
               uint32_t *out_vertex_agree) {
    if (!S.loaded) { set_error("no graph loaded"); return GB_ESTATE; }
    if (num_trees < 0 || num_trees > (1ll << 30) - 1) { set_error("num_trees out of range"); return GB_EINVAL; }
    if ((S.g.m > 0 && !out_edge_flip_counts) || !out_vertex_agree) { set_error("NULL output"); return GB_EINVAL; }
    if (!S.d_cnt || S.cnt_cap_m < std::max<int64_t>(S.g.m, 1) || S.cnt_cap_n < S.g.n) {
        if (S.d_cnt) cudaFree(S.d_cnt);
        if (S.d_agree) cudaFree(S.d_agree);
        S.d_cnt = S.d_agree = nullptr;
        S.cnt_cap_m = S.cnt_cap_n = 0;
        GB_CUDA_TRY(cudaMalloc(&S.d_cnt, sizeof(int32_t) * std::max<int64_t>(S.g.m, 1)));
        GB_CUDA_TRY(cudaMalloc(&S.d_agree, sizeof(int32_t) * S.g.n));
        S.cnt_cap_m = std::max<int64_t>(S.g.m, 1);
        S.cnt_cap_n = S.g.n;
    }
    GB_CUDA_TRY(cudaMemsetAsync(S.d_cnt, 0, sizeof(int32_t) * std::max<int64_t>(S.g.m, 1), S.stream));
    GB_CUDA_TRY(cudaMemsetAsync(S.d_agree, 0, sizeof(int32_t) * S.g.n, S.stream));
    int rc = balance_range(0, num_trees, 1, seed, S.d_cnt, S.d_agree, S.stream);
    if (rc) return rc;
    if (S.g.m)
        GB_CUDA_TRY(cudaMemcpyAsync(out_edge_flip_counts, S.d_cnt, sizeof(int32_t) * S.g.m,
                                    cudaMemcpyDeviceToHost, S.stream));
    GB_CUDA_TRY(cudaMemcpyAsync(out_vertex_agree, S.d_agree, sizeof(int32_t) * S.g.n,
                                cudaMemcpyDeviceToHost, S.stream));
    GB_CUDA_TRY(cudaStreamSynchronize(S.stream));
    return GB_OK;
}

int gb_tree_debug(int64_t t, uint64_t seed, int32_t *parent, int32_t *dist, int32_t *pre,
                  int32_t *size, uint8_t *flip, uint64_t *sum_cycle_len, int64_t *num_cycles) {
    if (!S.loaded) { set_error("no graph loaded"); return GB_ESTATE; }
    if (t < 0 || t > (1ll << 30) - 1) { set_error("bad tree index"); return GB_EINVAL; }
    int rc = run_single_tree(t, seed, nullptr);
    if (rc) return rc;
    const int64_t n = S.g.n;
    int32_t *d_tmp = nullptr;
    GB_CUDA_TRY(cudaMalloc(&d_tmp, sizeof(int32_t) * 4 * n));
    rc = debug_tree_views(S.g, S.ws, walk_descent(), d_tmp, d_tmp + n, d_tmp + 2 * n, d_tmp + 3 * n, S.stream);
    if (rc) { cudaFree(d_tmp); return rc; }
    std::vector<int32_t> h(4 * n);
    cudaError_t ce = cudaMemcpy(h.data(), d_tmp, sizeof(int32_t) * 4 * n, cudaMemcpyDeviceToHost);
    cudaFree(d_tmp);
    GB_CUDA_TRY(ce);
    if (parent) std::copy(h.begin(), h.begin() + n, parent);
    if (dist) std::copy(h.begin() + n, h.begin() + 2 * n, dist);
    if (size) std::copy(h.begin() + 2 * n, h.begin() + 3 * n, size);
    if (pre) std::copy(h.begin() + 3 * n, h.end(), pre);
    if (flip) { rc = copy_flips(flip); if (rc) return rc; }
    return copy_cycle_stats(sum_cycle_len, num_cycles);
}

int gb_balance_given_tree(const int32_t *parent, uint8_t *flip, uint64_t *sum_cycle_len,
                          int64_t *num_cycles) {
    if (!S.loaded) { set_error("no graph loaded"); return GB_ESTATE; }
    if (!parent) { set_error("NULL parent"); return GB_EINVAL; }
    const int64_t n = S.g.n;
    if ((int64_t)S.h_comp.size() != n) {   // component of every vertex, copied once per graph
        S.h_comp.resize(n);
        GB_CUDA_TRY(cudaMemcpy(S.h_comp.data(), S.g.comp, sizeof(int32_t) * n, cudaMemcpyDeviceToHost));
    }
    std::vector<int32_t> roots(S.g.ncomp, 0);
    for (int64_t v = 0; v < n; v++) {
        if (parent[v] == -1) roots[S.h_comp[v]]++;
        else if (parent[v] < 0 || parent[v] >= n || parent[v] == v) {
            set_error("parent entry out of range");
            return GB_EINVAL;
        }
    }
    for (int64_t c = 0; c < S.g.ncomp; c++)
        if (roots[c] != 1) { set_error("need exactly one root (-1) per connected component"); return GB_EINVAL; }
    if (!S.d_given || S.given_cap < n) {
        if (S.d_given) cudaFree(S.d_given);
        S.d_given = nullptr;
        S.given_cap = 0;
        GB_CUDA_TRY(cudaMalloc(&S.d_given, sizeof(int32_t) * n));
        S.given_cap = n;
    }
    GB_CUDA_TRY(cudaMemcpy(S.d_given, parent, sizeof(int32_t) * n, cudaMemcpyHostToDevice));
    int rc = run_single_tree(0, 0, S.d_given);
    if (rc) return rc;
    if (flip) { rc = copy_flips(flip); if (rc) return rc; }
    return copy_cycle_stats(sum_cycle_len, num_cycles);
}

int gb_get_stats(int64_t *ints, int n_ints, double *phase_ms, int n_phase) {
    if (finalize_stats()) return GB_ECUDA;
    const Stats &T = S.st;
    int64_t v[11] = {T.trees, (int64_t)T.sumk, (int64_t)T.cycles, T.launches, T.batches,
                     T.max_depth, T.batch_used, T.group_used, T.harary_bad, T.sub_used, T.bfs_group_used};
    int k = 0;
    for (; ints && k < n_ints && k < 11; k++) ints[k] = v[k];
    for (int i = 0; phase_ms && i < n_phase && i < GB_NPHASE; i++) phase_ms[i] = T.phase_ms[i];
    return k;
}

// BFS phase timestamps of the last batch (option "msprof"): [256][4] ns
int gb_msbfs_profile(uint64_t *out) {
    if (!S.ws.msprof) { set_error("msprof option not set"); return GB_ESTATE; }
    GB_CUDA_TRY(cudaMemcpy(out, S.ws.msprof, sizeof(uint64_t) * 1024, cudaMemcpyDeviceToHost));
    return GB_OK;
}

int gb_label_profile(uint64_t *out) {
    if (!S.ws.msprof) { set_error("msprof option not set"); return GB_ESTATE; }
    GB_CUDA_TRY(cudaMemcpy(out, S.ws.msprof + 1024, sizeof(uint64_t) * 1024, cudaMemcpyDeviceToHost));
    return GB_OK;
}

int64_t gb_cloud_states(uint64_t *sig, uint64_t *count, int64_t max_states) {
    if (finalize_stats()) return GB_ECUDA;
    const Stats &T = S.st;
    if (!S.d_rec_stats || T.nrec == 0) return 0;
    if (!S.d_states) {
        cudaError_t e = cudaMalloc(&S.d_states, sizeof(unsigned long long) * (2 * kStateSlots + 1));
        if (e != cudaSuccess) { set_error(std::string("cudaMalloc states: ") + cudaGetErrorString(e)); S.d_states = nullptr; return GB_ENOMEM; }
    }
    cudaStream_t st = S.stream;
    if (cudaMemsetAsync(S.d_states, 0, sizeof(unsigned long long) * (2 * kStateSlots + 1), st) != cudaSuccess) return GB_ECUDA;
    k_cloud_states<<<(unsigned)((T.nrec + 255) / 256), 256, 0, st>>>(S.d_rec_stats, T.nrec, S.d_states, kStateSlots,
                                                                     S.d_states + 2 * kStateSlots);
    std::vector<unsigned long long> tab(2 * kStateSlots + 1);
    if (cudaMemcpyAsync(tab.data(), S.d_states, sizeof(unsigned long long) * tab.size(), cudaMemcpyDeviceToHost, st) != cudaSuccess ||
        cudaStreamSynchronize(st) != cudaSuccess) {
        set_error("gb_cloud_states: copy failed");
        return GB_ECUDA;
    }
    int64_t k = 0;
    if (tab[2 * kStateSlots]) {
        if (k < max_states) { if (sig) sig[k] = 0; if (count) count[k] = tab[2 * kStateSlots]; }
        k++;
    }
    for (int64_t h = 0; h < kStateSlots; h++) {
        if (!tab[2 * h]) continue;
        if (k < max_states) { if (sig) sig[k] = tab[2 * h]; if (count) count[k] = tab[2 * h + 1]; }
        k++;
    }
    return k;
}

int64_t gb_tree_stats(uint64_t *out, int64_t *tree_ids, int64_t max_trees) {
    if (finalize_stats()) return GB_ECUDA;
    const Stats &T = S.st;
    int64_t k = std::min<int64_t>(max_trees, (int64_t)T.tree_ids.size());
    for (int64_t i = 0; i < k; i++) {
        if (out) for (int j = 0; j < 4; j++) out[4 * i + j] = T.per_tree[4 * i + j];
        if (tree_ids) tree_ids[i] = T.tree_ids[i];
    }
    return k;
}

}  // extern "C"
