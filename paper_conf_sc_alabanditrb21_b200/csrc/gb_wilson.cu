// gb_wilson.cu -- §8 row f.3: Alg. 2 with M = random (L130; L168): uniform
// random spanning forests, option "sampler" = 1.  Everything downstream
// (Alg. 4 labels, the cycle walk, Harary agree, accumulation) is the hot
// path's, unchanged; only the tree builder differs.
//
// Reading R17: Wilson's algorithm driven by a random stack per vertex -- the
// j-th departure from u goes to N(u)[mix64(tkey + W*(u*2^32 + j)) mod deg u].
// With fixed stacks the resulting tree does not depend on the order in which
// the loop-erased walks are run; equivalently it is what "cycle popping"
// leaves: every vertex points at the top of its stack, and as long as the
// pointer graph has a cycle, the cycle is popped (each of its vertices moves
// to its next stack entry).  Popping is order-free, so all cycles present at
// a time can be popped at once -- a data-parallel algorithm that reproduces
// the sequential oracle (oracle.c or_wilson_tree) bit for bit:
//
//   repeat
//     D(u) = "u reaches a root through the pointers"   (pointer doubling)
//     cycle vertices = { J(u) : u not done },  J = pointer^(2^K), 2^K > #active
//     pop every cycle vertex: stack index + 1, pointer = its next entry
//   until every vertex is done
//
// Vertices that reach a root are final (popping only touches cycles).
#include "gb_internal.cuh"
#include "../../include/graphb.h"

#include <algorithm>
#include <cstdio>
#include <cstdlib>

namespace gb {

constexpr uint64_t kWMul = 0xD6E8FEB86659FD93ull;

struct WParams {
    const uint32_t *row_ptr, *adj;
    const int32_t *coff, *cverts;
    int64_t n, ncomp;
    const uint64_t *tkey;
    uint32_t *s, *nxt;
    uint8_t *done, *cyc;
    unsigned long long *active;
};

__device__ __forceinline__ uint32_t w_next(const WParams &P, uint64_t tk, uint32_t u, uint32_t j) {
    const uint32_t rs = P.row_ptr[u], deg = P.row_ptr[u + 1] - rs;
    const uint64_t h = mix64(tk + kWMul * (((uint64_t)u << 32) | j));
    return P.adj[rs + (uint32_t)(h % deg)] & kIdMask;
}

__global__ void k_w_init(WParams P) {
    const uint64_t tk = *P.tkey;
    for (int64_t u = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; u < P.n;
         u += (int64_t)gridDim.x * blockDim.x) {
        P.s[u] = 0;
        P.done[u] = 0;
        P.cyc[u] = 0;
        const bool iso = P.row_ptr[u + 1] == P.row_ptr[u];
        P.nxt[u] = iso ? (uint32_t)u : w_next(P, tk, (uint32_t)u, 0);
    }
}

// roots (reading R4, the BFS sampler's): done, pointing at themselves
__global__ void k_w_roots(WParams P) {
    const uint64_t tk = *P.tkey;
    for (int64_t C = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; C < P.ncomp;
         C += (int64_t)gridDim.x * blockDim.x) {
        const uint32_t sz = (uint32_t)(P.coff[C + 1] - P.coff[C]);
        const uint32_t r = (uint32_t)P.cverts[P.coff[C] + (int64_t)(root_key(tk, C) % sz)];
        P.done[r] = 1;
        P.nxt[r] = r;
    }
}

__global__ void k_w_jump_init(WParams P, uint32_t *J, uint8_t *D) {
    for (int64_t u = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; u < P.n;
         u += (int64_t)gridDim.x * blockDim.x) {
        J[u] = P.nxt[u];
        D[u] = P.done[u];
    }
}

// one doubling step: D'(u) = D(u) or D(J(u)), J'(u) = J(J(u))
__global__ void k_w_jump(int64_t n, const uint32_t *__restrict__ Jin, const uint8_t *__restrict__ Din,
                         uint32_t *__restrict__ Jout, uint8_t *__restrict__ Dout) {
    for (int64_t u = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; u < n;
         u += (int64_t)gridDim.x * blockDim.x) {
        uint8_t d = Din[u];
        uint32_t j = Jin[u];
        if (!d) {
            d = Din[j];
            j = Jin[j];
        }
        Dout[u] = d;
        Jout[u] = j;
    }
}

// vertices that reach a root are final; J(u) of the others lies on a cycle
__global__ void k_w_mark(WParams P, const uint32_t *__restrict__ J, const uint8_t *__restrict__ D) {
    for (int64_t u = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; u < P.n;
         u += (int64_t)gridDim.x * blockDim.x) {
        if (D[u]) P.done[u] = 1;
        else P.cyc[J[u]] = 1;
    }
}

// pop every cycle: the next entry of each cycle vertex's stack
__global__ void k_w_pop(WParams P) {
    const uint64_t tk = *P.tkey;
    unsigned long long act = 0;
    for (int64_t u = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; u < P.n;
         u += (int64_t)gridDim.x * blockDim.x) {
        if (P.done[u]) continue;
        act++;
        if (P.cyc[u]) {
            const uint32_t j = ++P.s[u];
            P.nxt[u] = w_next(P, tk, (uint32_t)u, j);
            P.cyc[u] = 0;
        }
    }
#pragma unroll
    for (int d = 16; d; d >>= 1) act += __shfl_xor_sync(0xFFFFFFFFu, act, d);
    if ((threadIdx.x & 31) == 0 && act) atomicAdd(P.active, act);
}

__global__ void k_w_parent(WParams P, int32_t *parent) {
    for (int64_t u = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; u < P.n;
         u += (int64_t)gridDim.x * blockDim.x)
        parent[u] = P.nxt[u] == (uint32_t)u ? -1 : (int32_t)P.nxt[u];
}

// ---------------------------------------------------------------------------
// The default sampler: Wilson's algorithm exactly as the oracle runs it, one
// GPU thread per tree (a batch of W trees at once).  The walks of one tree
// are sequential (each loop-erased walk ends on the tree the previous ones
// built), so the parallelism is across trees; per tree the state is a byte
// (in tree), the stack depth and the last exit of every vertex.
// ---------------------------------------------------------------------------
struct WSeqParams {
    const uint32_t *row_ptr, *adj;
    const int32_t *coff, *cverts;
    int64_t n, ncomp;
    int W;
    const uint64_t *tkey;    // [W]
    uint8_t *in_tree;        // [W][n]
    uint32_t *dep;           // [W][n]
    int32_t *nxt;            // [W][n] -> parent (-1 at the roots)
};

__global__ void k_ws_init(WSeqParams P) {
    const int64_t total = (int64_t)P.W * P.n;
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < total;
         i += (int64_t)gridDim.x * blockDim.x) {
        P.in_tree[i] = 0;
        P.dep[i] = 0;
        P.nxt[i] = -1;
    }
}

__global__ void k_ws_roots(WSeqParams P) {
    const int64_t total = (int64_t)P.W * P.ncomp;
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < total;
         i += (int64_t)gridDim.x * blockDim.x) {
        const int b = (int)(i / P.ncomp);
        const int64_t C = i - (int64_t)b * P.ncomp;
        const uint32_t sz = (uint32_t)(P.coff[C + 1] - P.coff[C]);
        const uint32_t r = (uint32_t)P.cverts[P.coff[C] + (int64_t)(root_key(P.tkey[b], C) % sz)];
        P.in_tree[(size_t)b * P.n + r] = 1;
    }
}

__global__ void k_ws_walks(WSeqParams P) {
    const int b = blockIdx.x * blockDim.x + threadIdx.x;
    if (b >= P.W) return;
    const uint64_t tk = P.tkey[b];
    uint8_t *in_tree = P.in_tree + (size_t)b * P.n;
    uint32_t *dep = P.dep + (size_t)b * P.n;
    int32_t *nxt = P.nxt + (size_t)b * P.n;
    for (int64_t v = 0; v < P.n; v++) {
        if (in_tree[v]) continue;
        // random walk from v until it hits the tree; nxt keeps the last exit
        uint32_t u = (uint32_t)v;
        while (!in_tree[u]) {
            const uint32_t rs = __ldg(P.row_ptr + u), deg = __ldg(P.row_ptr + u + 1) - rs;
            const uint32_t j = dep[u]++;
            const uint64_t h = mix64(tk + kWMul * (((uint64_t)u << 32) | j));
            const uint32_t w = __ldg(P.adj + rs + (uint32_t)(h % deg)) & kIdMask;
            nxt[u] = (int32_t)w;
            u = w;
        }
        // the loop-erased path joins the tree
        for (u = (uint32_t)v; !in_tree[u]; u = (uint32_t)nxt[u]) in_tree[u] = 1;
    }
}

static unsigned wgrid(int64_t work, int sms) {
    return (unsigned)std::max<int64_t>(1, std::min<int64_t>((work + 255) / 256, (int64_t)sms * 8));
}

int run_wilson(const Graph &g, Workspace &ws, cudaStream_t st, int64_t *launches, int32_t *parent,
               int64_t *rounds_out) {
    const int64_t n = g.n;
    if (!ws.wbuf) {
        // s, nxt, J0, J1 (u32) + done, cyc, D0, D1 (u8) + counter
        const size_t bytes = 16 * (size_t)n + 4 * (size_t)n + 64;
        GB_CUDA_TRY(cudaMalloc(&ws.wbuf, bytes));
    }
    uint32_t *base = reinterpret_cast<uint32_t *>(ws.wbuf);
    WParams P;
    P.row_ptr = g.row_ptr; P.adj = g.adj; P.coff = g.coff; P.cverts = g.cverts;
    P.n = n; P.ncomp = g.ncomp; P.tkey = ws.tkey;
    P.s = base; P.nxt = base + n;
    uint32_t *J0 = base + 2 * n, *J1 = base + 3 * n;
    uint8_t *b8 = reinterpret_cast<uint8_t *>(base + 4 * n);
    P.done = b8; P.cyc = b8 + n;
    uint8_t *D0 = b8 + 2 * n, *D1 = b8 + 3 * n;
    P.active = reinterpret_cast<unsigned long long *>(((uintptr_t)(b8 + 4 * n) + 7) & ~(uintptr_t)7);
    const int sms = g.num_sms;
    const unsigned gn = wgrid(n, sms);
    k_w_init<<<gn, 256, 0, st>>>(P);
    k_w_roots<<<wgrid(g.ncomp, sms), 256, 0, st>>>(P);
    *launches += 2;
    int64_t active = n - g.ncomp, rounds = 0;
    static const bool trace = getenv("GB_WILSON_TRACE") != nullptr;
    while (active > 0) {
        if (++rounds > (1 << 22)) { set_error("wilson: cycle popping did not finish"); return GB_ECUDA; }
        int K = 1;
        while ((1ll << K) <= active) K++;
        k_w_jump_init<<<gn, 256, 0, st>>>(P, J0, D0);
        uint32_t *Ja = J0, *Jb = J1;
        uint8_t *Da = D0, *Db = D1;
        for (int k = 0; k < K; k++) {
            k_w_jump<<<gn, 256, 0, st>>>(n, Ja, Da, Jb, Db);
            std::swap(Ja, Jb);
            std::swap(Da, Db);
        }
        k_w_mark<<<gn, 256, 0, st>>>(P, Ja, Da);
        GB_CUDA_TRY(cudaMemsetAsync(P.active, 0, sizeof(unsigned long long), st));
        k_w_pop<<<gn, 256, 0, st>>>(P);
        *launches += K + 3;
        unsigned long long h = 0;
        GB_CUDA_TRY(cudaMemcpyAsync(&h, P.active, sizeof(h), cudaMemcpyDeviceToHost, st));
        GB_CUDA_TRY(cudaStreamSynchronize(st));
        active = (int64_t)h;
        if (trace && (rounds < 64 || (rounds & (rounds - 1)) == 0 || active < 64))
            fprintf(stderr, "wilson round %lld K %d active %lld\n", (long long)rounds, K, (long long)active);
    }
    if (trace) fprintf(stderr, "wilson rounds %lld\n", (long long)rounds);
    k_w_parent<<<gn, 256, 0, st>>>(P, parent);
    ++*launches;
    if (rounds_out) *rounds_out = rounds;
    GB_CUDA_TRY(cudaGetLastError());
    return GB_OK;
}

// ---------------------------------------------------------------------------
// Alg. 2 with M = DFS (reading R18), one GPU thread per tree: iterative DFS
// from the R4 root of every component; the scan of u's neighbours starts at
// mix64(tkey ^ D*(u+1)) mod deg(u) and wraps around.
// ---------------------------------------------------------------------------
constexpr uint64_t kDMul = 0x8CB92BA72F3D8DD7ull;

struct DfsParams {
    const uint32_t *row_ptr, *adj;
    const int32_t *coff, *cverts;
    int64_t n, ncomp;
    int W;
    const uint64_t *tkey;    // [W]
    int32_t *parent;         // [W][n]
    uint32_t *pos;           // [W][n] neighbours scanned so far
    uint8_t *seen;           // [W][n]
    uint32_t *stack;         // [W][n]
};

__global__ void k_ds_init(DfsParams P) {
    const int64_t total = (int64_t)P.W * P.n;
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < total;
         i += (int64_t)gridDim.x * blockDim.x) {
        P.parent[i] = -1;
        P.pos[i] = 0;
        P.seen[i] = 0;
    }
}

__global__ void k_ds_dfs(DfsParams P) {
    const int b = blockIdx.x * blockDim.x + threadIdx.x;
    if (b >= P.W) return;
    const uint64_t tk = P.tkey[b];
    const size_t o = (size_t)b * P.n;
    int32_t *parent = P.parent + o;
    uint32_t *pos = P.pos + o, *stack = P.stack + o;
    uint8_t *seen = P.seen + o;
    for (int64_t C = 0; C < P.ncomp; C++) {
        const uint32_t sz = (uint32_t)(P.coff[C + 1] - P.coff[C]);
        const uint32_t r = (uint32_t)P.cverts[P.coff[C] + (int64_t)(root_key(tk, C) % sz)];
        int64_t top = 0;
        seen[r] = 1;
        stack[top++] = r;
        while (top > 0) {
            const uint32_t u = stack[top - 1];
            const uint32_t rs = __ldg(P.row_ptr + u), deg = __ldg(P.row_ptr + u + 1) - rs;
            const uint32_t p = pos[u];
            if (p == deg) { top--; continue; }
            const uint32_t s0 = (uint32_t)(mix64(tk ^ (kDMul * ((uint64_t)u + 1))) % deg);
            const uint32_t k = s0 + p >= deg ? s0 + p - deg : s0 + p;
            pos[u] = p + 1;
            const uint32_t w = __ldg(P.adj + rs + k) & kIdMask;
            if (!seen[w]) {
                seen[w] = 1;
                parent[w] = (int32_t)u;
                stack[top++] = w;
            }
        }
    }
}

static int ensure_sampler_state(const Graph &g, Workspace &ws, int W) {
    if (ws.wseq_cap < W) {
        if (ws.wseq) cudaFree(ws.wseq);
        ws.wseq = nullptr;
        ws.wseq_cap = 0;
        GB_CUDA_TRY(cudaMalloc(&ws.wseq, (size_t)W * 13 * (size_t)g.n + 64));
        ws.wseq_cap = W;
    }
    return GB_OK;
}

int run_dfs_batch(const Graph &g, Workspace &ws, int W, cudaStream_t st, int64_t *launches) {
    const int64_t n = g.n;
    int rc = ensure_sampler_state(g, ws, W);
    if (rc) return rc;
    DfsParams P;
    P.row_ptr = g.row_ptr; P.adj = g.adj; P.coff = g.coff; P.cverts = g.cverts;
    P.n = n; P.ncomp = g.ncomp; P.W = W; P.tkey = ws.wtkey;
    char *base = reinterpret_cast<char *>(ws.wseq);
    P.parent = reinterpret_cast<int32_t *>(base);
    P.pos = reinterpret_cast<uint32_t *>(base + 4 * (size_t)W * n);
    P.seen = reinterpret_cast<uint8_t *>(base + 8 * (size_t)W * n);
    P.stack = reinterpret_cast<uint32_t *>(base + ((9 * (size_t)W * n + 15) & ~(size_t)15));
    k_ds_init<<<wgrid((int64_t)W * n, g.num_sms), 256, 0, st>>>(P);
    k_ds_dfs<<<(unsigned)W, 1, 0, st>>>(P);
    *launches += 2;
    GB_CUDA_TRY(cudaGetLastError());
    return GB_OK;
}

int run_wilson_batch(const Graph &g, Workspace &ws, int W, cudaStream_t st, int64_t *launches) {
    const int64_t n = g.n;
    int rc0 = ensure_sampler_state(g, ws, W);
    if (rc0) return rc0;
    WSeqParams P;
    P.row_ptr = g.row_ptr; P.adj = g.adj; P.coff = g.coff; P.cverts = g.cverts;
    P.n = n; P.ncomp = g.ncomp; P.W = W; P.tkey = ws.wtkey;
    char *base = reinterpret_cast<char *>(ws.wseq);
    P.nxt = reinterpret_cast<int32_t *>(base);
    P.dep = reinterpret_cast<uint32_t *>(base + 4 * (size_t)W * n);
    P.in_tree = reinterpret_cast<uint8_t *>(base + 8 * (size_t)W * n);
    const int sms = g.num_sms;
    k_ws_init<<<wgrid((int64_t)W * n, sms), 256, 0, st>>>(P);
    k_ws_roots<<<wgrid((int64_t)W * g.ncomp, sms), 256, 0, st>>>(P);
    k_ws_walks<<<(unsigned)W, 1, 0, st>>>(P);   // one tree per SM-resident thread
    *launches += 3;
    GB_CUDA_TRY(cudaGetLastError());
    return GB_OK;
}

}  // namespace gb
