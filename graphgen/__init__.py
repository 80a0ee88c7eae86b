"""Seeded synthetic signed-graph generators (input recipes only).

This module is shared by the oracle side (``oracle/``) and the CUDA side
(``paper_conf_sc_alabanditrb21_b200``).  It holds NO arithmetic of the
balancing method: it only draws graphs and signs, builds the symmetric CSR
that the C-ABI ``gb_load_csr`` takes, and extracts the largest connected
component (the paper processes only the LCC, §5).

Recipes (DESIGN.md §"Input recipe"; shapes from PAPER.md Table 1,
Table 5, Table 6):

* C1  ``er``      Erdos-Renyi G(n, m): m distinct uniform pairs, 30 % negative.
* C2  ``slashdot`` Chung-Lu power law, LCC, Slashdot shape (82,140 / 549,202,
                   max degree ~2.5k), 23 % negative.
* C3  ``amazon``  bipartite users x items Chung-Lu, LCC, Amazon-Books shape
                   (9.97 M / 22.27 M, max degree ~43 k), 50 % negative.
* C4  ``epinions`` Chung-Lu power law, LCC, Epinions shape (119,130 / 704,267,
                   max degree ~3.5 k), 15 % negative; ``wikielec`` secondary.
* C5  ``rmat``    Graph500 RMAT (0.57, 0.19, 0.19, 0.05), scale 26, edge
                   factor 16, symmetrised, de-duplicated, loops dropped,
                   all components kept, 50 % negative.

Every generator is a pure function of its seed.  Vertex ids are randomly
permuted (seeded) so that no artificial locality is left in the ids.
"""
from __future__ import annotations

import dataclasses
import numpy as np

__all__ = [
    "SignedCSR", "csr_from_edges", "er", "chung_lu", "bipartite_chung_lu",
    "rmat", "rmat_gpu", "largest_cc", "permute", "config", "CONFIGS",
    "ring", "path", "star", "complete", "grid2d", "diamond", "planted_signs",
    "random_tiny", "from_edge_list",
]


@dataclasses.dataclass
class SignedCSR:
    """Symmetric simple signed graph in CSR form (the gb_load_csr layout).

    row_ptr int64[n+1]; col int32[2m] (rows strictly increasing);
    sign int8[2m] in {+1,-1} with sign(u,v) == sign(v,u).
    """
    n: int
    m: int
    row_ptr: np.ndarray
    col: np.ndarray
    sign: np.ndarray
    name: str = ""

    def edges(self):
        """Undirected edge list (u < v), in CSR order of upper slots."""
        rows = np.repeat(np.arange(self.n, dtype=np.int64), np.diff(self.row_ptr))
        up = self.col > rows
        return rows[up], self.col[up].astype(np.int64), self.sign[up]

    def degrees(self):
        return np.diff(self.row_ptr)


def _canon(u, v):
    a = np.minimum(u, v).astype(np.int64)
    b = np.maximum(u, v).astype(np.int64)
    keep = a != b
    return a[keep], b[keep]


def _sorted_unique(key):
    key = np.sort(key)
    if len(key) == 0:
        return key
    keep = np.empty(len(key), bool)
    keep[0] = True
    np.not_equal(key[1:], key[:-1], out=keep[1:])
    return key[keep]


def _dedup(n, a, b):
    key = _sorted_unique(a * np.int64(n) + b)
    return key // n, key % n


def csr_from_edges(n, u, v, neg, name=""):
    """Build the symmetric CSR from an undirected simple edge list.

    ``neg`` is a boolean per undirected edge (True = negative sign).  One sort
    of packed keys ((src*n + dst) << 1 | neg) builds both directions.
    """
    u = np.asarray(u, dtype=np.int64)
    v = np.asarray(v, dtype=np.int64)
    neg = np.asarray(neg, dtype=np.int64)
    m = len(u)
    nn = np.int64(n)
    key = np.empty(2 * m, np.int64)
    np.multiply(u, nn, out=key[:m]); key[:m] += v
    np.multiply(v, nn, out=key[m:]); key[m:] += u
    key <<= 1
    key[:m] |= neg
    key[m:] |= neg
    key.sort(kind="stable")
    sg = np.where((key & 1).astype(bool), -1, 1).astype(np.int8)
    key >>= 1
    src = key // nn
    dst = (key - src * nn).astype(np.int32)
    del key
    row_ptr = np.zeros(n + 1, dtype=np.int64)
    np.cumsum(np.bincount(src, minlength=n), out=row_ptr[1:])
    return SignedCSR(n, m, row_ptr, dst, sg, name)


def from_edge_list(n, edges, name=""):
    """Tiny-graph helper: ``edges`` = iterable of (u, v, sign) with sign +1/-1."""
    edges = list(edges)
    if not edges:
        return SignedCSR(n, 0, np.zeros(n + 1, np.int64), np.zeros(0, np.int32),
                         np.zeros(0, np.int8), name)
    u = np.array([min(e[0], e[1]) for e in edges], np.int64)
    v = np.array([max(e[0], e[1]) for e in edges], np.int64)
    neg = np.array([e[2] < 0 for e in edges], bool)
    return csr_from_edges(n, u, v, neg, name)


def permute(g: SignedCSR, seed: int) -> SignedCSR:
    """Relabel vertices by a seeded random permutation (signs follow edges)."""
    u, v, s = g.edges()
    return _finish(g.n, u, v, s < 0, seed, g.name, lcc=False)


def _lcc_edges(n, u, v, neg):
    """Restrict an edge list to its largest connected component (PAPER.md
    L333: only the LCC is processed); vertex ids compacted in old-id order."""
    import scipy.sparse as sp
    from scipy.sparse.csgraph import connected_components
    a = sp.coo_matrix((np.ones(len(u), np.int8), (u, v)), shape=(n, n)).tocsr()
    nc, lab = connected_components(a, directed=False)
    if nc == 1:
        return n, u, v, neg
    big = np.bincount(lab).argmax()
    keep = lab == big
    newid = np.full(n, -1, np.int64)
    nk = int(keep.sum())
    newid[keep] = np.arange(nk)
    k = keep[u]
    return nk, newid[u[k]], newid[v[k]], neg[k]


def _finish(n, u, v, neg, seed, name, lcc):
    if lcc:
        n, u, v, neg = _lcc_edges(n, u, v, neg)
    rng = np.random.default_rng([seed, 0x5EED])
    perm = rng.permutation(n).astype(np.int64)
    pu, pv = perm[u], perm[v]
    return csr_from_edges(n, np.minimum(pu, pv), np.maximum(pu, pv), neg, name)


def largest_cc(g: SignedCSR) -> SignedCSR:
    """Keep only the largest connected component."""
    u, v, s = g.edges()
    n, u, v, neg = _lcc_edges(g.n, u, v, s < 0)
    return csr_from_edges(n, u, v, neg, g.name)


def _signs(rng, m, p_neg):
    return rng.random(m) < p_neg


# --------------------------------------------------------------------------
# Generators
# --------------------------------------------------------------------------

def er(n, m, p_neg, seed, name="er"):
    """G(n, m): m distinct uniform vertex pairs (no loops, no duplicates)."""
    rng = np.random.default_rng([seed, 1])
    a = np.zeros(0, np.int64)
    b = np.zeros(0, np.int64)
    while len(a) < m:
        need = int((m - len(a)) * 1.05) + 16
        x = rng.integers(0, n, need)
        y = rng.integers(0, n, need)
        x, y = _canon(x, y)
        a, b = _dedup(n, np.concatenate([a, x]), np.concatenate([b, y]))
    if len(a) > m:
        sel = np.sort(rng.choice(len(a), m, replace=False))
        a, b = a[sel], b[sel]
    return _finish(n, a, b, _signs(rng, m, p_neg), seed, name, lcc=False)


def _powerlaw_weights(N, beta, offset):
    return (np.arange(N, dtype=np.float64) + offset) ** (-beta)


def _wsum(N, beta, i0):
    """sum_{i<N} (i+i0)^-beta by Euler-Maclaurin (integral + end corrections)."""
    a, b = i0, N - 1 + i0
    integ = (b ** (1 - beta) - a ** (1 - beta)) / (1 - beta)
    return integ + 0.5 * (a ** -beta + b ** -beta) + beta / 12.0 * (a ** (-beta - 1) - b ** (-beta - 1))


def _solve_offset(N, beta, total_deg, dmax):
    """Offset i0 such that the expected degree of the heaviest vertex is dmax."""
    lo, hi = 1e-3, float(N)
    for _ in range(200):
        mid = np.sqrt(lo * hi)
        d0 = total_deg * mid ** (-beta) / _wsum(N, beta, mid)
        if d0 > dmax:
            lo = mid
        else:
            hi = mid
    return np.sqrt(lo * hi)


def _sample(rng, cdf, k):
    """k i.i.d. draws from the discrete distribution with cumulative weights
    ``cdf``.  Sorted uniforms (normalised exponential spacings) make the
    search cache-friendly; a random permutation restores i.i.d. order."""
    s = np.cumsum(rng.standard_exponential(k + 1))
    q = s[:k] * (cdf[-1] / s[k])
    idx = np.searchsorted(cdf, q, side="right")
    np.minimum(idx, len(cdf) - 1, out=idx)
    return idx[rng.permutation(k)]


def chung_lu(n, m, dmax, beta, p_neg, seed, lcc=True, name="chung_lu"):
    """Chung-Lu power-law graph: endpoints drawn proportional to (i+i0)^-beta."""
    rng = np.random.default_rng([seed, 2])
    i0 = _solve_offset(n, beta, 2.0 * m, dmax)
    cdf = np.cumsum(_powerlaw_weights(n, beta, i0))
    a = np.zeros(0, np.int64)
    b = np.zeros(0, np.int64)
    while len(a) < m:
        need = int((m - len(a)) * 1.1) + 16
        x, y = _canon(_sample(rng, cdf, need), _sample(rng, cdf, need))
        a, b = _dedup(n, np.concatenate([a, x]), np.concatenate([b, y]))
    if len(a) > m:
        sel = np.sort(rng.choice(len(a), m, replace=False))
        a, b = a[sel], b[sel]
    return _finish(n, a, b, _signs(rng, m, p_neg), seed, name, lcc)


def bipartite_chung_lu(n_users, n_items, m, dmax_users, dmax_items, beta_users,
                       beta_items, p_neg, seed, lcc=True, local_frac=0.0,
                       local_width=1, name="bipartite"):
    """Users x items ratings graph (Amazon-like, Table 1 'Amazon
    Ratings'): every edge joins a user to an item; both sides power law.

    A fraction ``local_frac`` of the edges is drawn "banded" instead: user x
    rates an item whose popularity rank is proportional to x's, within
    +-``local_width`` ranks.  This gives the sparse, chain-like periphery that
    makes the paper's Amazon BFS trees deep (15-19 levels, Table 6)
    while the Chung-Lu part keeps the hubs (max degree ~43k, Table 1).
    """
    rng = np.random.default_rng([seed, 3])
    cu = np.cumsum(_powerlaw_weights(n_users, beta_users,
                                     _solve_offset(n_users, beta_users, m, dmax_users)))
    ci = np.cumsum(_powerlaw_weights(n_items, beta_items,
                                     _solve_offset(n_items, beta_items, m, dmax_items)))
    n = n_users + n_items
    m_local = int(m * local_frac)
    a = np.zeros(0, np.int64)
    b = np.zeros(0, np.int64)
    if m_local:
        x = rng.integers(0, n_users, m_local)
        y = (x * (n_items / n_users)).astype(np.int64) + rng.integers(-local_width, local_width + 1, m_local)
        np.clip(y, 0, n_items - 1, out=y)
        a, b = _dedup(n, x, y + n_users)
    while len(a) < m:
        need = int((m - len(a)) * 1.05) + 16
        x = _sample(rng, cu, need)
        y = _sample(rng, ci, need) + n_users
        a, b = _dedup(n, np.concatenate([a, x]), np.concatenate([b, y]))
    if len(a) > m:
        sel = np.sort(rng.choice(len(a), m, replace=False))
        a, b = a[sel], b[sel]
    return _finish(n, a, b, _signs(rng, m, p_neg), seed, name, lcc)


def rmat(scale, edge_factor, p_neg, seed, abcd=(0.57, 0.19, 0.19, 0.05),
         name="rmat", chunk=1 << 25):
    """Graph500 R-MAT: 2^scale vertices, edge_factor*2^scale generated edges,
    symmetrised, de-duplicated, self loops dropped, all components kept."""
    rng = np.random.default_rng([seed, 4])
    n = 1 << scale
    total = edge_factor * n
    a, b, c, _ = abcd
    keys = []
    done = 0
    while done < total:
        k = min(chunk, total - done)
        src = np.zeros(k, np.int64)
        dst = np.zeros(k, np.int64)
        for bit in range(scale):
            r = rng.random(k)
            sbit = r >= a + b            # quadrants c, d -> source bit 1
            dbit = ((r >= a) & (r < a + b)) | (r >= a + b + c)
            src |= sbit.astype(np.int64) << bit
            dst |= dbit.astype(np.int64) << bit
        x, y = _canon(src, dst)
        keys.append(_sorted_unique(x * np.int64(n) + y))
        done += k
    key = _sorted_unique(np.concatenate(keys))
    u, v = key // n, key % n
    return _finish(n, u, v, _signs(rng, len(u), p_neg), seed, name, lcc=False)


def rmat_gpu(scale, edge_factor, p_neg, seed, abcd=(0.57, 0.19, 0.19, 0.05),
             name="rmat", chunk=1 << 26, device="cuda"):
    """Graph500 R-MAT generated with torch on a CUDA device (the same recipe as
    ``rmat``; a different random stream, so a different -- equally seeded --
    graph).  For scale 26 the numpy version needs many minutes of host time.
    Returns a SignedCSR with host (numpy) arrays."""
    import torch
    gen = torch.Generator(device=device)
    gen.manual_seed(int(seed) * 1000003 + 4)
    n = 1 << scale
    total = edge_factor * n
    a, b, c, _ = abcd
    keys = []
    done = 0
    while done < total:
        k = min(chunk, total - done)
        src = torch.zeros(k, dtype=torch.int64, device=device)
        dst = torch.zeros(k, dtype=torch.int64, device=device)
        for bit in range(scale):
            r = torch.rand(k, generator=gen, device=device)
            src |= (r >= a + b).to(torch.int64) << bit
            dst |= (((r >= a) & (r < a + b)) | (r >= a + b + c)).to(torch.int64) << bit
        lo = torch.minimum(src, dst)
        hi = torch.maximum(src, dst)
        keep = lo != hi
        keys.append(torch.unique(lo[keep] * n + hi[keep]))
        del src, dst, lo, hi, keep
        done += k
    key = torch.unique(torch.cat(keys))
    del keys
    m = key.numel()
    neg = (torch.rand(m, generator=gen, device=device) < p_neg).to(torch.int64)
    perm = torch.randperm(n, generator=gen, device=device)
    u = perm[key // n]
    v = perm[key % n]
    del key
    lo = torch.minimum(u, v)
    hi = torch.maximum(u, v)
    del u, v
    both = torch.cat([(lo * n + hi) * 2 + neg, (hi * n + lo) * 2 + neg])
    del lo, hi, neg
    both, _ = torch.sort(both)
    sg = torch.where((both & 1).bool(), -1, 1).to(torch.int8)
    both >>= 1
    srcv = both // n
    col = (both - srcv * n).to(torch.int32)
    del both
    cnt = torch.bincount(srcv, minlength=n)
    del srcv
    row_ptr = torch.zeros(n + 1, dtype=torch.int64, device=device)
    row_ptr[1:] = torch.cumsum(cnt, 0)
    out = SignedCSR(n, m, row_ptr.cpu().numpy(), col.cpu().numpy(), sg.cpu().numpy(), name)
    del row_ptr, col, sg, cnt
    torch.cuda.empty_cache()
    return out


# --------------------------------------------------------------------------
# Tiny / structured graphs for tests
# --------------------------------------------------------------------------

def ring(n, neg_edges=(), name="ring"):
    negs = set(neg_edges)
    return from_edge_list(n, [(i, (i + 1) % n, -1 if i in negs else 1) for i in range(n)], name)


def path(n, name="path"):
    return from_edge_list(n, [(i, i + 1, 1) for i in range(n - 1)], name)


def star(n, name="star"):
    return from_edge_list(n, [(0, i, 1) for i in range(1, n)], name)


def complete(n, sign_fn=lambda u, v: 1, name="complete"):
    return from_edge_list(n, [(u, v, sign_fn(u, v)) for u in range(n) for v in range(u + 1, n)], name)


def grid2d(r, c, p_neg=0.0, seed=0, name="grid"):
    rng = np.random.default_rng([seed, 5])
    es = []
    for i in range(r):
        for j in range(c):
            x = i * c + j
            if j + 1 < c:
                es.append((x, x + 1))
            if i + 1 < r:
                es.append((x, x + c))
    neg = rng.random(len(es)) < p_neg
    return from_edge_list(r * c, [(a, b, -1 if s else 1) for (a, b), s in zip(es, neg)], name)


def diamond(name="diamond"):
    """K4 minus an edge, only the shared diagonal (1,2) negative: the
    reconstruction of PAPER.md Fig. 1(a) used in SURVEY Appendix A."""
    return from_edge_list(4, [(0, 1, 1), (0, 2, 1), (1, 2, -1), (1, 3, 1), (2, 3, 1)], name)


def planted_signs(g: SignedCSR, seed):
    """Re-sign ``g`` as a balanced graph: draw a random 2-colouring and make an
    edge negative iff its endpoints have different colours.  Returns
    (graph, colour)."""
    rng = np.random.default_rng([seed, 6])
    col = rng.integers(0, 2, g.n).astype(np.int8)
    u, v, _ = g.edges()
    neg = col[u] != col[v]
    return csr_from_edges(g.n, u, v, neg, g.name + "_planted"), col


def random_tiny(n, m, p_neg, seed, connected=True, name="tiny"):
    """Random simple graph with n vertices and m edges (connected if asked:
    a random spanning tree is drawn first)."""
    rng = np.random.default_rng([seed, 7])
    edges = set()
    if connected:
        order = rng.permutation(n)
        for i in range(1, n):
            a, b = int(order[i]), int(order[rng.integers(0, i)])
            edges.add((min(a, b), max(a, b)))
    allpairs = [(a, b) for a in range(n) for b in range(a + 1, n) if (a, b) not in edges]
    rng.shuffle(allpairs)
    for p in allpairs:
        if len(edges) >= m:
            break
        edges.add(p)
    edges = sorted(edges)
    neg = rng.random(len(edges)) < p_neg
    return from_edge_list(n, [(a, b, -1 if s else 1) for (a, b), s in zip(edges, neg)], name)


# --------------------------------------------------------------------------
# The BASELINE.json configs
# --------------------------------------------------------------------------

CONFIGS = {
    # name: (builder, trees, description)
    "c1": (lambda seed=1: er(10_000, 50_000, 0.30, seed, name="c1_er_10k_50k"), 1,
           "Erdos-Renyi 10k vertices / 50k edges, 30% negative, 1 tree, seed 1"),
    "c2": (lambda seed=1: chung_lu(82_140, 549_202, 2_548, 0.75, 0.23, seed,
                                   name="c2_slashdot"), 100,
           "Slashdot-shaped power law, LCC of 82,140 / 549,202 generated, 100 trees"),
    "c3": (lambda seed=1: bipartite_chung_lu(8_400_000, 2_330_066, 22_280_000, 3_000, 64_500,
                                             0.5, 0.8, 0.5, seed, local_frac=0.4, local_width=1,
                                             name="c3_amazon"), 100,
           "Amazon-Books-shaped bipartite users x items, ~10M / ~22M (LCC), random signs, 100 trees"),
    "c4": (lambda seed=1: chung_lu(119_130, 704_267, 3_558, 0.75, 0.15, seed,
                                   name="c4_epinions"), 1000,
           "Epinions-shaped power law, LCC of 119,130 / 704,267 generated, 1000 trees"),
    "c4w": (lambda seed=1: chung_lu(7_539, 112_058, 1_079, 0.6, 0.22, seed,
                                    name="c4w_wikielec"), 1000,
            "wiki-Elec-shaped power law, LCC of 7,539 / 112,058 generated, 1000 trees"),
    "c5": (lambda seed=1: rmat_gpu(26, 16, 0.5, seed, name="c5_rmat26"), 10,
           "RMAT scale 26, edge factor 16 (~1B generated edges, GPU-generated), random signs, 10 trees"),
}


def config(name, seed=1):
    """Return (graph, default_num_trees, description) for a BASELINE config."""
    builder, trees, desc = CONFIGS[name]
    return builder(seed), trees, desc
