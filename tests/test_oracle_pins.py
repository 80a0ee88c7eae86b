"""Pins of the CPU oracle against what PAPER.md and the mathematics fix
(never against the oracle itself, never against the CUDA path).

Each test names the passage or fact it pins.  Tiny brute force lives in
tests/_brute.py (independent Python)."""
from __future__ import annotations

import os
from collections import deque

import numpy as np
import pytest

import graphgen
import oracle
from tests import _brute as bf
from tests.test_oracle_spec_pins import spec_rkey

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def _golden(name):
    rows = []
    with open(os.path.join(GOLDEN, name)) as f:
        for line in f:
            line = line.strip()
            if line and not line.startswith("#"):
                rows.append(line.split())
    return rows


def _tiny_graphs():
    out = [graphgen.diamond(), graphgen.ring(5, [0]), graphgen.ring(6, [1, 2, 4]),
           graphgen.complete(5, lambda u, v: -1 if (u + v) % 3 == 0 else 1),
           graphgen.grid2d(3, 3, 0.4, seed=3), graphgen.star(6), graphgen.path(5)]
    for s in range(40):
        n = 3 + s % 5
        m = min(n * (n - 1) // 2, n - 1 + s % 6)
        out.append(graphgen.random_tiny(n, m, 0.4, seed=100 + s, connected=(s % 7 != 0)))
    return out


# --------------------------------------------------------------------------
# Hash (reading R4) -- public SplitMix64 test vector
# --------------------------------------------------------------------------

def test_splitmix64_kat():
    kat = [int(v, 16) for _, v in _golden("splitmix64_kat.txt")]
    assert oracle.splitmix64_stream(0, len(kat)) == kat
    # tkey(seed, t) is the (t+1)-th output from state = seed
    assert [oracle.tkey(0, t) for t in range(len(kat))] == kat


def test_pscore_is_symmetric_and_spread():
    """The parent score depends on the unordered edge only, and its 32-bit
    values are spread (ties are rare; they fall back to the smaller id)."""
    rng = np.random.default_rng(3)
    vals = set()
    for _ in range(3000):
        a, b = (int(x) for x in rng.integers(0, 2**31 - 1, 2))
        s1 = oracle.pscore(9, 4, a, b)
        assert s1 == oracle.pscore(9, 4, b, a)
        vals.add(s1)
    assert len(vals) >= 2990
    # the score is the high word of mix64 over the packed pair (pinned mix64)
    a, b = 5, 77
    z = (oracle.tkey(1, 0) + 0x9E3779B97F4A7C15 * ((a << 32) | b)) % 2**64
    assert oracle.pscore(1, 0, a, b) == oracle.mix64(z) >> 32


def test_mix64_is_a_bijection_sample():
    xs = np.random.default_rng(1).integers(0, 2**63, 20000, dtype=np.int64)
    ys = {oracle.mix64(int(x)) for x in xs}
    assert len(ys) == len(set(int(x) for x in xs))


# --------------------------------------------------------------------------
# Table 1 identity and the cycle count (L112)
# --------------------------------------------------------------------------

def test_table1_cycles_identity():
    for name, n, m, cyc in _golden("table1_cycles.txt"):
        assert int(cyc) == int(m) - int(n) + 1, name


@pytest.mark.parametrize("seed", [1, 2, 3])
def test_cycle_count_is_m_minus_n_plus_c(seed):
    for g in [graphgen.er(300, 900, 0.3, seed), graphgen.er(200, 150, 0.5, seed),
              graphgen.grid2d(7, 9, 0.3, seed)]:
        og = oracle.Graph.from_csr(g)
        for t in range(3):
            parent, _, _ = og.bfs_tree(seed, t)
            flip, sk, ncyc, _ = og.balance_tree(parent)
            assert ncyc == g.m - g.n + og.ncomp


# --------------------------------------------------------------------------
# BFS tree (reading R4): textbook BFS distances, brute-force argmin parent
# --------------------------------------------------------------------------

@pytest.mark.parametrize("seed", [1, 7])
def test_bfs_dist_and_minhash_parent(seed):
    g = graphgen.er(400, 1000, 0.3, seed)
    og = oracle.Graph.from_csr(g)
    comp, coff, cverts = og.components()
    edges = bf.edge_list(g)
    eid = {(u, v): i for i, (u, v, _) in enumerate(edges)}
    for t in range(4):
        parent, dist, peid = og.bfs_tree(seed, t)
        # roots: cverts_C[rkey mod |C|], rkey restated from reading R4
        roots = []
        for c in range(og.ncomp):
            sz = int(coff[c + 1] - coff[c])
            roots.append(int(cverts[int(coff[c]) + spec_rkey(seed, t, c) % sz]))
        assert sorted(roots) == sorted(np.flatnonzero(parent == -1).tolist())
        # textbook multi-source BFS
        d = [-1] * g.n
        dq = deque()
        for r in roots:
            d[r] = 0
            dq.append(r)
        while dq:
            x = dq.popleft()
            for j in range(g.row_ptr[x], g.row_ptr[x + 1]):
                y = int(g.col[j])
                if d[y] < 0:
                    d[y] = d[x] + 1
                    dq.append(y)
        assert list(dist) == d
        # every edge spans at most one level (BFS-tree property)
        for u, v, _ in edges:
            assert abs(d[u] - d[v]) <= 1
        # brute-force argmin of (pscore, u) over neighbours one level up
        for w in range(g.n):
            if d[w] == 0:
                continue
            cands = [int(u) for u in g.col[g.row_ptr[w]:g.row_ptr[w + 1]] if d[u] == d[w] - 1]
            best = min(cands, key=lambda u: (oracle.pscore(seed, t, u, w), u))
            assert parent[w] == best
            assert peid[w] == eid[(min(best, w), max(best, w))]
        # spanning forest: n - c edges, acyclic (union-find)
        par = list(range(g.n))

        def find(x):
            while par[x] != x:
                par[x] = par[par[x]]
                x = par[x]
            return x
        k = 0
        for w in range(g.n):
            if parent[w] >= 0:
                a, b = find(w), find(int(parent[w]))
                assert a != b
                par[a] = b
                k += 1
        assert k == g.n - og.ncomp


# --------------------------------------------------------------------------
# Alg. 1: tree edges never switch (L102-L104); closed form of the new sign
# (L214: the cycle becomes even); balanced result (L79, L216); Sigma k (L230)
# --------------------------------------------------------------------------

def _check_tree_result(g, og, parent, flip, sumk):
    edges = bf.edge_list(g)
    n = g.n
    negmap = {(u, v): neg for u, v, neg in edges}
    pneg = [0] * n
    for v in range(n):
        if parent[v] >= 0:
            p = int(parent[v])
            pneg[v] = negmap[(min(p, v), max(p, v))]
    pi = bf.root_parity(n, [int(x) for x in parent], pneg)
    depth = [0] * n
    for v in range(n):
        x, d = v, 0
        while parent[x] >= 0:
            x = int(parent[x])
            d += 1
        depth[v] = d
    tot = 0
    new_edges = []
    for e, (u, v, neg) in enumerate(edges):
        tree = parent[u] == v or parent[v] == u
        if tree:
            assert flip[e] == 0                      # L102: only non-tree edges
        else:
            assert flip[e] == (pi[u] ^ pi[v] ^ neg)   # closed form: cycle even
            # k = d(u)+d(v)-2 d(lca)+1  <= d(u)+d(v)+1 (L230)
            a, b = u, v
            anc = set()
            x = a
            while True:
                anc.add(x)
                if parent[x] < 0:
                    break
                x = int(parent[x])
            y = b
            while y not in anc:
                y = int(parent[y])
            k = depth[u] + depth[v] - 2 * depth[y] + 1
            assert k <= depth[u] + depth[v] + 1
            tot += k
        new_edges.append((u, v, neg ^ int(flip[e])))
    assert tot == sumk
    assert bf.is_balanced(n, new_edges)               # L79: Sigma_T balanced
    return new_edges


@pytest.mark.parametrize("seed", [1, 2, 3, 4])
def test_alg1_closed_form_and_balance(seed):
    for g in [graphgen.er(300, 1200, 0.3, seed), graphgen.grid2d(8, 8, 0.5, seed),
              graphgen.chung_lu(500, 2000, 80, 0.75, 0.3, seed)]:
        og = oracle.Graph.from_csr(g)
        for t in range(3):
            parent, _, _ = og.bfs_tree(seed, t)
            flip, sk, ncyc, _ = og.balance_tree(parent)
            _check_tree_result(g, og, parent, flip, sk)


def test_all_cycles_even_after_balancing():
    """L216/L222: once the fundamental cycles are balanced every cycle is."""
    for g in _tiny_graphs()[:25]:
        og = oracle.Graph.from_csr(g)
        parent, _, _ = og.bfs_tree(5, 0)
        flip, _, _, _ = og.balance_tree(parent)
        edges = bf.edge_list(g)
        for cyc in bf.simple_cycles(g.n, edges):
            negs = sum(edges[i][2] ^ int(flip[i]) for i in cyc)
            assert negs % 2 == 0


def test_nearest_no_proper_subset_balances():
    """L81: a state is nearest if no subset of the switches yields balance."""
    for g in _tiny_graphs():
        og = oracle.Graph.from_csr(g)
        edges = bf.edge_list(g)
        for t in range(2):
            parent, _, _ = og.bfs_tree(11, t)
            flip, _, _, _ = og.balance_tree(parent)
            fl = [i for i in range(g.m) if flip[i]]
            if len(fl) > 10:
                continue
            for r in range(len(fl)):
                import itertools
                for sub in itertools.combinations(fl, r):
                    s = set(sub)
                    cand = [(u, v, neg ^ (i in s)) for i, (u, v, neg) in enumerate(edges)]
                    assert not bf.is_balanced(g.n, cand)


def test_frustration_index_bounds_over_all_trees():
    """L81: Fr(Sigma) = min number of negations; every tree's switch count is
    >= Fr, and the minimum over ALL spanning trees equals Fr."""
    checked = 0
    for g in _tiny_graphs():
        if g.n > 7 or g.m > 12:
            continue
        og = oracle.Graph.from_csr(g)
        edges = bf.edge_list(g)
        comp, c = bf.components(g.n, edges)
        roots = [min(v for v in range(g.n) if comp[v] == k) for k in range(c)]
        fr = bf.frustration_index(g.n, edges)
        best = None
        for tree in bf.spanning_trees(g.n, edges):
            parent = bf.parent_array(g.n, tree, roots)
            flip, _, _, _ = og.balance_tree(np.array(parent, np.int32))
            k = int(flip.sum())
            assert k >= fr
            best = k if best is None else min(best, k)
        assert best == fr
        checked += 1
    assert checked >= 20


# --------------------------------------------------------------------------
# Special cases with closed-form answers (SURVEY §8c "Special cases")
# --------------------------------------------------------------------------

def test_all_positive_and_planted_balanced_inputs():
    g = graphgen.er(500, 2000, 0.0, 3)
    og = oracle.Graph.from_csr(g)
    T = 5
    cnt, agree = og.balance(T, 9)
    assert cnt.sum() == 0 and np.all(agree == 2 * T)
    gb, colour = graphgen.planted_signs(graphgen.er(501, 2000, 0.0, 4), 5)
    og = oracle.Graph.from_csr(gb)
    cnt, agree = og.balance(T, 9)
    assert cnt.sum() == 0
    ones = int(colour.sum())
    zeros = gb.n - ones
    for v in range(gb.n):
        mine = ones if colour[v] else zeros
        exp = 2 * T if mine > gb.n - mine else (T if 2 * mine == gb.n else 0)
        assert agree[v] == exp


def test_bipartite_all_negative_has_no_flips():
    # every cycle of a bipartite graph is even, so all-negative is balanced
    g = graphgen.bipartite_chung_lu(300, 200, 900, 40, 60, 0.5, 0.6, 1.0, 2)
    og = oracle.Graph.from_csr(g)
    cnt, _ = og.balance(4, 1)
    assert cnt.sum() == 0


def test_tree_input_has_no_cycles():
    g = graphgen.path(50)
    og = oracle.Graph.from_csr(g)
    parent, _, _ = og.bfs_tree(1, 0)
    flip, sk, ncyc, _ = og.balance_tree(parent)
    assert ncyc == 0 and sk == 0 and flip.sum() == 0


@pytest.mark.parametrize("negs", [[0], [0, 1, 2], [3, 5, 6, 7, 9]])
def test_odd_ring_flips_exactly_once_per_tree(negs):
    g = graphgen.ring(11, negs)
    og = oracle.Graph.from_csr(g)
    T = 7
    cnt, _ = og.balance(T, 3)
    assert cnt.sum() == T


def test_triangle_flips_edge_opposite_root():
    g = graphgen.from_edge_list(3, [(0, 1, 1), (1, 2, -1), (0, 2, 1)])
    og = oracle.Graph.from_csr(g)
    for t in range(6):
        parent, dist, _ = og.bfs_tree(2, t)
        root = int(np.flatnonzero(parent == -1)[0])
        flip, _, _, _ = og.balance_tree(parent)
        u, v, _ = og.edges()
        opp = [e for e in range(3) if root not in (u[e], v[e])][0]
        assert flip.tolist() == [1 if e == opp else 0 for e in range(3)]


def test_switching_invariance():
    """Negating every edge across a vertex cut leaves each tree's switch set
    unchanged (cycle signs are switching invariant; the tree ignores signs)."""
    g = graphgen.er(300, 1000, 0.3, 8)
    rng = np.random.default_rng(0)
    side = rng.integers(0, 2, g.n)
    rows = np.repeat(np.arange(g.n), np.diff(g.row_ptr))
    sign2 = np.where(side[rows] != side[g.col], -g.sign, g.sign).astype(np.int8)
    g2 = graphgen.SignedCSR(g.n, g.m, g.row_ptr, g.col, sign2)
    c1, _ = oracle.Graph.from_csr(g).balance(6, 4)
    c2, _ = oracle.Graph.from_csr(g2).balance(6, 4)
    assert np.array_equal(c1, c2)


# --------------------------------------------------------------------------
# Labels (Alg. 3 steps 1-2, Alg. 4): pre-order permutation, laminar ranges
# --------------------------------------------------------------------------

@pytest.mark.parametrize("seed", [1, 2])
def test_preorder_labels(seed):
    g = graphgen.er(300, 700, 0.3, seed)   # sparse: several components
    og = oracle.Graph.from_csr(g)
    comp, coff, _ = og.components()
    parent, _, _ = og.bfs_tree(seed, 0)
    pre, size = og.preorder(parent)
    assert sorted(pre.tolist()) == list(range(g.n))
    for v in range(g.n):
        if parent[v] < 0:
            assert pre[v] == coff[comp[v]]                    # reading R6
    kids = [[] for _ in range(g.n)]
    for v in range(g.n):
        if parent[v] >= 0:
            kids[parent[v]].append(v)
    for p in range(g.n):
        assert size[p] == 1 + sum(size[c] for c in kids[p])
        nxt = pre[p] + 1
        for c in sorted(kids[p]):                             # reading R5
            assert pre[c] == nxt                              # Alg. 4
            nxt += size[c]
    # range of p contains exactly p's subtree (ancestor test used by Alg. 3)
    for v in range(g.n):
        anc = set()
        x = v
        while x >= 0:
            anc.add(x)
            x = int(parent[x])
        for a in range(g.n):
            inside = pre[a] <= pre[v] <= pre[a] + size[a] - 1
            assert inside == (a in anc)


# --------------------------------------------------------------------------
# Harary bipartition (L224) vs the root-parity shortcut, and delta (L144)
# --------------------------------------------------------------------------

@pytest.mark.parametrize("seed", [1, 2, 3])
def test_harary_matches_root_parity(seed):
    g = graphgen.er(250, 600, 0.4, seed)
    og = oracle.Graph.from_csr(g)
    comp, coff, _ = og.components()
    edges = bf.edge_list(g)
    negmap = {(u, v): neg for u, v, neg in edges}
    for t in range(3):
        parent, _, _ = og.bfs_tree(seed, t)
        flip, _, _, _ = og.balance_tree(parent)
        side, d2 = og.harary(flip)
        pneg = [0] * g.n
        for v in range(g.n):
            if parent[v] >= 0:
                p = int(parent[v])
                pneg[v] = negmap[(min(p, v), max(p, v))]
        pi = bf.root_parity(g.n, [int(x) for x in parent], pneg)
        for c in range(og.ncomp):
            vs = np.flatnonzero(comp == c)
            # same bipartition (up to naming the sides)
            a = [side[v] for v in vs]
            b = [pi[v] for v in vs]
            assert a == b or a == [1 - x for x in b]
            s1 = sum(b)
            s0 = len(vs) - s1
            for v in vs:
                mine = s1 if pi[v] else s0
                other = len(vs) - mine
                assert d2[v] == (2 if mine > other else (1 if mine == other else 0))


def test_harary_rejects_unbalanced():
    g = graphgen.from_edge_list(3, [(0, 1, 1), (1, 2, -1), (0, 2, 1)])
    og = oracle.Graph.from_csr(g)
    with pytest.raises(oracle.OracleError):
        og.harary(np.zeros(3, np.uint8))


# --------------------------------------------------------------------------
# The Fig. 1-3 example (reconstruction; consistency with the prose)
# --------------------------------------------------------------------------

def test_diamond_frustration_cloud():
    facts = {r[0]: r[1:] for r in _golden("diamond.txt")}
    g = graphgen.diamond()
    og = oracle.Graph.from_csr(g)
    edges = bf.edge_list(g)
    trees = list(bf.spanning_trees(g.n, edges))
    assert len(trees) == int(facts["spanning_trees"][0])          # L116
    states = {}
    agree = np.zeros(g.n, np.int64)
    for tree in trees:
        parent = bf.parent_array(g.n, tree, [0])
        flip, _, _, _ = og.balance_tree(np.array(parent, np.int32))
        key = tuple(int(neg) ^ int(f) for (_, _, neg), f in zip(edges, flip))  # signs of Sigma_T
        states[key] = states.get(key, 0) + 1
        _, d2 = og.harary(flip)
        agree += d2
    assert len(states) == int(facts["unique_states"][0])          # L81, L86
    # f.2: the state signature separates exactly the distinct states
    sigs = {}
    for tree in trees:
        parent = bf.parent_array(g.n, tree, [0])
        flip, _, _, _ = og.balance_tree(np.array(parent, np.int32))
        sigs.setdefault(oracle.state_signature(flip), set()).add(tuple(flip.tolist()))
    assert len(sigs) == len(states) and all(len(v) == 1 for v in sigs.values())
    assert max(states.values()) == int(facts["top_state_count"][0])  # L112
    assert states[tuple([0] * g.m)] == int(facts["top_state_count"][0])  # all-positive state
    assert agree.tolist() == [int(x) for x in facts["agree"]]     # L144 (6/8)


# --------------------------------------------------------------------------
# Validation (boundary error list) and sharding invariance (L248)
# --------------------------------------------------------------------------

def test_oracle_rejects_invalid_csr():
    g = graphgen.diamond()
    bad = []
    rp = g.row_ptr.copy(); rp[-1] += 1
    bad.append((rp, g.col, g.sign))                        # row_ptr[n] != 2m
    c = g.col.copy(); c[0] = c[1]
    bad.append((g.row_ptr, c, g.sign))                     # duplicate / unsorted
    s = g.sign.copy(); s[0] = -s[0]
    bad.append((g.row_ptr, g.col, s))                      # asymmetric sign
    s = g.sign.copy(); s[0] = 0
    bad.append((g.row_ptr, g.col, s))                      # sign not +-1
    c = g.col.copy(); c[0] = 0
    bad.append((g.row_ptr, c, g.sign))                     # self loop
    c = g.col.copy(); c[0] = 99
    bad.append((g.row_ptr, c, g.sign))                     # out of range
    for rp, c, s in bad:
        with pytest.raises(oracle.OracleError):
            oracle.Graph(rp, c, s)


def test_state_signature_definition():
    """f.2 signature: XOR-linear over switched edges, empty set -> 0."""
    assert oracle.state_signature(np.zeros(5, np.uint8)) == 0
    a = np.array([1, 0, 1, 0, 0], np.uint8)
    b = np.array([0, 0, 1, 1, 0], np.uint8)
    ab = a ^ b
    assert oracle.state_signature(a) ^ oracle.state_signature(b) == oracle.state_signature(ab)
    one = np.array([0, 0, 0, 1], np.uint8)
    assert oracle.state_signature(one) == oracle.mix64(3 ^ 0x5851F42D4C957F2D)


def test_tree_sharding_is_additive():
    g = graphgen.er(400, 1500, 0.3, 5)
    og = oracle.Graph.from_csr(g)
    T = 12
    c_all, a_all = og.balance(T, 77)
    for W in (2, 3, 4):
        cs = np.zeros_like(c_all); as_ = np.zeros_like(a_all)
        for r in range(W):
            c, a = og.balance(T, 77, t_begin=r, stride=W)
            cs += c; as_ += a
        assert np.array_equal(cs, c_all) and np.array_equal(as_, a_all)


def test_balance_given_tree_rejects_non_forests():
    g = graphgen.ring(5, [0])
    og = oracle.Graph.from_csr(g)
    with pytest.raises(oracle.OracleError):
        og.balance_tree(np.array([-1, 0, 1, 2, 3 if False else -1], np.int32))  # 2 roots
    with pytest.raises(oracle.OracleError):
        og.balance_tree(np.array([-1, 0, 3, 2, 0], np.int32))                   # cycle 2<->3
    with pytest.raises(oracle.OracleError):
        og.balance_tree(np.array([-1, 0, 0, 2, 3], np.int32))                   # 0-2 not an edge


# --------------------------------------------------------------------------
# f.3: Alg. 2 with M = random (L130): uniform spanning trees by Wilson's
# algorithm with per-vertex random stacks (reading R17).  Pins: the tree does
# not depend on the order of the start vertices (cycle-popping theorem), the
# sampled trees are exactly the spanning trees (count by Kirchhoff's
# matrix-tree theorem) and uniformly distributed (chi-square), roots follow R4.
# --------------------------------------------------------------------------

def _tree_key(parent):
    return tuple(sorted((min(v, int(p)), max(v, int(p))) for v, p in enumerate(parent) if p >= 0))


def _matrix_tree_count(g):
    n = g.n
    Lap = np.zeros((n, n))
    for u, v, _ in bf.edge_list(g):
        Lap[u, v] -= 1; Lap[v, u] -= 1; Lap[u, u] += 1; Lap[v, v] += 1
    return int(round(np.linalg.det(Lap[1:, 1:])))


@pytest.mark.parametrize("which", ["er", "chung_lu", "forest", "grid", "ring"])
def test_wilson_order_independent_spanning_forest(which):
    g = {"er": lambda: graphgen.er(400, 1500, 0.3, 3),
         "chung_lu": lambda: graphgen.chung_lu(600, 2400, 90, 0.75, 0.3, 2),
         "forest": lambda: graphgen.er(500, 300, 0.4, 2),
         "grid": lambda: graphgen.grid2d(9, 11, 0.5, 4),
         "ring": lambda: graphgen.ring(50)}[which]()
    og = oracle.Graph.from_csr(g)
    edges = {(u, v) for u, v, _ in bf.edge_list(g)}
    for t in range(5):
        p0, pops = og.wilson_tree(7, t, 0)
        p1, _ = og.wilson_tree(7, t, 1)
        assert np.array_equal(p0, p1), "Wilson tree depends on the start order"
        bfs_parent, dist, _ = og.bfs_tree(7, t)
        assert np.array_equal(np.flatnonzero(p0 < 0), np.flatnonzero(dist == 0))   # R4 roots
        for v in range(g.n):
            if p0[v] >= 0:
                assert (min(v, int(p0[v])), max(v, int(p0[v]))) in edges
        # acyclic: every vertex reaches a root within n steps
        for v in range(g.n):
            x, k = v, 0
            while p0[x] >= 0:
                x = int(p0[x]); k += 1
                assert k <= g.n
        assert int(pops.sum()) >= 0


@pytest.mark.parametrize("g,ntrees", [(graphgen.complete(4), 16), (graphgen.diamond(), 8),
                                      (graphgen.ring(6), 6)])
def test_wilson_uniform_over_all_spanning_trees(g, ntrees):
    from scipy.stats import chisquare
    assert _matrix_tree_count(g) == ntrees
    og = oracle.Graph.from_csr(g)
    counts = {}
    S = 400 * ntrees
    for t in range(S):
        p, _ = og.wilson_tree(11, t, 0)
        k = _tree_key(p)
        counts[k] = counts.get(k, 0) + 1
    assert len(counts) == ntrees
    assert chisquare(list(counts.values())).pvalue > 1e-4


def test_wilson_cloud_balances_every_tree():
    g = graphgen.er(200, 700, 0.4, 9)
    og = oracle.Graph.from_csr(g)
    for t in range(4):
        parent, _ = og.wilson_tree(3, t)
        flip, sk, nc, _ = og.balance_tree(parent)
        _check_tree_result(g, og, parent, flip, sk)
    cnt, agree, st = og.balance(4, 3, with_stats=True, sampler=1)
    assert int(st[:, 1].sum()) == 4 * (g.m - g.n + og.ncomp)


# --------------------------------------------------------------------------
# f.3: Alg. 2 with M = DFS (L130), reading R18.  Pins: the defining property
# of an undirected DFS tree -- every non-tree edge joins an ancestor and a
# descendant (no cross edges) -- plus closed shapes: DFS trees of complete
# graphs and rings are Hamiltonian paths; roots follow R4.
# --------------------------------------------------------------------------

def _ancestors(parent, v):
    out = set()
    while parent[v] >= 0:
        v = int(parent[v])
        out.add(v)
    return out


@pytest.mark.parametrize("which", ["er", "chung_lu", "forest", "grid"])
def test_dfs_tree_has_no_cross_edges(which):
    g = {"er": lambda: graphgen.er(300, 1100, 0.3, 3),
         "chung_lu": lambda: graphgen.chung_lu(400, 1600, 60, 0.75, 0.3, 2),
         "forest": lambda: graphgen.er(400, 250, 0.4, 2),
         "grid": lambda: graphgen.grid2d(9, 11, 0.5, 4)}[which]()
    og = oracle.Graph.from_csr(g)
    for t in range(4):
        parent = og.dfs_tree(5, t)
        _, dist, _ = og.bfs_tree(5, t)
        assert np.array_equal(np.flatnonzero(parent < 0), np.flatnonzero(dist == 0))   # R4 roots
        anc = [_ancestors(parent, v) for v in range(g.n)]
        for u, v, _ in bf.edge_list(g):
            assert u in anc[v] or v in anc[u], "cross edge: not a DFS tree"
        for v in range(g.n):
            if parent[v] >= 0:
                assert (min(v, int(parent[v])), max(v, int(parent[v]))) in {(a, b) for a, b, _ in bf.edge_list(g)}


@pytest.mark.parametrize("g", [graphgen.complete(9), graphgen.ring(17)])
def test_dfs_tree_of_complete_and_ring_is_a_path(g):
    og = oracle.Graph.from_csr(g)
    for t in range(5):
        parent = og.dfs_tree(2, t)
        depth = [len(_ancestors(parent, v)) for v in range(g.n)]
        assert sorted(depth) == list(range(g.n))          # one vertex per level: a path
