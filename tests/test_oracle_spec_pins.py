"""Pins of the oracle's seed-defined hash definitions against independent
Python restatements of their specification text.

PAPER.md is silent on the root, the BFS tie rule and the randomness of the
other samplers (Alg. 2 "e.g., BFS, DFS, random"; L479 "random BFS
trees"; L248 "a subset of the tree roots").  The build fixes them in
DESIGN.md §3 (readings R4, R17, R18); those sentences are the specification,
so the only possible pin is a second implementation written from them.  The
restatements below share nothing with oracle/oracle.c: SplitMix64 is written
out here from its public definition and checked against the public test
vector (tests/golden/splitmix64_kat.txt), and every tree builder is a plain
Python loop over the reading's words.

  R4   tkey(seed,t) = SplitMix64 output t+1 from state seed;
       root of component C = C's vertices ascending [mix64(tkey ^ K(C+1)) mod |C|],
       K = 0xD1B54A32D192ED03;
       parent(w) = the neighbour u one level up minimising (pscore(u,w), u),
       pscore = high 32 bits of mix64(tkey + G (min(u,w) 2^32 + max(u,w))).
  R17  the j-th departure of Wilson's walk from u goes to
       N(u)[mix64(tkey + W (u 2^32 + j)) mod deg u], W = 0xD6E8FEB86659FD93;
       walks start at the vertices in ascending order.
  R18  DFS: at u the neighbours are scanned cyclically from position
       mix64(tkey ^ D (u+1)) mod deg u, D = 0x8CB92BA72F3D8DD7; the first
       unvisited one is descended into; returning resumes the scan.
"""
from __future__ import annotations

import os
from collections import deque

import numpy as np
import pytest

import graphgen
import oracle

M64 = (1 << 64) - 1
G = 0x9E3779B97F4A7C15          # SplitMix64 increment (public definition)
K_ROOT = 0xD1B54A32D192ED03      # R4
W_WALK = 0xD6E8FEB86659FD93      # R17
D_DFS = 0x8CB92BA72F3D8DD7       # R18
GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def spec_mix64(z):
    """SplitMix64 output function (Steele, Lea, Flood 2014), written out."""
    z &= M64
    z = ((z ^ (z >> 30)) * 0xBF58476D1CE4E5B9) & M64
    z = ((z ^ (z >> 27)) * 0x94D049BB133111EB) & M64
    return z ^ (z >> 31)


def spec_tkey(seed, t):
    return spec_mix64(seed + G * (t + 1))


def spec_rkey(seed, t, c):
    return spec_mix64(spec_tkey(seed, t) ^ ((K_ROOT * (c + 1)) & M64))


def spec_pscore(seed, t, a, b):
    lo, hi = min(a, b), max(a, b)
    return spec_mix64(spec_tkey(seed, t) + G * ((lo << 32) | hi)) >> 32


def spec_wdraw(seed, t, u, j):
    return spec_mix64(spec_tkey(seed, t) + W_WALK * ((u << 32) | j))


def spec_dstart(seed, t, u):
    return spec_mix64(spec_tkey(seed, t) ^ ((D_DFS * (u + 1)) & M64))


def _adj(g):
    return [[int(x) for x in g.col[g.row_ptr[u]:g.row_ptr[u + 1]]] for u in range(g.n)]


def _components(adj):
    """components ranked by their minimum vertex; vertices ascending"""
    n = len(adj)
    comp = [-1] * n
    groups = []
    for s in range(n):
        if comp[s] >= 0:
            continue
        c = len(groups)
        comp[s] = c
        members, dq = [s], deque([s])
        while dq:
            x = dq.popleft()
            for y in adj[x]:
                if comp[y] < 0:
                    comp[y] = c
                    members.append(y)
                    dq.append(y)
        groups.append(sorted(members))
    return groups


def spec_roots(adj, seed, t):
    return [cv[spec_rkey(seed, t, c) % len(cv)] for c, cv in enumerate(_components(adj))]


def spec_bfs_tree(adj, seed, t):
    roots = spec_roots(adj, seed, t)
    dist = [-1] * len(adj)
    dq = deque()
    for r in roots:
        dist[r] = 0
        dq.append(r)
    while dq:
        x = dq.popleft()
        for y in adj[x]:
            if dist[y] < 0:
                dist[y] = dist[x] + 1
                dq.append(y)
    parent = [-1] * len(adj)
    for w in range(len(adj)):
        cands = [u for u in adj[w] if dist[u] == dist[w] - 1]
        if cands:
            parent[w] = min(cands, key=lambda u: (spec_pscore(seed, t, u, w), u))
    return parent, dist


def spec_wilson_tree(adj, seed, t):
    n = len(adj)
    in_tree = [False] * n
    for r in spec_roots(adj, seed, t):
        in_tree[r] = True
    departures = [0] * n
    nxt = [-1] * n
    for v in range(n):
        u = v
        while not in_tree[u]:
            k = spec_wdraw(seed, t, u, departures[u]) % len(adj[u])
            departures[u] += 1
            nxt[u] = adj[u][k]
            u = nxt[u]
        u = v
        while not in_tree[u]:
            in_tree[u] = True
            u = nxt[u]
    return nxt


def spec_dfs_tree(adj, seed, t):
    n = len(adj)
    parent = [-1] * n
    seen = [False] * n
    for r in spec_roots(adj, seed, t):
        seen[r] = True
        stack = [(r, 0)]
        while stack:
            u, i = stack[-1]
            deg = len(adj[u])
            if i == deg:
                stack.pop()
                continue
            stack[-1] = (u, i + 1)
            w = adj[u][(spec_dstart(seed, t, u) % deg + i) % deg]
            if not seen[w]:
                seen[w] = True
                parent[w] = u
                stack.append((w, 0))
    return parent


def _graphs():
    return [graphgen.er(120, 300, 0.3, 5), graphgen.er(90, 70, 0.3, 6),   # forest-ish, many comps
            graphgen.grid2d(6, 7, 0.3, 2), graphgen.diamond(), graphgen.ring(9, [0, 3]),
            graphgen.complete(7), graphgen.star(8),
            graphgen.chung_lu(400, 1200, 60, 0.75, 0.2, 3, lcc=False)]


# --------------------------------------------------------------------------
# the hash itself
# --------------------------------------------------------------------------

def test_spec_mix64_matches_public_vector():
    rows = []
    with open(os.path.join(GOLDEN, "splitmix64_kat.txt")) as f:
        for line in f:
            line = line.strip()
            if line and not line.startswith("#"):
                rows.append(line.split())
    state, outs = 0, []
    for _ in range(len(rows)):
        state = (state + G) & M64
        outs.append(spec_mix64(state))
    assert [int(r[-1], 16) for r in rows] == outs
    assert [spec_tkey(0, i) for i in range(len(rows))] == outs


def test_tkey_rkey_wdraw_dstart_match_spec():
    """or_tkey / or_rkey / or_wdraw / or_dstart equal the R4 / R17 / R18
    sentences on random inputs (a wrong constant, C for C+1, + for ^ or a
    swapped shift fails here)."""
    rng = np.random.default_rng(11)
    for _ in range(400):
        seed = int(rng.integers(0, 2**63)) * 2 + int(rng.integers(0, 2))
        t = int(rng.integers(0, 2**30 - 1))
        c = int(rng.integers(0, 2**31 - 1))
        u = int(rng.integers(0, 2**31 - 1))
        j = int(rng.integers(0, 2**32 - 1))
        assert oracle.tkey(seed, t) == spec_tkey(seed, t)
        assert oracle.rkey(seed, t, c) == spec_rkey(seed, t, c)
        assert oracle.wdraw(seed, t, u, j) == spec_wdraw(seed, t, u, j)
        assert oracle.dstart(seed, t, u) == spec_dstart(seed, t, u)
        v = int(rng.integers(0, 2**31 - 1))
        assert oracle.pscore(seed, t, u, v) == spec_pscore(seed, t, u, v)
    # small arguments, where an off-by-one in (t+1), (C+1), (u+1) shows most
    for seed in (0, 1, 2**64 - 1):
        for t in range(4):
            for c in range(4):
                assert oracle.rkey(seed, t, c) == spec_rkey(seed, t, c)
                assert oracle.dstart(seed, t, c) == spec_dstart(seed, t, c)
                assert oracle.wdraw(seed, t, c, t) == spec_wdraw(seed, t, c, t)


def test_root_choice_is_uniform_over_the_component():
    """R4 draws the root of a component uniformly (chi-square over trees)."""
    sz = 7
    counts = np.zeros(sz)
    T = 2800
    for t in range(T):
        counts[spec_rkey(1, t, 0) % sz] += 1
    exp = T / sz
    chi2 = float(((counts - exp) ** 2 / exp).sum())
    assert chi2 < 22.46   # 6 dof, p = 0.001


# --------------------------------------------------------------------------
# the trees the definitions produce
# --------------------------------------------------------------------------

@pytest.mark.parametrize("gi", range(8))
def test_oracle_bfs_tree_equals_spec(gi):
    g = _graphs()[gi]
    adj = _adj(g)
    og = oracle.Graph.from_csr(g)
    for seed in (1, 9):
        for t in range(4):
            parent, dist, _ = og.bfs_tree(seed, t)
            sp, sd = spec_bfs_tree(adj, seed, t)
            assert list(parent) == sp
            assert list(dist) == sd


@pytest.mark.parametrize("gi", range(8))
def test_oracle_wilson_tree_equals_spec(gi):
    g = _graphs()[gi]
    adj = _adj(g)
    og = oracle.Graph.from_csr(g)
    for t in range(3):
        parent, _ = og.wilson_tree(5, t)
        assert list(parent) == spec_wilson_tree(adj, 5, t)


@pytest.mark.parametrize("gi", range(8))
def test_oracle_dfs_tree_equals_spec(gi):
    g = _graphs()[gi]
    adj = _adj(g)
    og = oracle.Graph.from_csr(g)
    for t in range(3):
        assert list(og.dfs_tree(3, t)) == spec_dfs_tree(adj, 3, t)
