"""Tiny-graph brute force, written independently of oracle/ and of the CUDA
library (plain Python loops; only for n <= ~8).  Used to pin the oracle
against what the paper and the mathematics fix."""
from __future__ import annotations

import itertools
from collections import deque


def edge_list(g):
    """(u, v, neg) with u < v in eid order (rank of (min,max))."""
    out = []
    for u in range(g.n):
        for j in range(g.row_ptr[u], g.row_ptr[u + 1]):
            v = int(g.col[j])
            if v > u:
                out.append((u, v, int(g.sign[j] < 0)))
    return out


def components(n, edges):
    adj = [[] for _ in range(n)]
    for u, v, _ in edges:
        adj[u].append(v)
        adj[v].append(u)
    comp = [-1] * n
    c = 0
    for s in range(n):
        if comp[s] >= 0:
            continue
        comp[s] = c
        dq = deque([s])
        while dq:
            x = dq.popleft()
            for y in adj[x]:
                if comp[y] < 0:
                    comp[y] = c
                    dq.append(y)
        c += 1
    return comp, c


def signed_two_colouring(n, edges_with_neg):
    """BFS 2-colouring where a negative edge demands different colours.
    Returns the colouring or None if some edge conflicts (unbalanced, L79)."""
    adj = [[] for _ in range(n)]
    for u, v, neg in edges_with_neg:
        adj[u].append((v, neg))
        adj[v].append((u, neg))
    col = [-1] * n
    for s in range(n):
        if col[s] >= 0:
            continue
        col[s] = 0
        dq = deque([s])
        while dq:
            x = dq.popleft()
            for y, neg in adj[x]:
                want = col[x] ^ neg
                if col[y] < 0:
                    col[y] = want
                    dq.append(y)
                elif col[y] != want:
                    return None
    return col


def is_balanced(n, edges_with_neg):
    return signed_two_colouring(n, edges_with_neg) is not None


def frustration_index(n, edges):
    """Fr(Sigma) (L81): minimum number of edge negations giving balance =
    min over 2-colourings of the number of violated edges."""
    best = len(edges)
    for mask in range(1 << (n - 1)):          # fix colour of vertex n-1
        bad = 0
        for u, v, neg in edges:
            cu = (mask >> u) & 1 if u < n - 1 else 0
            cv = (mask >> v) & 1 if v < n - 1 else 0
            if (cu ^ cv) != neg:
                bad += 1
        best = min(best, bad)
    return best


def spanning_trees(n, edges):
    """All spanning forests with one tree per component, as parent arrays
    rooted at each component's smallest vertex (n-c edges, acyclic)."""
    comp, c = components(n, edges)
    k = n - c
    for sub in itertools.combinations(range(len(edges)), k):
        par = list(range(n))

        def find(x):
            while par[x] != x:
                par[x] = par[par[x]]
                x = par[x]
            return x
        ok = True
        for i in sub:
            a, b = find(edges[i][0]), find(edges[i][1])
            if a == b:
                ok = False
                break
            par[a] = b
        if not ok:
            continue
        yield [edges[i] for i in sub]


def parent_array(n, tree_edges, roots):
    adj = [[] for _ in range(n)]
    for u, v, _ in tree_edges:
        adj[u].append(v)
        adj[v].append(u)
    parent = [-2] * n
    for r in roots:
        parent[r] = -1
        dq = deque([r])
        while dq:
            x = dq.popleft()
            for y in adj[x]:
                if parent[y] == -2:
                    parent[y] = x
                    dq.append(y)
    return parent


def simple_cycles(n, edges):
    """All simple cycles (as edge-index lists), by DFS from each start vertex
    with the start as the smallest vertex on the cycle."""
    adj = [[] for _ in range(n)]
    for i, (u, v, _) in enumerate(edges):
        adj[u].append((v, i))
        adj[v].append((u, i))
    seen = set()
    out = []

    def dfs(start, x, visited, path_e):
        for y, i in adj[x]:
            if i in path_e:
                continue
            if y == start and len(path_e) >= 2:
                key = frozenset(path_e + [i])
                if key not in seen:
                    seen.add(key)
                    out.append(list(key))
            elif y > start and y not in visited:
                visited.add(y)
                dfs(start, y, visited, path_e + [i])
                visited.discard(y)
    for s in range(n):
        dfs(s, s, {s}, [])
    return out


def root_parity(n, parent, pneg):
    """pi(v) = XOR of negative bits on the tree path root -> v."""
    pi = [None] * n

    def get(v):
        chain = []
        x = v
        while pi[x] is None and parent[x] >= 0:
            chain.append(x)
            x = parent[x]
        if pi[x] is None:
            pi[x] = 0
        base = pi[x]
        for y in reversed(chain):
            base ^= pneg[y]
            pi[y] = base
        return pi[v]
    for v in range(n):
        get(v)
    return pi
