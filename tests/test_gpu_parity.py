"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle on the
same seeded inputs.  Everything here is integer work, so the bar is
bit-exact: edge flip counts, vertex agree counts, per-tree sums of cycle
lengths and cycle counts, and every stage of single trees (parent, dist,
size, flips).  Pre-order IDs are not unique (the sibling order is free,
reading R5), so they are checked for validity instead."""
from __future__ import annotations

import os

import numpy as np
import pytest

import graphgen
import oracle
from paper_conf_sc_alabanditrb21_b200 import graphb

pytestmark = pytest.mark.gpu


@pytest.fixture(autouse=True)
def _reset_options():
    yield
    graphb.set_option("reset", 0)


def check_cloud(g, T, seed, **opts):
    for k, v in opts.items():
        graphb.set_option(k, v)
    graphb.load_graph(g)
    cnt, agree = graphb.balance_host(T, seed)
    st = graphb.stats()
    ids, per = graphb.tree_stats()
    og = oracle.Graph.from_csr(g)
    ocnt, oagree, ostats = og.balance(T, seed, with_stats=True, sampler=opts.get("sampler", 0))
    assert np.array_equal(cnt, ocnt), "edge flip counts"
    assert np.array_equal(agree, oagree), "vertex agree"
    assert list(ids) == list(range(T))
    assert np.array_equal(per[:, 0], ostats[:, 0]), "per-tree sum of cycle lengths"
    assert np.array_equal(per[:, 1], ostats[:, 1]), "per-tree cycles"
    assert np.array_equal(per[:, 2], ostats[:, 2]), "per-tree depth"
    assert np.array_equal(per[:, 3], ostats[:, 3]), "per-tree state signature (f.2)"
    assert st["cycles"] == T * (g.m - g.n + og.ncomp)     # L112
    return st


def valid_preorder(parent, size, pre, comp_off_of_root):
    n = len(parent)
    assert sorted(pre.tolist()) == list(range(n))
    roots = np.flatnonzero(parent < 0)
    for r in roots:
        assert pre[r] == comp_off_of_root[r]
    ch = np.flatnonzero(parent >= 0)
    p = parent[ch]
    # child's range nested strictly inside the parent's (Alg. 4)
    assert np.all(pre[ch] > pre[p])
    assert np.all(pre[ch] + size[ch] <= pre[p] + size[p])
    # siblings' ranges disjoint and tile the parent's range: sort children by pre
    order = np.lexsort((pre[ch], p))
    cs, ps = ch[order], p[order]
    first = np.ones(len(cs), bool)
    first[1:] = ps[1:] != ps[:-1]
    exp = np.where(first, pre[ps] + 1, 0)
    prev_end = np.r_[0, pre[cs][:-1] + size[cs][:-1]]
    exp = np.where(first, exp, prev_end)
    assert np.array_equal(pre[cs], exp)


def check_tree_debug(g, seed, trees, walk=0):
    graphb.set_option("walk", walk)
    graphb.load_graph(g)
    og = oracle.Graph.from_csr(g)
    comp, coff, _ = og.components()
    for t in trees:
        d = graphb.tree_debug(t, seed)
        parent, dist, _ = og.bfs_tree(seed, t)
        flip, sk, nc, _ = og.balance_tree(parent)
        opre, osize = og.preorder(parent)
        assert np.array_equal(d["parent"], parent)
        assert np.array_equal(d["dist"], dist)
        assert np.array_equal(d["size"], osize)
        assert np.array_equal(d["flip"], flip)
        assert d["sum_cycle_len"] == sk and d["num_cycles"] == nc
        valid_preorder(d["parent"], d["size"], d["pre"], coff[comp])


# ---------------------------------------------------------------------------

def test_c1_config_exact():
    """BASELINE configs[0]: ER 10k / 50k, 30% negative, 1 tree, seed 1."""
    g, T, _ = graphgen.config("c1")
    st = check_cloud(g, T, 1)
    assert st["trees"] == 1


@pytest.mark.parametrize("walk", [0, 1, 2, 3])
def test_tree_stages_match_oracle(walk):
    g = graphgen.er(3000, 12000, 0.3, 4)
    check_tree_debug(g, 5, range(6), walk=walk)


@pytest.mark.parametrize("walk,linear", [(0, 0), (1, 0), (1, 1), (2, 0), (3, 0)])
def test_power_law_hubs_multi_batch(walk, linear):
    """Hubs (Chung-Lu, children lists of thousands) + several batches + cycle
    groups smaller than a batch; walk 1 with 32-ary pivots and with linear
    int4 ballot rounds, walk 2 = the paper's partitioned two-word edge lists
    (L238-L244)."""
    g = graphgen.chung_lu(20000, 90000, 2500, 0.75, 0.25, 3)
    check_cloud(g, 37, 11, batch=16, cycle_group=5, walk=walk, desc_linear=linear)


@pytest.mark.parametrize("ept", [2, 4])
def test_walk_edges_per_thread(ept):
    """Walk 0 with 2 / 4 edges per thread climbed interleaved (option
    walk_ept), cycle groups and a ragged last word (m not a multiple of 32)."""
    g = graphgen.chung_lu(20000, 90001, 2500, 0.75, 0.25, 3)
    check_cloud(g, 37, 11, batch=16, cycle_group=5, walk_ept=ept)
    check_cloud(graphgen.er(5000, 3000, 0.4, 2), 9, 3, walk_ept=ept)


def test_msbfs_128_tree_pass():
    """One multi-source BFS pass holds up to 128 trees (two 64-bit halves per
    vertex): 130 trees = a 128-tree batch + a 2-tree batch on a graph with
    hubs (multi-chunk vertices, phase C) and isolated vertices; the whole
    cloud and every per-tree statistic against the oracle."""
    g = graphgen.chung_lu(6000, 30000, 1500, 0.75, 0.3, 21, lcc=False)
    st = check_cloud(g, 130, 4)
    assert st["batch"] == 128 and st["batches"] == 2


@pytest.mark.parametrize("walk", [0, 1, 2, 3])
def test_paper_walks_on_forests_and_degenerate_trees(walk):
    """Walks 1 and 2 on a forest with isolated vertices (roots without a
    parent edge) and on a star (one hub with every vertex as a child)."""
    check_cloud(graphgen.er(5000, 3000, 0.4, 2), 9, 3, walk=walk)
    check_cloud(graphgen.star(300), 4, 1, walk=walk)
    check_cloud(graphgen.complete(40, lambda u, v: -1 if (u * v) % 3 == 1 else 1), 6, 2, walk=walk, desc_linear=1)


@pytest.mark.parametrize("jump,recpass,sub", [(1, 0, 0), (1, 1, 1), (2, 1, 0), (2, 0, 3), (4, 1, 1), (4, 0, 0)])
def test_walk_records_and_label_passes(jump, recpass, sub):
    """Walk 0 with 1-, 2- and 4-level ancestor records (option "jump"), the
    records scattered inside or after the top-down pass ("recpass"), and
    labelling launches of 1, 3 or all trees ("sub"): all bit-exact."""
    g = graphgen.chung_lu(30000, 120000, 3000, 0.75, 0.3, 8)
    check_cloud(g, 21, 3, batch=8, cycle_group=3, jump=jump, recpass=recpass, sub=sub)


@pytest.mark.parametrize("which", ["er", "chung_lu", "forest", "diamond", "planted", "grid"])
def test_harary_l224_procedure_on_gpu(which):
    """f.2 (L224): Harary sides from the paper's procedure on the GPU --
    CCs of the positive edges of Sigma_T, collapse, BFS level parity -- give
    the same agree counts as the oracle (which runs L224 literally), and every
    edge of every Sigma_T is consistent with the bipartition (L216)."""
    g = {"er": lambda: graphgen.er(4000, 16000, 0.3, 6),
         "chung_lu": lambda: graphgen.chung_lu(20000, 90000, 2500, 0.75, 0.5, 4),
         "forest": lambda: graphgen.er(5000, 3000, 0.4, 2),
         "diamond": lambda: graphgen.diamond(),
         "planted": lambda: graphgen.planted_signs(graphgen.er(3000, 12000, 0.0, 3), 5)[0],
         "grid": lambda: graphgen.grid2d(40, 50, 0.5, 7)}[which]()
    st = check_cloud(g, 13, 2, harary=1, batch=5)
    assert st["harary_violations"] == 0


def _uniform_graphs():
    return {"er": graphgen.er(3000, 12000, 0.3, 4),
            "chung_lu": graphgen.chung_lu(8000, 32000, 900, 0.75, 0.3, 5),
            "forest": graphgen.er(4000, 2500, 0.4, 2),
            "grid": graphgen.grid2d(30, 40, 0.5, 3),
            "ring": graphgen.ring(300, neg_edges=(0, 7, 11))}


@pytest.mark.parametrize("wilson", [0, 1])
@pytest.mark.parametrize("which", ["er", "chung_lu", "forest", "grid", "ring"])
def test_uniform_sampler_trees_match_oracle(which, wilson):
    """f.3 (Alg. 2 M = random, reading R17): the GPU's parallel cycle popping
    returns exactly the oracle's sequential Wilson tree, and every later stage
    (labels, walk, flips, cycle lengths) matches on it."""
    g = _uniform_graphs()[which]
    graphb.set_option("sampler", 1)
    graphb.set_option("wilson", wilson)     # 0: thread per tree, 1: parallel cycle popping
    graphb.load_graph(g)
    og = oracle.Graph.from_csr(g)
    comp, coff, _ = og.components()
    for t in range(4):
        d = graphb.tree_debug(t, 9)
        parent, _ = og.wilson_tree(9, t)
        assert np.array_equal(d["parent"], parent), "uniform tree differs from the oracle's"
        flip, sk, nc, _ = og.balance_tree(parent)
        opre, osize = og.preorder(parent)
        assert np.array_equal(d["size"], osize)
        assert np.array_equal(d["flip"], flip)
        assert d["sum_cycle_len"] == sk and d["num_cycles"] == nc
        valid_preorder(d["parent"], d["size"], d["pre"], coff[comp])


@pytest.mark.parametrize("wilson", [0, 1])
@pytest.mark.parametrize("which", ["er", "chung_lu", "forest"])
def test_uniform_sampler_cloud(which, wilson):
    """f.3: the frustration cloud over uniform spanning trees = the oracle's
    (several sampling chunks: T = 6 with at most 4 trees per chunk below)."""
    check_cloud(_uniform_graphs()[which], 6, 4, sampler=1, wilson=wilson)


@pytest.mark.parametrize("which", ["er", "chung_lu", "forest", "grid", "ring"])
def test_dfs_sampler_trees_match_oracle(which):
    """f.3 (Alg. 2 M = DFS, reading R18): the GPU's DFS tree equals the
    oracle's, and labels / walk / flips / cycle lengths match on it."""
    g = _uniform_graphs()[which]
    graphb.set_option("sampler", 2)
    graphb.load_graph(g)
    og = oracle.Graph.from_csr(g)
    comp, coff, _ = og.components()
    for t in range(3):
        d = graphb.tree_debug(t, 5)
        parent = og.dfs_tree(5, t)
        assert np.array_equal(d["parent"], parent), "DFS tree differs from the oracle's"
        flip, sk, nc, _ = og.balance_tree(parent)
        opre, osize = og.preorder(parent)
        assert np.array_equal(d["size"], osize)
        assert np.array_equal(d["flip"], flip)
        assert d["sum_cycle_len"] == sk and d["num_cycles"] == nc
        valid_preorder(d["parent"], d["size"], d["pre"], coff[comp])


@pytest.mark.parametrize("which", ["er", "forest"])
def test_dfs_sampler_cloud(which):
    """f.3: the frustration cloud over DFS trees = the oracle's."""
    check_cloud(_uniform_graphs()[which], 5, 6, sampler=2)


@pytest.mark.parametrize("sampler,walk,harary", [(1, 1, 0), (2, 1, 0), (1, 0, 1), (2, 0, 1), (1, 3, 0), (2, 3, 1)])
def test_samplers_with_descent_walk_and_l224_sides(sampler, walk, harary):
    """f.3 samplers combined with Alg. 3's descent walk (walk 1) and with the
    paper's L224 Harary procedure (f.2): still the oracle's cloud."""
    g = graphgen.chung_lu(6000, 24000, 700, 0.75, 0.35, 12)
    st = check_cloud(g, 5, 8, sampler=sampler, walk=walk, harary=harary)
    if harary:
        assert st["harary_violations"] == 0


def test_frustration_cloud_distinct_states():
    """f.2 (Fig. 2, L81/L86): distinct nearest balanced states over many
    trees, counted from the per-tree state signatures, equal the oracle's."""
    g = graphgen.random_tiny(7, 11, 0.4, seed=3)
    check_cloud(g, 200, 5)
    states = graphb.cloud_states()
    og = oracle.Graph.from_csr(g)
    _, _, ostats = og.balance(200, 5, with_stats=True)
    assert len(states) == len(set(int(x) for x in ostats[:, 3]))
    assert sum(states.values()) == 200
    assert len(states) > 1


def test_disconnected_forest_with_isolated_vertices():
    g = graphgen.er(5000, 3000, 0.4, 2)     # many components, isolated vertices
    check_cloud(g, 9, 3)
    check_tree_debug(g, 3, range(3))


@pytest.mark.parametrize("name", ["path", "star", "ring", "complete", "grid", "single", "pair",
                                  "empty", "diamond", "bipartite_neg"])
def test_degenerate_graphs(name):
    g = {
        "path": lambda: graphgen.path(100),
        "star": lambda: graphgen.star(3000),
        "ring": lambda: graphgen.ring(101, [0, 5, 7]),
        "complete": lambda: graphgen.complete(40, lambda u, v: -1 if (u * v) % 3 == 1 else 1),
        "grid": lambda: graphgen.grid2d(40, 50, 0.3, 1),
        "single": lambda: graphgen.from_edge_list(1, []),
        "pair": lambda: graphgen.from_edge_list(2, [(0, 1, -1)]),
        "empty": lambda: graphgen.from_edge_list(7, []),
        "diamond": graphgen.diamond,
        "bipartite_neg": lambda: graphgen.bipartite_chung_lu(500, 300, 2000, 50, 80, 0.5, 0.6, 1.0, 1),
    }[name]()
    check_cloud(g, 12, 7)


def test_deep_path_many_levels():
    """A long path: depth ~ n/2 levels in one cooperative kernel."""
    g = graphgen.path(20000)
    check_cloud(g, 3, 1)


def test_balanced_inputs_closed_form():
    gb, colour = graphgen.planted_signs(graphgen.largest_cc(graphgen.er(4001, 20000, 0.0, 9)), 2)
    graphb.load_graph(gb)
    T = 10
    cnt, agree = graphb.balance_host(T, 5)
    assert cnt.sum() == 0
    ones = int(colour.sum())
    big = 1 if ones > gb.n - ones else 0
    exp = np.where(colour == big, 2 * T, 0)
    assert np.array_equal(agree, exp)


def test_given_trees_match_oracle():
    """Alg. 3 on arbitrary (non-BFS) spanning trees."""
    g = graphgen.er(2000, 7000, 0.35, 6)
    graphb.load_graph(g)
    og = oracle.Graph.from_csr(g)
    rng = np.random.default_rng(0)
    u, v, _ = og.edges()
    for trial in range(4):
        # random spanning forest via union-find over shuffled edges
        par = np.arange(g.n)

        def find(x):
            while par[x] != x:
                par[x] = par[par[x]]
                x = par[x]
            return x
        adj = [[] for _ in range(g.n)]
        for e in rng.permutation(g.m):
            a, b = find(u[e]), find(v[e])
            if a != b:
                par[a] = b
                adj[u[e]].append(v[e]); adj[v[e]].append(u[e])
        parent = np.full(g.n, -2, np.int32)
        for s in range(g.n):
            if parent[s] != -2:
                continue
            parent[s] = -1
            stack = [s]
            while stack:
                x = stack.pop()
                for y in adj[x]:
                    if parent[y] == -2:
                        parent[y] = x
                        stack.append(y)
        flip, sk, nc = graphb.balance_given_tree(parent)
        oflip, osk, onc, _ = og.balance_tree(parent)
        assert np.array_equal(flip, oflip) and sk == osk and nc == onc
    # invalid trees are rejected
    bad = parent.copy()
    bad[np.flatnonzero(bad >= 0)[0]] = -1          # two roots in one component
    with pytest.raises(graphb.GraphBError):
        graphb.balance_given_tree(bad)
    bad = parent.copy()
    x = int(np.flatnonzero(bad >= 0)[0])
    nonadj = [w for w in range(g.n) if w != x and w not in set(g.col[g.row_ptr[x]:g.row_ptr[x + 1]])]
    bad[x] = nonadj[0]                              # parent not adjacent
    with pytest.raises(graphb.GraphBError):
        graphb.balance_given_tree(bad)


def test_invalid_csr_rejected():
    g = graphgen.diamond()
    cases = []
    c = g.col.copy(); c[0] = c[1]; cases.append((g.row_ptr, c, g.sign))
    s = g.sign.copy(); s[0] = -s[0]; cases.append((g.row_ptr, g.col, s))
    s = g.sign.copy(); s[0] = 0; cases.append((g.row_ptr, g.col, s))
    c = g.col.copy(); c[0] = 0; cases.append((g.row_ptr, c, g.sign))
    c = g.col.copy(); c[0] = 77; cases.append((g.row_ptr, c, g.sign))
    rp = g.row_ptr.copy(); rp[1], rp[2] = rp[2], rp[1]; cases.append((rp, g.col, g.sign))
    for rp, c, s in cases:
        with pytest.raises(graphb.GraphBError) as ei:
            graphb.load_csr(rp, c, s)
        assert ei.value.rc == graphb.GB_EINVAL


def test_sharded_ranges_sum_to_full():
    """L248: disjoint tree subsets add up (simulated sharding on one GPU)."""
    import torch
    g = graphgen.chung_lu(8000, 40000, 900, 0.75, 0.2, 5)
    graphb.load_graph(g)
    T = 24
    full_c, full_a = graphb.balance_host(T, 3)
    for W in (2, 3, 8):
        cnt = torch.zeros(g.m, dtype=torch.int32, device="cuda")
        agr = torch.zeros(g.n, dtype=torch.int32, device="cuda")
        for r in range(W):
            graphb.balance_range(r, T, W, 3, cnt, agr)
        torch.cuda.synchronize()
        assert np.array_equal(cnt.cpu().numpy().astype(np.uint32), full_c)
        assert np.array_equal(agr.cpu().numpy().astype(np.uint32), full_a)


def test_deterministic_repeat():
    g = graphgen.chung_lu(10000, 50000, 1500, 0.75, 0.3, 8)
    graphb.load_graph(g)
    a = graphb.balance_host(20, 9)
    b = graphb.balance_host(20, 9)
    assert np.array_equal(a[0], b[0]) and np.array_equal(a[1], b[1])


# ---------------------------------------------------------------------------
# BASELINE config sizes (the launch configuration bench.py times)
# ---------------------------------------------------------------------------

def test_c2_slashdot_full_cloud():
    g, T, _ = graphgen.config("c2")
    check_cloud(g, T, 1)


def test_c4_epinions_tree_subset():
    """C4 at full size: a strided subset of the 1000 trees, bit-exact."""
    import torch
    g, T, _ = graphgen.config("c4")
    graphb.load_graph(g)
    cnt = torch.zeros(g.m, dtype=torch.int32, device="cuda")
    agr = torch.zeros(g.n, dtype=torch.int32, device="cuda")
    graphb.balance_range(3, T, 97, 1, cnt, agr)      # trees 3, 100, 197, ...
    torch.cuda.synchronize()
    oc, oa = oracle.Graph.from_csr(g).balance(T, 1, t_begin=3, stride=97)
    assert np.array_equal(cnt.cpu().numpy().astype(np.uint32), oc)
    assert np.array_equal(agr.cpu().numpy().astype(np.uint32), oa)


@pytest.mark.slow
def test_c3_amazon_sampled_trees():
    """C3 (10M / 22M) at full size in bench's launch configuration (one step:
    100 trees in one 128-wide MS-BFS pass, four trees per labelling launch):
    per-tree statistics of all trees against invariants, and four sampled
    trees (first / last of each batch) bit-exact against the oracle -- cycle
    lengths, depth and the signature of the switched edge set."""
    g, T, _ = graphgen.config("c3")
    assert T == 100
    graphb.load_graph(g)
    cnt, agree = graphb.balance_host(T, 1)      # bench's step: one batch of 100 trees
    st = graphb.stats()
    assert st["batch"] == 100 and st["batches"] == 1 and st["sub"] == 4
    ids, per = graphb.tree_stats()
    og = oracle.Graph.from_csr(g)
    c = og.ncomp
    assert np.all(per[:, 1] == g.m - g.n + c)                  # L112
    assert np.all(agree <= 2 * T) and cnt.max() <= T
    # sampled trees of both 64-tree halves of the pass (first / last of
    # each): cycle lengths, depth and the signature of the switched edge set
    for t in (0, 63, 64, 99):
        parent, dist, _ = og.bfs_tree(1, t)
        flip, sk, nc, md = og.balance_tree(parent)
        assert per[t, 0] == sk and per[t, 2] == md
        assert per[t, 3] == oracle.state_signature(flip)
    d = graphb.tree_debug(5, 1)
    parent, _, _ = og.bfs_tree(1, 5)
    assert np.array_equal(d["parent"], parent)
    assert np.array_equal(d["flip"], og.balance_tree(parent)[0])


@pytest.mark.slow
def test_c3_amazon_cloud_subset_bit_exact():
    """C3 (10M / 22M) at full size: a strided subset of the bench step's 100
    trees (3, 27, 51, 75, 99) through gb_balance_range into device counters;
    every edge flip count and every vertex agree count equals the oracle's
    (Alg. 1 L96-L108 on the same trees, the L224 Harary procedure)."""
    import torch
    g, T, _ = graphgen.config("c3")
    graphb.load_graph(g)
    cnt = torch.zeros(g.m, dtype=torch.int32, device="cuda")
    agr = torch.zeros(g.n, dtype=torch.int32, device="cuda")
    graphb.balance_range(3, T, 24, 1, cnt, agr)
    torch.cuda.synchronize()
    st = graphb.stats()
    assert st["trees"] == 5
    oc, oa, ost = oracle.Graph.from_csr(g).balance(T, 1, t_begin=3, stride=24, with_stats=True)
    assert np.array_equal(cnt.cpu().numpy().astype(np.uint32), oc)
    assert np.array_equal(agr.cpu().numpy().astype(np.uint32), oa)
    ids, per = graphb.tree_stats()
    assert list(ids) == [3, 27, 51, 75, 99]
    assert np.array_equal(per, ost)        # sum k, cycles, depth, state signature


def test_rmat20_full_cloud_bit_exact():
    """Graph500 R-MAT scale 20 (the C5 recipe at 1/64 of the size): the whole
    frustration cloud of 8 trees, every counter, against the oracle."""
    g = graphgen.rmat(20, 16, 0.5, 3, name="rmat20")
    check_cloud(g, 8, 2)


@pytest.mark.parametrize("which", ["er", "forest", "c2"])
def test_ingest_edge_ids_and_components(which):
    """§8 a.1: edge table by eid (rank of (min,max)), eid of every slot, and
    component ranks (by minimum vertex) equal the oracle's plain definitions."""
    g = {"er": lambda: graphgen.er(3000, 9000, 0.3, 1),
         "forest": lambda: graphgen.er(5000, 3000, 0.4, 2),
         "c2": lambda: graphgen.config("c2")[0]}[which]()
    graphb.load_graph(g)
    eu, ev, en, se, comp = graphb.graph_debug()
    og = oracle.Graph.from_csr(g)
    ou, ov, on = og.edges()
    oc, _, _ = og.components()
    assert np.array_equal(eu, ou) and np.array_equal(ev, ov) and np.array_equal(en, on)
    rows = np.repeat(np.arange(g.n), np.diff(g.row_ptr))
    key = np.minimum(rows, g.col).astype(np.int64) * g.n + np.maximum(rows, g.col)
    okey = ou.astype(np.int64) * g.n + ov
    assert np.array_equal(se, np.searchsorted(okey, key))
    assert np.array_equal(comp, oc)
    assert graphb.graph_info()[2] == og.ncomp


def _climb_checks(g, d, sample_edges, rng):
    """Closed-form checks of sampled edges of one tree (any size): tree edges
    never flip; a non-tree edge flips iff pi(u) ^ pi(v) ^ neg(e) with pi the
    XOR of negative bits on the root path (L214); the cycle length is
    d(u) + d(v) - 2 d(lca) + 1 (L230)."""
    parent, dist, flip = d["parent"], d["dist"], d["flip"]
    rows = np.searchsorted(g.row_ptr, sample_edges, side="right") - 1
    u = rows.astype(np.int64)
    v = g.col[sample_edges].astype(np.int64)
    neg = (g.sign[sample_edges] < 0).astype(np.int64)
    keep = u < v
    u, v, neg, slots = u[keep], v[keep], neg[keep], sample_edges[keep]
    # eid of each sampled slot (a.1 ingest, itself checked against the oracle
    # on smaller graphs by test_ingest_edge_ids_and_components)
    eid = graphb.graph_debug(edges=False, comp=False)[3][slots].astype(np.int64)

    def neg_of_parent_edge(x):
        p = parent[x]
        out = np.zeros(len(x), np.int64)
        ok = p >= 0
        xs, ps = x[ok], p[ok].astype(np.int64)
        # sign of edge (x, p): search p in row x
        pos = np.array([g.row_ptr[a] + np.searchsorted(g.col[g.row_ptr[a]:g.row_ptr[a + 1]], b)
                        for a, b in zip(xs, ps)], np.int64)
        out[ok] = (g.sign[pos] < 0)
        return out
    tree = (parent[v] == u) | (parent[u] == v)
    assert np.all(flip[eid[tree]] == 0)
    a, b = u[~tree].copy(), v[~tree].copy()
    ne = neg[~tree]
    c = np.zeros(len(a), np.int64)
    k = np.ones(len(a), np.int64)
    da, db = dist[a].astype(np.int64), dist[b].astype(np.int64)
    while True:
        live = a != b
        if not live.any():
            break
        mova = live & (da >= db)
        movb = live & ~mova
        c[mova] ^= neg_of_parent_edge(a[mova]); a[mova] = parent[a[mova]]; da[mova] -= 1
        c[movb] ^= neg_of_parent_edge(b[movb]); b[movb] = parent[b[movb]]; db[movb] -= 1
        k[live] += 1
    assert np.array_equal(flip[eid[~tree]], (c ^ ne).astype(np.uint8))
    return int((~tree).sum()), k


def _c5_golden():
    rows = {"trees": []}
    with open(os.path.join(os.path.dirname(__file__), "golden", "c5_rmat26_trees.txt")) as f:
        for line in f:
            w = line.split()
            if not w or w[0].startswith("#"):
                continue
            if w[0] == "graph":
                rows["graph"] = (int(w[1]), int(w[2]), w[3], w[4])
            elif w[0] == "tree":
                rows["trees"].append((int(w[1]), int(w[2]), int(w[3]), int(w[4]), int(w[5], 16), w[6], w[7]))
    return rows


@pytest.mark.slow
def test_c5_rmat26_capacity_and_sampled_cycles():
    """C5 (RMAT scale 26, ~1 B generated edges) on one B200: loads, balances
    whole trees, per-tree cycle count m - n + c (L112), counters bounded, and
    sampled edges of one tree against the closed forms."""
    g, T, _ = graphgen.config("c5")
    graphb.load_graph(g)
    n, m, c = graphb.graph_info()
    assert (n, m) == (g.n, g.m)
    cnt, agree = graphb.balance_host(2, 1)
    ids, per = graphb.tree_stats()
    assert np.all(per[:, 1] == m - n + c)
    assert cnt.max() <= 2 and agree.max() <= 4
    d = graphb.tree_debug(0, 1)
    assert per[0, 0] == d["sum_cycle_len"]
    rng = np.random.default_rng(5)
    deg = np.diff(g.row_ptr)
    # the parent rule on sampled low-degree vertices (oracle's pscore)
    cand_v = rng.integers(0, g.n, 4000)
    for w in cand_v[(deg[cand_v] > 0) & (deg[cand_v] < 200)][:300]:
        w = int(w)
        if d["parent"][w] < 0:
            continue
        nb = g.col[g.row_ptr[w]:g.row_ptr[w + 1]]
        cands = [int(x) for x in nb if d["dist"][x] == d["dist"][w] - 1]
        best = min(cands, key=lambda x: (oracle.pscore(1, 0, x, w), x))
        assert d["parent"][w] == best
    nonc, _ = _climb_checks(g, d, rng.integers(0, len(g.col), 20000), rng)
    assert nonc > 1000
    # whole trees bit-exact against the oracle: tests/golden/c5_rmat26_trees.txt
    # holds the oracle's one-tree counters (sha256) and statistics, written by
    # tools/make_c5_golden.py (graphgen + oracle/ only); its graph line pins
    # the generated input
    import hashlib
    import torch
    gold = _c5_golden()
    sha = lambda a: hashlib.sha256(np.ascontiguousarray(a).tobytes()).hexdigest()
    assert gold["graph"] == (g.n, g.m, sha(g.col.astype("<i4")), sha(g.sign.astype("i1")))
    assert len(gold["trees"]) >= 2
    cnt_d = torch.zeros(m, dtype=torch.int32, device="cuda")
    agr_d = torch.zeros(n, dtype=torch.int32, device="cuda")
    for t, sk, nc, dep, sig, hc, ha in gold["trees"]:
        cnt_d.zero_()
        agr_d.zero_()
        graphb.balance_range(t, t + 1, 1, 1, cnt_d, agr_d)
        torch.cuda.synchronize()
        _, per1 = graphb.tree_stats()
        assert tuple(int(x) for x in per1[0]) == (sk, nc, dep, sig)
        assert sha(cnt_d.cpu().numpy().astype("<u4")) == hc
        assert sha(agr_d.cpu().numpy().astype("<u4")) == ha


def _sweep_case(i):
    """Case i of the randomized sweep: a seeded graph family and size, a tree
    count that straddles the 64- and 128-tree MS-BFS widths, and random
    batching / walk options (none of them may change a result)."""
    rng = np.random.default_rng(1000 + i)
    kind = ["er", "chung_lu", "bipartite", "forest", "grid", "rmat"][i % 6]
    n = int(rng.integers(40, 2500))
    if kind == "er":
        g = graphgen.er(n, int(n * rng.uniform(1.2, 4.0)), float(rng.uniform(0.0, 0.6)), 50 + i)
    elif kind == "chung_lu":
        g = graphgen.chung_lu(n, int(n * rng.uniform(2.0, 6.0)), max(8, n // 5), 2.2, float(rng.uniform(0.1, 0.5)),
                              50 + i, lcc=bool(i % 2))
    elif kind == "bipartite":
        nu = n // 2
        g = graphgen.bipartite_chung_lu(nu, n - nu, int(n * 2.2), 16, max(8, n // 6), 2.5, 2.1, 0.5, 50 + i)
    elif kind == "forest":
        g = graphgen.er(n, int(n * rng.uniform(0.3, 0.9)), 0.4, 50 + i)
    elif kind == "grid":
        g = graphgen.grid2d(int(rng.integers(3, 30)), int(rng.integers(3, 30)), float(rng.uniform(0, 0.5)), 50 + i)
    else:
        g = graphgen.rmat(int(rng.integers(7, 11)), 8, 0.3, 50 + i)
    T = int(rng.choice([1, 2, 31, 63, 64, 65, 100, 127, 128, 129, 140]))
    opts = {"walk": int(rng.choice([0, 0, 3, 1, 2])), "push_parent": int(rng.integers(0, 2)),
            "batch": int(rng.choice([0, 0, 1, 7, 64, 65, 128])),
            "cycle_group": int(rng.choice([0, 1, 3])),
            "sub": int(rng.choice([0, 1, 3]))}
    return g, T, int(rng.integers(1, 1 << 30)), opts


@pytest.mark.parametrize("i", range(48))
def test_randomized_sweep_bit_exact(i):
    """48 seeded (graph, trees, seed, options) cases against the oracle: flip
    counts, agree counts and every per-tree statistic bit for bit."""
    g, T, seed, opts = _sweep_case(i)
    check_cloud(g, T, seed, **opts)
