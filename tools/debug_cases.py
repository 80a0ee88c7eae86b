"""Ad-hoc GPU debugging: run named cases with progress output."""
import sys, time
import numpy as np
sys.path.insert(0, ".")
import graphgen, oracle
from paper_conf_sc_alabanditrb21_b200 import graphb

def run(name, g, T, seed=1, **opts):
    for k, v in opts.items():
        graphb.set_option(k, v)
    t0 = time.time()
    graphb.load_graph(g)
    cnt, agree = graphb.balance_host(T, seed)
    st = graphb.stats()
    dt = time.time() - t0
    oc, oa = oracle.Graph.from_csr(g).balance(T, seed)
    ok = np.array_equal(cnt, oc) and np.array_equal(agree, oa)
    print(f"{name}: ok={ok} {dt:.2f}s batch={st['batch']} group={st['cycle_group']} depth={st['max_depth']}", flush=True)
    for k in opts:
        graphb.set_option(k, 0)

cases = sys.argv[1:]
for c in cases:
    if c == "cl_b64":
        run(c, graphgen.chung_lu(5000, 20000, 500, 0.75, 0.3, 1), 64)
    if c == "cl_b64_g1":
        run(c, graphgen.chung_lu(5000, 20000, 500, 0.75, 0.3, 1), 64, cycle_group=1)
    if c == "cl_b32":
        run(c, graphgen.chung_lu(5000, 20000, 500, 0.75, 0.3, 1), 32)
    if c == "cl_b17":
        run(c, graphgen.chung_lu(5000, 20000, 500, 0.75, 0.3, 1), 17, batch=17)
    if c == "path200":
        run(c, graphgen.path(200), 3)
    if c == "path2000":
        run(c, graphgen.path(2000), 3)
    if c == "path20000":
        run(c, graphgen.path(20000), 1)
    if c == "c2":
        g, T, _ = graphgen.config("c2")
        run(c, g, T)
    if c == "path20000x3":
        run(c, graphgen.path(20000), 3)
    if c == "path8000":
        run(c, graphgen.path(8000), 3)
    if c == "disc":
        run(c, graphgen.er(5000, 3000, 0.4, 2), 9)
    if c == "disc1":
        run(c, graphgen.er(5000, 3000, 0.4, 2), 1)
    if c == "disc_s3":
        run(c, graphgen.er(5000, 3000, 0.4, 2), 9, seed=3)
    if c == "disc_dbg":
        g = graphgen.er(5000, 3000, 0.4, 2)
        graphb.load_graph(g)
        for t in range(3):
            d = graphb.tree_debug(t, 3)
            print("tree_debug", t, d["num_cycles"], flush=True)
    if c == "ingest":
        for gg in [graphgen.er(5000, 3000, 0.4, 2), graphgen.config("c2")[0], graphgen.er(100, 300, 0.3, 1)]:
            graphb.load_graph(gg)
            eu, ev, en, se, comp = graphb.graph_debug()
            og = oracle.Graph.from_csr(gg)
            ou, ov, on = og.edges()
            oc, _, _ = og.components()
            rows = np.repeat(np.arange(gg.n), np.diff(gg.row_ptr))
            a = np.minimum(rows, gg.col); b = np.maximum(rows, gg.col)
            key = a.astype(np.int64) * gg.n + b
            okey = ou.astype(np.int64) * gg.n + ov
            oslot = np.searchsorted(okey, key)
            print("ingest", gg.n, gg.m, "edges_u", np.array_equal(eu, ou), "edges_v", np.array_equal(ev, ov),
                  "neg", np.array_equal(en, on), "slot_eid", np.array_equal(se, oslot), "comp", np.array_equal(comp, oc),
                  "bad_e", int((eu != ou).sum()), "first_bad", int(np.flatnonzero(eu != ou)[0]) if (eu != ou).any() else -1, flush=True)
    if c == "cc":
        gg = graphgen.er(5000, 3000, 0.4, 2)
        graphb.load_graph(gg)
        eu, ev, en, se, comp = graphb.graph_debug()
        og = oracle.Graph.from_csr(gg)
        oc, coff, _ = og.components()
        bad = np.flatnonzero(comp != oc)
        print("ncomp gpu", comp.max() + 1, "oracle", oc.max() + 1, "nbad", len(bad))
        deg = np.diff(gg.row_ptr)
        for v in bad[:10]:
            print("v", v, "deg", deg[v], "gpu", comp[v], "oracle", oc[v])
        # first index where sorted-unique roots differ
        import collections
        print("gpu comp counts head", np.bincount(comp)[:10], "oracle", np.bincount(oc)[:10])
