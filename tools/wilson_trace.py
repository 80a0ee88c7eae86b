import sys, time; sys.path.insert(0, ".")
import graphgen, oracle
from paper_conf_sc_alabanditrb21_b200 import graphb
g,_,_ = graphgen.config("c2")
graphb.set_option("sampler", 1); graphb.load_graph(g)
t0=time.time(); d = graphb.tree_debug(0, 1); print("gpu tree", time.time()-t0, flush=True)
og = oracle.Graph.from_csr(g)
t0=time.time(); p,pops = og.wilson_tree(1, 0); print("oracle tree", time.time()-t0, "max pops", pops.max(), "sum pops", pops.sum(), flush=True)
