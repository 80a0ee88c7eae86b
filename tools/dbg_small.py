import sys
sys.path.insert(0, ".")
import numpy as np
import graphgen, oracle
from paper_conf_sc_alabanditrb21_b200 import graphb
for name, g, T in [("er", graphgen.er(2000, 8000, 0.3, 1), 8),
                   ("cl", graphgen.chung_lu(6000, 30000, 1500, 0.75, 0.3, 21, lcc=False), 20),
                   ("cl100", graphgen.chung_lu(6000, 30000, 1500, 0.75, 0.3, 21, lcc=False), 100)]:
    graphb.load_graph(g)
    try:
        c, a = graphb.balance_host(T, 3)
    except Exception as e:
        print(name, "ERR", e, flush=True)
        raise
    oc, oa = oracle.Graph.from_csr(g).balance(T, 3)
    print(name, np.array_equal(c, oc), np.array_equal(a, oa), flush=True)
