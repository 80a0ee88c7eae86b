"""Per-level phase times of the multi-source BFS: python tools/msprof.py CONFIG [TREES]"""
import sys
sys.path.insert(0, ".")
import torch
import graphgen
from paper_conf_sc_alabanditrb21_b200 import graphb

cfg = sys.argv[1]
T = int(sys.argv[2]) if len(sys.argv) > 2 else 64
g, _, _ = graphgen.config(cfg)
graphb.load_graph(g)
n, m, c = graphb.graph_info()
cnt = torch.zeros(m, dtype=torch.int32, device="cuda")
agr = torch.zeros(n, dtype=torch.int32, device="cuda")
graphb.balance_range(0, T, 1, 7, cnt, agr)
torch.cuda.synchronize()
graphb.set_option("msprof", 1)
graphb.set_option("timing", 1)
graphb.balance_range(0, T, 1, 1, cnt, agr)
torch.cuda.synchronize()
st = graphb.stats()
print(cfg, "trees", T, "phase_ms", {k: round(v, 3) for k, v in st["phase_ms"].items()})
tot = [0.0, 0.0, 0.0]
for L, a, b, c3 in graphb.msbfs_profile():
    print(f"  L{L:3d}  A {a:7.3f}  B {b:7.3f}  C+sync {c3:7.3f}")
    tot[0] += a; tot[1] += b; tot[2] += c3
print("  sum   A %.3f  B %.3f  C %.3f ms" % tuple(tot))
