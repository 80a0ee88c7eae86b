"""Per-level Alg. 4 times of the last labelling launch:
python tools/lprof.py CONFIG [TREES] [key=value options...]"""
import sys
sys.path.insert(0, ".")
import torch
import graphgen
from paper_conf_sc_alabanditrb21_b200 import graphb

cfg = sys.argv[1]
T = int(sys.argv[2]) if len(sys.argv) > 2 else 64
for kv in sys.argv[3:]:
    k, v = kv.split("=")
    graphb.set_option(k, int(v))
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
print(cfg, "trees", T, sys.argv[3:], "phase_ms", {k: round(v, 3) for k, v in st["phase_ms"].items()})
sb = st_ = 0.0
for L, nv, bu, td in graphb.label_profile():
    print(f"  L{L:3d} {nv:9d}  up {1000 * bu:8.1f} us  down {1000 * td:8.1f} us")
    sb += bu; st_ += td
print(f"  sum up {1000 * sb:.1f} us  down {1000 * st_:.1f} us (last launch)")
