"""Profiling driver: load a config, warm up, then one balance call (the one
to capture).  Usage: python tools/prof_run.py CONFIG TREES [BATCH] [WALK]"""
import sys, time
sys.path.insert(0, ".")
import torch
import graphgen
from paper_conf_sc_alabanditrb21_b200 import graphb

cfg = sys.argv[1]
T = int(sys.argv[2])
batch = int(sys.argv[3]) if len(sys.argv) > 3 else 0
walk = int(sys.argv[4]) if len(sys.argv) > 4 else 0
g, _, _ = graphgen.config(cfg)
graphb.set_option("batch", batch)
graphb.set_option("walk", walk)
graphb.load_graph(g)
n, m, c = graphb.graph_info()
cnt = torch.zeros(m, dtype=torch.int32, device="cuda")
agr = torch.zeros(n, dtype=torch.int32, device="cuda")
graphb.balance_range(0, T, 1, 7, cnt, agr)      # warm-up (same shape)
torch.cuda.synchronize()
graphb.set_option("timing", 1)
t0 = time.time()
graphb.balance_range(0, T, 1, 1, cnt, agr)      # the profiled call
torch.cuda.synchronize()
st = graphb.stats()
print("trees", T, "batch", st["batch"], "phase_ms", {k: round(v, 3) for k, v in st["phase_ms"].items()},
      "wall_ms", round(1000 * (time.time() - t0), 2), flush=True)
