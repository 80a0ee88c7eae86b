import sys, time
sys.path.insert(0, ".")
import numpy as np, torch, graphgen
from paper_conf_sc_alabanditrb21_b200 import graphb
g,_,_ = graphgen.config("c3")
pin = lambda a: torch.from_numpy(np.ascontiguousarray(a)).pin_memory().numpy()
hrp, hcol, hsg = pin(g.row_ptr), pin(g.col), pin(g.sign)
graphb.load_csr(hrp, hcol, hsg)
n, m, _ = graphb.graph_info()
cnt = torch.zeros(m, dtype=torch.int32, device="cuda"); agr = torch.zeros(n, dtype=torch.int32, device="cuda")
st = torch.cuda.current_stream()
graphb.balance_range(0, 100, 1, 1, cnt, agr, stream=st); torch.cuda.synchronize()
h_cnt = torch.empty(m, dtype=torch.int32).pin_memory(); h_agr = torch.empty(n, dtype=torch.int32).pin_memory()
for it in range(3):
    t0 = time.perf_counter(); graphb.load_csr(hrp, hcol, hsg); torch.cuda.synchronize(); t1 = time.perf_counter()
    cnt.zero_(); agr.zero_(); graphb.balance_range(0, 100, 1, 2 + it, cnt, agr, stream=st); torch.cuda.synchronize(); t2 = time.perf_counter()
    h_cnt.copy_(cnt); h_agr.copy_(agr); torch.cuda.synchronize(); t3 = time.perf_counter()
    print(f"load {t1-t0:.3f}s balance {t2-t1:.3f}s d2h {t3-t2:.3f}s", graphb.stats()["batch"], flush=True)
