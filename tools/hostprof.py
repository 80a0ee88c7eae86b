import sys, time
sys.path.insert(0, ".")
import torch, graphgen
from paper_conf_sc_alabanditrb21_b200 import graphb
g,_,_ = graphgen.config("c1")
graphb.load_graph(g)
n,m,_ = graphb.graph_info()
cnt = torch.zeros(m, dtype=torch.int32, device="cuda"); agr = torch.zeros(n, dtype=torch.int32, device="cuda")
for i in range(3): graphb.balance_range(0, 1, 1, 1, cnt, agr)
torch.cuda.synchronize()
import ctypes
L = graphb.lib()
t=time.perf_counter()
for i in range(50): graphb.balance_range(0, 1, 1, 1+i, cnt, agr)
torch.cuda.synchronize(); print("balance_range avg ms", (time.perf_counter()-t)/50*1e3)
t=time.perf_counter()
for i in range(50): L.gb_balance_range(0, 1, 1, 1+i, ctypes.c_void_p(cnt.data_ptr()), ctypes.c_void_p(agr.data_ptr()), None)
torch.cuda.synchronize(); print("raw gb_balance_range (own stream) avg ms", (time.perf_counter()-t)/50*1e3)
free = ctypes.c_size_t(); tot = ctypes.c_size_t()
cr = ctypes.CDLL("libcudart.so") if False else None
t=time.perf_counter()
for i in range(50): torch.cuda.mem_get_info()
print("cudaMemGetInfo avg ms", (time.perf_counter()-t)/50*1e3)
g3,_,_ = graphgen.config("c3")
for i in range(3):
    t=time.perf_counter(); graphb.load_graph(g3); torch.cuda.synchronize(); print("c3 load_csr s", time.perf_counter()-t)
