python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
GB_E2E_TRACE=1 timeout 300 python bench.py --config c2 --steps 5 --no-cpu-baseline > gpurun_out/e2e_c2.log 2>&1
grep "e2e step" gpurun_out/e2e_c2.log
GB_E2E_TRACE=1 timeout 300 python bench.py --config c3 --steps 3 --no-cpu-baseline > gpurun_out/e2e_c3.log 2>&1
grep "e2e step" gpurun_out/e2e_c3.log
timeout 300 python - <<'PY'
import time, sys
sys.path.insert(0, '.')
import numpy as np, graphgen
from paper_conf_sc_alabanditrb21_b200 import graphb
g,_,_ = graphgen.config('c2')
for i in range(4):
    t0=time.perf_counter(); graphb.load_graph(g); t1=time.perf_counter()
    c,a = graphb.balance_host(100, 7); t2=time.perf_counter()
    print(f"load {1e3*(t1-t0):.1f} ms balance_host {1e3*(t2-t1):.1f} ms")
PY
