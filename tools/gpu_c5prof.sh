python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 600 python tools/msprof.py c5 10 > gpurun_out/msprof_c5.log 2>&1; cat gpurun_out/msprof_c5.log | head -30
timeout 600 python -c "
import graphgen, numpy as np
g,_,_ = graphgen.config('c5')
deg = np.diff(g.row_ptr)
print('maxdeg', deg.max(), 'heavy>8', (deg>8).sum(), '>256', (deg>256).sum(), 'slots>256', deg[deg>256].sum(), 'iso', (deg==0).sum())
"
