timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -2
run() { timeout 600 python bench.py --config $CFG --no-cpu-baseline --no-e2e --steps 2 --warmup 3 "$@" 2>&1 | tail -1 | python -c "
import json,sys; d=json.loads(sys.stdin.read()); print('$LBL $CFG $*', round(d['value']/1e9,4), round(d['ms_per_step'],1), {k:round(v,1) for k,v in d['phase_ms_per_step'].items()}, d['config']['max_depth'], d['config']['avg_cycle_len'])" ; }
CFG=c2 run --opt sampler=2 --trees 20
python -c "
import sys,time; sys.path.insert(0,'.')
import graphgen, oracle
for c in ['c2']:
    g,_,_=graphgen.config(c); og=oracle.Graph.from_csr(g); t=time.time(); og.balance(1,1,sampler=2); print(c,'oracle dfs s/tree',(time.time()-t))
"
