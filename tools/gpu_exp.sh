timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -2
run() { timeout 600 python bench.py --config $CFG --no-cpu-baseline --no-e2e --steps 2 --warmup 3 "$@" 2>&1 | tail -1 | python -c "
import json,sys; d=json.loads(sys.stdin.read()); print('$LBL $CFG $*', round(d['value']/1e9,4), round(d['ms_per_step'],1), {k:round(v,1) for k,v in d['phase_ms_per_step'].items()}, d['config']['max_depth'], d['config']['avg_cycle_len'])" ; }
CFG=c2 run --opt sampler=1 --trees 100
CFG=c4 run --opt sampler=1 --trees 100
python -c "
import sys,time; sys.path.insert(0,'.')
import graphgen, oracle
for c in ['c2','c4']:
    g,_,_=graphgen.config(c); og=oracle.Graph.from_csr(g); t=time.time(); og.balance(2,1,sampler=1); print(c,'oracle uniform s/tree',(time.time()-t)/2)
"
