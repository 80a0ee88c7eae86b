run() { timeout 300 python bench.py --config c3 --no-cpu-baseline --no-e2e --steps 3 "$@" 2>&1 | tail -1 | python -c "
import json,sys; d=json.loads(sys.stdin.read()); print('$LBL', round(d['value']/1e9,3), round(d['ms_per_step'],1), {k:round(v,1) for k,v in d['phase_ms_per_step'].items()})" ; }
LBL=ilp4 run
for v in v1 v2 v3; do LBL=$v GRAPHB_LIB=$PWD/paper_conf_sc_alabanditrb21_b200/libgraphb_$v.so run; done
