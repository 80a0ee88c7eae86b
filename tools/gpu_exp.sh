timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -3
run() { timeout 300 python bench.py --config $CFG --no-cpu-baseline --no-e2e --steps 3 "$@" 2>&1 | tail -1 | python -c "
import json,sys; d=json.loads(sys.stdin.read()); print('$LBL $CFG $*', round(d['value']/1e9,3), round(d['ms_per_step'],1), {k:round(v,1) for k,v in d['phase_ms_per_step'].items()})" ; }
CFG=c2 run --opt harary=1
CFG=c2 run
