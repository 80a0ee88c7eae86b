run() { timeout 300 python bench.py --config c3 --no-cpu-baseline --no-e2e --steps 3 "$@" 2>&1 | tail -1 | python -c "
import json,sys; d=json.loads(sys.stdin.read()); print('$*', round(d['value']/1e9,3), round(d['ms_per_step'],1), {k:round(v,1) for k,v in d['phase_ms_per_step'].items()})" ; }
run --opt cycle_group=2
run --walk 1
