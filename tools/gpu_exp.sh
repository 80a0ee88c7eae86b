timeout 900 python -m pytest tests/test_gpu_parity.py -x -q 2>&1 | tail -1
run() { timeout 300 python bench.py --config $CFG --no-cpu-baseline --no-e2e --steps 3 "$@" 2>&1 | tail -1 | python -c "
import json,sys; d=json.loads(sys.stdin.read()); print('$LBL $CFG', round(d['value']/1e9,3), round(d['ms_per_step'],1), {k:round(v,1) for k,v in d['phase_ms_per_step'].items()})" ; }
for CFG in c3 c4 c2; do run; done
python tools/msprof.py c3 64 | tail -18
