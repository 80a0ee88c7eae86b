timeout 900 python -m pytest tests -m gpu -x -q -k "walk or stages or samplers or c3" > gpurun_out/pytest_w3.log 2>&1; echo pytest $?
tail -5 gpurun_out/pytest_w3.log
for c in c3 c4 c2; do for w in 0 3; do timeout 300 python bench.py --config $c --walk $w --no-cpu-baseline --no-e2e > gpurun_out/bench_${c}_w$w.log 2>&1; python -c "
import json; d=json.loads(open('gpurun_out/bench_${c}_w$w.log').read().strip().splitlines()[-1]); print('$c w$w', round(d['value']/1e9,2), round(d['ms_per_step'],2), {k:round(v,2) for k,v in d['phase_ms_per_step'].items()}, d['roofline']['frac'])"; done; done
