timeout 900 python -m pytest tests -m gpu -x -q -k "randomized or stages or c3 or c4 or forest or distinct or given or degenerate or samplers" > gpurun_out/pytest_exp.log 2>&1; echo pytest $?
tail -1 gpurun_out/pytest_exp.log
run() { tag=$1; shift; timeout 300 python bench.py --no-cpu-baseline --no-e2e "$@" > gpurun_out/bench_$tag.log 2>&1; python -c "
import json; d=json.loads(open('gpurun_out/bench_$tag.log').read().strip().splitlines()[-1]); print('$tag', round(d['value']/1e9,2), round(d['ms_per_step'],2), {k:round(v,2) for k,v in d['phase_ms_per_step'].items()}, round(d['roofline']['frac'],3))" || tail -3 gpurun_out/bench_$tag.log; }
for c in c3 c4 c2; do run ${c}_$TAG --config $c; done
run c5_$TAG --config c5 --steps 2
