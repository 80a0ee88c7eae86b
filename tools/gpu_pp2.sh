timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_pp2.log 2>&1; echo pytest $?
tail -2 gpurun_out/pytest_pp2.log
run() { tag=$1; shift; timeout 300 python bench.py --no-cpu-baseline --no-e2e "$@" > gpurun_out/bench_$tag.log 2>&1; python -c "
import json; d=json.loads(open('gpurun_out/bench_$tag.log').read().strip().splitlines()[-1]); print('$tag', round(d['value']/1e9,2), round(d['ms_per_step'],2), {k:round(v,2) for k,v in d['phase_ms_per_step'].items()})" || tail -3 gpurun_out/bench_$tag.log; }
run c5_w --config c5 --steps 2
run c1_w --config c1 --steps 400
timeout 600 python tools/msprof.py c5 10 > gpurun_out/msp_c5w.log 2>&1; cat gpurun_out/msp_c5w.log
