python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1; echo smoke $?; tail -1 gpurun_out/smoke.log
timeout 1200 python -m pytest tests -m gpu -x -q -k "not c5" > gpurun_out/pytest_gpu.log 2>&1; echo pytest $?
tail -3 gpurun_out/pytest_gpu.log
run() { timeout ${TO:-300} python bench.py --no-cpu-baseline --no-e2e $@ > gpurun_out/b.log 2>&1
  python -c "
import json,sys; d=json.loads(open('gpurun_out/b.log').read().strip().splitlines()[-1]); print('$*', round(d['value']/1e9,3), round(d['ms_per_step'],2), {k:round(v,2) for k,v in d['phase_ms_per_step'].items()})" || tail -3 gpurun_out/b.log; }
run --config c3
run --config c3 --sub 1
run --config c4 --steps 20
