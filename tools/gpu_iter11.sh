python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "not c5 and not c3" > gpurun_out/pytest_gpu.log 2>&1; echo pytest $?
tail -2 gpurun_out/pytest_gpu.log
run() { timeout ${TO:-300} python bench.py --no-cpu-baseline --no-e2e $@ > gpurun_out/b.log 2>&1
  python -c "
import json,sys; d=json.loads(open('gpurun_out/b.log').read().strip().splitlines()[-1]); print('$*', round(d['value']/1e9,3), round(d['ms_per_step'],2), {k:round(v,2) for k,v in d['phase_ms_per_step'].items()})" || tail -3 gpurun_out/b.log; }
run --config c3
TO=900 run --config c5 --steps 3 --warmup 3
run --config c4 --steps 20
