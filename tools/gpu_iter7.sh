python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1; echo smoke $?; tail -1 gpurun_out/smoke.log
timeout 300 python tools/dbg_small.py 2>&1 | tail -4
timeout 1500 python -m pytest tests -m gpu -x -q -k "not c5" > gpurun_out/pytest_gpu.log 2>&1; echo pytest $?
tail -3 gpurun_out/pytest_gpu.log
timeout 600 python bench.py > gpurun_out/b3.json 2> gpurun_out/b3.err; echo c3 $?
timeout 600 python bench.py --config c4 --steps 40 --no-cpu-baseline > gpurun_out/b4.json 2> gpurun_out/b4.err; echo c4 $?
timeout 900 python bench.py --config c5 --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/b5.json 2> gpurun_out/b5.err; echo c5 $?
for f in b3 b4 b5; do python -c "
import json; d=json.loads(open('gpurun_out/$f.json').read().strip().splitlines()[-1])
print('$f', round(d['value']/1e9,3), round(d['ms_per_step'],2), {k:round(v,2) for k,v in d['phase_ms_per_step'].items()}, 'e2e', round(d['e2e']['value']/1e9,3), d['roofline']['kernel_name'], round(d['roofline']['frac'],3), round(d['roofline']['path_frac'],3))"; done
