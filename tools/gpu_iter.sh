# one build-measure iteration: GPU parity, then bench lines (phase split)
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1; echo smoke $?; tail -1 gpurun_out/smoke.log
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo pytest $?
tail -4 gpurun_out/pytest_gpu.log
for spec in "c3" "c4 --steps 20" "c2 --steps 50" ${EXTRA}; do
  timeout 300 python bench.py --no-cpu-baseline --no-e2e --config $spec > gpurun_out/b.log 2>&1
  python -c "
import json,sys; d=json.loads(open('gpurun_out/b.log').read().strip().splitlines()[-1]); print('$spec', round(d['value']/1e9,3), round(d['ms_per_step'],2), {k:round(v,2) for k,v in d['phase_ms_per_step'].items()})" || tail -5 gpurun_out/b.log
done
