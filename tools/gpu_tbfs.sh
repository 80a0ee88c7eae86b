# tree-parallel BFS: parity + timings against the multi-source BFS
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1; echo smoke $?
tail -2 gpurun_out/smoke.log
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo pytest $?
tail -15 gpurun_out/pytest_gpu.log
for o in "bfs=1" "bfs_group=1" "bfs_group=2" "bfs_group=4" "bfs_group=8" "bfs_group=4 --opt push_k=2" "bfs_group=4 --opt push_k=8" "bfs_group=4 --opt push_k=1024"; do
  timeout 300 python bench.py --no-cpu-baseline --no-e2e --steps 3 --opt $o > gpurun_out/b.log 2>&1
  python -c "
import json,sys; d=json.loads(open('gpurun_out/b.log').read().strip().splitlines()[-1]); print('$o', round(d['value']/1e9,3), round(d['ms_per_step'],2), {k:round(v,2) for k,v in d['phase_ms_per_step'].items()})" || tail -5 gpurun_out/b.log
done
timeout 300 python tools/msprof.py c3 4 > gpurun_out/msprof_tb.log 2>&1; cat gpurun_out/msprof_tb.log
