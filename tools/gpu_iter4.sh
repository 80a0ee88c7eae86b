python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
run() { timeout ${TO:-300} python bench.py --no-cpu-baseline --no-e2e $@ > gpurun_out/b.log 2>&1
  python -c "
import json,sys; d=json.loads(open('gpurun_out/b.log').read().strip().splitlines()[-1]); print('$*', round(d['value']/1e9,3), round(d['ms_per_step'],2), {k:round(v,2) for k,v in d['phase_ms_per_step'].items()}, d['config']['batch'])" || tail -3 gpurun_out/b.log; }
run --config c3
run --config c3 --sub 8
run --config c3 --sub 16
TO=900 run --config c5 --steps 3 --warmup 3
timeout 300 python tools/msprof.py c3 64 > gpurun_out/msprof_c3.log 2>&1; head -20 gpurun_out/msprof_c3.log
timeout 600 ncu --set full --clock-control none --import-source on -k regex:'k_bottom_up|k_top_down|k_cycles_irec' -c 3 -o gpurun_out/full_r2b -f python tools/prof_run.py c3 4 > gpurun_out/ncu_full.log 2>&1; echo ncufull $?
