run() { tag=$1; shift; timeout 300 python bench.py --no-cpu-baseline --no-e2e "$@" > gpurun_out/bench_$tag.log 2>&1; python -c "
import json; d=json.loads(open('gpurun_out/bench_$tag.log').read().strip().splitlines()[-1]); print('$tag', round(d['value']/1e9,3), round(d['ms_per_step'],3), {k:round(v,3) for k,v in d['phase_ms_per_step'].items()})" || tail -3 gpurun_out/bench_$tag.log; }
for gsz in 0 444 296 148 74; do
 if [ $gsz = 0 ]; then unset GB_MS_GRID; else export GB_MS_GRID=$gsz; fi
 run c1_g$gsz --config c1 --steps 400
 run c2_g$gsz --config c2 --steps 100
 run c4_g$gsz --config c4 --steps 10
done
unset GB_MS_GRID
