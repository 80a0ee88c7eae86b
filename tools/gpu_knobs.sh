run() { tag=$1; shift; timeout 300 python bench.py --no-cpu-baseline --no-e2e "$@" > gpurun_out/bench_$tag.log 2>&1; python -c "
import json; d=json.loads(open('gpurun_out/bench_$tag.log').read().strip().splitlines()[-1]); print('$tag', round(d['value']/1e9,2), round(d['ms_per_step'],2), {k:round(v,2) for k,v in d['phase_ms_per_step'].items()})" || tail -3 gpurun_out/bench_$tag.log; }
run base
run cg2 --opt cycle_group=2
run cg4 --opt cycle_group=4
run sub2 --opt sub=2
run sub8 --opt sub=8
run c4base --config c4 
run c4cg8 --config c4 --opt cycle_group=8
run c4cg64 --config c4 --opt cycle_group=64
