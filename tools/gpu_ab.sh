timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_ab.log 2>&1; echo pytest $?; tail -1 gpurun_out/pytest_ab.log
run() { tag=$1; shift; timeout 300 python bench.py --no-cpu-baseline --no-e2e "$@" > gpurun_out/bench_$tag.log 2>&1; python -c "
import json; d=json.loads(open('gpurun_out/bench_$tag.log').read().strip().splitlines()[-1]); print('$tag', round(d['value']/1e9,2), round(d['ms_per_step'],2), {k:round(v,2) for k,v in d['phase_ms_per_step'].items()})" || tail -3 gpurun_out/bench_$tag.log; }
for r in 1 2; do
run c4_new$r --config c4
GRAPHB_LIB=$PWD/paper_conf_sc_alabanditrb21_b200/libgraphb_prev.so run c4_prev$r --config c4
run c2_new$r --config c2
done
run c5_new --config c5 --steps 2
run c3_new
