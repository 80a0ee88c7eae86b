timeout 900 python -m pytest tests -m gpu -x -q -k "walk or stages or samplers or c3 or c4 or c5 or forest" > gpurun_out/pytest_lca.log 2>&1; echo pytest $?
tail -3 gpurun_out/pytest_lca.log
run() { tag=$1; shift; timeout 300 python bench.py --no-cpu-baseline --no-e2e "$@" > gpurun_out/bench_$tag.log 2>&1; python -c "
import json; d=json.loads(open('gpurun_out/bench_$tag.log').read().strip().splitlines()[-1]); print('$tag', round(d['value']/1e9,2), round(d['ms_per_step'],2), {k:round(v,2) for k,v in d['phase_ms_per_step'].items()}, round(d['roofline']['frac'],3))" || tail -3 gpurun_out/bench_$tag.log; }
for c in c3 c4 c2; do
run ${c}_m8 --config $c
GRAPHB_LIB=$PWD/paper_conf_sc_alabanditrb21_b200/libgraphb_w6.so run ${c}_m6 --config $c
done
