run() { tag=$1; shift; timeout 300 python bench.py --no-cpu-baseline --no-e2e "$@" > gpurun_out/bench_$tag.log 2>&1; python -c "
import json; d=json.loads(open('gpurun_out/bench_$tag.log').read().strip().splitlines()[-1]); print('$tag', round(d['value']/1e9,2), round(d['ms_per_step'],2), {k:round(v,2) for k,v in d['phase_ms_per_step'].items()})" || tail -3 gpurun_out/bench_$tag.log; }
for c in c3 c4; do
run ${c}_base --config $c
GRAPHB_LIB=$PWD/paper_conf_sc_alabanditrb21_b200/libgraphb_m5.so run ${c}_m5 --config $c
GRAPHB_LIB=$PWD/paper_conf_sc_alabanditrb21_b200/libgraphb_c256.so run ${c}_c256 --config $c
done
