run() { tag=$1; shift; timeout 300 python bench.py --no-cpu-baseline --no-e2e "$@" > gpurun_out/bench_$tag.log 2>&1; python -c "
import json; d=json.loads(open('gpurun_out/bench_$tag.log').read().strip().splitlines()[-1]); print('$tag', round(d['value']/1e9,2), round(d['ms_per_step'],2), {k:round(v,2) for k,v in d['phase_ms_per_step'].items()})" || tail -3 gpurun_out/bench_$tag.log; }
python -c "import torch; p=torch.cuda.get_device_properties(0); print('L2', p.L2_cache_size, 'persist max', getattr(p,'persisting_l2_cache_max_size',None))"
run wp0
for b in 16000000 32000000 64000000 96000000; do run wp$b --opt wpersist=$b; done
timeout 300 python bench.py --config c1 --steps 4000 > gpurun_out/bench_c1_long.json 2> gpurun_out/bench_c1_long.err; echo c1 $?
