#!/bin/bash
# build here, run tests + quick benches on the GPU box, summarise
cd /root/repo
python -c "from paper_conf_sc_alabanditrb21_b200 import _build; _build.build()" || exit 1
timeout 2400 /usr/local/graft/bin/gpurun --timeout ${T:-1500} -- "bash tools/gpu_quick.sh" 2>&1 | grep -v "^{" | tail -${TAILN:-4}
for c in c3 c2 c4; do python -c "
import json; d=json.loads(open('gpurun_out/bench_$c.log').read().strip().splitlines()[-1]); print('$c', round(d['value']/1e9,2), round(d['ms_per_step'],2), {k:round(v,2) for k,v in d['phase_ms_per_step'].items()}, d['config']['batch'], d['config']['max_depth'])" 2>/dev/null || tail -3 gpurun_out/bench_$c.log; done
