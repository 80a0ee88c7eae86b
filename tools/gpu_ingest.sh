timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_ing.log 2>&1; echo pytest $?; tail -2 gpurun_out/pytest_ing.log
python tools/e2eprof.py
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_ing.csv python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > /dev/null 2>&1; echo ncu $?
timeout 600 python bench.py --no-cpu-baseline > gpurun_out/bench_ing_c3.log 2>&1; tail -1 gpurun_out/bench_ing_c3.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('c3', d['value']/1e9, d['e2e']['value']/1e9)"
timeout 900 python bench.py --config c5 --steps 2 --warmup 3 --no-cpu-baseline > gpurun_out/bench_ing_c5.log 2>&1; tail -1 gpurun_out/bench_ing_c5.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('c5', d['value']/1e9, d['e2e']['value']/1e9, d['config']['components'])"
