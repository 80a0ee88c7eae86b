timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo pytest $?
tail -30 gpurun_out/pytest_gpu.log
for c in c3 c2 c4; do timeout 300 python bench.py --config $c --no-cpu-baseline --no-e2e > gpurun_out/bench_$c.log 2>&1; tail -1 gpurun_out/bench_$c.log | cut -c1-600; done
for c in c3 c4; do timeout 300 python tools/msprof.py $c 64 | tail -1; done
