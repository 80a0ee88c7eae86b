timeout 900 python bench.py --config c5 --no-cpu-baseline --no-e2e --steps 2 --warmup 3 > gpurun_out/bench_c5.log 2>&1; echo c5 $?
tail -3 gpurun_out/bench_c5.log | cut -c1-300
timeout 600 python -m pytest tests -m gpu -x -q -k "c5 or rmat" > gpurun_out/pytest_c5.log 2>&1; echo pytest $?; tail -3 gpurun_out/pytest_c5.log
