set -x
nvidia-smi -L
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1; echo smoke $?
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo pytest $?
tail -3 gpurun_out/pytest_gpu.log
timeout 300 python bench.py --no-cpu-baseline > gpurun_out/bench_c3.log 2>&1; echo bench $?
tail -1 gpurun_out/bench_c3.log | cut -c1-900
timeout 300 python tools/msprof.py c3 64 > gpurun_out/msprof_c3.log 2>&1
timeout 300 python tools/lprof.py c3 1 > gpurun_out/lprof_c3.log 2>&1
cat gpurun_out/msprof_c3.log gpurun_out/lprof_c3.log
