set -x
nvidia-smi -L
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1; echo smoke $?
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo pytest $?
tail -3 gpurun_out/pytest_gpu.log
timeout 600 python bench.py > gpurun_out/bench_c3.log 2>&1; echo bench $?
tail -1 gpurun_out/bench_c3.log
for c in c2 c4; do timeout 300 python bench.py --config $c --no-cpu-baseline > gpurun_out/bench_$c.log 2>&1; tail -1 gpurun_out/bench_$c.log | cut -c1-400; done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_c3.csv python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/ncu_launch.log 2>&1; echo ncu $?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:'k_bfs|k_cycles|k_top_down|k_bottom_up' -c 4 -o gpurun_out/prof_c3 python tools/prof_run.py c3 2 2 > gpurun_out/ncu_full.log 2>&1; echo ncufull $?
