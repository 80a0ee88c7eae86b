python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1; echo smoke $?
timeout 900 python bench.py > gpurun_out/bench_c3_full.log 2>&1; echo bench $?
for c in c2 c4; do timeout 600 python bench.py --config $c > gpurun_out/bench_${c}_full.log 2>&1; echo bench $c $?; done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_c3.csv python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/ncu_launch.log 2>&1; echo ncu $?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_msbfs -c 1 -o gpurun_out/full_k_msbfs python tools/prof_run.py c3 64 > gpurun_out/ncu_full_k_msbfs.log 2>&1; echo ncufull msbfs $?
