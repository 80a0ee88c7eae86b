# round-2 final measurements: GPU suite, smoke, bench lines (driver-style), launch list, ncu full captures
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
mkdir -p gpurun_out/fin
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/fin/pytest_gpu.log 2>&1; echo pytest $?; tail -2 gpurun_out/fin/pytest_gpu.log
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/fin/smoke.log 2>&1; echo smoke $?
timeout 900 python bench.py > gpurun_out/fin/bench_c3.json 2> gpurun_out/fin/bench_c3.err; echo c3 $?
timeout 600 python bench.py --config c4 --steps 40 > gpurun_out/fin/bench_c4.json 2> gpurun_out/fin/bench_c4.err; echo c4 $?
timeout 600 python bench.py --config c2 --steps 400 > gpurun_out/fin/bench_c2.json 2> gpurun_out/fin/bench_c2.err; echo c2 $?
timeout 600 python bench.py --config c1 --steps 4000 > gpurun_out/fin/bench_c1.json 2> gpurun_out/fin/bench_c1.err; echo c1 $?
timeout 900 python bench.py --config c5 --steps 3 --warmup 3 > gpurun_out/fin/bench_c5.json 2> gpurun_out/fin/bench_c5.err; echo c5 $?
timeout 900 python bench.py --impl reference --steps 2 --warmup 3 > gpurun_out/fin/ref_c3.json 2> gpurun_out/fin/ref_c3.err; echo ref $?
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/fin/launches_c3.csv python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/fin/ncu_launch.log 2>&1; echo ncu $?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_msbfs -c 1 -o gpurun_out/fin/full_k_msbfs -f python tools/prof_run.py c3 100 > gpurun_out/fin/ncu_full_msbfs.log 2>&1; echo ncufull $?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:'k_bottom_up|k_top_down|k_cycles_irec' -c 3 -o gpurun_out/fin/full_rest -f python tools/prof_run.py c3 4 > gpurun_out/fin/ncu_full_rest.log 2>&1; echo ncufull2 $?
