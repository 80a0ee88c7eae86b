# round-2 final measurements: bench lines (driver-style), launch list, ncu full captures
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
mkdir -p gpurun_out/ck2
timeout 900 python bench.py > gpurun_out/ck2/bench_c3.json 2> gpurun_out/ck2/bench_c3.err; echo c3 $?
timeout 600 python bench.py --config c4 --steps 40 > gpurun_out/ck2/bench_c4.json 2> gpurun_out/ck2/bench_c4.err; echo c4 $?
timeout 600 python bench.py --config c2 --steps 400 > gpurun_out/ck2/bench_c2.json 2> gpurun_out/ck2/bench_c2.err; echo c2 $?
timeout 600 python bench.py --config c1 --steps 400 > gpurun_out/ck2/bench_c1.json 2> gpurun_out/ck2/bench_c1.err; echo c1 $?
timeout 900 python bench.py --config c5 --steps 3 --warmup 3 > gpurun_out/ck2/bench_c5.json 2> gpurun_out/ck2/bench_c5.err; echo c5 $?
timeout 900 python bench.py --impl reference --steps 2 --warmup 1 > gpurun_out/ck2/ref_c3.json 2> gpurun_out/ck2/ref_c3.err; echo ref $?
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/ck2/launches_c3.csv python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/ck2/ncu_launch.log 2>&1; echo ncu $?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_msbfs -c 1 -o gpurun_out/ck2/full_k_msbfs -f python tools/prof_run.py c3 100 > gpurun_out/ck2/ncu_full_msbfs.log 2>&1; echo ncufull $?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:'k_bottom_up|k_top_down|k_cycles_irec' -c 3 -o gpurun_out/ck2/full_rest -f python tools/prof_run.py c3 4 > gpurun_out/ck2/ncu_full_rest.log 2>&1; echo ncufull2 $?
