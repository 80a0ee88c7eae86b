timeout 600 ncu --set full --clock-control none --import-source on -k regex:'k_bottom_up|k_top_down|k_cycles_irec' -s 6 -c 3 -o gpurun_out/full_lab_r2 -f python tools/prof_run.py c3 8 > gpurun_out/ncu_full_lab.log 2>&1; echo ncufull $?
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_c3.csv python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/ncu_launch.log 2>&1; echo ncu $?
free -g | head -2; nproc
