for k in k_rec_scatter k_top_down k_bottom_up; do
timeout 600 ncu --set full --clock-control none --import-source on -k regex:$k -s 3 -c 1 -o gpurun_out/s1_$k python tools/prof_run.py c3 8 > gpurun_out/ncu_s1_$k.log 2>&1; echo $k $?
done
