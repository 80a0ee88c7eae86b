python tools/msprof.py c3 100 > gpurun_out/msp_c3.log 2>&1
python tools/msprof.py c4 128 > gpurun_out/msp_c4.log 2>&1
timeout 600 python tools/msprof.py c5 10 > gpurun_out/msp_c5.log 2>&1
cat gpurun_out/msp_c3.log gpurun_out/msp_c4.log gpurun_out/msp_c5.log
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_msbfs -c 1 -o gpurun_out/full_k_msbfs -f python tools/prof_run.py c3 100 > gpurun_out/ncu_full_msbfs.log 2>&1; echo ncufull $?
