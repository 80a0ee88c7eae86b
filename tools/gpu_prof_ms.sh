timeout 900 ncu --set full --clock-control none --import-source on -k regex:'k_msbfs' -s 1 -c 1 -o gpurun_out/prof_ms python tools/prof_run.py ${1:-c3} 64 > gpurun_out/ncu_ms.log 2>&1; echo ncu $?
tail -3 gpurun_out/ncu_ms.log
