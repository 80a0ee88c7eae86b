python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 300 python tools/lprof.py c3 4 > gpurun_out/lprof_c3.log 2>&1; cat gpurun_out/lprof_c3.log
timeout 300 python tools/lprof.py c3 4 sub=1 > gpurun_out/lprof_c3s1.log 2>&1; tail -20 gpurun_out/lprof_c3s1.log
