timeout 600 python -m pytest tests/test_dist_gpu.py -x -q > gpurun_out/pytest_dist.log 2>&1; echo pytest_dist $?
tail -5 gpurun_out/pytest_dist.log
timeout 300 python bench.py --no-cpu-baseline --steps 5 > gpurun_out/b.log 2>&1; echo bench $?
tail -1 gpurun_out/b.log | cut -c1-1500
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_msbfs -c 1 -o gpurun_out/full_k_msbfs_r2a -f python tools/prof_run.py c3 64 > gpurun_out/ncu_full.log 2>&1; echo ncufull $?
tail -3 gpurun_out/ncu_full.log
