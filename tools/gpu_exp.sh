for sub in 8 64; do timeout 300 python bench.py --config c3 --no-cpu-baseline --no-e2e --sub $sub --steps 3 > gpurun_out/exp_sub$sub.log 2>&1; done
