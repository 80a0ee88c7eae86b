python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "tree_parallel" > gpurun_out/pytest_gpu.log 2>&1; echo pytest $?
tail -15 gpurun_out/pytest_gpu.log
