python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 300 python tools/dbg_small.py 2>&1 | tail -5
timeout 600 compute-sanitizer --tool memcheck --show-backtrace no --print-limit 5 python tools/dbg_small.py 2>&1 | tail -30
