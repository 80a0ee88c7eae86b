for c in ${@:-c3 c4}; do timeout 300 python tools/msprof.py $c 64; done
