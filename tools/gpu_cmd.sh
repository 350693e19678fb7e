for v in tools/var_*.so; do echo "== $v"; CUSAN_LIBRARY=$v timeout 300 python tools/quick_timing.py 5,4,3 4096 2>&1 | cut -c1-90; done
