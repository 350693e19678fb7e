# guided-tail sweep (profiles/range_sweep_r01.md): CUSAN_TAIL_PCT / CUSAN_TAIL_DIV at run time
python __graft_entry__.py build > /dev/null
for cfg in "$@"; do set -- $(echo $cfg | tr / ' '); echo "== tail $1% /$2"; CUSAN_TAIL_PCT=$1 CUSAN_TAIL_DIV=$2 timeout 300 python tools/quick_timing.py 3,4,5 4096 2>&1 | sed -E "s/ races.*//" | sed -E "s/lower.*kernel/kernel/" | sed -E "s/run .* checked;/|/" | cut -c1-120; done
