python __graft_entry__.py build > /dev/null
for v in default rpw2 rpw4 rpw8 rpa256 rpw2rpa256; do
  if [ $v = default ]; then unset CUSAN_LIBRARY; else export CUSAN_LIBRARY=$PWD/build_variants/libcusan_$v.so; fi
  echo "== $v"; timeout 300 python tools/quick_timing.py 3,4,5 4096 2>&1 | sed -E 's/ races.*//' | cut -c1-160
done
