for v in v42e9a0c v2b392a9 vc51b012 cur; do
  if [ $v = cur ]; then unset SASSI_LIB; else export SASSI_LIB=paper_conf_isca_stephensonhlejn15_b200/lib/variants/$v/libsassi.so; fi
  echo "== $v"; timeout 600 compute-sanitizer --tool synccheck python tools/synccheck_min.py 4 2>&1 | tail -2
done
