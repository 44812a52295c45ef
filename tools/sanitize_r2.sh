for tool in memcheck racecheck synccheck initcheck; do
  echo "### $tool (SANITIZE_PART=r2)"; SANITIZE_PART=r2 timeout 1200 compute-sanitizer --tool $tool --num-cuda-barriers 8192 python tools/sanitize_run.py 2>&1 | tail -3
  echo "### $tool (SANITIZE_PART=base)"; SANITIZE_PART=base timeout 1800 compute-sanitizer --tool $tool --num-cuda-barriers 8192 python tools/sanitize_run.py 2>&1 | tail -3
done
