# ncu --set full of the fold on c2 and c3 (current build) -> per-line and per-opcode summaries
mkdir -p /tmp/rep gpurun_out/prof
for w in c2 c3; do
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:consume_kernel -s 1 -c 1 -o /tmp/rep/p_$w python tools/prof_consume.py $w 2 > /dev/null 2>&1
  ncu -i /tmp/rep/p_$w.ncu-rep --page source --csv --print-source cuda,sass > gpurun_out/prof/src_$w.csv 2>/dev/null
  python tools/summarize_ncu.py /tmp/rep/p_$w.ncu-rep tmp_p_$w > /dev/null 2>&1; cp profiles/tmp_p_$w.md gpurun_out/prof/
done
