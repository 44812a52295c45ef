mkdir -p /tmp/rep gpurun_out/prof5
timeout 1500 ncu --set full --clock-control none --import-source on -k regex:consume_kernel -s 1 -c 1 -o /tmp/rep/consume_c5 python tools/prof_consume.py c5 2 > gpurun_out/prof5/ncu.log 2>&1
python tools/summarize_ncu.py /tmp/rep/consume_c5.ncu-rep ncu_consume_c5 > /dev/null 2>&1
cp profiles/ncu_consume_c5.json profiles/ncu_consume_c5.md gpurun_out/prof5/
python tools/ncu_toplines.py /tmp/rep/consume_c5.ncu-rep consume.cu 40 > gpurun_out/prof5/toplines_c5.txt 2>&1
