#!/bin/bash
# one GPU iteration: parity tests, a short bench line, and an ncu capture of the consume kernel
# usage: tools/gpu_iter.sh TAG [workload]
TAG=${1:-iter}; WL=${2:-c3}
timeout 600 python -m pytest tests -m gpu -q -x 2>&1 | tail -4
timeout 300 python bench.py --workload $WL --no-e2e --no-cpu-baseline --steps 10 2>&1 | tail -1 > gpurun_out/bench_$TAG.json
python -c "import json; d=json.load(open('gpurun_out/bench_$TAG.json')); print('value %.3e rec/s  consume %.3f ms  %.0f GB/s  frac %.3f  clocks %s' % (d['value'], d['roofline']['consume_ms_avg'], d['roofline']['achieved'], d['roofline']['frac'], d['clocks']))"
timeout 600 ncu --set full --clock-control none --import-source on -k regex:consume_kernel -s 1 -c 1 -o gpurun_out/prof_${WL}_$TAG python tools/prof_consume.py $WL 2 > /dev/null 2>&1
ls gpurun_out | grep $TAG
