#!/bin/bash
# Round-2 evidence on one B200: GPU tests, bench lines (c3 default, c2 / c4 / c5), the launch list
# of a short bench run, ncu --set full captures of the fold (c3, c2, c4) summarised for profiles/.
# usage (on the box): bash tools/evidence_r2.sh TAG   -> gpurun_out/ev_TAG/...
TAG=${1:-r2}; O=gpurun_out/ev_$TAG; mkdir -p $O /tmp/rep
nvidia-smi --query-gpu=name,clocks.max.sm,power.limit --format=csv > $O/gpu.txt
timeout 2400 python -m pytest tests/ -m gpu -q 2>&1 | tail -3 > $O/pytest_gpu.txt
timeout 1200 python bench.py > $O/bench.json 2> $O/bench.err
for w in c2 c4 c5; do
  timeout 1500 python bench.py --workload $w --steps 10 --no-slowdown --no-injection --no-cpu-baseline >> $O/bench_configs.jsonl 2>> $O/bench_configs.err
done
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches.csv \
  python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu-baseline --no-slowdown --no-injection > /dev/null 2>&1
python tools/launch_list.py $O/launches.csv $O/launches.md > /dev/null 2>&1
for w in c3 c2 c4; do
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:consume_kernel -s 1 -c 1 \
    -o /tmp/rep/consume_$w python tools/prof_consume.py $w 2 > /dev/null 2>&1
  python tools/summarize_ncu.py /tmp/rep/consume_$w.ncu-rep ncu_consume_$w > /dev/null 2>&1
  cp profiles/ncu_consume_$w.json profiles/ncu_consume_$w.md $O/
  python tools/ncu_toplines.py /tmp/rep/consume_$w.ncu-rep consume.cu 40 > $O/toplines_$w.txt 2>&1
done
ls $O
timeout 600 python tools/paper_report.py $O/paper_report.md > /dev/null 2>&1
timeout 1200 python tools/fuzz_parity.py 300 11 > $O/fuzz_parity.txt 2>&1
timeout 900 python tools/fuzz_inline.py > $O/fuzz_inline.txt 2>&1
SASSI_BENCH_SCALING_EXTRAS=1 timeout 900 python bench.py --workload c5 --steps 10 > $O/bench_c5_scaling_extras.json 2>&1
ls $O
