# quick ncu metric comparison of library variants on one workload: bash tools/ncu_cmp.sh "prev va" "c5 c3"
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,smsp__inst_executed.sum,smsp__inst_issued.sum,sm__inst_executed_pipe_alu.avg.pct_of_peak_sustained_active,smsp__issue_active.avg.pct_of_peak_sustained_active,launch__registers_per_thread,smsp__average_warp_latency_issue_stalled_long_scoreboard.ratio,smsp__average_warp_latency_issue_stalled_wait.ratio,smsp__average_warp_latency_issue_stalled_short_scoreboard.ratio,smsp__average_warp_latency_issue_stalled_no_instruction.ratio,smsp__average_warp_latency_issue_stalled_branch_resolving.ratio
mkdir -p gpurun_out/ncmp
for v in $1; do for w in $2; do
SASSI_LIB=paper_conf_isca_stephensonhlejn15_b200/lib/variants/$v/libsassi.so timeout 600 ncu --metrics $M --clock-control none -k regex:consume_kernel -s 1 -c 1 --csv python tools/prof_consume.py $w 2 > gpurun_out/ncmp/${v}_$w.csv 2>&1
done; done
