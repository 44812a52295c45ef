"""Summarise an ncu --set full report of the consume kernel into profiles/ (JSON + markdown).

usage: python tools/summarize_ncu.py REPORT.ncu-rep NAME [algorithmic_bytes]
Writes profiles/NAME.json and profiles/NAME.md; when NAME starts with ncu_consume_ the JSON carries
dram_bytes_per_launch, which bench.py reports as roofline.traffic.
"""
import csv
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
UNITS = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12,
         "ns": 1e-9, "us": 1e-6, "usecond": 1e-6, "ms": 1e-3, "msecond": 1e-3, "s": 1.0}
KEYS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "smsp__inst_issued.sum",
        "smsp__issue_active.avg.pct_of_peak_sustained_active",
        "sm__warps_active.avg.pct_of_peak_sustained_active", "launch__registers_per_thread",
        "launch__grid_size", "launch__block_size", "launch__occupancy_limit_registers",
        "launch__occupancy_limit_shared_mem", "sm__cycles_elapsed.avg.per_second",
        "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum", "lts__t_sectors_srcunit_tex_op_read.sum",
        "smsp__inst_executed_op_shared_atom.sum", "smsp__inst_executed_op_global_red.sum",
        # L2 and atomic throughput (north_star asks for both next to the DRAM figure)
        "lts__throughput.avg.pct_of_peak_sustained_elapsed", "lts__t_sector_hit_rate.pct",
        "lts__t_sectors_srcunit_tex_op_red.sum", "lts__t_sectors_srcunit_tex_op_atom.sum",
        "lts__d_atomic_input_cycles_active.avg.pct_of_peak_sustained_elapsed",
        "l1tex__data_pipe_lsu_wavefronts_mem_shared_op_atom.sum",
        "l1tex__data_pipe_lsu_wavefronts_mem_shared_op_atom.sum.pct_of_peak_sustained_elapsed",
        "l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_atom.sum",
        # which pipe is busiest (the fold is integer / warp-vote work)
        "sm__inst_executed_pipe_alu.avg.pct_of_peak_sustained_active",
        "sm__inst_executed_pipe_xu.avg.pct_of_peak_sustained_active",
        "sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active",
        "sm__inst_executed_pipe_fma.avg.pct_of_peak_sustained_active",
        "sm__throughput.avg.pct_of_peak_sustained_elapsed"]


def raw(report):
    out = subprocess.run(["ncu", "-i", report, "--page", "raw", "--csv"], capture_output=True,
                         text=True, check=True).stdout
    rows = list(csv.reader(out.splitlines()))
    return rows[0], rows[1], rows[2]


def main():
    report, name = sys.argv[1], sys.argv[2]
    alg = float(sys.argv[3]) if len(sys.argv) > 3 else None
    h, u, v = raw(report)
    m = {}
    for k, un, x in zip(h, u, v):
        if k in KEYS or ("stall" in k and k.endswith("_per_issue_active.ratio")):
            try:
                val = float(x.replace(",", ""))
            except ValueError:
                continue
            if un in UNITS:
                val *= UNITS[un]
            m[k] = val
    dur = m.get("gpu__time_duration.sum")
    rd, wr = m.get("dram__bytes_read.sum", 0.0), m.get("dram__bytes_write.sum", 0.0)
    summary = {
        "report": os.path.basename(report), "kernel": "consume_kernel",
        "duration_s": dur, "dram_bytes_read": rd, "dram_bytes_write": wr,
        "dram_bytes_per_launch": rd + wr,
        "dram_gbs": (rd + wr) / dur / 1e9 if dur else None,
        "algorithmic_bytes_per_launch": alg,
        "traffic_over_algorithmic": (rd + wr) / alg if alg else None,
        "metrics": m,
        "note": "ncu --set full --clock-control none, one launch, cold-ish caches, serialised",
    }
    os.makedirs(os.path.join(ROOT, "profiles"), exist_ok=True)
    json.dump(summary, open(os.path.join(ROOT, "profiles", name + ".json"), "w"), indent=1)
    stalls = sorted(((k.replace("smsp__average_warps_issue_stalled_", "").replace(
        "_per_issue_active.ratio", ""), x) for k, x in m.items() if "stall" in k),
        key=lambda t: -t[1])
    with open(os.path.join(ROOT, "profiles", name + ".md"), "w") as f:
        f.write("# %s\n\nSource: `%s` (ncu --set full --clock-control none).\n\n" % (name, report))
        f.write("| metric | value |\n|---|---|\n")
        f.write("| duration | %.3f ms |\n" % (1e3 * dur) if dur else "")
        f.write("| DRAM read / write | %.3f GB / %.1f MB |\n" % (rd / 1e9, wr / 1e6))
        if alg:
            f.write("| algorithmic bytes | %.3f GB (traffic / algorithmic = %.3f) |\n" % (alg / 1e9, (rd + wr) / alg))
        if dur:
            f.write("| DRAM bandwidth (traffic / duration) | %.0f GB/s |\n" % ((rd + wr) / dur / 1e9))
        for k in KEYS[3:]:
            if k in m:
                f.write("| %s | %s |\n" % (k, ("%.4g" % m[k])))
        f.write("\nWarp stall reasons (per issued instruction):\n\n")
        for k, x in stalls:
            if x >= 0.05:
                f.write("- %s: %.2f\n" % (k, x))
    print(json.dumps({k: summary[k] for k in ("duration_s", "dram_bytes_per_launch", "dram_gbs",
                                                "traffic_over_algorithmic")}))


if __name__ == "__main__":
    main()
