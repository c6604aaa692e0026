"""Summarise an ncu report (raw page) or a launch-list CSV.
Usage: python scripts/ncu_summary.py REPORT.ncu-rep | LAUNCHES.csv"""
import csv
import subprocess
import sys

METRICS = ["gpu__time_duration.sum", "sm__inst_executed_pipe_alu.avg.pct_of_peak_sustained_active",
           "sm__inst_executed_pipe_fma.avg.pct_of_peak_sustained_active",
           "sm__inst_executed_pipe_fmaheavy.avg.pct_of_peak_sustained_active",
           "sm__issue_active.avg.pct_of_peak_sustained_active", "smsp__inst_executed.sum",
           "smsp__thread_inst_executed_per_inst_executed.ratio", "sm__warps_active.avg.pct_of_peak_sustained_active",
           "smsp__sass_average_branch_targets_threads_uniform.pct", "dram__bytes_read.sum", "dram__bytes_write.sum",
           "launch__registers_per_thread", "sm__cycles_elapsed.avg"]


def main(path):
    if path.endswith(".csv"):
        rows = list(csv.reader(open(path)))
        h = next(i for i, r in enumerate(rows) if "Kernel Name" in r)
        hdr, data = rows[h], rows[h + 1:]
        ki, vi = hdr.index("Kernel Name"), hdr.index("Metric Value")
        tot = 0.0
        for r in data:
            v = float(r[vi].replace(",", ""))
            tot += v
            print("%-44s %10.1f us" % (r[ki].split("(")[0][:44], v / 1e3))
        print("%-44s %10.1f us" % ("total", tot / 1e3))
        return
    out = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(out.splitlines()))
    hdr, units = rows[0], rows[1]
    for r in rows[2:]:
        print(r[hdr.index("Kernel Name")].split("(")[0])
        for m in METRICS:
            if m in hdr:
                i = hdr.index(m)
                print("   %-70s %14s %s" % (m, r[i], units[i]))


if __name__ == "__main__":
    main(sys.argv[1])
