"""Write profiles/<TAG>_*.md from a scripts/checkpoint.sh run's gpurun_out/
files: the launch lists (headline, SGEMM-B200), the ncu --set full metrics of
k_tile_eval<A>/<B>, the tail kernels and the prefix-stage levels, and the bench lines' key numbers.
Usage: python scripts/summarize_checkpoint.py TAG"""
import csv
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
OUT = os.path.join(ROOT, "gpurun_out")
PROF = os.path.join(ROOT, "profiles")
KEYS = [("gpu__time_duration.sum", "duration"), ("dram__bytes_read.sum", "DRAM read"),
        ("dram__bytes_write.sum", "DRAM write"), ("sm__throughput.avg.pct_of_peak_sustained_elapsed", "SM throughput %"),
        ("smsp__issue_active.avg.pct_of_peak_sustained_active", "issue active %"),
        ("sm__inst_executed_pipe_alu.avg.pct_of_peak_sustained_active", "ALU pipe %"),
        ("sm__inst_executed_pipe_fma.avg.pct_of_peak_sustained_active", "FMA pipe %"),
        ("smsp__inst_executed.sum", "warp instructions"),
        ("smsp__thread_inst_executed_per_inst_executed.ratio", "SIMT efficiency (of 32)"),
        ("sm__warps_active.avg.pct_of_peak_sustained_active", "achieved occupancy %"),
        ("launch__registers_per_thread", "registers / thread"), ("launch__grid_size", "grid")]


def raw_table(path):
    rows = list(csv.reader(open(path)))
    hdr, units, data = rows[0], rows[1], rows[2:]
    ki = hdr.index("Kernel Name")
    names = [r[ki].split("(")[0].replace("void ", "").replace("beast::", "") for r in data]
    lines = ["| metric | " + " | ".join("`%s`" % n for n in names) + " |", "|---" * (len(names) + 1) + "|"]
    for k, lbl in KEYS:
        if k not in hdr:
            continue
        i = hdr.index(k)
        u = units[i]
        lines.append("| %s%s | %s |" % (lbl, " (%s)" % u if u and u != "%" else "", " | ".join(r[i] for r in data)))
    return "\n".join(lines)


def main():
    tag = sys.argv[1]
    parts = ["# %s — round-2 checkpoint (one B200, `scripts/checkpoint.sh %s`)\n" % (tag, tag)]
    for wl in ("headline", "b200_S"):
        p = os.path.join(OUT, "%s_%s_launches.csv" % (tag, wl))
        if os.path.exists(p):
            md = subprocess.run([sys.executable, os.path.join(ROOT, "scripts", "summarize_launches.py"), p, "--md"],
                                capture_output=True, text=True).stdout
            parts.append("## Launch list, %s (ncu `gpu__time_duration.sum --clock-control none`, one pass of "
                         "`scripts/prof_run.py %s`; cold-cache and serialised: compare shares)\n\n%s" % (wl, wl, md))
    for r, what in (("headline_keval", "k_tile_eval<A>, k_tile_eval<B>, scan, placement + write-out, headline"),
                    ("b200_S_keval", "k_tile_eval<A>, k_tile_eval<B>, SGEMM-B200"),
                    ("headline_seglvl", "prefix-stage levels, headline")):
        p = os.path.join(OUT, "%s_%s_raw.csv" % (tag, r))
        if os.path.exists(p):
            parts.append("## ncu --set full: %s\n\n%s\n" % (what, raw_table(p)))
    for wl, f in (("headline", "bench_default"), ("b200_S", "bench_b200_S")):
        p = os.path.join(OUT, "%s_%s.json" % (tag, f))
        if os.path.exists(p):
            try:
                d = json.load(open(p))
            except Exception:
                continue
            r = d["roofline"]
            parts.append("## bench line, %s\n\nms/step %.4f, value %.4g points/s, k_tile_eval<A> %.4f ms = %.3f of the derived "
                         "issue peak, %.3f of the measured packed-scan ceiling; count %.4f ms; e2e %.4g points/s; "
                         "write-out %s; clocks %s\n" % (
                             wl, d["ms_per_step"], d["value"], r["avg_launch_ms"], r["frac"], r["frac_measured_scan"],
                             d["count"]["ms_per_step"], d["e2e"]["value"],
                             "%.4f ms = %.2f of HBM" % (d["write_out"]["avg_launch_ms"], d["write_out"]["frac"])
                             if d.get("write_out") else "-", d["clocks"]))
            with open(os.path.join(PROF, "%s_bench_%s.json" % (tag, wl)), "w") as g:
                json.dump(d, g)
    with open(os.path.join(PROF, "%s_summary.md" % tag), "w") as f:
        f.write("\n".join(parts))
    print("wrote profiles/%s_summary.md" % tag)


if __name__ == "__main__":
    main()
