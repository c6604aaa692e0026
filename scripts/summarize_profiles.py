"""Build profiles/<tag>_* summaries from gpurun_out/ captures of
scripts/profile_round.sh.  Usage: python scripts/summarize_profiles.py TAG WORKLOAD..."""
import csv
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
OUT = os.path.join(ROOT, "gpurun_out")
PROF = os.path.join(ROOT, "profiles")

KEYS = [
    ("gpu__time_duration.sum", "duration"),
    ("dram__bytes_read.sum", "DRAM read"),
    ("dram__bytes_write.sum", "DRAM write"),
    ("sm__issue_active.avg.pct_of_peak_sustained_active", "issue slots busy (% of peak)"),
    ("sm__inst_executed_pipe_alu.avg.pct_of_peak_sustained_active", "ALU pipe (% of peak)"),
    ("sm__inst_executed_pipe_fma.avg.pct_of_peak_sustained_active", "FMA pipe (% of peak)"),
    ("sm__inst_executed_pipe_fmaheavy.avg.pct_of_peak_sustained_active", "FMA-heavy pipe (% of peak)"),
    ("smsp__inst_executed.sum", "warp instructions executed"),
    ("smsp__thread_inst_executed_per_inst_executed.ratio", "SIMT efficiency (threads / warp instr, of 32)"),
    ("smsp__sass_average_branch_targets_threads_uniform.pct", "branch targets uniform (%)"),
    ("sm__warps_active.avg.pct_of_peak_sustained_active", "achieved occupancy (%)"),
    ("launch__registers_per_thread", "registers / thread"),
    ("launch__grid_size", "grid size"),
    ("sm__cycles_elapsed.avg", "SM cycles elapsed"),
    ("smsp__cycles_active.avg", "SMSP cycles active"),
]


def launches(tag, wl):
    path = os.path.join(OUT, "%s_%s_launches.csv" % (tag, wl))
    rows = list(csv.reader(open(path)))
    h = next(i for i, r in enumerate(rows) if "Kernel Name" in r)
    hdr, data = rows[h], rows[h + 1:]
    ki, vi = hdr.index("Kernel Name"), hdr.index("Metric Value")
    names = [r[ki].split("(")[0].replace("void ", "").replace("beast::", "") for r in data]
    vals = [float(r[vi].replace(",", "")) for r in data]
    # one step = the last run of launches starting at the first-level count kernel
    starts = [i for i, n in enumerate(names) if n.startswith(("k_seg_count<", "k_seg_level<")) and ("PairsSeg" in n or "PairRowsSeg" in n)]
    bounds = list(zip(starts, starts[1:] + [len(names)]))
    # the last canonical pass (the bench also times the factorised path)
    a, b = [(a, b) for a, b in bounds if any(n.startswith("k_eval<") for n in names[a:b])][-1]
    step = list(zip(names[a:b], vals[a:b]))
    pub = [i for i, (n, _) in enumerate(step) if n.startswith("k_publish")]
    if pub:
        step = step[:pub[0] + 1]
    # drop non-pipeline kernels (torch flush etc.)
    step = [(n, v) for n, v in step if n.startswith("k_")]
    tot = sum(v for _, v in step)
    lines = ["# %s — %s: ncu launch list of one bench step" % (tag, wl), "",
             "`ncu --metrics gpu__time_duration.sum --clock-control none` over "
             "`python bench.py --steps 3 --warmup 3 --workload %s`; the last step's pipeline kernels "
             "(cold-cache, serialised: compare shares, not absolutes; the bench value is taken without ncu)." % wl,
             "", "| # | kernel | µs | share |", "|---|---|---|---|"]
    for i, (n, v) in enumerate(step):
        lines.append("| %d | `%s` | %.1f | %.1f%% |" % (i + 1, n, v / 1e3, 100 * v / tot))
    lines.append("| | **total** | **%.1f** | 100%% |" % (tot / 1e3))
    open(os.path.join(PROF, "%s_%s_launches.md" % (tag, wl)), "w").write("\n".join(lines) + "\n")
    return {n: v for n, v in step}, tot


def keval(tag, wl):
    rep = os.path.join(OUT, "%s_%s_keval.ncu-rep" % (tag, wl))
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(out.splitlines()))
    hdr, units, r = rows[0], rows[1], rows[2]
    lines = ["# %s — %s: `ncu --set full` of k_eval<A> (one launch)" % (tag, wl), "",
             "Kernel: `%s`" % r[hdr.index("Kernel Name")], "", "| metric | value | unit | ncu name |",
             "|---|---|---|---|"]
    vals = {}
    for key, label in KEYS:
        if key in hdr:
            i = hdr.index(key)
            vals[key] = (r[i], units[i])
            lines.append("| %s | %s | %s | `%s` |" % (label, r[i], units[i], key))
    open(os.path.join(PROF, "%s_%s_keval_ncu.md" % (tag, wl)), "w").write("\n".join(lines) + "\n")
    def to_bytes(v, u):
        x = float(v.replace(",", ""))
        return x * {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}.get(u, 1)
    rd = to_bytes(*vals["dram__bytes_read.sum"])
    wr = to_bytes(*vals["dram__bytes_write.sum"])
    return rd + wr


def main():
    tag, wls = sys.argv[1], sys.argv[2:]
    os.makedirs(PROF, exist_ok=True)
    traffic_path = os.path.join(PROF, "k_eval_traffic.json")
    traffic = json.load(open(traffic_path)) if os.path.exists(traffic_path) else {}
    for wl in wls:
        launches(tag, wl)
        traffic[wl] = keval(tag, wl)
        print(wl, "traffic bytes/launch", traffic[wl])
    json.dump(traffic, open(traffic_path, "w"), indent=1, sort_keys=True)


if __name__ == "__main__":
    main()
