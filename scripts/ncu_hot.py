"""Per-instruction hot spots of one kernel in an ncu report (source page).
Usage: python scripts/ncu_hot.py REPORT.ncu-rep KERNEL_SUBSTRING [min_exec]"""
import csv
import subprocess
import sys

rep, sub = sys.argv[1], sys.argv[2]
thresh = int(sys.argv[3]) if len(sys.argv) > 3 else 300000
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                     capture_output=True, text=True).stdout
secs, cur = [], None
for r in csv.reader(out.splitlines()):
    if r and r[0] == "Kernel Name":
        cur = [r[1], []]
        secs.append(cur)
    elif cur is not None:
        cur[1].append(r)
for name, body in secs:
    if sub in name:
        hdr = body[0]
        data = [x for x in body[1:] if len(x) == len(hdr)]
        ie, src = hdr.index("Instructions Executed"), hdr.index("Source")
        st = hdr.index("Warp Stall Sampling (All Samples)")
        vals = [(x, int(x[ie])) for x in data if x[ie].isdigit()]
        print(name[:80], "total inst", sum(v for _, v in vals),
              "stall samples", sum(int(x[st]) for x, _ in vals if x[st].isdigit()))
        for x, v in vals:
            if v >= thresh or (x[st].isdigit() and int(x[st]) > 400):
                print("  %s %10d %6s  %s" % (x[0][-5:], v, x[st], x[src][:90]))
        break
