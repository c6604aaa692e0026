"""Runs of consecutive SASS instructions with equal execution counts (basic
blocks, roughly) from an `ncu --page source --csv --print-source sass` export:
start address, executions, instructions in the run, their total, stall
samples, first opcode.  Usage: python scripts/sass_runs.py FILE [section] [min_total]"""
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
secn = int(sys.argv[2]) if len(sys.argv) > 2 else 0
thr = float(sys.argv[3]) if len(sys.argv) > 3 else 5e5
sec, cur = [], None
for r in rows:
    if r and r[0] == "Kernel Name":
        cur = [r[1]]
        sec.append(cur)
        continue
    if cur is not None:
        cur.append(r)
body = sec[secn]
print(body[0][:100])
hdr = body[1]
ie, src, st = hdr.index("Instructions Executed"), hdr.index("Source"), hdr.index("Warp Stall Sampling (All Samples)")
data = [(r[0][-5:], r[src].strip(), int(r[ie] or 0), int(r[st] or 0)) for r in body[2:] if len(r) == len(hdr)]
tot = sum(d[2] for d in data)
stot = sum(d[3] for d in data) or 1
print("total %.2fM warp instructions, %d stall samples" % (tot / 1e6, stot))
runs = []
for a, s, n, sl in data:
    if runs and runs[-1][1] == n:
        runs[-1][2] += 1
        runs[-1][3] += n
        runs[-1][4] += sl
        runs[-1][6].append(s.split()[0] if not s.startswith("@") else s.split()[1])
    else:
        runs.append([a, n, 1, n, sl, s[:60], [s.split()[0] if not s.startswith("@") else s.split()[1]]])
for a, n, k, t, sl, s, ops in runs:
    if t >= thr:
        print("%s exec %9d x %3d = %7.2fM (%4.1f%%) stalls %4.1f%%  %s" % (a, n, k, t / 1e6, 100 * t / tot, 100 * sl / stot, s))
