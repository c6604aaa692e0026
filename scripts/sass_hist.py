"""Summarise an `ncu --page source --csv --print-source sass` export: total
instructions, the hottest lines and per-region sums (regions split at
branch targets).  Usage: python scripts/sass_hist.py FILE [min_count]"""
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
thr = float(sys.argv[2]) if len(sys.argv) > 2 else 2e5
hdr = next(r for r in rows if "Source" in r)
i_src, i_ie = hdr.index("Source"), hdr.index("Instructions Executed")
i_st = hdr.index("Warp Stall Sampling (All Samples)")
data = []
for r in rows[rows.index(hdr) + 1:]:
    if len(r) < len(hdr):
        continue
    data.append((r[0][-4:], r[i_src].strip(), int(r[i_ie] or 0), int(r[i_st] or 0)))
tot = sum(d[2] for d in data)
stot = sum(d[3] for d in data) or 1
print("total warp instructions %.2fM, stall samples %d" % (tot / 1e6, stot))
kinds = {}
for a, s, ie, st in data:
    op = s.split()[0] if not s.startswith("@") else s.split()[1]
    op = op.split(".")[0]
    kinds[op] = kinds.get(op, 0) + ie
for op, n in sorted(kinds.items(), key=lambda x: -x[1])[:25]:
    print("  %-10s %7.2fM  %5.1f%%" % (op, n / 1e6, 100 * n / tot))
for a, s, ie, st in data:
    if ie > thr or st > stot * 0.01:
        print("%s %8.3fM %5.1f%% %s" % (a, ie / 1e6, 100 * st / stot, s[:80]))
