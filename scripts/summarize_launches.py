"""Print the per-kernel launch list (ncu gpu__time_duration.sum CSV) of one
pass captured by scripts/prof_run.py.  Usage: python scripts/summarize_launches.py CSV [--md]"""
import csv
import sys


def rows(path):
    data = list(csv.reader(open(path)))
    h = next(i for i, r in enumerate(data) if "Kernel Name" in r)
    hdr, body = data[h], data[h + 1:]
    ki, vi, ui = hdr.index("Kernel Name"), hdr.index("Metric Value"), hdr.index("Metric Unit")
    out = []
    for r in body:
        if len(r) <= vi:
            continue
        name = r[ki].split("(")[0].replace("void ", "").replace("beast::", "")
        v = float(r[vi].replace(",", ""))
        unit = r[ui]
        us = v / 1e3 if unit in ("nsecond", "ns") else v if unit in ("usecond", "us") else v * 1e3
        out.append((name, us))
    return out


def main():
    path = sys.argv[1]
    md = "--md" in sys.argv
    r = rows(path)
    tot = sum(us for _, us in r)
    if md:
        print("| # | kernel | µs | share |\n|---|---|---|---|")
    for i, (n, us) in enumerate(r, 1):
        if md:
            print("| %d | `%s` | %.1f | %.1f%% |" % (i, n, us, 100 * us / tot))
        else:
            print("%2d %-42s %8.1f us %5.1f%%" % (i, n, us, 100 * us / tot))
    print(("| | **total** | **%.1f** | 100%% |" if md else "   total %.1f us") % tot)


if __name__ == "__main__":
    main()
