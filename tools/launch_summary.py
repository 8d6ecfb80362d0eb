"""Summarise an ncu --metrics gpu__time_duration.sum --csv launch list: per kernel launches, total ms, share."""
import collections
import csv
import re
import sys

SCALE = {"ns": 1e-6, "nsecond": 1e-6, "us": 1e-3, "usecond": 1e-3, "ms": 1.0, "msecond": 1.0}


def main(path, skip=()):
    rows = [r for r in csv.reader(open(path)) if len(r) > 5]
    h = rows[0]
    ki, vi, ui = h.index("Kernel Name"), h.index("Metric Value"), h.index("Metric Unit")
    agg = collections.OrderedDict()
    for r in rows[1:]:
        name = re.sub(r"\(.*", "", r[ki]).replace("void ", "").replace("olap::", "")
        if any(s in name for s in skip):
            continue
        a = agg.setdefault(name, [0, 0.0])
        a[0] += 1
        a[1] += float(r[vi].replace(",", "")) * SCALE[r[ui]]
    tot = sum(a[1] for a in agg.values())
    for k, (n, t) in sorted(agg.items(), key=lambda x: -x[1][1]):
        print(f"{k[:44]:44s} launches {n:3d} total {t:10.3f} ms share {100 * t / tot:6.2f}%")


if __name__ == "__main__":
    main(sys.argv[1], tuple(sys.argv[2:]))
