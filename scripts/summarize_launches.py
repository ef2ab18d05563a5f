"""Summarise an ncu launch list (--metrics gpu__time_duration.sum --csv) per kernel."""
import csv, sys
from collections import OrderedDict

SCALE = {"ns": 1e-3, "nsecond": 1e-3, "us": 1.0, "usecond": 1.0, "ms": 1e3, "msecond": 1e3}


def summarize(path):
    rows = list(csv.reader(open(path)))
    hdr, agg = None, OrderedDict()
    for r in rows:
        if r and r[0] == "ID":
            hdr = r
            continue
        if not hdr or len(r) != len(hdr):
            continue
        d = dict(zip(hdr, r))
        if d.get("Metric Name") != "gpu__time_duration.sum":
            continue
        name = d["Kernel Name"].split("(")[0].replace("void ", "").split("::")[-1]
        t = float(d["Metric Value"].replace(",", "")) * SCALE.get(d.get("Metric Unit", "ns"), 1e-3)
        a = agg.setdefault(name, [0, 0.0])
        a[0] += 1
        a[1] += t
    return agg


if __name__ == "__main__":
    agg = summarize(sys.argv[1])
    tot = sum(v[1] for v in agg.values())
    print("# per-kernel totals from %s (ncu gpu__time_duration.sum, cold-cache, serialised)" % sys.argv[1])
    print("%-44s %8s %11s %9s %7s" % ("kernel", "launches", "total_us", "avg_us", "share"))
    for k, (n, t) in sorted(agg.items(), key=lambda x: -x[1][1]):
        print("%-44s %8d %11.1f %9.2f %6.1f%%" % (k, n, t, t / n, 100 * t / tot))
