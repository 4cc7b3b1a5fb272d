"""Per-kernel totals of an ncu launch list (--metrics gpu__time_duration.sum --csv)."""
import collections
import csv
import sys


def summary(path, top=16):
    rows = list(csv.reader(open(path)))
    h, agg = None, collections.defaultdict(lambda: [0, 0.0])
    scale = {"ns": 1e-6, "nsecond": 1e-6, "us": 1e-3, "usecond": 1e-3, "ms": 1.0, "msecond": 1.0, "s": 1e3, "second": 1e3}
    for r in rows:
        if "Kernel Name" in r:
            h = r
            continue
        if h is None or len(r) != len(h):
            continue
        x = dict(zip(h, r))
        if x.get("Metric Name") != "gpu__time_duration.sum":
            continue
        v = float(x["Metric Value"].replace(",", "")) * scale.get(x["Metric Unit"], 1.0)
        a = agg[x["Kernel Name"].split("(")[0]]
        a[0] += 1
        a[1] += v
    tot = sum(a[1] for a in agg.values())
    out = [f"total {tot:.1f} ms over {sum(a[0] for a in agg.values())} launches"]
    for k, a in sorted(agg.items(), key=lambda t: -t[1][1])[:top]:
        out.append(f"{a[1]:10.1f} ms {a[1] / tot:6.3f} n={a[0]:6d} {k}")
    return "\n".join(out)


if __name__ == "__main__":
    print(summary(sys.argv[1]))
