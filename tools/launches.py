"""Summarise an ncu --metrics gpu__time_duration.sum --csv launch list by kernel."""
import collections
import csv
import sys


def summarise(path, top=30):
    rows = list(csv.reader(open(path)))
    hi = [i for i, r in enumerate(rows) if "Kernel Name" in r][0]
    h = rows[hi]
    ki, vi = h.index("Kernel Name"), h.index("Metric Value")
    agg = collections.defaultdict(lambda: [0, 0.0])
    for r in rows[hi + 1:]:
        if len(r) <= vi:
            continue
        name = r[ki].replace("<unnamed>::", "").replace("(anonymous namespace)::", "")
        name = name.split("(")[0].split("<")[0].replace("void ", "")
        try:
            v = float(r[vi].replace(",", ""))
        except ValueError:
            continue
        agg[name][0] += 1
        agg[name][1] += v
    tot = sum(v[1] for v in agg.values())
    out = []
    for k, (c, v) in sorted(agg.items(), key=lambda x: -x[1][1])[:top]:
        out.append(f"{k:42s} {c:6d} {v / 1e6:9.3f} ms {100 * v / tot:5.1f}%")
    out.append(f"total {tot / 1e6:.3f} ms over {sum(c for c, _ in agg.values())} launches")
    return "\n".join(out)


if __name__ == "__main__":
    print(summarise(sys.argv[1]))
