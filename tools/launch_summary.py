"""Per-kernel summary of an ncu launch list CSV (gpu__time_duration.sum, dram bytes): launches,
total ms, share, DRAM GB/s (diagnostic; profiles/ summaries are made with it)."""
import collections
import csv
import sys


def main(path, top=40):
    rows = list(csv.reader(open(path)))
    hi = [i for i, r in enumerate(rows) if "Kernel Name" in r][0]
    h = rows[hi]
    ki, mi, vi, ii = h.index("Kernel Name"), h.index("Metric Name"), h.index("Metric Value"), h.index("ID")
    per = {}
    for r in rows[hi + 1:]:
        if len(r) <= vi:
            continue
        d = per.setdefault(int(r[ii]), {"name": r[ki]})
        try:
            d[r[mi]] = float(r[vi].replace(",", ""))
        except ValueError:
            pass
    agg = collections.defaultdict(lambda: [0, 0.0, 0.0])
    for d in per.values():
        n = d["name"].replace("(anonymous namespace)::", "").replace("buffalo::", "").split("(")[0].replace("void ", "")
        a = agg[n]
        a[0] += 1
        a[1] += d.get("gpu__time_duration.sum", 0.0)
        a[2] += d.get("dram__bytes_read.sum", 0.0) + d.get("dram__bytes_write.sum", 0.0)
    tot = sum(v[1] for v in agg.values())
    print(f"# {path}: {len(per)} launches, {tot / 1e6:.3f} ms serialised (ncu, --clock-control none)")
    print(f"{'kernel':64s} {'launches':>8s} {'ms':>9s} {'share':>6s} {'DRAM GB/s':>10s}")
    for k, (c, t, b) in sorted(agg.items(), key=lambda x: -x[1][1])[:top]:
        print(f"{k[:64]:64s} {c:8d} {t / 1e6:9.3f} {t / tot:6.3f} {b / t if t else 0:10.1f}")


if __name__ == "__main__":
    main(sys.argv[1])
