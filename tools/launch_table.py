"""Per-launch table (time, DRAM bytes, GB/s) of an ncu --metrics ... --csv launch list."""
import collections
import csv
import sys


def main(path):
    rows = list(csv.reader(open(path)))
    hi = [i for i, r in enumerate(rows) if "Kernel Name" in r][0]
    h = rows[hi]
    ki, mi, vi, ii = h.index("Kernel Name"), h.index("Metric Name"), h.index("Metric Value"), h.index("ID")
    per = collections.OrderedDict()
    for r in rows[hi + 1:]:
        if len(r) <= vi:
            continue
        try:
            v = float(r[vi].replace(",", ""))
        except ValueError:
            continue
        d = per.setdefault(int(r[ii]), {"name": r[ki]})
        d[r[mi]] = v
    for i, d in per.items():
        t = d.get("gpu__time_duration.sum", 0.0)
        rd, wr = d.get("dram__bytes_read.sum", 0.0), d.get("dram__bytes_write.sum", 0.0)
        nm = d["name"].split("(")[0].replace("void ", "").replace("buffalo::", "").replace("<unnamed>::", "")
        print(f"{i:6d} {nm[:44]:44s} {t / 1e3:9.1f} us  R {rd / 1e6:8.1f} MB  W {wr / 1e6:8.1f} MB  "
              f"{(rd + wr) / max(t, 1):6.0f} GB/s")


if __name__ == "__main__":
    main(sys.argv[1])
