"""Hot SASS lines of one kernel from `ncu --page source --csv --print-source sass` output
(warp-stall samples and executed instructions per line).  Diagnostic only."""
import csv
import sys


def main(path, top=30):
    rows = list(csv.reader(open(path)))
    hi = [i for i, r in enumerate(rows) if r and r[0] == "Address"][0]
    h = rows[hi]
    si, ws, ie = h.index("Source"), h.index("Warp Stall Sampling (All Samples)"), h.index("Instructions Executed")
    stall_cols = [i for i, k in enumerate(h) if k.startswith("stall_") and "Not Issued" not in k]

    def num(x):
        try:
            return int(x)
        except ValueError:
            return 0
    data = [r for r in rows[hi + 1:] if len(r) > max(si, ws, ie)]
    tot = sum(num(r[ws]) for r in data) or 1
    print("samples", tot, "instructions", sum(num(r[ie]) for r in data))
    for i, r in sorted(enumerate(data), key=lambda x: -num(x[1][ws]))[:top]:
        st = sorted(((num(r[c]), h[c][6:]) for c in stall_cols), reverse=True)[:2]
        print(f"{i:5d} {num(r[ws]):7d} {100 * num(r[ws]) / tot:5.1f}% {num(r[ie]):10d} {st}  {r[si].strip()[:70]}")


if __name__ == "__main__":
    main(sys.argv[1], int(sys.argv[2]) if len(sys.argv) > 2 else 30)
