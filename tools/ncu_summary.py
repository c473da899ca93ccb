"""Key metrics of an ncu --set full report (per launch)."""
import csv
import io
import subprocess
import sys

KEYS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "lts__t_sector_hit_rate.pct",
        "lts__t_bytes.sum", "sm__warps_active.avg.pct_of_peak_sustained_active",
        "launch__registers_per_thread", "sm__throughput.avg.pct_of_peak_sustained_elapsed",
        "l1tex__t_bytes.sum", "sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed",
        "TPC.TriageCompute.sm__pipe_tensor_cycles_active_realtime.avg.pct_of_peak_sustained_elapsed",
        "smsp__inst_executed.sum", "launch__grid_size", "launch__block_size",
        "lts__throughput.avg.pct_of_peak_sustained_elapsed"]


def main(path):
    out = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    h, units = rows[0], rows[1]
    for r in rows[2:]:
        print(r[h.index("Kernel Name")][:70])
        for k in KEYS:
            if k in h:
                print(f"  {k:75s} {r[h.index(k)]} {units[h.index(k)]}")
        stalls = [(h[i], r[i]) for i in range(len(h))
                  if h[i].startswith("smsp__average_warp_latency_issue_stalled") or
                  (h[i].startswith("smsp__pcsamp_warps_issue_stalled") and not h[i].endswith("not_issued"))]
        vals = []
        for k, v in stalls:
            try:
                vals.append((float(v.replace(",", "")), k))
            except ValueError:
                pass
        for v, k in sorted(vals, reverse=True)[:8]:
            print(f"  stall {k:70s} {v}")


if __name__ == "__main__":
    main(sys.argv[1])
