"""Print the key ncu metrics of a .ncu-rep (speed of light, issue, stalls, memory)."""
import csv
import io
import subprocess
import sys

rep = sys.argv[1]
raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(raw)))
h, u = rows[0], rows[1]
keys = ["gpu__time_duration.sum", "sm__throughput.avg.pct_of_peak_sustained_elapsed",
        "smsp__issue_active.avg.pct_of_peak_sustained_active", "smsp__inst_executed.sum",
        "sm__warps_active.avg.pct_of_peak_sustained_active", "launch__registers_per_thread",
        "l1tex__t_sector_hit_rate.pct", "lts__t_sector_hit_rate.pct", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active",
        "sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active", "smsp__thread_inst_executed_per_inst_executed.ratio",
        "l1tex__throughput.avg.pct_of_peak_sustained_active"]
for r in rows[2:]:
    d = dict(zip(h, r))
    print("kernel:", d.get("Kernel Name", "")[:80])
    for k in keys:
        if k in d:
            print(f"  {k:70s} {d[k]} {u[h.index(k)]}")
    st = [(k, float(d[k])) for k in h if k.startswith("smsp__average_warp_latency_issue_stalled") or
          (k.startswith("smsp__pcsamp_warps_issue_stalled") and not k.endswith("not_issued"))]
    st = [(k, v) for k, v in st if v > 0]
    tot = sum(v for _, v in st) or 1
    for k, v in sorted(st, key=lambda x: -x[1])[:12]:
        print(f"  stall {k.replace('smsp__pcsamp_warps_issue_stalled_', ''):60s} {100 * v / tot:5.1f}%")
