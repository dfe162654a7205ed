"""Summarise ncu evidence into profiles/ (committed).

python scripts/make_profile_summary.py <tag>
  reads gpurun_out/launches_<tag>.csv, force_<tag>.ncu-rep, build_<tag>.ncu-rep,
  bench_<tag>.json and writes profiles/<tag>_launches.md, <tag>_force_ncu.json,
  <tag>_kernels_ncu.md, <tag>_bench.json.
"""
import collections
import csv
import io
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
OUT = os.path.join(ROOT, "gpurun_out")
PROF = os.path.join(ROOT, "profiles")

METRICS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
           "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "sm__throughput.avg.pct_of_peak_sustained_elapsed",
           "smsp__issue_active.avg.pct_of_peak_sustained_active", "smsp__inst_executed.sum",
           "sm__warps_active.avg.pct_of_peak_sustained_active", "launch__registers_per_thread",
           "sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active", "l1tex__t_sector_hit_rate.pct",
           "lts__t_sector_hit_rate.pct", "smsp__thread_inst_executed_per_inst_executed.ratio"]


def raw(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    h, u = rows[0], rows[1]
    res = []
    for r in rows[2:]:
        d = dict(zip(h, r))
        res.append({"kernel": d.get("Kernel Name", ""), **{m: d.get(m) for m in METRICS},
                    "units": {m: u[h.index(m)] for m in METRICS if m in h}})
    return res


def to_bytes(v, unit):
    f = float(v)
    return f * {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}.get(unit, 1)


def main(tag):
    os.makedirs(PROF, exist_ok=True)
    # launch list: share of the step per kernel (cold-cache, serialised)
    lp = os.path.join(OUT, f"launches_{tag}.csv")
    if os.path.exists(lp):
        txt = open(lp).read()
        txt = txt[txt.index('"ID"'):] if '"ID"' in txt else txt
        rows = list(csv.DictReader(io.StringIO(txt)))
        dur = collections.defaultdict(float)
        cnt = collections.Counter()
        for r in rows:
            if r.get("Metric Name") != "gpu__time_duration.sum":
                continue
            name = r["Kernel Name"].split("(")[0].split("::")[-1]
            v = float(r["Metric Value"].replace(",", ""))
            unit = r.get("Metric Unit", "ns")
            v *= {"ns": 1e-6, "us": 1e-3, "usecond": 1e-3, "nsecond": 1e-6, "msecond": 1.0, "ms": 1.0}.get(unit, 1e-6)
            dur[name] += v
            cnt[name] += 1
        tot = sum(dur.values())
        with open(os.path.join(PROF, f"{tag}_launches.md"), "w") as f:
            f.write(f"# ncu launch list ({tag}): `ncu --metrics gpu__time_duration.sum --clock-control none` of "
                    f"`python bench.py --steps 2 --warmup 1 --no-cpu-baseline --no-e2e`\n\n"
                    "Cold-cache, serialised per-launch times: compare shares, not absolutes.\n\n"
                    "| kernel | launches | total ms | share |\n|---|---|---|---|\n")
            for k, v in sorted(dur.items(), key=lambda x: -x[1]):
                f.write(f"| {k} | {cnt[k]} | {v:.3f} | {100 * v / tot:.1f}% |\n")
            f.write(f"| **all** | {sum(cnt.values())} | {tot:.3f} | 100% |\n")
    fr = os.path.join(OUT, f"force_{tag}.ncu-rep")
    if os.path.exists(fr):
        k = raw(fr)[0]
        u = k["units"]
        traffic = to_bytes(k["dram__bytes_read.sum"], u["dram__bytes_read.sum"]) + \
            to_bytes(k["dram__bytes_write.sum"], u["dram__bytes_write.sum"])
        d = {"tag": tag, "kernel": k["kernel"], "command": "ncu --set full --clock-control none --import-source on "
             "-k regex:k_force -s 1 -c 1 python scripts/run_pass.py --passes 2 (disks N=1e7, theta=0.5)",
             "dram_bytes_per_launch": traffic, "metrics": {m: k[m] for m in METRICS}, "units": u,
             # the configuration of the capture (bench.py uses a capture's traffic only for the same one)
             "config": {"workload": "disks", "n": 10_000_000, "theta": 0.5, "precision": 32, "multipole": 1,
                        "key_bits": 16}}
        with open(os.path.join(PROF, f"{tag}_force_ncu.json"), "w") as f:
            json.dump(d, f, indent=1)
    br = os.path.join(OUT, f"build_{tag}.ncu-rep")
    if os.path.exists(br):
        ks = raw(br)
        with open(os.path.join(PROF, f"{tag}_kernels_ncu.md"), "w") as f:
            f.write(f"# ncu --set full of the non-force kernels ({tag}), disks N=1e7\n\n"
                    "| kernel | ms | DRAM read MB | DRAM write MB | DRAM % of peak | issue % | regs |\n"
                    "|---|---|---|---|---|---|---|\n")
            for k in ks:
                u = k["units"]
                ms = float(k["gpu__time_duration.sum"]) * {"ms": 1, "msecond": 1, "us": 1e-3, "usecond": 1e-3,
                                                           "ns": 1e-6, "nsecond": 1e-6}.get(
                    u.get("gpu__time_duration.sum"), 1)
                f.write(f"| {k['kernel'].split('(')[0].split('::')[-1][:40]} | {ms:.3f} | "
                        f"{to_bytes(k['dram__bytes_read.sum'], u['dram__bytes_read.sum']) / 1e6:.1f} | "
                        f"{to_bytes(k['dram__bytes_write.sum'], u['dram__bytes_write.sum']) / 1e6:.1f} | "
                        f"{k['gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed']} | "
                        f"{k['smsp__issue_active.avg.pct_of_peak_sustained_active']} | "
                        f"{k['launch__registers_per_thread']} |\n")
    bj = os.path.join(OUT, f"bench_{tag}.json")
    if os.path.exists(bj):
        line = open(bj).read().strip().splitlines()[-1]
        with open(os.path.join(PROF, f"{tag}_bench.json"), "w") as f:
            f.write(line + "\n")


if __name__ == "__main__":
    main(sys.argv[1])
