"""Per-instruction execution counts / stall samples from an ncu report (source page, SASS)."""
import csv
import io
import subprocess
import sys

rep = sys.argv[1]
thr = float(sys.argv[2]) if len(sys.argv) > 2 else 0.002
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"], capture_output=True,
                     text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
h = rows[1]
data = rows[2:]
iS, iE = h.index("Source"), h.index("Instructions Executed")
iW, iT = h.index("Warp Stall Sampling (All Samples)"), h.index("Avg. Threads Executed")
num = lambda x: int(x) if x.isdigit() else 0
tot = sum(num(r[iE]) for r in data)
totw = sum(num(r[iW]) for r in data)
print("total inst", tot, "samples", totw, "sass lines", len(data))
for r in data:
    e, w = num(r[iE]), num(r[iW])
    if e > tot * thr or w > totw * 0.01:
        print(f"{e / tot * 100:5.2f}% {w / totw * 100:5.1f}%s thr={r[iT]:>5} {r[iS][:100]}")
