"""Per CUDA source line: executed instructions and stall samples (from ncu --print-source cuda,sass)."""
import csv
import io
import subprocess
import sys

rep = sys.argv[1]
thr = float(sys.argv[2]) if len(sys.argv) > 2 else 0.01
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
h = rows[2]
iE, iW = h.index("Instructions Executed"), h.index("Warp Stall Sampling (All Samples)")
num = lambda x: int(x) if x.isdigit() else 0
lines = [(r[0], r[1], num(r[iE]), num(r[iW])) for r in rows[3:] if len(r) > iE and r[0] not in ("", "Line No")]
tot = sum(e for _, _, e, _ in lines) or 1
totw = sum(w for _, _, _, w in lines) or 1
print(f"total inst {tot:.3e} samples {totw}")
for ln, src, e, w in lines:
    if e > tot * thr or w > totw * thr:
        print(f"{ln:>5} {100 * e / tot:5.1f}% {100 * w / totw:5.1f}%s  {src.strip()[:100]}")
