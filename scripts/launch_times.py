"""Per-launch GPU times of a command under ncu (cold, serialised; for the
kernel SHARE of a step only).  usage: python scripts/launch_times.py CMD..."""
import csv
import io
import subprocess
import sys

cmd = ["ncu", "--metrics", "gpu__time_duration.sum", "--clock-control", "none", "--csv"] + sys.argv[1:]
out = subprocess.run(cmd, capture_output=True, text=True).stdout
rows = [r for r in csv.reader(io.StringIO("\n".join(l for l in out.splitlines() if l.startswith('"'))))]
if not rows:
    print(out[-2000:])
    sys.exit(1)
hdr = rows[0]
ki, vi, ui, gi, bi = (hdr.index(k) for k in ("Kernel Name", "Metric Value", "Metric Unit", "Grid Size", "Block Size"))
for r in rows[1:]:
    v = float(r[vi].replace(",", ""))
    us = v / 1e3 if r[ui] == "ns" else v * 1e3 if r[ui] == "ms" else v
    print(f"{us:10.1f} us  grid {r[gi]:>14} block {r[bi]:>12}  {r[ki][:90]}")
