"""Top SASS instructions of an ncu source page (sass) by stall samples.
usage: ncu -i R --page source --csv --print-source=sass > s.csv; python scripts/ncu_hot.py s.csv [N]"""
import csv
import sys
from collections import Counter

rows = list(csv.reader(open(sys.argv[1])))
hdr = rows[1]
idx = {h: i for i, h in enumerate(hdr)}
data = [r for r in rows[2:] if len(r) >= len(hdr) - 1]
N = int(sys.argv[2]) if len(sys.argv) > 2 else 40
S = idx["Warp Stall Sampling (All Samples)"]
tot = sum(int(r[S] or 0) for r in data)
stall_cols = [h for h in hdr if h.startswith("stall_") and "Not Issued" not in h]
print(f"total samples {tot}, instructions {len(data)}")
cls, ex = Counter(), Counter()
for r in data:
    toks = r[idx["Source"]].split()
    if not toks:
        continue
    op = toks[1] if toks[0].startswith("@") and len(toks) > 1 else toks[0]
    op = op.split(".")[0]
    cls[op] += int(r[S] or 0)
    ex[op] += int(r[idx["Instructions Executed"]] or 0)
print("by opcode (samples, warp-instr executed):")
for op, s in cls.most_common(25):
    print(f"  {op:10s} {s:8d} {100*s/tot:5.1f}%  exec {ex[op]}")
data.sort(key=lambda r: -int(r[S] or 0))
for r in data[:N]:
    s = int(r[S] or 0)
    st = sorted(((int(r[idx[h]] or 0), h[6:]) for h in stall_cols), reverse=True)[:3]
    print(f"{r[0][-5:]} {s:7d} {100*s/tot:5.1f}%  {r[idx['Source']].strip()[:60]:60s} {st}")
