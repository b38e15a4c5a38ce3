"""Attribute an ncu source capture of the fused kernel to warp roles.
usage: python scripts/ncu_roles.py REPORT  (needs -lineinfo + --import-source)
Each SASS instruction is mapped to the k_fused.cuh line it came from (inlined
helpers inherit the role of the nearest preceding k_fused.cuh instruction)."""
import csv
import io
import subprocess
import sys

ROLES = [(1, 232, None), (233, 242, "setup"), (243, 399, "PCR"), (400, 410, "handoff-only"), (411, 509, "TC"),
         (510, 628, "TR"), (629, 10000, "TB")]

rep = sys.argv[1]
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                     capture_output=True, text=True).stdout
cur_file, cur_line = None, None
inst = []  # (addr, file, line, exec, samples, sass)
hdr = None
for row in csv.reader(io.StringIO(out)):
    if not row:
        continue
    if row[0] == "File Path":
        cur_file = row[1]
        continue
    if row[0] == "Line No":
        hdr = row
        continue
    if hdr is None:
        continue
    if row[0] not in ("", "-"):
        if row[0].isdigit():
            cur_line = int(row[0])
        continue
    if row[2] in ("...", "-", ""):
        continue
    try:
        ex = int(row[hdr.index("Instructions Executed")])
        smp = int(row[hdr.index("Warp Stall Sampling (All Samples)")])
    except ValueError:
        continue
    reasons = {h[6:]: int(v) for h, v in zip(hdr, row) if h.startswith("stall_") and "Not Issued" not in h
               and v.isdigit() and int(v) > 0}
    inst.append((int(row[2], 16), cur_file, cur_line, ex, smp, row[3], reasons))
# an inlined instruction is listed once per source line it maps to: keep one
# entry per address, preferring the k_fused.cuh attribution
best = {}
for t in inst:
    if t[0] not in best or (t[1].endswith("k_fused.cuh") and not best[t[0]][1].endswith("k_fused.cuh")):
        best[t[0]] = t
inst = sorted(best.values())
role_of = {}
last = "setup"
for addr, f, ln, ex, smp, sass, *_ in inst:
    if f.endswith("k_fused.cuh"):
        for lo, hi, name in ROLES:
            if lo <= ln <= hi:
                last = name or last  # helpers (None) inherit the caller's role
                break
    role_of[addr] = last
WAITOPS = ("TRYWAIT", "NANOSLEEP", "PHASECHK", "YIELD")
for addr, f, ln, ex, smp, sass, *_ in inst:
    if any(w in sass for w in WAITOPS):
        role_of[addr] = "wait-loops"
tot = {}
for addr, f, ln, ex, smp, sass, *_ in inst:
    r = role_of[addr]
    t = tot.setdefault(r, [0, 0, 0, 0])
    t[0] += ex
    t[1] += smp
    if sass.split()[0].lstrip("@!P0123456789T ").startswith(("DFMA", "DMUL", "DADD")) or " DFMA" in sass or " DMUL" in sass or " DADD" in sass:
        t[2] += ex
    if "SHFL" in sass:
        t[3] += ex
rs = {}
for addr, f, ln, ex, smp, sass, why in inst:
    d = rs.setdefault(role_of[addr], {})
    for k, v in why.items():
        d[k] = d.get(k, 0) + v
S = sum(t[1] for t in tot.values())
print(f"{'role':14s} {'warp-inst':>12s} {'fp64':>12s} {'shfl':>10s} {'samples%':>9s}")
for r, t in sorted(tot.items(), key=lambda kv: -kv[1][0]):
    top = sorted(rs.get(r, {}).items(), key=lambda kv: -kv[1])[:5]
    print(f"{r:14s} {t[0]:12d} {t[2]:12d} {t[3]:10d} {100 * t[1] / max(1, S):8.1f}%  " +
          " ".join(f"{k}:{v}" for k, v in top))

if len(sys.argv) > 2:
    want = sys.argv[2]
    rows = [(ex, smp, addr, ln, sass) for addr, f, ln, ex, smp, sass, *_ in inst if role_of[addr] == want]
    rows.sort(reverse=True)
    for ex, smp, addr, ln, sass in rows[:int(sys.argv[3]) if len(sys.argv) > 3 else 40]:
        print(f"{ex:10d} {smp:6d} {hex(addr)[-5:]} L{ln:<5} {sass}")
