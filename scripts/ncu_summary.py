"""Summarise an ncu report (.ncu-rep) into a short text file for profiles/.
usage: python scripts/ncu_summary.py REPORT OUT.txt [traffic_json n m k [variant [layout]]]"""
import csv
import io
import json
import subprocess
import sys

rep, out = sys.argv[1], sys.argv[2]
raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(raw)))
hdr, units = rows[0], rows[1]
keys = ["Kernel Name", "gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "dram__throughput.avg.pct_of_peak_sustained_elapsed", "sm__throughput.avg.pct_of_peak_sustained_elapsed",
        "sm__inst_executed_pipe_fp64.avg.pct_of_peak_sustained_active", "sm__warps_active.avg.pct_of_peak_sustained_active",
        "launch__registers_per_thread", "launch__grid_size", "launch__block_size",
        "smsp__inst_executed.sum", "l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum",
        "lts__t_sectors_srcunit_tex_op_read.sum", "launch__shared_mem_per_block_dynamic"]
lines = []
for r in rows[2:]:
    d = dict(zip(hdr, r))
    u = dict(zip(hdr, units))
    lines.append("kernel: " + d.get("Kernel Name", "?"))
    for k in keys[1:]:
        if k in d:
            lines.append(f"  {k} = {d[k]} {u.get(k, '')}")
    stalls = []
    for h, v in d.items():
        if h.startswith("smsp__pcsamp_warps_issue_stalled_") and not h.endswith("not_issued"):
            try:
                stalls.append((float(v), h.replace("smsp__pcsamp_warps_issue_stalled_", "")))
            except ValueError:
                pass
    tot = sum(v for v, _ in stalls) or 1
    lines.append("  stall samples: " + ", ".join(f"{n} {v / tot:.0%}" for v, n in sorted(stalls, reverse=True)[:8]))
open(out, "w").write("\n".join(lines) + "\n")
print("\n".join(lines))
if len(sys.argv) > 3:
    # the solve's DRAM bytes: every launch in the report (profile exactly one solve's launches)
    scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}
    tb, names = 0.0, []
    for r in rows[2:]:
        d = dict(zip(hdr, r))
        u = dict(zip(hdr, units))
        tb += sum(float(d[k].replace(",", "")) * scale.get(u[k], 1) for k in ("dram__bytes_read.sum", "dram__bytes_write.sum"))
        names.append(d["Kernel Name"])
    rec = {"source": rep, "kernels": names, "dram_bytes_per_launch": tb, "n": int(sys.argv[4]), "m": int(sys.argv[5]),
           "k": int(sys.argv[6])}
    if len(sys.argv) > 7:
        rec["variant"] = int(sys.argv[7])
    if len(sys.argv) > 8:
        rec["layout"] = int(sys.argv[8])
    json.dump(rec, open(sys.argv[3], "w"), indent=1)
