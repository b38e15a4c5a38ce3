"""Run SPLIT at every k on one shape, one process per k (a device fault kills
only that process); prints k, launches, plan, status and max rel err vs SCAN."""
import subprocess
import sys

ROOT = __file__.rsplit("/scripts/", 1)[0]
CODE = r'''
import sys, numpy as np, torch
sys.path.insert(0, "{root}")
import paper_conf_icpp_kimwch11_b200 as tri
n, m, layout, dt, k, tma = {n}, {m}, {layout}, "{dt}", {k}, {tma}
torch.manual_seed(0)
tdt = torch.float64 if dt == "f64" else torch.float32
N = n * m
a = torch.rand(N, dtype=torch.float64) - 0.5; c = torch.rand(N, dtype=torch.float64) - 0.5
b = 2.0 + torch.rand(N, dtype=torch.float64); d = torch.rand(N, dtype=torch.float64)
dev = [t.to(tdt).cuda() for t in (a, b, c, d)]
ref = tri.Plan(n, m, tri.F64 if dt == "f64" else tri.F32, layout)
xr = ref.solve(*dev).double().cpu()
p = tri.Plan(n, m, tri.F64 if dt == "f64" else tri.F32, layout)
p.set_option(tri.OPT_TMA, tma)
p.variant = tri.VARIANT_SPLIT
p.k = k
x = p.solve(*dev)
torch.cuda.synchronize()
err = float(((x.double().cpu() - xr).abs() / xr.abs().clamp_min(1e-30)).max())
print("k", k, "launches", p.launches, "err %.2e" % err, p.describe())
'''
n, m, layout, dt = int(sys.argv[1]), int(sys.argv[2]), int(sys.argv[3]), sys.argv[4]
tma = int(sys.argv[5]) if len(sys.argv) > 5 else 1
ks = range(0, n.bit_length())
for k in ks:
    r = subprocess.run([sys.executable, "-c", CODE.format(root=ROOT, n=n, m=m, layout=layout, dt=dt, k=k, tma=tma)],
                       capture_output=True, text=True, timeout=300)
    out = r.stdout.strip() or [l for l in r.stderr.strip().splitlines() if "Error" in l or "error" in l][-3:]
    print(k, "rc", r.returncode, out, flush=True)
