"""One SPLIT solve (n m layout dtype k [tma]) + synchronize; for compute-sanitizer."""
import sys
import torch
sys.path.insert(0, __file__.rsplit("/scripts/", 1)[0])
import paper_conf_icpp_kimwch11_b200 as tri  # noqa: E402
n, m, layout, dt, k = int(sys.argv[1]), int(sys.argv[2]), int(sys.argv[3]), sys.argv[4], int(sys.argv[5])
tma = int(sys.argv[6]) if len(sys.argv) > 6 else 1
tdt = torch.float64 if dt == "f64" else torch.float32
N = n * m
g = torch.Generator().manual_seed(0)
a, c = (torch.rand(N, generator=g, dtype=torch.float64) - 0.5 for _ in range(2))
b, d = 2.0 + torch.rand(N, generator=g, dtype=torch.float64), torch.rand(N, generator=g, dtype=torch.float64)
dev = [t.to(tdt).cuda() for t in (a, b, c, d)]
p = tri.Plan(n, m, tri.F64 if dt == "f64" else tri.F32, layout)
p.set_option(tri.OPT_TMA, tma)
p.variant = tri.VARIANT_SPLIT
p.k = k
print(p.describe(), flush=True)
x = p.solve(*dev)
torch.cuda.synchronize()
print("ok", float(x.double().abs().max()))
