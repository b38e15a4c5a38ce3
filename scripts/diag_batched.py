"""Diagnostics: one BATCHED-layout shape per process (n ms nb dtype): max rel err."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import oracle  # noqa: E402
import trigen  # noqa: E402
import paper_conf_icpp_kimwch11_b200 as tri  # noqa: E402

n, ms, nb, dt = int(sys.argv[1]), int(sys.argv[2]), int(sys.argv[3]), sys.argv[4]
arrs = trigen.generate(n, ms * nb, dt, 0, "dd")
grid = [np.ascontiguousarray(t.reshape(nb, ms, n).transpose(0, 2, 1)).reshape(-1) for t in arrs]
plan = tri.Plan.batched(n, ms, nb, tri.F64 if dt == "f64" else tri.F32)
print(plan.describe(), flush=True)
xg = plan.solve(*(torch.from_numpy(t).cuda() for t in grid)).cpu().numpy()
x = np.ascontiguousarray(xg.reshape(nb, n, ms).transpose(0, 2, 1)).reshape(-1)
xo = oracle.solve_batch(n, ms * nb, *arrs)
print(n, ms, nb, dt, "err", float(np.max(np.abs(x - xo) / np.abs(xo))), flush=True)
