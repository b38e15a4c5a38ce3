"""Diagnostics: SCAN over a list of (n, m, layout) shapes (max rel err, bad rows/systems)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import oracle  # noqa: E402
import trigen  # noqa: E402
import paper_conf_icpp_kimwch11_b200 as tri  # noqa: E402

shapes = [(2048, 300, 0), (2048, 296, 0), (1024, 1024, 1), (1024, 300, 1), (1024, 298, 1), (896, 600, 1), (1152, 600, 1)]
for (n, m, lay) in shapes:
    arrs = trigen.generate(n, m, "f64", lay, "dd")
    plan = tri.Plan(n, m, tri.F64, lay)
    plan.variant = tri.VARIANT_SCAN
    x = plan.solve(*(torch.from_numpy(t).cuda() for t in arrs)).cpu().numpy()
    xo = oracle.solve_batch(n, m, *arrs, layout=lay)
    e = (np.abs(x - xo) / np.abs(xo))
    e2 = e.reshape(n, m).T if lay == 1 else e.reshape(m, n)
    bad = np.argwhere(e2 > 1e-10)
    print(n, m, lay, os.environ.get("TRI_SCAN_DELTA", "8"), f"err={e.max():.2e}", "bad systems", sorted(set(bad[:, 0].tolist()))[:10],
          len(set(bad[:, 0].tolist())), "rows", sorted(set(bad[:, 1].tolist()))[:6], flush=True)
