"""Small solves of every kernel family for compute-sanitizer runs."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402
import torch  # noqa: E402

from paper_conf_sc_asahilbpbgo24_b200 import GREVILLE, HERMITE, PERIODIC, SplineBuilder, inputs  # noqa: E402

cases = [(3, 1000, PERIODIC, "uniform", 257, "batch"), (5, 996, HERMITE, "sin", 96, "batch"),
         (5, 1000, GREVILLE, "sin", 64, "batch"), (3, 1024, PERIODIC, "uniform", 70, "point"),
         (3, 3000, PERIODIC, "uniform", 33, "batch"), (3, 16, PERIODIC, "uniform", 8, "batch"),
         (3, 1000, PERIODIC, "uniform", 37, "batch")]
for p, npts, bc, mesh, B, layout in cases:
    N = inputs.n_cells(p, npts, bc)
    sb = SplineBuilder(p, npts, bc, inputs.breakpoints(N, mesh))
    b = inputs.rhs(sb.n, B, seed=3, degree=p, bc=bc)
    for dt in (np.float64, np.float32):
        t = torch.from_numpy((b if layout == "batch" else np.ascontiguousarray(b.T)).astype(dt)).cuda()
        sb.solve_(t)
torch.cuda.synchronize()
print("sanitize run done")
