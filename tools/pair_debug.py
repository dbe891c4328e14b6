"""Diagnostic: run the pair tile kernel (SB_TILE_PAIR=2) on growing batches and
report parity against the oracle (2+ tiles per cluster)."""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import oracle  # noqa: E402
from paper_conf_sc_asahilbpbgo24_b200 import SplineBuilder, inputs, last_kernel  # noqa: E402

for deg, npts, bc, mesh in [(3, 1000, 0, "uniform"), (5, 1000, 1, "sin")]:
    N = inputs.n_cells(deg, npts, bc)
    x = inputs.breakpoints(N, mesh)
    sb = SplineBuilder(deg, npts, bc, x)
    o = oracle.Oracle(deg, npts, bc, x)
    for B in (64, 96, 32 * 74, 32 * 74 * 2 + 5, 100000):
        b = inputs.rhs(sb.n, B, seed=5, degree=deg, bc=bc)
        t = torch.from_numpy(b).cuda()
        sb.solve_(t)
        torch.cuda.synchronize()
        got = t.cpu().numpy()
        idx = np.unique(np.r_[0, B - 1, np.random.default_rng(1).choice(B, min(B, 300), replace=False)])
        err = oracle.rel_coef_error(got[:, idx], o.solve(np.ascontiguousarray(b[:, idx])))
        print(deg, bc, B, last_kernel(), f"{err:.2e}", flush=True)
