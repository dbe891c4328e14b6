"""ncu driver: a few device-side refactorisations (spline_builder_update_device)
of the C3 Greville shape (p = 5, n = 1000), alternating two meshes."""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_sc_asahilbpbgo24_b200 import GREVILLE, SplineBuilder, inputs  # noqa: E402

N = inputs.n_cells(5, 1000, GREVILLE)
u = np.arange(N + 1) / N
xs = [inputs.breakpoints(N, "sin"), u + 0.3 * np.sin(2 * np.pi * u) / (2 * np.pi)]
xs[1][0], xs[1][-1] = 0.0, 1.0
sb = SplineBuilder(5, 1000, GREVILLE, xs[0], device_update=True)
d = [torch.from_numpy(x).cuda() for x in xs]
for i in range(int(sys.argv[1]) if len(sys.argv) > 1 else 4):
    sb.update_device_(d[i % 2])
    sb.update_status()
torch.cuda.synchronize()
print("done")
