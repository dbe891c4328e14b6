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
# advection (uniform stencil and non-uniform BSPLVB), both layouts
for mesh in ("uniform", "sin"):
    sb = SplineBuilder(3, 1024, PERIODIC, inputs.breakpoints(1024, mesh))
    b = inputs.rhs(sb.n, 45, seed=5)
    sh = torch.linspace(-0.3, 0.7, 45, dtype=torch.float64).cuda()
    for dt in (np.float64, np.float32):
        sb.advect_(torch.from_numpy(np.ascontiguousarray(b.T).astype(dt)).cuda(), sh)
        sb.advect_(torch.from_numpy(b.astype(dt)).cuda(), sh)
# slabs (3-D TMA) and the 2-D tensor-product builder (warp pass + slab pass)
sb = SplineBuilder(5, 200, GREVILLE, inputs.breakpoints(inputs.n_cells(5, 200, GREVILLE), "sin"))
f = torch.from_numpy(np.random.default_rng(1).uniform(-1, 1, (3, sb.n, 40))).cuda()
sb.solve_slabs_(f, 40, 40, 3, sb.n * 40)
h1 = SplineBuilder(3, 128, PERIODIC)
h2 = SplineBuilder(5, 96, GREVILLE, inputs.breakpoints(inputs.n_cells(5, 96, GREVILLE), "sin"))
from paper_conf_sc_asahilbpbgo24_b200 import solve_2d_  # noqa: E402
solve_2d_(h1, h2, torch.from_numpy(np.random.default_rng(2).uniform(-1, 1, (5, h2.n, h1.n))).cuda())
# mixed boundary conditions (Hermite at one end, Greville at the other)
from paper_conf_sc_asahilbpbgo24_b200 import bc_mixed  # noqa: E402
bcm = bc_mixed(HERMITE, GREVILLE)
sb = SplineBuilder(5, 300, bcm, inputs.breakpoints(inputs.n_cells(5, 300, bcm), "sin"))
sb.solve_(torch.from_numpy(np.random.default_rng(3).uniform(-1, 1, (sb.n, 50))).cuda())
# spline_builder_update: a handle moved to a new mesh, then solved and advected
sb = SplineBuilder(3, 1000, PERIODIC)
for mesh in ("sin", "jitter"):
    sb.update(inputs.breakpoints(1000, mesh))
    b = inputs.rhs(sb.n, 65, seed=7)
    sb.solve_(torch.from_numpy(b).cuda())
    sb.advect_(torch.from_numpy(b).cuda(), torch.linspace(-0.3, 0.7, 65, dtype=torch.float64).cuda())
# device-side refactorisation (refactor + commit kernels), then solves on the new mesh
for p, npts, bc in ((3, 1000, PERIODIC), (5, 1000, GREVILLE), (5, 996, HERMITE)):
    N = inputs.n_cells(p, npts, bc)
    sb = SplineBuilder(p, npts, bc, inputs.breakpoints(N, "sin"), device_update=True)
    kn = torch.from_numpy(inputs.breakpoints(N, "jitter")).cuda()
    sb.update_device_(kn)
    sb.update_status()
    b = inputs.rhs(sb.n, 40, seed=8, degree=p, bc=bc)
    sb.solve_(torch.from_numpy(b).cuda())
torch.cuda.synchronize()
print("sanitize run done")
