"""Diagnostic: per-warp clock64 timeline of the tile kernel (library built
with -DSB_TRACE, loaded through SB_LIB_PATH).  Prints, per compute warp, the
mean cycles from tile start to each trace point, relative to the B2 release."""
import ctypes
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

import bench  # noqa: E402
from paper_conf_sc_asahilbpbgo24_b200 import SplineBuilder, _lib, inputs  # noqa: E402

wl = sys.argv[1] if len(sys.argv) > 1 else "C3G"
deg, npts, bc, mesh, B, dt, layout, desc = bench.WORKLOADS[wl]
n = inputs.nbasis(deg, npts, bc)
sb = SplineBuilder(deg, npts, bc, inputs.breakpoints(inputs.n_cells(deg, npts, bc), mesh))
x = torch.from_numpy(bench.make_rhs(deg, n, bc, B, 0, layout, dt)).cuda()
for _ in range(3):
    sb.solve_(x)
torch.cuda.synchronize()
NB, NT, NW, NP = 4, 8, 16, 9
OUT = os.environ.get("TRACE_OUT")
buf = np.zeros(NB * NT * NW * NP, dtype=np.int64)
import paper_conf_sc_asahilbpbgo24_b200 as pkg
lib = pkg.load_library()
rc = lib.sb_trace_dump(ctypes.c_void_p(buf.ctypes.data), ctypes.c_size_t(buf.nbytes))
assert rc == 0, rc
t = buf.reshape(NB, NT, NW, NP).astype(np.float64)
if OUT:
    np.save(OUT, buf.reshape(NB, NT, NW, NP))
names = ["start", "loaded", "gamma", "preB2", "postB2", "preB3", "postB3", "end", "fullwait"]
order = [0, 8, 1, 2, 3, 4, 5, 6, 7]
live = t[0, 1, :, 0] != 0
nw = int(live.sum()) - 1  # the last traced warp is the corner/producer warp
print(wl, "compute warps", nw)
# relative to the B2 release of the same tile (max over warps of postB2)
for b in range(NB):
    for it in range(1, NT):
        ref = t[b, it, :nw, 4].max()
        tile0 = t[b, it, :nw, 0].min()
        print(f"block {b} tile {it}: tile len {t[b, it, :nw, 7].max() - tile0:.0f} cyc, start->B2 {ref - tile0:.0f}")
print("mean over blocks/tiles 1..7, cycles relative to B2 release:")
print("warp " + " ".join(f"{names[o]:>8s}" for o in order))
for w in range(nw):
    rel = [np.mean([t[b, it, w, o] - t[b, it, :nw, 4].max() for b in range(NB) for it in range(1, NT)]) for o in order]
    print(f"{w:4d} " + " ".join(f"{r:8.0f}" for r in rel))
cw = nw
print("corner warp (start, TMA issued, x1 done) relative to the compute warps' B2 arrival max of the same tile and of tile+1:")
for b in range(NB):
    for it in range(1, NT - 1):
        r0 = t[b, it, :nw, 3].max()
        print(f"b{b} it{it}: start {t[b, it, cw, 0] - r0:7.0f} issued {t[b, it, cw, 8] - r0:7.0f} cfull {t[b, it, cw, 2] - r0:7.0f} spmv {t[b, it, cw, 3] - r0:7.0f} x1 {t[b, it, cw, 1] - r0:7.0f}"
              f" | gamma-warp loaded(it) {t[b, it, 0, 1] - r0:7.0f} gamma(it) {t[b, it, 0, 2] - r0:7.0f}")
