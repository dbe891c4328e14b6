"""The paper's Table V grid and Fig. 2 sweep on one B200.

Table V: spline-building bandwidth for the six periodic
variants -- uniform / non-uniform x degree 3, 4, 5 -- at (Nx, Nv) =
(1000, 100000), fp64.  The paper's bandwidth counts 8 B per element
("Bandwidth = Nx x Nv x 8 / t"); we print that figure next to ours
(16 B per element: one read + one write).
Fig. 2: one Algorithm-2 advection step, GLUPS = Nx Nv 1e-9 / t
(Eq. 7), Nx = 1024, Nv = 100 ... 100000, the same six variants.

Non-uniform = the sin-map mesh.  Timing: CUDA
events on the launching stream around K back-to-back launches after W
warm-ups; the input is restored and L2 flushed (256 MB) before each timed
group, outside the events.  Prints one JSON object per line; with --out the
lines are also written to a file.

  python tools/table5.py [--steps 40] [--warmup 3] [--out profiles/r02/table5.jsonl]
"""
from __future__ import annotations

import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

from paper_conf_sc_asahilbpbgo24_b200 import PERIODIC, SplineBuilder, inputs  # noqa: E402

# the paper's A100 column of Table V (GB/s at 8 B per element), context only
PAPER_A100 = {("uniform", 3): 268.6, ("uniform", 4): 252.6, ("uniform", 5): 251.3,
              ("sin", 3): 208.4, ("sin", 4): 169.9, ("sin", 5): 142.2}


def time_launches(fn, x, pristine, steps, warmup):
    """ms per launch: `steps` launches captured in one CUDA graph and replayed
    (Python's per-call overhead would otherwise dominate the small batches)."""
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    for _ in range(warmup):
        fn(x)
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g):
        for _ in range(steps):
            fn(x)
    x.copy_(pristine)
    flush.fill_(1)
    s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize()
    s.record()
    g.replay()
    e.record()
    torch.cuda.synchronize()
    return s.elapsed_time(e) / steps


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--steps", type=int, default=40)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--out", default=None)
    ap.add_argument("--nv", default="100,1000,10000,100000")
    args = ap.parse_args()
    out = open(args.out, "w") if args.out else None

    def emit(d):
        line = json.dumps(d)
        print(line, flush=True)
        if out:
            out.write(line + "\n")

    torch.cuda.set_device(0)
    # ---- Table V: solve only (the build), Nx = 1000, batch-contiguous; Nv = 1e5 is the
    # paper's point, the sweep over Nv (100 ... 1e5) the build-only batch sweep
    from paper_conf_sc_asahilbpbgo24_b200 import last_kernel
    nx = 1000
    for mesh in ("uniform", "sin"):
        for p in (3, 4, 5):
            sb = SplineBuilder(p, nx, PERIODIC, inputs.breakpoints(nx, mesh))
            info = sb.info()
            for nv in [int(v) for v in args.nv.split(",")]:
                pristine = torch.from_numpy(inputs.rhs(sb.n, nv, seed=1234)).cuda()
                x = pristine.clone()
                ms = time_launches(sb.solve_, x, pristine, args.steps, args.warmup)
                emit({"table": "V", "mesh": "uniform" if mesh == "uniform" else "non-uniform (sin map)",
                      "degree": p, "nx": nx, "nv": nv, "ms": ms, "rhs_per_s": nv / (ms / 1e3),
                      "gbs_16B": 16.0 * nx * nv / (ms / 1e3) / 1e9, "gbs_paper_8B": 8.0 * nx * nv / (ms / 1e3) / 1e9,
                      "paper_a100_gbs_8B": PAPER_A100[(mesh, p)] if nv == 100000 else None,
                      "q_band": [info["q_kl"], info["q_ku"]], "k": info["k"], "layout": "batch-contiguous",
                      "kernel": last_kernel()})
                del x, pristine
    # ---- Fig. 2: one advection step, Nx = 1024, Nv sweep, x contiguous
    nx = 1024
    for mesh in ("uniform", "sin"):
        for p in (3, 4, 5):
            sb = SplineBuilder(p, nx, PERIODIC, inputs.breakpoints(nx, mesh))
            for nv in [int(v) for v in args.nv.split(",")]:
                pristine = torch.from_numpy(np.ascontiguousarray(inputs.rhs(sb.n, nv, seed=1234).T)).cuda()
                x = pristine.clone()
                v = -1.0 + 2.0 * np.arange(nv) / nv
                shift = torch.from_numpy(v * 2.5 / nx).cuda()
                ms = time_launches(lambda t: sb.advect_(t, shift), x, pristine, args.steps, args.warmup)
                ms_solve = time_launches(sb.solve_, x, pristine, args.steps, args.warmup)
                emit({"figure": "2", "mesh": "uniform" if mesh == "uniform" else "non-uniform (sin map)",
                      "degree": p, "nx": nx, "nv": nv, "ms": ms, "glups": nx * nv * 1e-9 / (ms / 1e3),
                      "gbs_16B": 16.0 * nx * nv / (ms / 1e3) / 1e9, "layout": "point-contiguous (x fastest)",
                      "ms_build_only": ms_solve, "q_band": [sb.info()["q_kl"], sb.info()["q_ku"]]})
                del x, pristine
    if out:
        out.close()


if __name__ == "__main__":
    main()
