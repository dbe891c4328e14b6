"""Minimal driver for ncu captures: W warm-up solves + K solves of one
bench workload (no timing, no oracle)."""
import argparse
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import bench  # noqa: E402
from paper_conf_sc_asahilbpbgo24_b200 import SplineBuilder, inputs  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--workload", default="C2")
ap.add_argument("--n", type=int, default=3)
ap.add_argument("--degree", type=int, default=None, help="override the workload's degree (periodic workloads)")
ap.add_argument("--solve", action="store_true", help="plain solve even for an advection workload")
args = ap.parse_args()
deg, npts, bc, mesh, B, dt, layout, desc = bench.WORKLOADS[args.workload]
if args.degree:
    deg = args.degree
n = inputs.nbasis(deg, npts, bc)
sb = SplineBuilder(deg, npts, bc, inputs.breakpoints(inputs.n_cells(deg, npts, bc), mesh))
x = torch.from_numpy(bench.make_rhs(deg, n, bc, B, 0, layout, dt)).cuda()
if args.workload in bench.ADVECT and not args.solve:
    sh = torch.from_numpy(bench.adv_shift(inputs.n_cells(deg, npts, bc), B)).cuda()
    for _ in range(args.n):
        sb.advect_(x, sh)
else:
    for _ in range(args.n):
        sb.solve_(x)
torch.cuda.synchronize()
print("done", args.workload)
