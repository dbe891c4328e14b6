#!/usr/bin/env python
"""Benchmark of the batched spline-coefficient build (BASELINE.json metric:
"RHS/s and achieved HBM GB/s (% of peak), cubic n=1000, 1e5 RHS, fp64").

A step = one in-place solve (Algorithm 1) of the whole
batch of one workload: default C2 = cubic uniform periodic, n = 1000,
1e5 RHS, fp64, batch-contiguous -- the configuration BASELINE.json's metric
is quoted on.  Inputs (800 MB) are larger than L2 (126 MB); solves are timed
in chunks of 40 back-to-back launches, the input restored and L2 flushed
between chunks outside the CUDA events.

  python bench.py [--gpus N --steps K --warmup W] [--workload C2|C3G|C3H|C4|C4F32|C5|C1]
  python bench.py --impl reference ...   # the CPU oracle, same metric/config

Multi-GPU (torchrun, one rank per GPU): weak scaling, each rank solves its
own slice [rank*B, (rank+1)*B) of a global batch (RHS index drives the RNG);
no collective on the data path, NCCL only for the barrier and the max-time
reduction.  Prints one JSON line on rank 0.
"""
from __future__ import annotations

import argparse
import json
import os
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

from paper_conf_sc_asahilbpbgo24_b200 import inputs  # noqa: E402

METRIC = "RHS/s and achieved HBM GB/s (% of peak), cubic n=1000, 1e5 RHS, fp64"
ADV_METRIC = "advection GLUPS (Eq. 7: Nx*Nv / step time), one Algorithm-2 step"
STRONG = {"C5"}            # total batch fixed, sharded over the ranks
ADVECT = {"ADV", "ADVNU"}  # one semi-Lagrangian step (Algorithm 2) per step, metric GLUPS (Eq. 7)
SLAB_W = 2048  # C4M: RHS per slab (the v*mu extent)
TWOD = {
    # name: ((degree, n_points, bc, mesh) along dim 1, same along dim 2, grids per GPU, dtype, description)
    "C6": ((3, 1024, 0, "uniform"), (3, 1024, 0, "uniform"), 64, "f64",
           "C6 2-D tensor-product build (P:59): 64 grids of 1024 x 1024, cubic uniform periodic x periodic, fp64"),
    "C6NU": ((3, 1024, 0, "sin"), (5, 1000, 1, "sin"), 64, "f64",
             "C6 2-D tensor-product build: 64 grids, dim 1 cubic non-uniform periodic n=1024 x dim 2 quintic "
             "non-uniform Greville n=1000, fp64"),
    "C6F32": ((3, 1024, 0, "uniform"), (3, 1024, 0, "uniform"), 64, "f32",
              "C6 2-D tensor-product build: 64 grids of 1024 x 1024, cubic uniform periodic, fp32"),
}
TWOD_METRIC = "2-D tensor-product build: grid points per second (n1*n2*grids / step time)"
DEVICE_INPUT_ELEMS = 4e8   # above this, inputs are generated on the device (inputs.rhs_device)
E2E_MAX_RHS = 1_000_000    # the e2e leg moves at most this many RHS through host memory

WORKLOADS = {
    # name: (degree, n_points, bc, mesh, batch per GPU (weak) or total (C5, strong), dtype, layout, description)
    "C1": (3, 16, 0, "uniform", 8, "f64", "batch", "C1 cubic uniform periodic n=16 batch=8 fp64"),
    "C2": (3, 1000, 0, "uniform", 100000, "f64", "batch",
           "C2 cubic uniform periodic n=1000 batch=1e5 fp64 batch-contiguous"),
    "C3G": (5, 1000, 1, "sin", 100000, "f64", "batch", "C3 degree-5 non-uniform (sin map) Greville n=1000 batch=1e5 fp64"),
    "C3H": (5, 996, 2, "sin", 100000, "f64", "batch", "C3 degree-5 non-uniform (sin map) Hermite n=1000 batch=1e5 fp64"),
    "C4": (3, 1024, 0, "uniform", 131072, "f64", "point",
           "C4 GYSELA slice f[64][64][32][x=1024] cubic periodic along x, x contiguous, fp64"),
    "C4F32": (3, 1024, 0, "uniform", 131072, "f32", "point",
              "C4 GYSELA slice f[64][64][32][x=1024] cubic periodic along x, x contiguous, fp32"),
    "ADV": (3, 1024, 0, "uniform", 100000, "f64", "point",
            "Algorithm 2 advection step: Nx=1024, Nv=1e5, cubic uniform periodic, x contiguous, fp64 (GLUPS)"),
    "ADVNU": (3, 1024, 0, "sin", 100000, "f64", "point",
              "Algorithm 2 advection step: Nx=1024, Nv=1e5, cubic non-uniform (sin map) periodic, fp64 (GLUPS)"),
    "C4M": (3, 1024, 0, "uniform", 131072, "f64", "slabs",
            "C4 second layout f[y=64][x=1024][v*mu=2048] cubic periodic along x (x in the middle: 64 slabs of "
            "(1024, 2048) batch-contiguous blocks, spline_builder_solve_slabs), fp64"),
    "C5": (3, 1000, 0, "uniform", 8000000, "f64", "batch",
           "C5 cubic uniform periodic n=1000, 8e6 RHS in total sharded over the GPUs (strong scaling) fp64"),
    "C5S8": (3, 1000, 0, "uniform", 1000000, "f64", "batch",
             "C5's per-GPU shard at 8 GPUs (1e6 RHS, 8 MB row pitch) on one GPU: the per-GPU rate the "
             "8-GPU strong-scaling run would see"),
}


# Practical in-place streaming ceilings on this pool (no-math read-modify-write
# kernels with the solver's access patterns, tools/stream_probe*.cu;
# profiles/r01/stream_probe*_session2.txt): batch-contiguous 16/32-RHS TMA tiles
# + st.cs writes, and flat contiguous rows (the point layout).
STREAM_CEILING_GBS = {"batch": 5681.0, "slabs": 5681.0, "point": 6372.0}


def load_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return float(d["hbm_gbs"]), "measured"
    return 6650.0, "fallback"


def load_traffic(workload):
    """dram bytes per launch from the committed ncu --set full capture."""
    p = os.path.join(ROOT, "profiles", "ncu_summary.json")
    if not os.path.exists(p):
        return None
    d = json.load(open(p))
    w = d.get(workload)
    return None if w is None else w.get("dram_bytes_per_launch")


class ClockSampler:
    """nvidia-smi clocks and throttle reasons during the timed region
    (streaming `nvidia-smi -lms`, the recipe's clocks line)."""

    Q = ("clocks.sm,clocks.max.sm,clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap,power.draw")

    def __init__(self, index=0, interval_ms=50):
        self.index = index
        self.interval_ms = interval_ms
        self.samples = []
        self._p = None
        self._t = None

    def _read(self):
        for line in self._p.stdout:
            parts = [x.strip() for x in line.strip().split(",")]
            if len(parts) == 7:
                self.samples.append(parts)

    def __enter__(self):
        try:
            self._p = subprocess.Popen(["nvidia-smi", "-i", str(self.index), f"--query-gpu={self.Q}",
                                        "--format=csv,noheader,nounits", f"-lms={self.interval_ms}"],
                                       stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self._t = threading.Thread(target=self._read, daemon=True)
            self._t.start()
            time.sleep(0.3)  # first samples before the timed region starts
        except Exception:
            self._p = None
        return self

    def __exit__(self, *a):
        if self._p is not None:
            time.sleep(0.1)
            self._p.terminate()
            try:
                self._p.wait(timeout=5)
            except Exception:
                self._p.kill()
            self._t.join(timeout=5)

    def summary(self):
        def num(x):
            try:
                return float(x)
            except ValueError:
                return None
        sm = [num(s[0]) for s in self.samples if num(s[0]) is not None]
        if not sm:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["unsampled"], "samples": 0}
        mx = [num(s[1]) for s in self.samples if num(s[1]) is not None]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[i] for s in self.samples for i in range(4) if s[2 + i].lower() == "active"})
        pw = [num(s[6]) for s in self.samples if num(s[6]) is not None]
        return {"sm_mhz": float(np.median(sm)), "sm_max_mhz": max(mx) if mx else None, "reasons": reasons,
                "samples": len(self.samples), "power_w_max": max(pw) if pw else None}


class ChunkRunner:
    """Runs m back-to-back steps.  With graphs (default) the m launches are
    captured once into a CUDA graph and replayed, so the timed region measures
    the GPU, not Python's per-call overhead (~10 us, which dominates the tiny
    C1 solve); the kernels and their arguments are identical."""

    def __init__(self, step, use_graph):
        self.step, self.use_graph, self.graphs = step, use_graph, {}

    def __call__(self, m):
        import torch
        if not self.use_graph:
            for _ in range(m):
                self.step()
            return
        g = self.graphs.get(m)
        if g is None:
            g = torch.cuda.CUDAGraph()
            with torch.cuda.graph(g):
                for _ in range(m):
                    self.step()
            self.graphs[m] = g
        g.replay()


def dist_env():
    ws = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return ws, rank, local


def use_dist(ws):
    """NCCL process group (barrier + max-over-ranks timing) when there is more
    than one rank; SB_BENCH_FORCE_DIST=1 takes the same path at world size 1
    (exercises the NCCL code on a one-GPU box)."""
    return ws > 1 or os.environ.get("SB_BENCH_FORCE_DIST") == "1"


def make_rhs(deg, n, bc, B, first, layout, dtype):
    b = inputs.rhs(n, B, seed=1234, degree=deg, bc=bc, first=first)  # (n, B) fp64
    if layout == "point":
        b = np.ascontiguousarray(b.T)
    elif layout == "slabs":  # f[y][x][v]: slab y = r // SLAB_W, column r % SLAB_W
        b = np.ascontiguousarray(b.reshape(n, B // SLAB_W, SLAB_W).transpose(1, 0, 2))
    return np.ascontiguousarray(b.astype(np.float32 if dtype == "f32" else np.float64))


def adv_shift(n_cells, B, first=0):
    """Displacements of the advection workloads: shift_j = dt * v_j with v_j
    on a uniform velocity grid in [-vmax, vmax), dt chosen so |shift| <= 2.5
    cells (a CFL number above 1, as semi-Lagrangian schemes allow)."""
    j = np.arange(first, first + B, dtype=np.float64)
    v = -1.0 + 2.0 * (j % 100000) / 100000.0
    return v * (2.5 / n_cells)


def cpu_oracle_rate(deg, npts, bc, knots, n, target_s=10.0, max_rhs=None, adv=False):
    """Time the oracle as it stands on a bounded sample; returns (RHS/s,
    threads, sample description).  adv: one Algorithm-2 step per RHS."""
    import oracle
    o = oracle.Oracle(deg, npts, bc, knots)
    threads = len(os.sched_getaffinity(0))

    def run(b):
        if adv:
            o.advect(b, adv_shift(o.N, b.shape[1]), nthreads=threads)
        else:
            o.solve_(b, nthreads=threads)
    probe = 256
    b = inputs.rhs(n, probe, seed=99, degree=deg, bc=bc)
    t0 = time.perf_counter()
    run(b.copy())
    dt = time.perf_counter() - t0
    m = int(max(probe, min(target_s / max(dt, 1e-6) * probe, 200000)))
    if max_rhs:
        m = min(m, max_rhs)
    b = inputs.rhs(n, m, seed=98, degree=deg, bc=bc)
    t0 = time.perf_counter()
    run(b)
    dt = time.perf_counter() - t0
    what = "solve + evaluation at the feet (Algorithm 2)" if adv else "dense GEPP oracle"
    return m / dt, threads, f"{m} RHS of the same workload (n={n}), {what}, {threads} OpenMP threads"


def run_2d(args):
    """2-D tensor-product workloads (NEXT row f3): a step = spline_builder_solve_2d
    over every grid of this rank.  Algorithmic bytes = one read + one write of
    every grid point (the single-pass minimum; two passes without L2 reuse
    would move twice that)."""
    import torch
    import torch.distributed as dist
    from paper_conf_sc_asahilbpbgo24_b200 import SplineBuilder, solve_2d_

    spec1, spec2, G, dt, desc = TWOD[args.workload]
    ws, rank, local = dist_env()
    torch.cuda.set_device(local)
    if use_dist(ws):
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    sbs = []
    for deg, npts, bc, mesh in (spec1, spec2):
        sbs.append(SplineBuilder(deg, npts, bc, inputs.breakpoints(inputs.n_cells(deg, npts, bc), mesh)))
    n1, n2 = sbs[0].n, sbs[1].n
    esz = 4 if dt == "f32" else 8
    tdt = torch.float32 if dt == "f32" else torch.float64
    host = inputs.rhs(n1, G * n2, seed=1234, first=rank * G * n2).T.reshape(G, n2, n1)
    host = np.ascontiguousarray(host.astype(np.float32 if dt == "f32" else np.float64))
    pristine = torch.from_numpy(host).cuda()
    x = pristine.clone()
    stream = torch.cuda.current_stream()

    def barrier():
        if use_dist(ws):
            dist.barrier()
        torch.cuda.synchronize()

    chunk_mb = int(os.environ.get("SB_2D_CHUNK_MB", "0"))
    per_chunk = G if chunk_mb <= 0 else max(1, (chunk_mb << 20) // (n1 * n2 * esz))
    launches_per_step = 2 * ((G + per_chunk - 1) // per_chunk)
    CHUNK = 20
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    for _ in range(args.warmup):
        solve_2d_(sbs[0], sbs[1], x)
    barrier()
    run_chunk = ChunkRunner(lambda: solve_2d_(sbs[0], sbs[1], x), not args.no_graph)
    nchunks = (args.steps + CHUNK - 1) // CHUNK
    for m in {min(CHUNK, args.steps - c * CHUNK) for c in range(nchunks)}:
        run_chunk(m) if not args.no_graph else None
    barrier()
    starts = [torch.cuda.Event(enable_timing=True) for _ in range(nchunks)]
    ends = [torch.cuda.Event(enable_timing=True) for _ in range(nchunks)]
    with ClockSampler(local) as clk:
        barrier()
        done = 0
        for c in range(nchunks):
            m = min(CHUNK, args.steps - done)
            x.copy_(pristine)
            flush.fill_(c & 0xFF)
            starts[c].record(stream)
            run_chunk(m)
            ends[c].record(stream)
            done += m
        barrier()
    total_ms = float(sum(s_.elapsed_time(e_) for s_, e_ in zip(starts, ends)))
    t_tensor = torch.tensor([total_ms], device="cuda", dtype=torch.float64)
    if use_dist(ws):
        dist.all_reduce(t_tensor, op=dist.ReduceOp.MAX)
    ms_per_step = float(t_tensor[0]) / args.steps
    pts = n1 * n2 * G
    value = ws * pts / (ms_per_step / 1e3)
    alg_bytes = 2.0 * pts * esz
    achieved = alg_bytes / (ms_per_step / 1e3) / 1e9
    peak, peak_kind = load_peaks()
    e2e = None
    if not args.no_e2e:
        hp = torch.from_numpy(host.copy()).pin_memory()
        dev = torch.empty_like(pristine)
        ts = []
        for _ in range(args.e2e_steps + 1):
            barrier()
            t0 = time.perf_counter()
            dev.copy_(hp, non_blocking=True)
            solve_2d_(sbs[0], sbs[1], dev)
            hp.copy_(dev, non_blocking=True)
            torch.cuda.synchronize()
            ts.append(time.perf_counter() - t0)
        te = torch.tensor([float(np.mean(ts[1:]))], device="cuda", dtype=torch.float64)
        if use_dist(ws):
            dist.all_reduce(te, op=dist.ReduceOp.MAX)
        e2e = {"value": ws * pts / float(te[0]), "unit": "points/s", "h2d_bytes_per_step": int(host.nbytes),
               "d2h_bytes_per_step": int(host.nbytes), "path": "H2D + spline_builder_solve_2d + D2H"}
    cpu = None
    if rank == 0 and ws == 1 and not args.no_cpu_baseline:
        import oracle
        o1 = oracle.Oracle(spec1[0], spec1[1], spec1[2], inputs.breakpoints(inputs.n_cells(*spec1[:3]), spec1[3]))
        o2 = oracle.Oracle(spec2[0], spec2[1], spec2[2], inputs.breakpoints(inputs.n_cells(*spec2[:3]), spec2[3]))
        threads = len(os.sched_getaffinity(0))
        t0 = time.perf_counter()
        oracle.solve_2d(o1, o2, host[:1].astype(np.float64), nthreads=threads)
        dt1 = time.perf_counter() - t0
        m = int(max(1, min(G, 10.0 / max(dt1, 1e-6))))
        t0 = time.perf_counter()
        oracle.solve_2d(o1, o2, host[:m].astype(np.float64), nthreads=threads)
        rate = m * n1 * n2 / (time.perf_counter() - t0)
        cpu = {"value": rate, "unit": "points/s", "cores": threads, "kind": "oracle",
               "sample": f"{m} of the {G} grids ({n1} x {n2}), dense GEPP oracle per dimension, {threads} threads"}
    if rank == 0:
        line = {
            "metric": TWOD_METRIC, "value": value, "unit": "points/s", "n_gpus": ws, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms_per_step, "higher_is_better": True, "scaling": "weak",
            "vs_baseline": None, "dtype": dt, "data": "synthetic (Philox U(-1,1) grids, seeded)",
            "config": {"workload": desc, "n1": n1, "n2": n2, "grids_per_gpu": G, "l2_chunk_mb": chunk_mb,
                       "l2": f"inputs {pts * esz / 1e6:.0f} MB per GPU > 126 MB L2; input restored + 256 MB L2 "
                             f"flush every {CHUNK} steps (untimed)", "parallelism": f"dp{ws} (grid shards)"},
            "achieved_gbs": achieved,
            "roofline": {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s", "frac": achieved / peak,
                         "traffic": None, "peak_kind": peak_kind, "kernel_ms": ms_per_step,
                         "algorithmic_bytes_per_launch": alg_bytes / launches_per_step,
                         "note": f"whole step ({launches_per_step} launches): one read + one write per point"},
            "clocks": clk.summary(), "e2e": e2e, "gpu_launches": launches_per_step * args.steps, "cpu_baseline": cpu,
        }
        print(json.dumps(line), flush=True)
    if use_dist(ws):
        dist.destroy_process_group()


def run_reference_2d(args):
    """Reference arm of the 2-D workloads: the oracle's solve_2d as it stands on
    a bounded sample of grids per step."""
    ws, rank, _ = dist_env()
    if rank != 0:
        return
    import oracle
    spec1, spec2, G, dt, desc = TWOD[args.workload]
    os_ = [oracle.Oracle(d, p, b, inputs.breakpoints(inputs.n_cells(d, p, b), m)) for d, p, b, m in (spec1, spec2)]
    n1, n2 = os_[0].n, os_[1].n
    threads = len(os.sched_getaffinity(0))
    g0 = inputs.rhs(n1, n2, seed=1234).T.reshape(1, n2, n1).copy()
    t0 = time.perf_counter()
    oracle.solve_2d(os_[0], os_[1], g0, nthreads=threads)
    dt1 = time.perf_counter() - t0
    per_step = int(max(1, min(G, 100.0 / max(1, args.steps + args.warmup) / max(dt1, 1e-6))))
    grids = inputs.rhs(n1, per_step * n2, seed=1234).T.reshape(per_step, n2, n1).copy()
    for _ in range(args.warmup):
        oracle.solve_2d(os_[0], os_[1], grids, nthreads=threads)
    times = []
    for _ in range(args.steps):
        t0 = time.perf_counter()
        oracle.solve_2d(os_[0], os_[1], grids, nthreads=threads)
        times.append(time.perf_counter() - t0)
    t = float(np.mean(times))
    val = per_step * n1 * n2 / t
    line = {
        "impl": "reference", "metric": TWOD_METRIC, "value": val, "unit": "points/s", "n_gpus": args.gpus,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": t * 1e3, "higher_is_better": True,
        "scaling": "weak", "vs_baseline": None, "dtype": dt, "data": "synthetic",
        "config": {"workload": desc, "n1": n1, "n2": n2, "grids_per_step": per_step},
        "cpu_baseline": {"value": val, "unit": "points/s", "cores": threads, "kind": "oracle",
                         "sample": f"{per_step} of the {G} grids per step"},
        "e2e": {"value": val, "unit": "points/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)


def run_reference(args, wl):
    ws, rank, _ = dist_env()
    if rank != 0:
        return
    deg, npts, bc, mesh, B, dt, layout, desc = wl
    n = inputs.nbasis(deg, npts, bc)
    knots = inputs.breakpoints(inputs.n_cells(deg, npts, bc), mesh)
    import oracle
    o = oracle.Oracle(deg, npts, bc, knots)
    threads = len(os.sched_getaffinity(0))
    # each step: a bounded sample sized so the whole run stays within minutes
    adv = args.workload in ADVECT
    rate0, _, _ = cpu_oracle_rate(deg, npts, bc, knots, n, target_s=2.0, adv=adv)
    per_step = max(64, int(rate0 * min(4.0, 120.0 / max(1, args.steps + args.warmup))))  # whole run ~2 min
    b0 = inputs.rhs(n, per_step, seed=1234, degree=deg, bc=bc)
    sh0 = adv_shift(o.N, per_step)

    def run(b):
        if adv:
            o.advect(b, sh0, nthreads=threads)
        else:
            o.solve_(b, nthreads=threads)
    for _ in range(args.warmup):
        run(b0.copy())
    times = []
    for _ in range(args.steps):
        b = b0.copy()
        t0 = time.perf_counter()
        run(b)
        times.append(time.perf_counter() - t0)
    t = float(np.mean(times))
    val = per_step / t
    esz = 4 if dt == "f32" else 8
    metric, unit, scale = (ADV_METRIC, "GLUPS", n / 1e9) if adv else (METRIC, "RHS/s", 1.0)
    line = {
        "impl": "reference", "metric": metric, "value": val * scale, "unit": unit, "n_gpus": args.gpus,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": t * 1e3, "higher_is_better": True,
        "scaling": "weak", "vs_baseline": None, "dtype": dt, "data": "synthetic",
        "config": {"workload": desc, "n": n, "batch_per_step": per_step, "degree": deg, "bc": bc},
        "achieved_gbs": val * 2 * n * esz / 1e9,
        "cpu_baseline": {"value": val * scale, "unit": unit, "cores": threads, "kind": "oracle",
                         "sample": f"{per_step} RHS per step of the workload (n={n}); the full batch would take "
                                   f"{B / val:.1f} s"},
        "e2e": {"value": val * scale, "unit": unit, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)


EXTRA_DEFAULT = "C1,C3G,C3H,C4,C4F32,C4M,ADV,ADVNU,C5,C5S8,C6"


def quick_measure(name, steps=20, warmup=3):
    """One device-timed measurement of another workload on this GPU (same
    protocol as the headline: CUDA graph of `steps` launches, input restored
    and L2 flushed before the timed chunk, CUDA events on the launching
    stream), for the `extra_workloads` record of the default run: so the
    round-end bench line carries every BASELINE config (C1-C5) and the NEXT
    rows, not only C2.  Returns a small dict (no e2e / CPU baseline)."""
    import torch
    from paper_conf_sc_asahilbpbgo24_b200 import SplineBuilder, last_kernel, solve_2d_
    stream = torch.cuda.current_stream()
    peak, _ = load_peaks()
    if name in TWOD:
        spec1, spec2, G, dt, desc = TWOD[name]
        sbs = [SplineBuilder(d, p_, b, inputs.breakpoints(inputs.n_cells(d, p_, b), m)) for d, p_, b, m in (spec1, spec2)]
        n1, n2 = sbs[0].n, sbs[1].n
        host = np.ascontiguousarray(inputs.rhs(n1, G * n2, seed=1234).T.reshape(G, n2, n1).astype(
            np.float32 if dt == "f32" else np.float64))
        pristine = torch.from_numpy(host).cuda()
        x = pristine.clone()
        step = lambda: solve_2d_(sbs[0], sbs[1], x)  # noqa: E731
        restore = lambda: x.copy_(pristine)  # noqa: E731
        units, unit, esz, n_el = n1 * n2 * G, "points/s", (4 if dt == "f32" else 8), n1 * n2 * G
        kern = "warp pass + tile slab pass"
    else:
        deg, npts, bc, mesh, B, dt, layout, desc = WORKLOADS[name]
        n = inputs.nbasis(deg, npts, bc)
        sb = SplineBuilder(deg, npts, bc, inputs.breakpoints(inputs.n_cells(deg, npts, bc), mesh))
        tdt = torch.float32 if dt == "f32" else torch.float64
        if n * B > DEVICE_INPUT_ELEMS and layout == "batch":
            x = inputs.rhs_device(n, B, seed=1234, dtype=tdt)
            restore = lambda: inputs.rhs_device(n, B, seed=1234, dtype=tdt, out=x)  # noqa: E731
        else:
            pristine = torch.from_numpy(make_rhs(deg, n, bc, B, 0, layout, dt)).cuda()
            x = pristine.clone()
            restore = lambda: x.copy_(pristine)  # noqa: E731
        if name in ADVECT:
            sh = torch.from_numpy(adv_shift(inputs.n_cells(deg, npts, bc), B)).cuda()
            step = lambda: sb.advect_(x, sh)  # noqa: E731
        elif layout == "slabs":
            step = lambda: sb.solve_slabs_(x, SLAB_W, SLAB_W, B // SLAB_W, n * SLAB_W)  # noqa: E731
        else:
            step = lambda: sb.solve_(x)  # noqa: E731
        esz = 4 if dt == "f32" else 8
        units, unit, n_el = B, "RHS/s", n * B
        if name in ADVECT:
            units, unit = B * n / 1e9, "GLUPS"
    for _ in range(warmup):
        step()
    kern = last_kernel() if name not in TWOD else kern
    runner = ChunkRunner(step, True)
    runner(steps)
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    restore()
    flush.fill_(1)
    torch.cuda.synchronize()
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    with ClockSampler(torch.cuda.current_device()) as clk:
        ev0.record(stream)
        runner(steps)
        ev1.record(stream)
        torch.cuda.synchronize()
    ms = ev0.elapsed_time(ev1) / steps
    gbs = 2.0 * n_el * esz / (ms / 1e3) / 1e9
    out = {"config": desc, "ms_per_step": ms, "value": units / (ms / 1e3), "unit": unit,
           "achieved_gbs": gbs, "frac_of_measured_peak": gbs / peak, "pct_of_8tbs": gbs / 8000.0,
           "kernel": kern, "steps": steps, "clocks": clk.summary()}
    del x
    torch.cuda.empty_cache()
    return out


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=200)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--workload", default="C2", choices=sorted(WORKLOADS) + sorted(TWOD))
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--e2e-steps", type=int, default=3)
    ap.add_argument("--no-graph", action="store_true", help="launch each step from Python instead of a CUDA graph")
    ap.add_argument("--split", default=None, help="force the Schur split LO,HI (default: chosen at create)")
    ap.add_argument("--extra", default=None,
                    help="comma-separated workloads measured after the headline into extra_workloads "
                         f"(default for the C2 run on one GPU: {EXTRA_DEFAULT}; 'none' to skip)")
    args = ap.parse_args()
    if args.workload in TWOD:
        if args.impl == "reference":
            return run_reference_2d(args)
        return run_2d(args)
    wl = WORKLOADS[args.workload]
    if args.impl == "reference":
        return run_reference(args, wl)

    import torch
    import torch.distributed as dist
    from paper_conf_sc_asahilbpbgo24_b200 import SplineBuilder

    ws, rank, local = dist_env()
    torch.cuda.set_device(local)
    if use_dist(ws):
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    from paper_conf_sc_asahilbpbgo24_b200.shard import shard_bounds, weak_bounds
    deg, npts, bc, mesh, Bspec, dt, layout, desc = wl
    strong = args.workload in STRONG
    first, last = shard_bounds(rank, ws, Bspec) if strong else weak_bounds(rank, Bspec)
    B = last - first                      # this rank's RHS
    B_total = Bspec if strong else ws * Bspec
    n = inputs.nbasis(deg, npts, bc)
    knots = inputs.breakpoints(inputs.n_cells(deg, npts, bc), mesh)
    split = tuple(int(v) for v in args.split.split(",")) if args.split else None
    sb = SplineBuilder(deg, npts, bc, knots, split=split)
    esz = 4 if dt == "f32" else 8
    tdt = torch.float32 if dt == "f32" else torch.float64
    on_device = n * B > DEVICE_INPUT_ELEMS and layout == "batch"
    if on_device:
        host = None
        x = inputs.rhs_device(n, B, seed=1234, first=first, dtype=tdt)
        pristine = None
        restore = lambda: inputs.rhs_device(n, B, seed=1234, first=first, dtype=tdt, out=x)  # noqa: E731
    else:
        host = make_rhs(deg, n, bc, B, first, layout, dt)
        pristine = torch.from_numpy(host).cuda()
        x = pristine.clone()
        restore = lambda: x.copy_(pristine)  # noqa: E731
    stream = torch.cuda.current_stream()
    adv = args.workload in ADVECT
    if adv:
        shift = torch.from_numpy(adv_shift(inputs.n_cells(deg, npts, bc), B, first)).cuda()
        step = lambda t: sb.advect_(t, shift)  # noqa: E731
    elif layout == "slabs":
        step = lambda t: sb.solve_slabs_(t, SLAB_W, SLAB_W, B // SLAB_W, n * SLAB_W)  # noqa: E731
    else:
        step = sb.solve_

    def barrier():
        if use_dist(ws):
            dist.barrier()
        torch.cuda.synchronize()

    # The solve is in place, so repeated solves compute A^-k b, which grows
    # like cond(A)^k: time chunks of CHUNK back-to-back solves, restoring the
    # input and flushing L2 (256 MB write) between chunks, outside the events.
    CHUNK = 40
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    for _ in range(args.warmup):
        step(x)
    from paper_conf_sc_asahilbpbgo24_b200 import last_kernel
    kernel_name = last_kernel()
    barrier()
    run_chunk = ChunkRunner(lambda: step(x), not args.no_graph)
    nchunks = (args.steps + CHUNK - 1) // CHUNK
    for m in {min(CHUNK, args.steps - c * CHUNK) for c in range(nchunks)}:
        run_chunk(m) if not args.no_graph else None  # capture outside the timed region (replay = extra warm-up)
    barrier()
    starts = [torch.cuda.Event(enable_timing=True) for _ in range(nchunks)]
    ends = [torch.cuda.Event(enable_timing=True) for _ in range(nchunks)]
    with ClockSampler(local) as clk:
        barrier()
        done = 0
        for c in range(nchunks):
            m = min(CHUNK, args.steps - done)
            restore()
            flush.fill_(c & 0xFF)
            starts[c].record(stream)
            run_chunk(m)  # m steps, one fused kernel launch each
            ends[c].record(stream)
            done += m
        barrier()
    total_ms = float(sum(s_.elapsed_time(e_) for s_, e_ in zip(starts, ends)))
    chunk_steps = [min(CHUNK, args.steps - c * CHUNK) for c in range(nchunks)]
    per_chunk = [s_.elapsed_time(e_) / m for s_, e_, m in zip(starts, ends, chunk_steps)]  # ms per step
    t_tensor = torch.tensor([total_ms, total_ms / args.steps], device="cuda", dtype=torch.float64)
    if use_dist(ws):
        dist.all_reduce(t_tensor, op=dist.ReduceOp.MAX)
    total_ms, kern_avg_ms = float(t_tensor[0]), float(t_tensor[1])
    ms_per_step = total_ms / args.steps
    value = B_total / (ms_per_step / 1e3)
    alg_bytes = 2.0 * n * B * esz
    achieved = alg_bytes / (kern_avg_ms / 1e3) / 1e9   # per GPU (the slowest rank's kernel time)
    peak, peak_kind = load_peaks()

    # end to end through the C ABI with host buffers (pinned), copies in the timed region
    e2e = None
    if not args.no_e2e:
        Be = min(B, E2E_MAX_RHS)
        hsrc = host if host is not None else np.ascontiguousarray(x[:, :Be].cpu().numpy())
        if layout == "batch":
            hsrc = np.ascontiguousarray(hsrc[:, :Be])
            hp = torch.from_numpy(hsrc.copy()).pin_memory()
            sb.solve_host_(hp)  # warm-up (allocates staging)
            barrier()
            ts = []
            for _ in range(args.e2e_steps):
                hp.copy_(torch.from_numpy(hsrc))
                barrier()
                t0 = time.perf_counter()
                sb.solve_host_(hp)
                ts.append(time.perf_counter() - t0)
            te = torch.tensor([float(np.mean(ts))], device="cuda", dtype=torch.float64)
            if use_dist(ws):
                dist.all_reduce(te, op=dist.ReduceOp.MAX)
            e2e = {"value": ws * Be / float(te[0]), "unit": "RHS/s", "h2d_bytes_per_step": int(hsrc.nbytes),
                   "d2h_bytes_per_step": int(hsrc.nbytes), "path": "spline_builder_solve_host (pinned, chunked)",
                   "rhs_per_gpu": Be}
        else:
            hp = torch.from_numpy(hsrc.copy()).pin_memory()
            dev = torch.empty_like(pristine)
            ts = []
            for _ in range(args.e2e_steps + 1):
                barrier()
                t0 = time.perf_counter()
                dev.copy_(hp, non_blocking=True)
                step(dev)
                hp.copy_(dev, non_blocking=True)
                torch.cuda.synchronize()
                ts.append(time.perf_counter() - t0)
            te = torch.tensor([float(np.mean(ts[1:]))], device="cuda", dtype=torch.float64)
            if use_dist(ws):
                dist.all_reduce(te, op=dist.ReduceOp.MAX)
            e2e = {"value": ws * B / float(te[0]) * (n / 1e9 if adv else 1.0), "unit": "GLUPS" if adv else "RHS/s",
                   "h2d_bytes_per_step": int(hsrc.nbytes), "d2h_bytes_per_step": int(hsrc.nbytes),
                   "path": "H2D + spline_builder_" + ("advect" if adv else "solve") + " + D2H",
                   "rhs_per_gpu": B}

    cpu = None
    if rank == 0 and ws == 1 and not args.no_cpu_baseline:
        rate, cores, sample = cpu_oracle_rate(deg, npts, bc, knots, n, target_s=10.0, adv=adv)
        cpu = {"value": rate * (n / 1e9 if adv else 1.0), "unit": "GLUPS" if adv else "RHS/s", "cores": cores,
               "kind": "oracle", "sample": sample}

    if rank == 0:
        line = {
            "metric": ADV_METRIC if adv else METRIC, "value": value * (n / 1e9 if adv else 1.0),
            "unit": "GLUPS" if adv else "RHS/s", "n_gpus": ws, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms_per_step, "higher_is_better": True, "scaling": "strong" if strong else "weak",
            "vs_baseline": None, "dtype": dt, "data": "synthetic (Philox U(-1,1) RHS, seeded)",
            "config": {"workload": desc, "n": n, "batch_per_gpu": B, "batch_total": B_total, "degree": deg,
                       "bc": ["periodic", "greville", "hermite"][bc],
                       "mesh": mesh, "layout": {"batch": "batch-contiguous", "point": "point-contiguous",
                                                "slabs": "slabs of batch-contiguous blocks"}[layout],
                       "l2": f"inputs {n * B * esz / 1e6:.0f} MB per GPU > 126 MB L2; input restored + 256 MB "
                             f"L2 flush every 40 steps (untimed)",
                       "inputs": "device Philox (inputs.rhs_device)" if on_device else "host Philox (inputs.rhs)",
                       "launch": "python per step" if args.no_graph else
                       f"CUDA graphs of up to {CHUNK} launches, replayed",
                       "kernel": kernel_name, "split": [sb.info()["split_lo"], sb.info()["split_hi"]],
                       "parallelism": f"dp{ws} (RHS shards)"},
            "ms_per_step_median": float(np.median(per_chunk)), "ms_per_step_best": float(min(per_chunk)),
            "timed_chunks": len(per_chunk),
            "achieved_gbs": achieved, "pct_of_8tbs": achieved / 8000.0,
            "roofline": {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s",
                         "frac": achieved / peak, "traffic": load_traffic(args.workload),
                         "stream_ceiling_gbs": STREAM_CEILING_GBS[layout],
                         "frac_of_stream_ceiling": achieved / STREAM_CEILING_GBS[layout],
                         "peak_kind": peak_kind, "kernel_ms": kern_avg_ms,
                         "algorithmic_bytes_per_launch": alg_bytes},
            "clocks": clk.summary(),
            "e2e": e2e,
            "gpu_launches": args.steps,
            "cpu_baseline": cpu,
        }
        extra = args.extra if args.extra is not None else (EXTRA_DEFAULT if (args.workload == "C2" and ws == 1) else "none")
        if extra and extra != "none":
            del x
            torch.cuda.empty_cache()
            line["extra_workloads"] = {}
            for w in [e for e in extra.split(",") if e]:
                try:
                    line["extra_workloads"][w] = quick_measure(w)
                except Exception as exc:  # report, do not lose the headline
                    line["extra_workloads"][w] = {"error": f"{type(exc).__name__}: {exc}"}
        print(json.dumps(line), flush=True)
    if use_dist(ws):
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
