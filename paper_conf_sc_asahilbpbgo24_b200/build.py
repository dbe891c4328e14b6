"""In-tree build of libsplinebuilder.so (C ABI + sm_100a kernels).

nvcc cross-compiles for sm_100a without a GPU.  The library links the shared
CUDA runtime (libcudart.so.12; when torch is loaded first, its copy of the
runtime is the one used) and never links torch.
"""
from __future__ import annotations

import os
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(HERE)
CSRC = os.path.join(HERE, "csrc")
BUILD = os.path.join(HERE, "_build")
LIB = os.path.join(HERE, "libsplinebuilder.so")
CUDA_HOME = os.environ.get("CUDA_HOME", "/usr/local/cuda")
NVCC = os.path.join(CUDA_HOME, "bin", "nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]

SOURCES = [
    ("host/plan.cpp", "cxx"),
    ("capi.cpp", "cxx"),
    ("solve_kernels.cu", "cu"),
    ("tile_f64.cu", "cu"),
    ("tile_f32.cu", "cu"),
    ("warp_f64.cu", "cu"),
    ("warp_f32.cu", "cu"),
    ("warp_adv_f64.cu", "cu"),
    ("warp_adv_f32.cu", "cu"),
    ("serial.cu", "cu"),
    ("refactor.cu", "cu"),
    ("tile_pair_f64.cu", "cu"),
]
HEADERS = ["host/plan.hpp", "device.hpp", "kernels.cuh", "refactor.hpp", "pair.cuh"]


def _newer(target: str, deps: list[str]) -> bool:
    if not os.path.exists(target):
        return True
    t = os.path.getmtime(target)
    return any(os.path.getmtime(d) > t for d in deps)


def build(force: bool = False, verbose: bool = False, extra_flags: tuple = (), lib: str = LIB, build_dir: str = BUILD,
          only: tuple = ()) -> str:
    """extra_flags / lib / build_dir: diagnostic variants (e.g. -DSB_TRACE) built beside the shipped library.
    only: compile just these sources in build_dir and link the shipped build's objects for the rest."""
    default_build = os.path.join(HERE, "_build")
    LIB, BUILD = lib, build_dir
    os.makedirs(BUILD, exist_ok=True)
    hdrs = [os.path.join(CSRC, h) for h in HEADERS] + [os.path.join(ROOT, "include", "spline_builder.h")]
    objs, jobs = [], []
    for src, kind in SOURCES:
        path = os.path.join(CSRC, src)
        if only and src not in only:
            objs.append(os.path.join(default_build, src.replace("/", "_") + ".o"))
            continue
        obj = os.path.join(BUILD, src.replace("/", "_") + ".o")
        objs.append(obj)
        if not (force or _newer(obj, [path] + hdrs)):
            continue
        if kind == "cxx":
            cmd = ["g++", "-std=c++17", "-O2", "-fno-fast-math", "-fPIC", "-Wall", "-Wno-unused-function",
                   "-I" + os.path.join(CUDA_HOME, "include"), "-c", path, "-o", obj]
        else:
            cmd = [NVCC, *ARCH, "-std=c++17", "-O3", "-lineinfo", "-Xptxas", "-v", "-Xcompiler", "-fPIC",
                   "--expt-relaxed-constexpr", *extra_flags, "-c", path, "-o", obj]
        if verbose:
            print(" ".join(cmd), file=sys.stderr)
        jobs.append((cmd, obj, kind))

    def run(job):
        cmd, obj, kind = job
        r = subprocess.run(cmd, capture_output=True, text=True)
        if r.returncode != 0:
            raise RuntimeError(f"compile failed: {' '.join(cmd)}\n{r.stdout}\n{r.stderr}")
        if kind == "cu":
            with open(obj + ".ptxas.txt", "w") as f:
                f.write(r.stderr)

    from concurrent.futures import ThreadPoolExecutor
    with ThreadPoolExecutor(max_workers=max(1, min(len(jobs), os.cpu_count() or 4))) as ex:
        list(ex.map(run, jobs))
    if force or _newer(LIB, objs):
        cmd = [NVCC, *ARCH, "-shared", "-cudart", "shared", "-Xlinker", "-rpath=" + os.path.join(CUDA_HOME, "lib64"),
               "-o", LIB + ".tmp", *objs, "-lpthread", "-ldl", "-lrt"]
        r = subprocess.run(cmd, capture_output=True, text=True)
        if r.returncode != 0:
            raise RuntimeError(f"link failed: {' '.join(cmd)}\n{r.stdout}\n{r.stderr}")
        os.replace(LIB + ".tmp", LIB)
    return LIB


if __name__ == "__main__":
    print(build(force="--force" in sys.argv, verbose=True))
