"""Build the CUDA C-ABI library libcapgpu.so in-tree (nvcc, sm_100a).

    python -m paper_conf_icpp_masw25_b200.build [--force]

Every translation unit is compiled with
``-gencode arch=compute_100a,code=sm_100a -O3 -lineinfo`` (parallel, one
process per unit) and linked with the shared CUDA runtime plus the NCCL that
ships with torch (site-packages/nvidia/nccl).  The host side is compiled with
``-ffp-contract=off`` so host-computed tables reproduce the oracle's formulas.
"""
from __future__ import annotations

import concurrent.futures as cf
import glob
import os
import subprocess
import sys

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
BUILD = os.path.join(PKG, "_build")
LIB = os.path.join(PKG, "libcapgpu.so")
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]


def nccl_dirs():
    import importlib.util
    spec = importlib.util.find_spec("nvidia")
    cands = []
    if spec and spec.submodule_search_locations:
        for p in spec.submodule_search_locations:
            cands.append(os.path.join(p, "nccl"))
    cands.append("/opt/prime-rl/.venv/lib/python3.12/site-packages/nvidia/nccl")
    for c in cands:
        if os.path.exists(os.path.join(c, "include", "nccl.h")):
            return os.path.join(c, "include"), os.path.join(c, "lib")
    raise RuntimeError("nccl.h not found (torch's nvidia-nccl wheel)")


def _cudart_dir():
    """torch's libcudart.so.12 (nvidia-cuda-runtime wheel)."""
    import importlib.util
    spec = importlib.util.find_spec("nvidia")
    for p in (spec.submodule_search_locations if spec else []) or []:
        d = os.path.join(p, "cuda_runtime", "lib")
        if os.path.exists(os.path.join(d, "libcudart.so.12")):
            return d
    return "/usr/local/cuda/lib64"


def cflags():
    inc, _ = nccl_dirs()
    return [*ARCH, "-O3", "-lineinfo", "-std=c++17", "-Xcompiler", "-fPIC", "-Xcompiler", "-ffp-contract=off",
            "-Xcompiler", "-fno-fast-math", f"-I{inc}", f"-I{os.path.join(ROOT, 'include')}",
            f"-I{os.path.join(ROOT, 'gen')}"]


def _deps():
    return (glob.glob(os.path.join(CSRC, "*.cuh")) + [os.path.join(ROOT, "include", "capgpu.h"),
                                                      os.path.join(ROOT, "gen", "capgpu_gen.h")])


VARIANTS = {
    # profiling build: per-phase cycle counters in the fused kernel (never the product library)
    "timing": (["-DCAPGPU_PHASE_TIMING"], "_build_timing", "libcapgpu_timing.so"),
    # A/B experiments: the working tree built beside the product library
    "exp": ([], "_build_exp", "libcapgpu_exp.so"),
    # k_period compiled for 12 resident warps per SM (read-only constants from global memory)
    "pw12": (["-DCAPGPU_PERIOD_WARPS=12"], "_build_pw12", "libcapgpu_pw12.so"),
}


def _compile(src: str, force: bool, verbose: bool, bdir: str = BUILD, extra=()) -> str:
    obj = os.path.join(bdir, os.path.basename(src).replace(".cu", ".o"))
    newest_dep = max(os.path.getmtime(d) for d in _deps() + [src])
    if not force and os.path.exists(obj) and os.path.getmtime(obj) >= newest_dep:
        return obj
    cmd = [NVCC, *cflags(), *extra, "-c", src, "-o", obj]
    if verbose:
        cmd.insert(1, "-Xptxas=-v")
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        raise RuntimeError(f"nvcc failed for {src}:\n{r.stderr[-8000:]}")
    if verbose:
        with open(obj + ".ptxas.txt", "w") as fh:
            fh.write(r.stderr)
    return obj


def build(force: bool = False, verbose: bool = False, jobs: int | None = None, variant: str | None = None,
          defs: tuple = ()) -> str:
    extra, bdir, lib = ((), BUILD, LIB)
    if variant and variant not in VARIANTS:  # ad-hoc experiment build: --variant=NAME --defs="-DX -DY"
        VARIANTS[variant] = (list(defs), f"_build_{variant}", f"libcapgpu_{variant}.so")
    if variant:
        flags, sub, name = VARIANTS[variant]
        extra, bdir, lib = (flags, os.path.join(PKG, sub), os.path.join(PKG, name))
    os.makedirs(bdir, exist_ok=True)
    srcs = sorted(glob.glob(os.path.join(CSRC, "*.cu")))
    # a library newer than every source is current even without its objects
    # (the object directory does not travel to the GPU box)
    if not force and os.path.exists(lib) and os.path.getmtime(lib) >= max(
            os.path.getmtime(d) for d in _deps() + srcs + [os.path.abspath(__file__)]):
        return lib
    only = [int(x) for x in os.environ.get("CAPGPU_ONLY_N", "").split(",") if x] if variant else []
    if only:  # experiment build with a subset of the knob counts (smaller library to ship)
        bdir = bdir + "_n" + "-".join(map(str, sorted(only)))  # objects depend on the subset
        os.makedirs(bdir, exist_ok=True)
        srcs = [s_ for s_ in srcs if not os.path.basename(s_).startswith("inst_n") or
                int(os.path.basename(s_)[6:-3]) in only]
        extra = list(extra) + ["-DCAPGPU_SUBSET"] + [
            f"-DCAPGPU_CASE_IF_{n}=" + (f"case {n}: return launchers_n{n}(M);" if n in only else "")
            for n in range(2, 17)]
    jobs = jobs or max(1, min(len(srcs), os.cpu_count() or 4))
    with cf.ThreadPoolExecutor(jobs) as ex:
        objs = list(ex.map(lambda s: _compile(s, force, verbose, bdir, extra), srcs))
    newest = max(os.path.getmtime(o) for o in objs)
    if force or not os.path.exists(lib) or os.path.getmtime(lib) < newest:
        _, libdir = nccl_dirs()
        # shared CUDA runtime (the one torch already maps into the process, else
        # the toolkit's): the product library carries no copy of the runtime
        cmd = [NVCC, *ARCH, "-shared", "-o", lib, *objs, "-cudart", "shared", f"-L{libdir}", "-l:libnccl.so.2",
               "-Xlinker", f"-rpath,{libdir}", "-Xlinker", f"-rpath,{_cudart_dir()}", "-Xlinker",
               "-rpath,/usr/local/cuda/lib64"]
        r = subprocess.run(cmd, capture_output=True, text=True)
        if r.returncode != 0:
            raise RuntimeError(f"link failed:\n{r.stderr[-8000:]}")
    return lib


if __name__ == "__main__":
    var = next((a.split("=", 1)[1] for a in sys.argv if a.startswith("--variant=")), None)
    defs = next((a.split("=", 1)[1].split() for a in sys.argv if a.startswith("--defs=")), [])
    print(build(force="--force" in sys.argv, verbose="-v" in sys.argv, variant=var, defs=tuple(defs)))
