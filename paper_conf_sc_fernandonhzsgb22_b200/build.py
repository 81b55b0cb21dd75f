"""Build libdgr.so in-tree: nvcc for sm_100a (cross-compiles without a GPU).

    python -m paper_conf_sc_fernandonhzsgb22_b200.build [-v]

Outputs paper_conf_sc_fernandonhzsgb22_b200/lib/libdgr.so.  Incremental: an
object is rebuilt when its source or any header is newer.
"""
from __future__ import annotations

import os
import shutil
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
CSRC = os.path.join(HERE, "csrc")
INC = os.path.join(os.path.dirname(HERE), "include")
LIBDIR = os.path.join(HERE, "lib")
OBJDIR = os.path.join(HERE, "lib", "obj")
LIB = os.path.join(LIBDIR, "libdgr.so")

CUDA_HOME = os.environ.get("CUDA_HOME", "/usr/local/cuda")
NVCC = os.path.join(CUDA_HOME, "bin", "nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
CU_FLAGS = ARCH + ["-O3", "-lineinfo", "-std=c++17", "--expt-relaxed-constexpr",
                   "-Xcompiler", "-fPIC,-ffp-contract=off", "-I", INC, "-I", CSRC]
CXX_FLAGS = ["-O2", "-fPIC", "-fopenmp", "-ffp-contract=off", "-std=c++17", "-I", INC, "-I", CSRC]

SOURCES_CU = ["api.cu", "kernels.cu", "unzip_kernel.cu", "rhs_kernel.cu", "rhs_kernel_fi.cu", "constraints_kernel.cu",
              "rhs_inputs.cu", "regrid.cu", "psi4.cu", "gen/rhs_alg.cu", "gen/psi4.cu"]
SOURCES_CXX = ["host_mesh.cpp"]


def _headers():
    hs = [os.path.join(CSRC, f) for f in os.listdir(CSRC) if f.endswith((".hpp", ".cuh", ".h"))]
    hs.append(os.path.join(INC, "dgr.h"))
    return hs


def _stale(obj, src):
    if not os.path.exists(obj):
        return True
    t = os.path.getmtime(obj)
    return any(os.path.getmtime(d) > t for d in [src] + _headers())


def _run(cmd, verbose):
    if verbose:
        print(" ".join(cmd), flush=True)
    r = subprocess.run(cmd, capture_output=True, text=True)
    if verbose and (r.stdout or r.stderr):
        print(r.stdout + r.stderr, flush=True)
    if r.returncode != 0:
        raise RuntimeError("build failed:\n" + " ".join(cmd) + "\n" + r.stdout + r.stderr)
    return r


def build(verbose: bool = False, ptxas_verbose: bool = False, variant: str = "") -> str:
    """variant="timing" builds lib/libdgr_timing.so with -DDGR_RHS_TIMING (per-stage
    cycle counters in k_rhs, for tools/rhs_stage_profile.py); any other variant
    builds lib/libdgr_<variant>.so with the -D flags in $DGR_EXTRA_DEFS (A/B
    experiments); never the product."""
    objdir = OBJDIR + (("_" + variant) if variant else "")
    lib = LIB if not variant else os.path.join(LIBDIR, f"libdgr_{variant}.so")
    defs = []
    if variant == "timing":
        defs = ["-DDGR_RHS_TIMING"]
    elif variant:   # experiment builds: -D flags from DGR_EXTRA_DEFS
        defs = os.environ.get("DGR_EXTRA_DEFS", "").split()
    os.makedirs(objdir, exist_ok=True)
    objs = []
    changed = False
    for s in SOURCES_CXX:
        src = os.path.join(CSRC, s)
        obj = os.path.join(objdir, s + ".o")
        objs.append(obj)
        if _stale(obj, src):
            _run([shutil.which("g++") or "g++"] + CXX_FLAGS + ["-c", src, "-o", obj], verbose)
            changed = True
    for s in SOURCES_CU:
        src = os.path.join(CSRC, s)
        obj = os.path.join(objdir, s.replace("/", "_") + ".o")
        objs.append(obj)
        if _stale(obj, src):
            extra = ["-Xptxas", "-v"] if ptxas_verbose else []
            _run([NVCC] + CU_FLAGS + defs + extra + ["-c", src, "-o", obj],
                 verbose or ptxas_verbose)
            changed = True
    if changed or not os.path.exists(lib):
        _run([NVCC] + ARCH + ["-shared", "-o", lib] + objs +
             ["-Xcompiler", "-fopenmp", "-lgomp", "-ldl"], verbose)
    return lib


if __name__ == "__main__":
    v = "-v" in sys.argv
    var = sys.argv[sys.argv.index("--variant") + 1] if "--variant" in sys.argv else ""
    print(build(verbose=v, ptxas_verbose="--ptxas" in sys.argv, variant=var))
