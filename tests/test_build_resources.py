"""Compiled-resource guard for the RHS kernels (CPU: reads the built library
with cuobjdump -res-usage, no device).

nvcc's inlining of the k_rhs lambdas is fragile: when it outlines point_work,
the kernel's captured per-point state moves to a local-memory frame of several
hundred bytes and the C3 step slows from ~26-31 ms to 59-72 ms (DESIGN.md §7,
"the option kernels").  Every instantiation the library launches — the default
k_rhs<fused, no radiative boundary, pre-pass, centred> and every k_rhs_fi —
must keep a frame of spills only.
"""
import re
import shutil
import subprocess

import pytest

import paper_conf_sc_fernandonhzsgb22_b200 as dgr

MAX_STACK = 256   # bytes; outlined lambdas give 460+


def _res_usage():
    exe = shutil.which("cuobjdump") or "/usr/local/cuda/bin/cuobjdump"
    out = subprocess.run([exe, "-res-usage", dgr.LIB_PATH], capture_output=True, text=True).stdout
    res = {}
    name = None
    for line in out.splitlines():
        m = re.search(r"Function (\S+):", line)
        if m:
            name = m.group(1)
            continue
        m = re.search(r"REG:(\d+) STACK:(\d+)", line)
        if m and name:
            res[name] = (int(m.group(1)), int(m.group(2)))
    return res


def test_launched_rhs_kernels_have_no_local_memory_frames():
    res = _res_usage()
    if not res:
        pytest.skip("cuobjdump unavailable or library without device code")
    launched = {k: v for k, v in res.items()
                if "k_rhs_fi" in k or k.startswith("_ZN3dgr5k_rhsILb1ELb0ELb1ELb0E")}
    # the default instantiation plus the force-inlined k_rhs_fi ones (rhs_kernel_fi.cu)
    assert len(launched) >= 12, sorted(launched)
    for k, (reg, stack) in launched.items():
        assert stack <= MAX_STACK, f"{k}: {stack} B stack frame (outlined lambda?)"
        assert reg <= 168, f"{k}: {reg} registers"
