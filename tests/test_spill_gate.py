"""The ptxas spill gate of SURVEY §4 T3 / §5, as a ratchet (CPU: `cuobjdump -res-usage` of the built library).

The paper's Fig 4 lesson: per-point workspaces in local memory cost 4x.  The default
corner-force kernels of the benchmark configs are listed with the local stack (spill) bytes measured when they
became the default; a change that makes any of them spill MORE fails here (a smaller value is welcome: lower the
bound).  Register counts are bounded too (the occupancy each design relies on)."""
import os
import re
import shutil
import subprocess

import pytest

LIB = os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "paper_conf_ipps_dongdkrtd14_b200",
                   "libblastcf.so")

# mangled kernel name -> (config, max STACK bytes, max registers)
DEFAULTS = {
    "_Z10kb1_v10_3dILi4ELi0ELi0ELi33554432ELi11EEv7KB1Args": ("C4 v10.wpx", 56, 128),
    "_Z10kb1_v11_3dILi8ELi2ELi467EEv7KB1Args": ("C5 v11.mbtsiet", 0, 128),
    "_Z9kb1_v2_3dILi2ELi1ELi12ELi2ELi6EEv7KB1Args": ("C3 v2.z1m12e", 40, 168),
    "_Z7kb1_p2dILi4ELi2ELi6EEv7KB1Args": ("C2 p2d.z2m6", 0, 80),
    "_Z10kb2_gatherILi3ELi8EEvPKdPKiS3_lllidPdS1_iS4_": ("KB2 3D", 0, 64),
}


def res_usage():
    if shutil.which("cuobjdump") is None or not os.path.exists(LIB):
        pytest.skip("cuobjdump or the built library missing")
    out = subprocess.run(["cuobjdump", "-res-usage", LIB], capture_output=True, text=True).stdout
    res, fn = {}, None
    for line in out.splitlines():
        m = re.match(r"\s*Function (\S+):", line)
        if m:
            fn = m.group(1)
            continue
        m = re.search(r"REG:(\d+) STACK:(\d+)", line)
        if m and fn:
            res[fn] = (int(m.group(1)), int(m.group(2)))
            fn = None
    return res


def test_default_kernels_do_not_spill_more():
    res = res_usage()
    for fn, (name, max_stack, max_reg) in DEFAULTS.items():
        if fn.startswith("_Z10kb2_gather"):
            fn = next((f for f in res if f.startswith("_Z10kb2_gatherILi3ELi8E")), fn)
        assert fn in res, f"{name}: kernel {fn} not in the library"
        reg, stack = res[fn]
        assert stack <= max_stack, f"{name}: local stack {stack} B > {max_stack} B (spills grew)"
        assert reg <= max_reg, f"{name}: {reg} registers > {max_reg}"
