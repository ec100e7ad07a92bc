"""Build libblastcf.so in-tree with nvcc for sm_100a (no JIT cache: the .so travels with the repo)."""
import os
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(HERE)
CSRC = os.path.join(HERE, "csrc")
LIB = os.path.join(HERE, "libblastcf.so")
SOURCES = [os.path.join(CSRC, "blast_cf.cu"), os.path.join(CSRC, "integrator.cu")]
OBJDIR = os.path.join(HERE, "build")
DEPS = [os.path.join(CSRC, f) for f in os.listdir(CSRC)] + [os.path.join(ROOT, "include", "blast_cf.h")]


def nccl_include():
    import importlib.util
    spec = importlib.util.find_spec("nvidia")
    for base in (spec.submodule_search_locations or []):
        inc = os.path.join(base, "nccl", "include")
        if os.path.exists(os.path.join(inc, "nccl.h")):
            return inc
    raise RuntimeError("nccl.h not found (nvidia-nccl wheel)")


def nccl_lib():
    inc = nccl_include()
    return os.path.join(os.path.dirname(inc), "lib", "libnccl.so.2")


NVCC_FLAGS = ["-gencode", "arch=compute_100a,code=sm_100a", "-O3", "-lineinfo", "-std=c++17",
              "-Xcompiler", "-fPIC", "-Xptxas", "-warn-spills"]


def build(force: bool = False, verbose: bool = False) -> str:
    if not force and os.path.exists(LIB):
        t = os.path.getmtime(LIB)
        if all(os.path.getmtime(d) <= t for d in DEPS):
            return LIB
    os.makedirs(OBJDIR, exist_ok=True)
    inc = ["-I", os.path.join(ROOT, "include"), "-I", nccl_include()]
    objs, procs = [], []
    for src in SOURCES:   # one object per translation unit, compiled in parallel
        obj = os.path.join(OBJDIR, os.path.basename(src) + f".{os.getpid()}.o")
        # BLAST_CF_NVCC_FLAGS: extra flags for experiments (e.g. -DBLAST_CF_DIAGNOSTICS, timing-only kernels)
        cmd = ["nvcc", *NVCC_FLAGS, *os.environ.get("BLAST_CF_NVCC_FLAGS", "").split(), *inc, "-c", "-o", obj, src]
        if verbose:
            cmd.insert(1, "-Xptxas=-v")
            print(" ".join(cmd))
        objs.append(obj)
        procs.append(subprocess.Popen(cmd))
    if any(p.wait() != 0 for p in procs):
        raise subprocess.CalledProcessError(1, "nvcc")
    tmp = LIB + f".tmp{os.getpid()}"
    subprocess.check_call(["nvcc", "-gencode", "arch=compute_100a,code=sm_100a", "-shared", "-o", tmp, *objs, "-ldl"])
    for o in objs:
        os.remove(o)
    os.replace(tmp, LIB)
    return LIB


if __name__ == "__main__":
    build(force="--force" in sys.argv, verbose="-v" in sys.argv)
    print(LIB)
