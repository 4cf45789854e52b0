"""Build libhisq_dslash.so in-tree with nvcc for sm_100a (used by __graft_entry__.build)."""
from __future__ import annotations

import glob
import os
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(HERE)
LIB = os.path.join(HERE, "libhisq_dslash.so")


def nccl_dir():
    import nvidia.nccl  # torch's bundled NCCL (headers + libnccl.so.2)
    d = os.path.dirname(nvidia.nccl.__file__) if nvidia.nccl.__file__ else list(nvidia.nccl.__path__)[0]
    return d


def sources():
    return sorted(glob.glob(os.path.join(HERE, "csrc", "*.cu")) + glob.glob(os.path.join(HERE, "csrc", "*.cuh"))
                  + glob.glob(os.path.join(HERE, "csrc", "*.h")) + [os.path.join(ROOT, "include", "hisq_dslash.h")])


ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]


def build(force: bool = False, verbose: bool = False, defines=(), out: str = None) -> str:
    """Compile every csrc/*.cu to an object in parallel (sm_100a, -lineinfo) and link the .so.

    defines / out (measurement aid for A/B runs): extra -D flags and another output path; such a
    variant builds in its own object directory and is loaded with HISQ_DSLASH_LIB=<out>."""
    lib = out or LIB
    if not force and os.path.exists(lib) and os.path.getmtime(lib) >= max(os.path.getmtime(s) for s in sources()):
        return lib
    from concurrent.futures import ThreadPoolExecutor

    nccl = nccl_dir()
    objdir = os.path.join(HERE, "build") if out is None else out + ".objs"
    os.makedirs(objdir, exist_ok=True)
    common = ["nvcc", *ARCH, "-lineinfo", "-O3", "-std=c++17", "-Xcompiler", "-fPIC,-fvisibility=hidden",
              "-I", os.path.join(nccl, "include"), "-I", os.path.join(ROOT, "include")]
    if verbose:
        common.append("-Xptxas=-v")
    common += ["-D" + d for d in defines]
    cus = sorted(glob.glob(os.path.join(HERE, "csrc", "*.cu")))
    objs = [os.path.join(objdir, os.path.basename(c)[:-3] + ".o") for c in cus]

    def compile_one(pair):
        src, obj = pair
        cmd = common + ["-c", src, "-o", obj]
        if verbose:
            print(" ".join(cmd), file=sys.stderr)
        return subprocess.run(cmd, capture_output=not verbose, text=True)

    with ThreadPoolExecutor(max_workers=min(len(cus), os.cpu_count() or 4)) as ex:
        results = list(ex.map(compile_one, zip(cus, objs)))
    for src, r in zip(cus, results):
        if r.returncode != 0:
            raise RuntimeError(f"nvcc failed on {src}:\n{r.stderr}")
    link = ["nvcc", *ARCH, "-shared", "-o", lib, *objs, "-L", os.path.join(nccl, "lib"), "-l:libnccl.so.2",
            "-Xlinker", "-rpath=" + os.path.join(nccl, "lib")]
    subprocess.check_call(link)
    if out is not None:
        return lib
    build_c_demo("c_api_demo")
    build_c_demo("c_p2p_demo")
    return LIB


def build_c_demo(name: str = "c_api_demo") -> str:
    """examples/<name>: the library used from plain C (the boundary is a C ABI).  c_api_demo: one
    rank; c_p2p_demo: a forked multi-rank P2P partition (no Python, no MPI)."""
    src = os.path.join(ROOT, "examples", name + ".c")
    exe = os.path.join(ROOT, "examples", name)
    if os.path.exists(src):
        subprocess.check_call(["gcc", "-std=gnu99", "-O2", src, "-I", os.path.join(ROOT, "include"), "-L", HERE,
                               "-lhisq_dslash", "-Wl,-rpath," + HERE, "-lpthread", "-lm", "-o", exe])
    return exe


if __name__ == "__main__":
    build(force="--force" in sys.argv, verbose=True)
