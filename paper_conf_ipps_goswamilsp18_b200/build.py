"""Build liblasagna.so in-tree: nvcc for sm_100a (-gencode arch=compute_100a,code=sm_100a).

The library is a plain C-ABI shared object (include/lasagna.h), loaded through ctypes by
paper_conf_ipps_goswamilsp18_b200.lasagna; no torch types cross the boundary.
"""
from __future__ import annotations

import glob
import os
import shutil
import subprocess

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
INCLUDE = os.path.join(ROOT, "include")
SO = os.path.join(PKG, "liblasagna.so")
# bounds-checked variant (-DLSG_CHECKS, common.cuh LSG_DCHECK): the GPU tests' stand-in for
# compute-sanitizer, which the GPU pool does not offer; loaded when LASAGNA_CHECKED=1
SO_CHECKED = os.path.join(PKG, "liblasagna_checked.so")

NVCC_FLAGS = [
    "-O3", "-std=c++17", "-lineinfo",
    "-gencode", "arch=compute_100a,code=sm_100a",
    "-Xcompiler", "-fPIC", "-Xcompiler", "-fvisibility=hidden",
    "-Xptxas", "-v",
]


def sources() -> list[str]:
    return sorted(glob.glob(os.path.join(CSRC, "*.cu")))


def headers() -> list[str]:
    return sorted(glob.glob(os.path.join(CSRC, "*.cuh"))) + [os.path.join(INCLUDE, "lasagna.h")]


def stale(checked: bool = False) -> bool:
    so = SO_CHECKED if checked else SO
    if not os.path.exists(so):
        return True
    t = os.path.getmtime(so)
    return any(os.path.getmtime(f) > t for f in sources() + headers())


def nvcc() -> str:
    for c in [shutil.which("nvcc"), "/usr/local/cuda/bin/nvcc"]:
        if c and os.path.exists(c):
            return c
    raise RuntimeError("nvcc not found: cannot build liblasagna.so")


def _compile(src: str, obj: str, extra: tuple = ()) -> subprocess.CompletedProcess:
    return subprocess.run([nvcc(), *NVCC_FLAGS, *extra, "-I", INCLUDE, "-c", "-o", obj, src],
                          capture_output=True, text=True)


def build(verbose: bool = False, force: bool = False, checked: bool = False) -> str:
    """Compile every csrc/*.cu to an object in parallel (one nvcc per translation unit; no
    device code crosses units), then link the shared library."""
    so = SO_CHECKED if checked else SO
    if not force and not stale(checked):
        return so
    from concurrent.futures import ThreadPoolExecutor

    objdir = os.path.join(PKG, ".obj_checked" if checked else ".obj")
    extra = ("-DLSG_CHECKS",) if checked else ()
    os.makedirs(objdir, exist_ok=True)
    srcs = sources()
    objs = [os.path.join(objdir, os.path.basename(f)[:-3] + ".o") for f in srcs]
    with ThreadPoolExecutor(max_workers=min(len(srcs), os.cpu_count() or 4)) as ex:
        results = list(ex.map(lambda f, o: _compile(f, o, extra), srcs, objs))
    logs = []
    for f, r in zip(srcs, results):
        logs.append(f"== {os.path.basename(f)}\n" + r.stdout + r.stderr)
        if r.returncode != 0:
            raise RuntimeError(f"nvcc failed on {f}:\n" + r.stdout + r.stderr)
    link = [nvcc(), "-shared", "-gencode", "arch=compute_100a,code=sm_100a", "-o", so + ".tmp", *objs]
    r = subprocess.run(link, capture_output=True, text=True)
    if r.returncode != 0:
        raise RuntimeError("link failed:\n" + r.stdout + r.stderr)
    os.replace(so + ".tmp", so)
    log = os.path.join(PKG, "build_checked.log" if checked else "build.log")
    with open(log, "w") as f:
        f.write(" ".join([nvcc(), *NVCC_FLAGS, "-c"]) + "\n" + "".join(logs))
    if verbose:
        print("".join(logs))
    return so


if __name__ == "__main__":
    print(build(verbose=True, force=True))
