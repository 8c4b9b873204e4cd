"""In-tree build of libmpspmm.so (CUDA sm_100a) with explicit nvcc commands.

The shared library lands next to this file so that it travels with the repo snapshot
to the GPU box.  Rebuilds only when a source or header is newer than the library.
"""
from __future__ import annotations

import glob
import os
import subprocess
import sys
from concurrent.futures import ThreadPoolExecutor

HERE = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(HERE)
CSRC = os.path.join(HERE, "csrc")
LIB = os.path.join(HERE, "libmpspmm.so")
OBJ = os.path.join(HERE, "build")
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
FLAGS = ["-O3", "-std=c++17", "-lineinfo", "-Xcompiler", "-fPIC", "-Xcompiler", "-O2",
         "-Xptxas", "-v", "--use_fast_math=false"]


def _sources():
    return sorted(glob.glob(os.path.join(CSRC, "*.cu")))


def _deps():
    return _sources() + sorted(glob.glob(os.path.join(CSRC, "*.cuh"))) + \
        [os.path.join(ROOT, "include", "mpspmm.h")]


def up_to_date() -> bool:
    if not os.path.exists(LIB):
        return False
    t = os.path.getmtime(LIB)
    return all(os.path.getmtime(d) <= t for d in _deps())


def build(force: bool = False, verbose: bool = False, lib: str = None, defines=()) -> str:
    """Build libmpspmm.so (or, for experiments, `lib` with extra -D `defines`)."""
    target = lib or LIB
    if not force and lib is None and up_to_date():
        return LIB
    obj_dir = OBJ if lib is None else OBJ + "_" + os.path.basename(lib).replace(".so", "")
    os.makedirs(obj_dir, exist_ok=True)
    flags = [f for f in FLAGS if f != "--use_fast_math=false"] + ["-D" + d for d in defines]

    def compile_one(src):
        obj = os.path.join(obj_dir, os.path.basename(src) + ".o")
        cmd = [NVCC, *ARCH, *flags, "-I", os.path.join(ROOT, "include"), "-c", src, "-o", obj]
        r = subprocess.run(cmd, capture_output=True, text=True)
        if r.returncode != 0:
            raise RuntimeError("nvcc failed for %s:\n%s\n%s" % (src, r.stdout, r.stderr))
        with open(obj + ".ptxas.txt", "w") as f:
            f.write(r.stderr)
        return obj

    with ThreadPoolExecutor(max_workers=min(8, os.cpu_count() or 1)) as ex:
        objs = list(ex.map(compile_one, _sources()))
    tmp = target + ".tmp%d" % os.getpid()
    cmd = [NVCC, *ARCH, "-shared", "-Xcompiler", "-fPIC", *objs, "-o", tmp]
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        raise RuntimeError("nvcc link failed:\n%s\n%s" % (r.stdout, r.stderr))
    os.replace(tmp, target)
    if verbose:
        print("built", target, file=sys.stderr)
    return target


if __name__ == "__main__":
    # python _build.py [--force] [--lib path.so -DNAME=VAL ...]
    args = sys.argv[1:]
    lib = None
    if "--lib" in args:
        lib = args[args.index("--lib") + 1]
    build(force="--force" in args, verbose=True, lib=lib,
          defines=[a[2:] for a in args if a.startswith("-D")])
