"""Build libmpx.so in-tree with nvcc for sm_100a (no JIT cache, no pip install).

    python -m paper_conf_sc_sojoodiasfga25_b200._build [--force]

The shared library is written to paper_conf_sc_sojoodiasfga25_b200/_lib/libmpx.so
(git-ignored; it travels to the GPU box with the gpurun snapshot).  cudart is linked
statically so the library does not depend on which libcudart torch loaded.
"""
from __future__ import annotations

import os
import subprocess
import sys

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
OUT_DIR = os.path.join(PKG, "_lib")
LIB = os.path.join(OUT_DIR, "libmpx.so")
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
SOURCES = ["model.cpp", "capi.cpp", "calib.cpp", "world.cpp", "coll.cpp", "topo.cpp", "engine.cu"]
HEADERS = ["model.h", "engine.h", "ctx.h"]


def _inputs():
    files = [os.path.join(CSRC, s) for s in SOURCES + HEADERS]
    files.append(os.path.join(ROOT, "include", "mp.h"))
    files.append(os.path.abspath(__file__))
    return files


def up_to_date() -> bool:
    if not os.path.exists(LIB):
        return False
    t = os.path.getmtime(LIB)
    return all(os.path.getmtime(f) <= t for f in _inputs())


def build(force: bool = False, verbose: bool = False, out: str = None, defines=()) -> str:
    """Build libmpx.so (default: the in-tree product library).  `out` + `defines`
    (e.g. ["MPX_STREAM_STAGES=6"]) build a variant elsewhere for design experiments;
    load it with MPX_LIB=<out>."""
    lib_path = out or LIB
    if not force and out is None and up_to_date():
        return LIB
    out_dir = os.path.dirname(lib_path)
    os.makedirs(out_dir, exist_ok=True)
    objs = []
    common = ["-O3", "-std=c++17", "-Xcompiler", "-fPIC", "-Xcompiler", "-Wall",
              "-I", os.path.join(ROOT, "include")] + [f"-D{d}" for d in defines]
    for s in SOURCES:
        src = os.path.join(CSRC, s)
        obj = os.path.join(out_dir, s + ".o")
        cmd = [NVCC] + ARCH + common + ["-lineinfo", "-c", src, "-o", obj]
        if s.endswith(".cu"):
            cmd += ["-Xptxas", "-v"] if verbose else []
        else:
            cmd = ["g++", "-O3", "-std=c++17", "-fPIC", "-Wall", "-I", os.path.join(ROOT, "include"),
                   "-I", "/usr/local/cuda/include", "-c", src, "-o", obj] + [f"-D{d}" for d in defines]
        subprocess.run(cmd, check=True)
        objs.append(obj)
    tmp = lib_path + ".tmp"
    subprocess.run([NVCC] + ARCH + ["-shared", "-cudart", "static", "-o", tmp] + objs, check=True)
    os.replace(tmp, lib_path)
    for o in objs:
        os.remove(o)
    return lib_path


if __name__ == "__main__":
    print(build(force="--force" in sys.argv, verbose="-v" in sys.argv))
