"""Build libctxb.so in-tree.  The library is host C++; the GPU kernels are
generated per IR program and compiled for sm_100a by NVRTC inside
ctxb_analyze (the bulk save/restore bandwidth kernels are generated the same
way, from an IR kernel, so they run the very same save/restore stubs)."""
from __future__ import annotations

import os
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
CSRC = os.path.join(HERE, "csrc")
SOURCES = ["ir.cpp", "analysis.cpp", "codegen.cpp", "driver.cpp", "api.cpp"]
OUT = os.path.join(HERE, "libctxb.so")
CUDA = os.environ.get("CUDA_HOME", "/usr/local/cuda")


def needs_build():
    if not os.path.exists(OUT):
        return True
    t = os.path.getmtime(OUT)
    deps = [os.path.join(CSRC, s) for s in SOURCES] + [os.path.join(CSRC, "ctxb_internal.h"),
                                                      os.path.join(CSRC, "driver.h"),
                                                      os.path.join(HERE, "..", "include", "ctxb.h")]
    return any(os.path.getmtime(d) > t for d in deps)


def build(force=False, verbose=True):
    if not force and not needs_build():
        return OUT
    cmd = ["g++", "-O2", "-g", "-std=c++17", "-fPIC", "-shared", "-Wall", "-Wno-format-truncation",
           f"-I{CUDA}/include", "-o", OUT + ".tmp"] + [os.path.join(CSRC, s) for s in SOURCES] + ["-ldl", "-pthread"]
    if verbose:
        print(" ".join(cmd), file=sys.stderr)
    subprocess.check_call(cmd)
    os.replace(OUT + ".tmp", OUT)
    return OUT


if __name__ == "__main__":
    build(force="--force" in sys.argv)
