"""Build libsigmo.so in-tree for sm_100a (nvcc cross-compiles without a GPU)."""
from __future__ import annotations

import os
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
CSRC = os.path.join(HERE, "csrc")
LIB = os.path.join(HERE, "libsigmo.so")
SOURCES = ["sigmo_abi.cu", "sigmo_kernels.cu", "sigmo_filter_lane.cu", "sigmo_jit.cu", "sigmo_load.cu"]
HEADERS = ["sigmo_internal.h", "lane_filter_types.h", "lane_filter_body.cuh", os.path.join("..", "..", "include", "sigmo.h")]
# headers embedded as raw strings for the NVRTC-specialised filter (sigmo_jit.cu)
EMBED = ["lane_filter_types.h", "lane_filter_body.cuh"]


def _embed() -> None:
    for h in EMBED:
        src = open(os.path.join(CSRC, h)).read()
        assert ")SIGMOSRC" not in src
        inc = os.path.join(CSRC, h.rsplit(".", 1)[0] + ".inc")
        body = 'R"SIGMOSRC(' + src + ')SIGMOSRC"\n'
        if not os.path.exists(inc) or open(inc).read() != body:
            with open(inc, "w") as f:
                f.write(body)

NVCC_FLAGS = ["-gencode", "arch=compute_100a,code=sm_100a", "-lineinfo", "-O3", "-std=c++17",
              "-Xcompiler", "-fPIC", "-Xcompiler", "-fvisibility=hidden", "-shared", "-cudart", "static",
              "--expt-relaxed-constexpr"]


def _stale() -> bool:
    if not os.path.exists(LIB):
        return True
    t = os.path.getmtime(LIB)
    files = [os.path.join(CSRC, f) for f in SOURCES + HEADERS] + [__file__]
    return any(os.path.getmtime(f) > t for f in files)


def build(force: bool = False, verbose: bool = False) -> str:
    if not force and not _stale():
        return LIB
    _embed()
    nvcc = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
    objs = []
    for src in SOURCES:
        obj = os.path.join(CSRC, src.replace(".cu", ".o"))
        cmd = [nvcc, *[f for f in NVCC_FLAGS if f != "-shared"], "-c", os.path.join(CSRC, src), "-o", obj]
        if verbose:
            cmd.insert(1, "-Xptxas=-v")
        subprocess.check_call(cmd)
        objs.append(obj)
    tmp = LIB + ".tmp"
    subprocess.check_call([nvcc, "-gencode", "arch=compute_100a,code=sm_100a", "-shared", "-cudart", "static",
                           "-Xcompiler", "-fPIC", *objs, "-o", tmp, "-ldl"])
    os.replace(tmp, LIB)
    return LIB


if __name__ == "__main__":
    print(build(force="--force" in sys.argv, verbose="-v" in sys.argv))
