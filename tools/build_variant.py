"""Build an experimental variant of libsigmo.so with extra nvcc flags into
build/variants/NAME/libsigmo.so (git-ignored; travels to the GPU box with
gpurun).  Run it with SIGMO_LIB=build/variants/NAME/libsigmo.so.
Usage: python tools/build_variant.py NAME -DFLAG=VALUE ..."""
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, os.path.join(ROOT, "paper_conf_sc_carocfc25_b200"))
import build as B  # noqa: E402

name, extra = sys.argv[1], sys.argv[2:]
out = os.path.join(ROOT, "build", "variants", name)
os.makedirs(out, exist_ok=True)
B._embed()
objs = []
for src in B.SOURCES:
    obj = os.path.join(out, src.replace(".cu", ".o"))
    subprocess.check_call([os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc"),
                           *[f for f in B.NVCC_FLAGS if f != "-shared"], *extra, "-c", os.path.join(B.CSRC, src),
                           "-o", obj])
    objs.append(obj)
subprocess.check_call(["/usr/local/cuda/bin/nvcc", "-gencode", "arch=compute_100a,code=sm_100a", "-shared", "-cudart",
                       "static", "-Xcompiler", "-fPIC", *objs, "-o", os.path.join(out, "libsigmo.so"), "-ldl"])
print(os.path.join(out, "libsigmo.so"))
