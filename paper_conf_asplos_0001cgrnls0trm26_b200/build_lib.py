"""Build libll.so in-tree: nvcc for sm_100a (-gencode arch=compute_100a,code=sm_100a)."""
import os
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
CSRC = os.path.join(HERE, "csrc")
INCLUDE = os.path.join(os.path.dirname(HERE), "include")
LIB = os.path.join(HERE, "libll.so")
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")


def _sources():
    return sorted(os.path.join(CSRC, f) for f in os.listdir(CSRC)
                  if f.endswith((".cpp", ".cu")))


def _deps():
    deps = _sources() + [os.path.join(CSRC, f) for f in os.listdir(CSRC) if f.endswith((".hpp", ".cuh"))]
    return deps + [os.path.join(INCLUDE, "ll.h"), os.path.abspath(__file__)]


def embed_template():
    src = open(os.path.join(CSRC, "ll_kernels.cuh")).read()
    out = os.path.join(CSRC, "ll_kernels_embed.inc")
    text = 'R"LLKERNELS(' + src + ')LLKERNELS"\n'
    if not os.path.exists(out) or open(out).read() != text:
        with open(out, "w") as f:
            f.write(text)


def build(force=False, verbose=False):
    if not force and os.path.exists(LIB):
        t = os.path.getmtime(LIB)
        if all(os.path.getmtime(d) <= t for d in _deps()):
            return LIB
    embed_template()
    cmd = [NVCC, "-shared", "-Xcompiler", "-fPIC", "-O3", "-std=c++17",
           "-gencode", "arch=compute_100a,code=sm_100a", "-lineinfo",
           "-I", INCLUDE, "-I", CSRC, "-o", LIB + ".tmp"] + _sources() + ["-lnvrtc", "-ldl", "-lcuda" if False else "-lcudart_static"]
    if verbose:
        print(" ".join(cmd))
    subprocess.run(cmd, check=True)
    os.replace(LIB + ".tmp", LIB)
    return LIB


if __name__ == "__main__":
    build(force="--force" in sys.argv, verbose=True)
