"""ctypes binding of the C++17/OpenMP oracle (oracle/ll_oracle.cpp) — TEST
INFRASTRUCTURE ONLY (same rules as oracle/ll_oracle.py: tests, smoke/build and
bench.py's cpu_baseline / --impl reference legs only).

build() compiles oracle/libll_oracle.so with g++ -O2 -fopenmp (no SIMD intrinsics, no
-ffast-math, FP contraction off); it is never linked into the product's libll.so.
Every function takes the layout as its columns (O.Layout.cols, or any list of logical
flat indices per input bit).
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess
from typing import Optional, Sequence

import numpy as np

HERE = os.path.dirname(os.path.abspath(__file__))
SRC = os.path.join(HERE, "ll_oracle.cpp")
LIB = os.path.join(HERE, "libll_oracle.so")
_lib = None


def build(force: bool = False) -> str:
    if not force and os.path.exists(LIB) and os.path.getmtime(LIB) >= os.path.getmtime(SRC):
        return LIB
    cmd = ["g++", "-O2", "-std=c++17", "-fopenmp", "-ffp-contract=off", "-fno-fast-math",
           "-shared", "-fPIC", SRC, "-o", LIB + ".tmp"]
    subprocess.run(cmd, check=True)
    os.replace(LIB + ".tmp", LIB)
    return LIB


def lib():
    global _lib
    if _lib is None:
        build()
        L = C.CDLL(LIB)
        U64P, I64P = C.POINTER(C.c_uint64), C.POINTER(C.c_int64)
        L.llo_threads.restype = C.c_int
        L.llo_apply.argtypes = [U64P, C.c_int, U64P, U64P, C.c_int64, C.c_int]
        L.llo_right_inverse.argtypes = [U64P, C.c_int, C.c_int, U64P]
        L.llo_preimage_min.argtypes = [U64P, C.c_int, C.c_int, I64P]
        L.llo_convert.argtypes = [U64P, C.c_int, U64P, C.c_int, C.c_int, C.c_int, C.c_void_p, C.c_void_p,
                                  C.c_uint64, C.c_int64, C.c_int]
        L.llo_gather.argtypes = [U64P, C.c_int, C.c_int, C.c_int, C.c_int, C.c_int, C.c_void_p,
                                 C.POINTER(C.c_int32), C.c_void_p, C.c_int]
        L.llo_reduce_fp32.argtypes = [U64P, C.c_int, C.c_int, C.c_int, C.c_int, C.c_int,
                                      C.POINTER(C.c_float), C.POINTER(C.c_float), C.c_int]
        L.llo_reduce_fp64.argtypes = [U64P, C.c_int, C.c_int, C.c_int, C.c_int, C.c_int,
                                      C.POINTER(C.c_float), C.POINTER(C.c_double), C.c_int]
        for f in ("llo_right_inverse", "llo_preimage_min", "llo_convert", "llo_gather",
                  "llo_reduce_fp32", "llo_reduce_fp64"):
            getattr(L, f).restype = C.c_int
        _lib = L
    return _lib


def _cols(cols: Sequence[int]):
    a = np.asarray([int(c) for c in cols], dtype=np.uint64)
    return a, a.ctypes.data_as(C.POINTER(C.c_uint64))


def max_threads() -> int:
    return int(lib().llo_threads())


def apply(cols, hs, threads: int = 0) -> np.ndarray:
    c, cp = _cols(cols)
    hs = np.ascontiguousarray(hs, dtype=np.uint64)
    out = np.empty_like(hs)
    lib().llo_apply(cp, len(c), hs.ctypes.data_as(C.POINTER(C.c_uint64)), out.ctypes.data_as(C.POINTER(C.c_uint64)),
                    hs.size, int(threads))
    return out


def right_inverse(cols, d_out: int):
    c, cp = _cols(cols)
    out = np.zeros(d_out, dtype=np.uint64)
    if lib().llo_right_inverse(cp, len(c), d_out, out.ctypes.data_as(C.POINTER(C.c_uint64))) != 0:
        raise ValueError("layout is not surjective; no right inverse (P:194)")
    return [int(v) for v in out]


def preimage_min(cols, d_out: int) -> np.ndarray:
    c, cp = _cols(cols)
    out = np.empty(1 << d_out, dtype=np.int64)
    if lib().llo_preimage_min(cp, len(c), d_out, out.ctypes.data_as(C.POINTER(C.c_int64))) != 0:
        raise ValueError("layout is not surjective")
    return out


def convert(colsA, colsB, d_out: int, w: int, src: np.ndarray, h0: int = 0, n: Optional[int] = None,
            threads: int = 0, out: Optional[np.ndarray] = None) -> np.ndarray:
    """dst[i] = src[A^+(B(h0 + i))] for i in [0, n) (O5); src packed in A."""
    a, ap = _cols(colsA)
    b, bp = _cols(colsB)
    if n is None:
        n = (1 << len(b)) - h0
    src = np.ascontiguousarray(src)
    assert src.itemsize * src.size >= (w << len(a))
    if out is None:
        out = np.empty(n * w, dtype=np.uint8)
    if lib().llo_convert(ap, len(a), bp, len(b), d_out, int(w), src.ctypes.data, out.ctypes.data, int(h0), int(n),
                         int(threads)) != 0:
        raise ValueError("A is not surjective")
    return out


def gather(cols, d_out: int, axis_shift: int, kbits: int, w: int, src: np.ndarray, idx: np.ndarray,
           threads: int = 0) -> np.ndarray:
    c, cp = _cols(cols)
    src = np.ascontiguousarray(src)
    idx = np.ascontiguousarray(idx, dtype=np.int32)
    out = np.empty_like(src)
    if lib().llo_gather(cp, len(c), d_out, axis_shift, kbits, w, src.ctypes.data,
                        idx.ctypes.data_as(C.POINTER(C.c_int32)), out.ctypes.data, int(threads)) != 0:
        raise ValueError("L is not surjective")
    return out


def reduce(cols, d_out: int, axis_shift: int, axis_bits: int, kbits: int, src: np.ndarray, fp64: bool = False,
           threads: int = 0) -> np.ndarray:
    c, cp = _cols(cols)
    src = np.ascontiguousarray(src, dtype=np.float32)
    n_out = 1 << (d_out - kbits)
    if fp64:
        out = np.empty(n_out, dtype=np.float64)
        r = lib().llo_reduce_fp64(cp, len(c), d_out, axis_shift, axis_bits, kbits,
                                  src.ctypes.data_as(C.POINTER(C.c_float)), out.ctypes.data_as(C.POINTER(C.c_double)),
                                  int(threads))
    else:
        out = np.empty(n_out, dtype=np.float32)
        r = lib().llo_reduce_fp32(cp, len(c), d_out, axis_shift, axis_bits, kbits,
                                  src.ctypes.data_as(C.POINTER(C.c_float)), out.ctypes.data_as(C.POINTER(C.c_float)),
                                  int(threads))
    if r != 0:
        raise ValueError("L is not surjective")
    return out


def cpu_model() -> str:
    try:
        with open("/proc/cpuinfo") as f:
            for line in f:
                if line.startswith("model name"):
                    return line.split(":", 1)[1].strip()
    except OSError:
        pass
    import platform
    return platform.processor() or "unknown"
